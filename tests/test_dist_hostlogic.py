"""a7 host logic on CPU: the slab partition and halo schedule of the C library,
driven for real through torch.distributed (gloo, world_size 2 and 3, one
process per rank): every rank holds only its slab + ghost planes, exchanges
the planes sdag_slab_halo() names with send/recv each sweep, sweeps its slab
with the oracle, and the gathered result equals the global oracle iteration
bit for bit.  This is the NCCL path's bookkeeping with gloo as the transport
and the oracle standing in for the kernel."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import paper_conf_ipps_rawatvsrps19_b200 as sdag


@pytest.mark.parametrize("gnz,rz,P", [(40, 1, 1), (40, 1, 2), (41, 4, 3), (64, 4, 8), (9, 4, 1), (10, 2, 5)])
def test_partition_covers_and_computes_exactly_the_interior(gnz, rz, P):
    owned, computed = [], []
    for r in range(P):
        s = sdag.slab_partition(gnz, rz, P, r)
        g0 = s["z0"] - rz
        assert s["nz_alloc"] == s["nz_own"] + 2 * rz
        owned.extend(range(s["z0"], s["z0"] + s["nz_own"]))
        computed.extend(g0 + k for k in range(s["k_lo"], s["k_hi"]))
        assert s["has_lower"] == (r > 0) and s["has_upper"] == (r < P - 1)
        sizes = [sdag.slab_partition(gnz, rz, P, q)["nz_own"] for q in range(P)]
        assert max(sizes) - min(sizes) <= 1 and sizes == sorted(sizes, reverse=True)
    assert owned == list(range(gnz))
    assert computed == list(range(rz, gnz - rz))


def test_halo_schedule_pairs_up():
    gnz, rz, P = 50, 3, 4
    for r in range(P - 1):
        a = sdag.slab_halo(gnz, rz, P, r)
        b = sdag.slab_halo(gnz, rz, P, r + 1)
        sa = sdag.slab_partition(gnz, rz, P, r)
        sb = sdag.slab_partition(gnz, rz, P, r + 1)
        ga, gb = sa["z0"] - rz, sb["z0"] - rz
        # what r sends up lands in r+1's lower ghosts, and vice versa, same global planes
        assert ga + a["up_send"] == gb + b["lo_recv"]
        assert gb + b["lo_send"] == ga + a["up_recv"]
    assert sdag.slab_halo(gnz, rz, P, 0)["lo_send"] == -1
    assert sdag.slab_halo(gnz, rz, P, P - 1)["up_send"] == -1


@pytest.mark.parametrize("gnz,rz,tt,P", [(40, 1, 2, 2), (41, 1, 3, 4), (50, 2, 2, 3), (64, 4, 2, 4)])
def test_time_tiled_partition_and_halo(gnz, rz, tt, P):
    """Ghost depth H = R_z t; the same owned planes as t = 1; exchanges of any
    planes <= H pair up between neighbours on the same global planes."""
    H = rz * tt
    for r in range(P):
        a = sdag.slab_partition(gnz, rz, P, r)
        b = sdag.slab_partition2(gnz, rz, tt, P, r)
        assert (b["z0"], b["nz_own"], b["halo"]) == (a["z0"], a["nz_own"], H)
        assert b["nz_alloc"] == b["nz_own"] + 2 * H
        g0 = b["z0"] - H
        assert (b["k_lo"] + g0, b["k_hi"] + g0) == (a["k_lo"] + a["z0"] - rz, a["k_hi"] + a["z0"] - rz)
    for planes in range(1, H + 1):
        for r in range(P - 1):
            x = sdag.slab_halo2(gnz, rz, tt, P, r, planes)
            y = sdag.slab_halo2(gnz, rz, tt, P, r + 1, planes)
            gx = sdag.slab_partition2(gnz, rz, tt, P, r)["z0"] - H
            gy = sdag.slab_partition2(gnz, rz, tt, P, r + 1)["z0"] - H
            assert gx + x["up_send"] == gy + y["lo_recv"] and gy + y["lo_send"] == gx + x["up_recv"]
            # the received planes sit right next to the owned range
            assert y["lo_recv"] + planes == H and x["up_recv"] == H + sdag.slab_partition2(gnz, rz, tt, P, r)["nz_own"]
    with pytest.raises(sdag.SdagError):
        sdag.slab_halo2(gnz, rz, tt, P, 0, H + 1)


def test_partition_errors():
    with pytest.raises(sdag.SdagError) as e:
        sdag.slab_partition(20, 4, 8, 0)  # 2 planes per rank < R_z
    assert e.value.code == "DOMAIN"
    with pytest.raises(sdag.SdagError):
        sdag.slab_partition(20, 1, 2, 2)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, P, port, gdims, T, q, tt=1):
    """One rank: its slab + ghosts; per launch of x sweeps (x <= time tile tt,
    the apply_iterated DP schedule) ONE exchange of x*R_z planes, then x oracle
    sweeps, the i-th on the owned range widened by (x-i)*R_z planes into the
    ghosts (the redundant computation of communication-avoiding fusion)."""
    import torch
    import torch.distributed as dist

    import oracle
    import paper_conf_ipps_rawatvsrps19_b200 as sd
    import synth
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=P)
    try:
        rz = 1
        A = synth.uniform(gdims, -1, 1, "gloo-slab")  # each rank regenerates the same global field
        w, nu = [-128 / 30, 14 / 30, 3 / 30, 1 / 30], 0.125
        s = sd.slab_partition2(gdims[0], rz, tt, P, rank)
        H = s["halo"]
        g0 = s["z0"] - H
        zr_lo, zr_hi = rz - g0, gdims[0] - rz - g0  # local planes of the global interior
        loc = np.zeros((s["nz_alloc"], *gdims[1:]))
        lo, hi = max(g0, 0), min(g0 + s["nz_alloc"], gdims[0])
        loc[lo - g0:hi - g0] = A[lo:hi]
        bufs = [loc, loc.copy()]
        sched = sd.fusion_schedule({1: 1.0, **({tt: 1.0 + 0.15 * (tt - 1)} if tt > 1 else {})}, T)[0]
        t = 0
        for x in sched:
            src = bufs[t & 1]
            h = sd.slab_halo2(gdims[0], rz, tt, P, rank, x * rz)
            n = h["planes"]
            reqs = []
            if h["lo_send"] >= 0:
                reqs.append(dist.isend(torch.from_numpy(src[h["lo_send"]:h["lo_send"] + n].copy()), rank - 1))
                rb = torch.empty((n, *gdims[1:]), dtype=torch.float64)
                reqs.append(("recv", dist.irecv(rb, rank - 1), rb, h["lo_recv"]))
            if h["up_send"] >= 0:
                reqs.append(dist.isend(torch.from_numpy(src[h["up_send"]:h["up_send"] + n].copy()), rank + 1))
                rb2 = torch.empty((n, *gdims[1:]), dtype=torch.float64)
                reqs.append(("recv", dist.irecv(rb2, rank + 1), rb2, h["up_recv"]))
            for r_ in reqs:
                if isinstance(r_, tuple):
                    r_[1].wait()
                    src[r_[3]:r_[3] + n] = r_[2].numpy()
                else:
                    r_.wait()
            for i in range(1, x + 1):
                src, dst = bufs[t & 1], bufs[(t + 1) & 1]
                ext = (x - i) * rz
                klo = max(s["k_lo"] - (ext if s["has_lower"] else 0), zr_lo)
                khi = min(s["k_hi"] + (ext if s["has_upper"] else 0), zr_hi)
                oracle.smooth27(src, w, nu, out=dst, krange=(klo, khi))
                t += 1
        res = bufs[T & 1][s["z0"] - g0:s["z0"] - g0 + s["nz_own"]]
        q.put((rank, s["z0"], res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P,tt,T", [(2, 1, 4), (3, 1, 4), (2, 2, 5), (3, 2, 6)])
def test_gloo_slab_iteration_equals_global_oracle(P, tt, T):
    """tt = 2: communication-avoiding temporal fusion (NEXT-1) -- one exchange of
    2 R_z planes per fused pair of sweeps -- still equals the global iteration."""
    gdims = (17, 9, 10)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, P, port, gdims, T, q, tt)) for r in range(P)]
    for p in procs:
        p.start()
    parts = [q.get(timeout=180) for _ in range(P)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import oracle
    import synth
    A = synth.uniform(gdims, -1, 1, "gloo-slab")
    ref = oracle.smooth27_iter(A, [-128 / 30, 14 / 30, 3 / 30, 1 / 30], 0.125, T)
    got = np.zeros(gdims)
    for _, z0, res in parts:
        got[z0:z0 + res.shape[0]] = res
    assert np.array_equal(got, ref)


def test_p2p_entry_points_fail_cleanly_without_a_device():
    """sdag_dist_p2p_* on a host-only slab: status codes, no crash (the peer
    path itself is tests/test_gpu_p2p.py)"""
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    d = sdag.Dist(sdag.spec_text("smooth27"), (30, 20, 22), 0, 2, device=-2)
    for call, code in ((lambda: d.p2p_alloc(), "DEVICE"), (lambda: d.p2p_handle(), "INVALID_ARG"),
                       (lambda: d.p2p_attach(1, b"\0" * 64), "INVALID_ARG"),
                       (lambda: d.p2p_apply_iterated(2, [0.0] * 5, stream=0), "INVALID_ARG")):
        with pytest.raises(sdag.SdagError) as e:
            call()
        assert e.value.code == code
    with pytest.raises(ValueError):
        d.p2p_attach(1, b"short")


def test_dist_from_a_local_plan_matches_the_global_form():
    """SURVEY 8(b)'s sdag_dist_create(local plan, ...): a plan of the owned slab
    (nz_own, ny, nx) gives the same slab layout and local plan as the global
    form with nz = nz_own * nranks, for every rank and ghost depth"""
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    for name, tt in (("smooth27", 1), ("smooth27", 2), ("lap25", 1)):
        spec = sdag.spec_text(name)
        local = sdag.Plan(spec, (24, 20, 22), device="none")
        for P in (1, 2, 3):
            for r in range(P):
                a = sdag.Dist.from_local_plan(local, r, P, time_tile=tt)
                b = sdag.Dist(spec, (24 * P, 20, 22), r, P, device="none", time_tile=tt)
                assert a.layout() == b.layout(), (name, tt, P, r)
                assert a.plan.info["variant"] == b.plan.info["variant"]
    prog = sdag.Program(sdag.fission(sdag.spec_text("rhs4center"), "trivial"), (20, 20, 20), device="none")
    with pytest.raises(sdag.SdagError) as e:
        sdag.Dist.from_local_plan(prog.stage(0), 0, 2)
    assert e.value.code == "UNSUPPORTED"
