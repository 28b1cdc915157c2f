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


def _worker(rank, P, port, gdims, T, q):
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
        s = sd.slab_partition(gdims[0], rz, P, rank)
        h = sd.slab_halo(gdims[0], rz, P, rank)
        g0 = s["z0"] - rz
        loc = np.zeros((s["nz_alloc"], *gdims[1:]))
        lo, hi = max(g0, 0), min(g0 + s["nz_alloc"], gdims[0])
        loc[lo - g0:hi - g0] = A[lo:hi]
        bufs = [loc, loc.copy()]
        for t in range(T):
            src, dst = bufs[t & 1], bufs[(t + 1) & 1]
            reqs = []
            if h["lo_send"] >= 0:
                reqs.append(dist.isend(torch.from_numpy(src[h["lo_send"]:h["lo_send"] + rz].copy()), rank - 1))
                rb = torch.empty((rz, *gdims[1:]), dtype=torch.float64)
                reqs.append(("recv", dist.irecv(rb, rank - 1), rb, h["lo_recv"]))
            if h["up_send"] >= 0:
                reqs.append(dist.isend(torch.from_numpy(src[h["up_send"]:h["up_send"] + rz].copy()), rank + 1))
                rb2 = torch.empty((rz, *gdims[1:]), dtype=torch.float64)
                reqs.append(("recv", dist.irecv(rb2, rank + 1), rb2, h["up_recv"]))
            for r_ in reqs:
                if isinstance(r_, tuple):
                    r_[1].wait()
                    src[r_[3]:r_[3] + rz] = r_[2].numpy()
                else:
                    r_.wait()
            oracle.smooth27(src, w, nu, out=dst, krange=(s["k_lo"], s["k_hi"]))
        res = bufs[T & 1][s["z0"] - g0:s["z0"] - g0 + s["nz_own"]]
        q.put((rank, s["z0"], res))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [2, 3])
def test_gloo_slab_iteration_equals_global_oracle(P):
    gdims, T = (17, 9, 10), 4
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, P, port, gdims, T, q)) for r in range(P)]
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
