"""Two ranks of the peer-memory halo path in two processes on cuda:0 (used by
tests/test_gpu_p2p.py): CUDA IPC handles all-gathered over gloo, T sweeps of
the 27-point smoother, each rank's owned planes compared bitwise with the
single-GPU iteration computed in the same process."""
import os
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, HERE)
sys.path.insert(0, os.path.dirname(HERE))

import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as tdist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def run(rank, world, q):
    try:
        import paper_conf_ipps_rawatvsrps19_b200 as sdag
        import synth
        tdist.init_process_group("gloo", rank=rank, world_size=world)
        torch.cuda.set_device(0)
        gdims, T, tt = (36, 24, 30), 9, 2
        ins, sc = synth.smooth27_inputs(gdims, cfg="slab")
        A = ins["A"]
        s = [sc[k] for k in ("w0", "w1", "w2", "w3", "nu")]
        spec = sdag.spec_text("smooth27")
        full = sdag.Plan(spec, gdims)
        f0 = torch.from_numpy(A).cuda()
        f1 = f0.clone()
        full.apply_iterated(f0, f1, T, scalars=s)
        ref = (f0 if T % 2 == 0 else f1).cpu().numpy()

        d = sdag.Dist(spec, gdims, rank, world, time_tile=tt)
        b0, b1 = d.p2p_alloc()
        (nza, ny, nx), g0 = d.layout()
        loc = np.zeros((nza, ny, nx))
        lo, hi = max(g0, 0), min(g0 + nza, gdims[0])
        loc[lo - g0:hi - g0] = A[lo:hi]
        b0.copy_(torch.from_numpy(loc))
        b1.copy_(torch.from_numpy(loc))
        torch.cuda.synchronize()
        hs = [None] * world
        tdist.all_gather_object(hs, d.p2p_handle())
        if rank > 0:
            d.p2p_attach(0, hs[rank - 1])
        if rank < world - 1:
            d.p2p_attach(1, hs[rank + 1])
        tdist.barrier()
        d.p2p_apply_iterated(T, scalars=s)
        torch.cuda.synchronize()
        res = (b0 if T % 2 == 0 else b1).cpu().numpy()
        part = sdag.slab_partition2(gdims[0], 1, tt, world, rank)
        z0, n = part["z0"], part["nz_own"]
        ok = np.array_equal(res[z0 - g0:z0 - g0 + n], ref[z0:z0 + n])
        tdist.barrier()  # keep the mappings alive until every rank has read its result
        d.close()
        q.put((rank, bool(ok), ""))
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, False, traceback.format_exc()))


if __name__ == "__main__":
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=run, args=(r, world, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = [q.get(timeout=500) for _ in range(world)]
    for p in ps:
        p.join(60)
    bad = False
    for rank, ok, err in sorted(res):
        print(f"rank {'ok' if ok else 'FAILED'} {rank}", err)
        bad |= not ok
    sys.exit(1 if bad else 0)
