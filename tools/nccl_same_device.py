"""Two ranks, one GPU: does NCCL accept a communicator whose ranks share a
device?  If it does, run the z-slab NCCL halo path (sdag_dist_apply_iterated,
ncclSend/ncclRecv) against the single-GPU iteration bitwise; either way the
outcome is printed (the round's GPU pool has one GPU per box)."""
import os
import sys
from pathlib import Path

import numpy as np
import torch
import torch.distributed as tdist

sys.path.insert(0, str(Path(__file__).resolve().parents[1]))
import paper_conf_ipps_rawatvsrps19_b200 as sdag  # noqa: E402
import synth  # noqa: E402

rank, world = int(os.environ["RANK"]), int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
tdist.init_process_group("gloo")
uid = [sdag.nccl_unique_id() if rank == 0 else None]
tdist.broadcast_object_list(uid, src=0)
try:
    comm = sdag.nccl_comm_create(uid[0], world, rank, 0)
except sdag.SdagError as e:
    print(f"rank {rank}: NCCL refused two ranks on one device: {e}", flush=True)
    sys.exit(0)
spec = sdag.spec_text("smooth27")
gdims, T = (40, 30, 34), 6
A = synth.uniform(gdims, -1.0, 1.0, "nccl", "A")
s = [synth.SMOOTH27_W[k] for k in ("w0", "w1", "w2", "w3", "nu")]
d = sdag.Dist(spec, gdims, rank, world, comm=comm, time_tile=2)
(nza, ny, nx), g0 = d.layout()
loc = np.zeros((nza, ny, nx))
lo, hi = max(g0, 0), min(g0 + nza, gdims[0])
loc[lo - g0:hi - g0] = A[lo:hi]
b0 = torch.from_numpy(loc).cuda()
b1 = b0.clone()
d.apply_iterated(b0, b1, T, scalars=s)
torch.cuda.synchronize()
full = sdag.Plan(spec, gdims)
r0 = torch.from_numpy(A).cuda()
r1 = r0.clone()
full.apply_iterated(r0, r1, T, scalars=s)
ref = (r0 if T % 2 == 0 else r1).cpu().numpy()
part = sdag.slab_partition2(gdims[0], 1, 2, world, rank)
got = (b0 if T % 2 == 0 else b1).cpu().numpy()[part["z0"] - g0:part["z0"] - g0 + part["nz_own"]]
ok = np.array_equal(got, ref[part["z0"]:part["z0"] + part["nz_own"]])
print(f"rank {rank}: NCCL halo over 2 ranks on one device, bitwise equal to one GPU: {ok}", flush=True)
tdist.barrier()
sdag.nccl_comm_destroy(comm)
