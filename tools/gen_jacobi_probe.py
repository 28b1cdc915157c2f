import os, sys, json
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import torch
import paper_conf_ipps_rawatvsrps19_b200 as sdag
t = sdag.spec_text("jacobi7").replace("#pragma stream k block (32,16) unroll j=2\n", "")
def timed(f, reps=20):
    for _ in range(3): f()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize(); e0.record()
    for _ in range(reps): f()
    e1.record(); torch.cuda.synchronize(); return e0.elapsed_time(e1) / reps
for dims, batch in (((512, 512, 512), 1), ((64, 64, 64), 128)):
    shape = (batch, *dims) if batch > 1 else dims
    A = torch.rand(shape, dtype=torch.float64, device="cuda"); B = torch.zeros_like(A)
    base = sdag.Plan(t, dims, batch=batch, variant="jit")
    for v in base.variants()[:5]:
        p = sdag.Plan(t, dims, batch=batch, variant=v)
        f = (lambda: p.apply_batched(batch, [B, A], [], [4.0, 0.5, 0.25])) if batch > 1 else (lambda: p.apply([B, A], [], [4.0, 0.5, 0.25]))
        print(json.dumps({"dims": dims, "batch": batch, "variant": v, "ms": round(timed(f), 4)}), flush=True)
