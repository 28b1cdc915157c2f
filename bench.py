#!/usr/bin/env python3
"""bench.py -- headline benchmark of the sdag hot path on B200.

Workload (BASELINE.json configs[1]): 25-point radius-4 FP64 Laplacian,
512^3 grid per GPU, one sweep per step.  At N GPUs the grid is weak-scaled
as z-slabs (512N x 512 x 512) with a per-step NCCL halo exchange (a7).
A step = parse/plan done once up front (a1-a3, host), then one sweep
(a4-a5) [+ exchange (a7) for N>1] over the resident input.

Prints ONE JSON line (rank 0).  --impl reference times the CPU oracle (the
reference arm of this tier) on the same metric/config.  --config selects
another BASELINE stencil for reporting (not the headline line).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "FP64 GFLOP/s and HBM GB/s per stencil, % of roofline, at 1/2/4/8 B200"

CONFIGS = {
    # name: (spec, dims per GPU, BASELINE config string, flops/pt)
    "lap25": ("lap25", (512, 512, 512), "3D 4th-order 25-point Laplacian (order 4), 512^3 FP64, single GPU"),
    "jacobi7": ("jacobi7", (64, 64, 64), "3D 7-point Jacobi (order 1), 64^3 FP64 grid, single sweep, 1 input/1 output"),
    "hypterm": ("hypterm", (320, 320, 320), "ExpCNS hypterm-style DAG (order 4, ~8 inputs, multiple outputs), 320^3 FP64"),
    "rhs4center": ("rhs4center", (320, 320, 320),
                   "SW4 rhs4th3fort-style elastic-wave stencil (order 2, multi-statement, ~300 FLOP/pt), 320^3 FP64"),
    "smooth27": ("smooth27", (1024, 1024, 1024),
                 "iterated 27-point order-2 stencil, 1024^3 FP64 weak-scaled as z-slabs with halo exchange"),
}


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return d.get("hbm_gbs", 6650.0), "measured"
    return 6650.0, "fallback"


def load_traffic(variant, dims, batch=1):
    """DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum) from a
    committed ncu --set full capture of this variant at this size, else None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f)
    key = variant + "@" + "x".join(str(x) for x in ([batch] if batch > 1 else []) + list(dims))
    return d.get(key)


class Clocks:
    """nvidia-smi sampler running during the timed region."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            p = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                  "-lms", "100"], stdout=subprocess.PIPE, text=True)
        except Exception:
            return
        while not self._stop.is_set():
            line = p.stdout.readline()
            if not line:
                break
            self.samples.append([x.strip() for x in line.split(",")])
        p.terminate()
        try:
            p.wait(timeout=2)
        except Exception:
            p.kill()

    def __enter__(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        time.sleep(0.3)
        return self

    def __exit__(self, *a):
        self._stop.set()
        self._t.join(timeout=3)

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for s in self.samples:
            for n, v in zip(names, s[3:7]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.samples)}


def cpu_baseline_lap25(A, c, seconds=10.0):
    """Time the oracle (as it stands) on the same 512^3 input: whole sweeps,
    repeated for ~`seconds` of CPU work (the bounded sample)."""
    import oracle
    cores = len(os.sched_getaffinity(0))
    nz, ny, nx = A.shape
    out = np.zeros_like(A)
    oracle.lap25(A, c, out=out, krange=(4, 6))  # warm (build + page-in)
    reps, t0 = 0, time.perf_counter()
    while True:
        oracle.lap25(A, c, out=out)
        reps += 1
        if time.perf_counter() - t0 >= seconds:
            break
    dt = time.perf_counter() - t0
    pts = reps * (nz - 8) * (ny - 8) * (nx - 8)
    return {"value": pts * 29 / dt / 1e9, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
            "sample": f"{reps} full 512^3 sweeps of the benchmark input ({pts} interior points), {dt:.1f} s, "
                      f"OpenMP over k with {cores} threads"}


def run_reference(args):
    """--impl reference: the CPU oracle (this tier's reference arm) on the host
    cores, same metric and config: each step is one full 512^3 sweep of the same
    seeded input (~0.1-0.3 s of CPU work per step)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import synth
    dims = CONFIGS["lap25"][1]
    ins, sc = synth.lap25_inputs(dims, cfg="cfg2")
    A = ins["A"]
    c = [sc[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    import oracle
    cores = len(os.sched_getaffinity(0))
    out = np.zeros_like(A)
    nz, ny, nx = dims
    oracle.lap25(A, c, out=out, krange=(4, 6))
    for _ in range(args.warmup):
        oracle.lap25(A, c, out=out)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        oracle.lap25(A, c, out=out)
    dt = time.perf_counter() - t0
    pts = args.steps * (nz - 8) * (ny - 8) * (nx - 8)
    val = pts * 29 / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": CONFIGS["lap25"][2], "stencil": "lap25", "grid": list(dims),
                       "step": "one full oracle sweep of the 512^3 input on the host cores"},
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": cores, "kind": "oracle",
                             "sample": f"{args.steps} full 512^3 sweeps (all interior points)"},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


def run_other(args):
    """One line for another BASELINE stencil at N=1 (recorded under profiles/, not the headline).
    Inputs: seeded torch generator on the device (timing is data-independent; parity of
    the same kernels on synth/ inputs is in tests/test_gpu_parity.py)."""
    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    name = args.config
    spec = sdag.spec_text(name)
    dims = CONFIGS[name][1]
    torch.cuda.set_device(0)
    g = torch.Generator(device="cuda").manual_seed(20190520)
    batch, T = 1, 1
    if name == "jacobi7":
        batch = 128  # config 1b: 128 independent 64^3 problems in one launch (latency-bound alone)
    # the non-headline lines use the measured (hierarchical tune=1) plan, as a
    # production user would; plan time is outside the timed region
    plan = sdag.Plan(spec, dims, batch=batch, tune=not args.no_tune, variant=args.variant)
    info = plan.info
    shape = (batch, *dims) if batch > 1 else dims
    scal = {"jacobi7": [4.0, 0.5, 0.25], "hypterm": [0.5, 0.25, 0.125, 0.8, -0.2, 4 / 105, -1 / 280],
            "rhs4center": [0.75, 1 / 6, 1 / 144, 1.0, 1.0], "smooth27": [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125]}[name]
    arrs = [torch.rand(shape, dtype=torch.float64, device="cuda", generator=g) + 0.5
            for _ in range(info["n_arrays3d"])]
    a1 = [torch.rand(dims[2 - q], dtype=torch.float64, device="cuda", generator=g) + 0.5
          for q in range(info["n_arrays1d"])]
    if name == "smooth27":
        T = 12  # config 5: iterated T = 12 sweeps (Table I "T", reading R5)
        b0, b1 = arrs[1], arrs[0]

        def step():
            plan.apply_iterated(b0, b1, T, scal)
    elif batch > 1:
        def step():
            plan.apply_batched(batch, arrs, a1, scal)
    else:
        def step():
            plan.apply(arrs, a1, scal)
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    l0 = sdag.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(0) as clk:
        torch.cuda.synchronize()
        e0.record()
        for _ in range(args.steps):
            step()
        e1.record()
        torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / args.steps
    launches = sdag.launch_count() - l0
    pts = info["points"] * batch * T
    flops = info["flops_per_point"] * pts
    byts = info["bytes_per_point"] * pts
    kms = ms / (launches / args.steps)
    hbm, src = load_peaks()
    if name == "rhs4center":
        fp64 = sdag.fp64_peak()
        achieved = info["flops_per_point"] * info["points"] / (kms * 1e-3) / 1e12
        roof = {"bound": "fp64", "achieved": achieved, "peak": fp64 / 1e12, "unit": "TFLOP/s", "frac": achieved * 1e12 / fp64,
                "peak_source": "measured DFMA micro-benchmark (sdag_measure_fp64_peak) in this run"}
    else:
        achieved = info["bytes_per_point"] * info["points"] * batch / (kms * 1e-3) / 1e9
        roof = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s", "frac": achieved / hbm,
                "peak_source": src}
    kernel = info["variant"]
    if name == "smooth27" and launches < T * args.steps:
        # temporal fusion (NEXT-1): the launches are 2-sweep kernels; one launch
        # reads its input and writes its output once, so its algorithmic bytes
        # are one sweep's -- the roofline below is the fused kernel's own
        fl = [ln for ln in plan.describe().splitlines() if "temporal fusion" in ln]
        kernel = fl[0].split(":", 1)[1].split()[0] if fl else kernel
        # per SURVEY 8(d)'s unit (one written point of one sweep): a launch processes
        # T / launches sweeps' units, so the sweep-equivalent rate can exceed the
        # HBM roofline of unfused sweeps -- the point of temporal fusion
        spl = T * args.steps / launches
        roof["sweep_equivalent"] = {"sweeps_per_launch": spl, "achieved": achieved * spl,
                                    "frac": achieved * spl / hbm}
    roof.update({"traffic": load_traffic(kernel, dims, batch), "kernel_ms": kms, "kernel": kernel})
    line = {"metric": METRIC, "value": flops / (ms * 1e-3) / 1e9, "unit": "GFLOP/s", "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded torch generator)",
            "config": {"workload": CONFIGS[name][2], "stencil": name, "grid": list(dims), "batch": batch,
                       "sweeps_per_step": T, "variant": kernel, "tuned": not args.no_tune,
                       "l2": "inputs > 126 MB L2 (no flush needed)",
                       "launches_per_step": launches // args.steps, "flops_per_point": info["flops_per_point"],
                       "bytes_per_point": info["bytes_per_point"]},
            "hbm_gbs": byts / (ms * 1e-3) / 1e9, "roofline": roof, "gpu_launches": launches,
            "clocks": clk.summary()}
    print(json.dumps(line))
    return 0


def run_slabs27(args):
    """Config 5 as BASELINE names it: the iterated 27-point smoother, 1024^3 per
    GPU, T = 12 sweeps per step, weak-scaled as z-slabs (one rank per GPU).
    --halo nccl: ghost planes exchanged by NCCL send/recv on a comm stream,
    overlapped with the interior launch (sdag_dist_apply_iterated);
    --halo p2p: the boundary launches store their planes straight into the
    neighbours' ghost planes over NVLink (sdag_dist_p2p_apply_iterated; CUDA IPC
    handles exchanged over the process group), no NCCL.  Ghost depth 2 R_z
    (time_tile 2): one exchange per fused 2-sweep launch.
    SDAG_BENCH_SAME_DEVICE=1 maps every rank to cuda:0 (plumbing check of the
    multi-process p2p path on one GPU; times are then not scaling numbers)."""
    import torch
    import torch.distributed as tdist
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = 0 if os.environ.get("SDAG_BENCH_SAME_DEVICE") else int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    halo = args.halo or "nccl"
    pg = None
    if world > 1:
        if halo == "p2p":
            tdist.init_process_group("gloo")  # host plumbing only: IPC handles, barrier, timing reduce
        else:
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
        pg = tdist
    name, T, tt = "smooth27", 12, 2
    spec = sdag.spec_text(name)
    n = int(os.environ.get("SDAG_BENCH_SLAB_N", "1024"))
    gdims = (n * world, n, n)
    scal = [-128 / 30, 14 / 30, 3 / 30, 1 / 30, 0.125]
    comm = None
    if halo == "nccl" and world > 1:
        uid = [sdag.nccl_unique_id() if rank == 0 else None]
        tdist.broadcast_object_list(uid, src=0)
        comm = sdag.nccl_comm_create(uid[0], world, rank, local)
    dd = sdag.Dist(spec, gdims, rank, world, comm=comm, time_tile=tt, variant=args.variant)
    (nza, ny, nx), g0 = dd.layout()
    part = sdag.slab_partition2(gdims[0], 1, tt, world, rank)
    stream = torch.cuda.current_stream()
    full = torch.from_numpy(__import__("synth").uniform((nza, ny, nx), -1.0, 1.0, "cfg5-slab", rank))
    if halo == "p2p":
        b0, b1 = dd.p2p_alloc()
        b0.copy_(full)
        b1.copy_(full)
        torch.cuda.synchronize()
        if world > 1:
            hs = [None] * world
            tdist.all_gather_object(hs, dd.p2p_handle())
            if rank > 0:
                dd.p2p_attach(0, hs[rank - 1])
            if rank < world - 1:
                dd.p2p_attach(1, hs[rank + 1])

        def step():
            dd.p2p_apply_iterated(T, scalars=scal, stream=stream)
    else:
        b0 = full.cuda()
        b1 = b0.clone()
        cs = torch.cuda.Stream()

        def step():
            dd.apply_iterated(b0, b1, T, scalars=scal, stream=stream, comm_stream=cs)
    del full
    info = dd.plan.info
    pts_rank = (part["k_hi"] - part["k_lo"]) * (ny - 2) * (nx - 2) * T
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if pg:
        tdist.barrier()
    l0 = sdag.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
    launches = sdag.launch_count() - l0
    ms = e0.elapsed_time(e1)
    red = torch.tensor([ms, float(pts_rank)], dtype=torch.float64)
    if pg:
        tdist.barrier()
        mx = red.clone()
        tdist.all_reduce(mx, op=tdist.ReduceOp.MAX)
        sm = red.clone()
        tdist.all_reduce(sm, op=tdist.ReduceOp.SUM)
        ms_max, total_pts = float(mx[0]), float(sm[1])
    else:
        ms_max, total_pts = ms, float(pts_rank)
    flops = total_pts * info["flops_per_point"] * args.steps
    if rank == 0:
        line = {"metric": METRIC, "value": flops / (ms_max * 1e-3) / 1e9, "unit": "GFLOP/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic (counter-based generator, per-rank slab)",
                "config": {"workload": CONFIGS[name][2], "stencil": name, "grid_per_gpu": [n, n, n],
                           "global_grid": list(gdims), "decomposition": f"z-slabs x{world}", "halo": halo,
                           "time_tile": tt, "sweeps_per_step": T, "variant": info["variant"],
                           "same_device": bool(os.environ.get("SDAG_BENCH_SAME_DEVICE")),
                           "l2": "8 GiB slab/GPU > 126 MB L2 (no flush needed)"},
                "hbm_gbs_sweep_equivalent": total_pts * info["bytes_per_point"] * args.steps / (ms_max * 1e-3) / 1e9,
                "gpu_launches": launches, "clocks": clk.summary()}
        print(json.dumps(line))
    if pg:
        tdist.barrier()
        tdist.destroy_process_group()
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="sdag", choices=["sdag", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--variant", default=None)
    ap.add_argument("--tune", action="store_true", help="headline: tune=1 plan (the --config lines tune by default)")
    ap.add_argument("--no-tune", action="store_true", help="--config lines: heuristic plan instead of tune=1")
    ap.add_argument("--force-dist", action="store_true",
                    help="take the z-slab/NCCL path even on one rank (plumbing check of the multi-GPU code)")
    ap.add_argument("--config", default="lap25", choices=list(CONFIGS),
                    help="lap25 = the headline line; the others record the remaining BASELINE stencils (N=1)")
    ap.add_argument("--halo", default=None, choices=["nccl", "p2p"],
                    help="z-slab halo path (default nccl); with --config smooth27: the z-slab run of config 5 "
                         "(BASELINE's multi-GPU workload)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)
    if args.config == "smooth27" and (args.halo or int(os.environ.get("WORLD_SIZE", "1")) > 1):
        return run_slabs27(args)
    if args.config != "lap25":
        return run_other(args)

    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = 0 if os.environ.get("SDAG_BENCH_SAME_DEVICE") else int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    p2p = args.halo == "p2p"
    dist = None
    if world > 1:
        import torch.distributed as tdist
        if p2p:  # host plumbing only (IPC handles, barriers, the timing reduce)
            tdist.init_process_group("gloo")
        else:
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
        dist = tdist
    red_dev = "cpu" if p2p else "cuda"
    name = "lap25"
    spec = sdag.spec_text(name)
    ldims = CONFIGS[name][1]
    gdims = (ldims[0] * world, ldims[1], ldims[2])
    use_dist = world > 1 or args.force_dist or args.halo == "p2p"
    ins, sc = synth.lap25_inputs(ldims, cfg="cfg2") if not use_dist else (None, dict(synth.LAP25_COEFS))
    c = [sc[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    stream = torch.cuda.current_stream()

    if not use_dist:
        plan = sdag.Plan(spec, ldims, tune=args.tune, variant=args.variant)
        A = ins["A"]
        dA = torch.from_numpy(A).cuda()
        dB = torch.zeros(ldims, dtype=torch.float64, device="cuda")
        arrays = [dB, dA]
        info = plan.info
        pts_rank = info["points"]

        def step():
            plan.apply(arrays, scalars=c, stream=stream)
    else:
        comm = None
        if not p2p:
            uid = [None]
            if rank == 0:
                try:
                    uid = [sdag.nccl_unique_id()]
                except sdag.SdagError as e:  # no usable NCCL: the peer-memory halo needs none
                    print(f"bench: NCCL halo unavailable ({e}); using the p2p halo", file=sys.stderr)
            if dist:
                dist.broadcast_object_list(uid, src=0)
            if uid[0] is None:
                p2p = True
            else:
                comm = sdag.nccl_comm_create(uid[0], world, rank, local)
        dd = sdag.Dist(spec, gdims, rank, world, comm=comm, tune=args.tune, variant=args.variant)
        (nza, ny, nx), g0 = dd.layout()
        part = sdag.slab_partition(gdims[0], 4, world, rank)
        # this rank's slab of the global synthetic input, regenerated from the counter-based generator
        full = synth.uniform((nza, ny, nx), -1.0, 1.0, "cfg2-slab", rank)
        if p2p:
            # --halo p2p: library-owned slab buffers; the input's ghost planes are
            # pushed over NVLink by the neighbours and flag-ordered (one sweep =
            # sdag_dist_p2p_apply_iterated with T = 1), no NCCL
            dA, dB = dd.p2p_alloc()
            dA.copy_(torch.from_numpy(full))
            dB.zero_()
            torch.cuda.synchronize()
            if dist:
                hs = [None] * world
                dist.all_gather_object(hs, dd.p2p_handle())
                if rank > 0:
                    dd.p2p_attach(0, hs[rank - 1])
                if rank < world - 1:
                    dd.p2p_attach(1, hs[rank + 1])
        else:
            dA = torch.from_numpy(full).cuda()
            dB = torch.zeros((nza, ny, nx), dtype=torch.float64, device="cuda")
        arrays = [dB, dA]
        plan = dd.plan
        info = plan.info
        pts_rank = (part["k_hi"] - part["k_lo"]) * (ny - 8) * (nx - 8)
        comm_stream = torch.cuda.Stream()

        def step():
            if p2p:
                dd.p2p_apply_iterated(1, scalars=c, stream=stream)
            else:
                dd.apply(arrays, scalars=c, stream=stream, comm_stream=comm_stream)

    flops_pt = info["flops_per_point"]
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    l0 = sdag.launch_count()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(args.steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
    launches = sdag.launch_count() - l0
    ms = e0.elapsed_time(e1)
    ms_t = torch.tensor([ms], dtype=torch.float64, device=red_dev)
    pts_t = torch.tensor([float(pts_rank)], dtype=torch.float64, device=red_dev)
    if dist:
        dist.barrier()
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
        dist.all_reduce(pts_t, op=dist.ReduceOp.SUM)
    ms_max = float(ms_t.item())
    total_pts = float(pts_t.item())
    gflops = total_pts * flops_pt * args.steps / (ms_max * 1e-3) / 1e9

    # dominant kernel: the sweep.  N=1: the step is exactly one launch.  N>1: time the
    # local sweep kernel alone (same stream, same launch configuration).
    kms = ms / max(1, launches) if not use_dist else None
    if use_dist:
        ka, kb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        lp = dd.plan
        ka.record(stream)
        for _ in range(args.steps):
            lp.apply(arrays, scalars=c, stream=stream)
        kb.record(stream)
        torch.cuda.synchronize()
        kms = ka.elapsed_time(kb) / args.steps
    peak, peak_src = load_peaks()
    bytes_launch = info["bytes_per_point"] * info["points"]
    achieved = bytes_launch / (kms * 1e-3) / 1e9
    traffic = load_traffic(info["variant"], ldims) if not use_dist else None

    e2e = None
    if not args.no_e2e and not use_dist:
        hA = torch.from_numpy(A).pin_memory().numpy()
        hB = torch.zeros(ldims, dtype=torch.float64).pin_memory().numpy()
        ee = []
        plan.apply_host([hB, hA], scalars=c, stream=stream)  # warm workspace
        up = down = 0
        for _ in range(max(3, min(args.steps, 5))):
            t0 = time.perf_counter()
            up, down = plan.apply_host([hB, hA], scalars=c, stream=stream)
            ee.append(time.perf_counter() - t0)
        t_e2e = statistics.median(ee)
        e2e = {"value": info["points"] * flops_pt / t_e2e / 1e9, "unit": "GFLOP/s", "h2d_bytes_per_step": up,
               "d2h_bytes_per_step": down, "ms_per_step": t_e2e * 1e3}
    elif not args.no_e2e and use_dist:
        # every rank: its slab (local layout, ghost planes included: the host holds
        # them, so no exchange) host -> device from pinned memory, the sweep of its
        # planes of the global interior, those planes device -> host, pipelined over
        # z-chunks (sdag_dist_apply_host); wall time per step, max over ranks
        hA = dA.cpu().pin_memory().numpy()
        hB = torch.zeros((nza, ny, nx), dtype=torch.float64).pin_memory().numpy()
        dd.apply_host([hB, hA], scalars=c, stream=stream)  # warm workspace
        ee = []
        up = down = 0
        for it in range(max(3, min(args.steps, 5))):
            if dist:
                dist.barrier()
            t0 = time.perf_counter()
            up, down = dd.apply_host([hB, hA], scalars=c, stream=stream)
            ee.append(time.perf_counter() - t0)
        t_loc = torch.tensor([statistics.median(ee)], dtype=torch.float64, device=red_dev)
        if dist:
            dist.all_reduce(t_loc, op=dist.ReduceOp.MAX)
        t_e2e = float(t_loc.item())
        e2e = {"value": total_pts * flops_pt / t_e2e / 1e9, "unit": "GFLOP/s", "h2d_bytes_per_step": int(up),
               "d2h_bytes_per_step": int(down), "ms_per_step": t_e2e * 1e3, "per_rank_bytes": True}

    cpu = None
    if rank == 0 and not use_dist and not args.no_cpu:
        cpu = cpu_baseline_lap25(A, c)

    if rank == 0:
        line = {
            "metric": METRIC, "value": gflops, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": CONFIGS[name][2], "stencil": name, "grid_per_gpu": list(ldims),
                       "global_grid": list(gdims), "decomposition": f"z-slabs x{world}" if use_dist else "none",
                       "halo": ("p2p" if p2p else "nccl") if use_dist else None,
                       "variant": info["variant"], "flops_per_point": flops_pt,
                       "bytes_per_point": info["bytes_per_point"],
                       "l2": "input 1 GiB/GPU > 126 MB L2 (no flush needed)"},
            "hbm_gbs": total_pts * info["bytes_per_point"] * args.steps / (ms_max * 1e-3) / 1e9,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic, "peak_source": peak_src,
                         "kernel": "sdag_sweep<Lap25> " + info["variant"], "kernel_ms": kms},
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "clocks": clk.summary(),
        }
        print(json.dumps(line))
    if dist:
        dist.barrier()
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
