#!/usr/bin/env python3
"""bench.py -- the BASELINE benchmark of the sdag hot path on B200.

BASELINE.json metric: "FP64 GFLOP/s and HBM GB/s per stencil, % of roofline,
at 1/2/4/8 B200".  One JSON line (rank 0):

  headline  (`value`, `roofline`, `e2e`, `cpu_baseline`): configs[1], the
            25-point radius-4 FP64 Laplacian on a 512^3 grid per GPU, one
            sweep per step (a4-a5 over inputs resident in HBM).  At N GPUs the
            grid is weak-scaled as z-slabs (512N x 512 x 512) with the per-sweep
            NCCL halo exchange (a7) inside the step.
  per_config (N = 1): every other BASELINE stencil in the same run -- 1 (64^3
            single sweep: latency), 1b (128 x 64^3 batched), 3 hypterm 320^3,
            4 rhs4center 320^3, 5 the iterated 27-point smoother 1024^3 x 12
            sweeps -- each with its own roofline, kernel time, traffic, clocks.
  per_config (N > 1): config 5 as z-slabs (1024^3 per GPU, T = 12, NCCL
            halo) with its weak-scaling efficiency E(N) = t_sweep(1) / t_sweep(N),
            t_sweep(1) measured in the same run on each rank's own GPU.

--gpus N without torchrun re-launches itself under torch.distributed.run with
N ranks (127.0.0.1); under torchrun WORLD_SIZE must equal N.
--impl reference times the CPU oracle (this tier's reference arm) on the
headline workload with an identical `config`.
Inputs: the synth/ recipes (counter-based generator), built on the device for
the BASELINE sizes -- the same values the parity tests feed the oracle.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "FP64 GFLOP/s and HBM GB/s per stencil, % of roofline, at 1/2/4/8 B200"
WORKLOAD = {
    "1": "3D 7-point Jacobi (order 1), 64^3 FP64 grid, single sweep, 1 input/1 output",
    "1b": "3D 7-point Jacobi (order 1), 64^3 FP64 grid, single sweep, batched: 128 independent problems per launch",
    "2": "3D 4th-order 25-point Laplacian (order 4), 512^3 FP64, single GPU",
    "3": "ExpCNS hypterm-style DAG (order 4, ~8 inputs, multiple outputs), 320^3 FP64",
    "4": "SW4 rhs4th3fort-style elastic-wave stencil (order 2, multi-statement, ~300 FLOP/pt), 320^3 FP64",
    "5": "iterated 27-point order-2 stencil, 1024^3 FP64 weak-scaled as z-slabs with halo exchange at 2/4/8 B200",
}
# config -> (stencil, dims per GPU, batch, sweeps per step)
CONFIGS = {"1": ("jacobi7", (64, 64, 64), 1, 1), "1b": ("jacobi7", (64, 64, 64), 128, 1),
           "2": ("lap25", (512, 512, 512), 1, 1), "3": ("hypterm", (320, 320, 320), 1, 1),
           "4": ("rhs4center", (320, 320, 320), 1, 1), "5": ("smooth27", (1024, 1024, 1024), 1, 12)}
# P100 numbers the paper prints, quoted as context (other hardware: never the target)
PAPER_P100 = {
    "3": {"value": 1.08e10 / 1e9, "unit": "GFLOP (per sweep, nvprof)", "note": "Table III P:1939 hypterm: 1.08e10 "
          "FP64 flops per sweep at 312^3 interior; best P100 variant (global memory, P:2167-2173)"},
    "4": {"value": 1.93e10 / 1e9, "unit": "GFLOP (per sweep, nvprof)", "note": "Table III P:1949 rhs4center: "
          "1.93e10 executed FP64 flops per sweep (nvcc CSE; 666 x 316^3 = 2.10e10 canonical)"},
}


def headline_config(world):
    """`config` of the headline line -- identical in both arms (same_config)."""
    n = 512
    return {"workload": WORKLOAD["2"], "stencil": "lap25", "grid_per_gpu": [n, n, n], "global_grid": [n * world, n, n],
            "decomposition": f"z-slabs x{world}" if world > 1 else "none",
            "l2": "input 1 GiB/GPU > 126 MB L2 (no flush needed)"}


# ---------------------------------------------------------------------------
# peaks, committed ncu counters, clocks
# ---------------------------------------------------------------------------

def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        if "hbm_gbs" in d:
            return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json copy bandwidth)"
    return 6650.0, "fallback (B200_PROFILING.md)"


def load_counters(variant, dims, batch=1):
    """Per-launch ncu counters of this variant at this size, from one committed
    `ncu --set full` capture (profiles/ncu_counters.json): DRAM bytes read+write
    and executed FP64 flops (2 x DFMA + DADD + DMUL thread instructions)."""
    key = variant + "@" + "x".join(str(x) for x in ([batch] if batch > 1 else []) + list(dims))
    out = {}
    for fn in ("ncu_counters.json", "ncu_traffic.json"):
        p = os.path.join(ROOT, "profiles", fn)
        if os.path.exists(p):
            with open(p) as f:
                d = json.load(f).get(key)
            if isinstance(d, dict):
                for k, v in d.items():
                    out.setdefault(k, v)
            elif d is not None:
                out.setdefault("dram_bytes", d)
    return out


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
                                  "-lms", "50"], stdout=subprocess.PIPE, text=True)
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
        mx = [float(s[1]) for s in self.samples if len(s) > 1 and s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for s in self.samples:
            for n, v in zip(names, s[3:7]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.samples)}


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


# ---------------------------------------------------------------------------
# device inputs (synth recipes, bit-identical to the parity tests' arrays)
# ---------------------------------------------------------------------------

def build_arrays(sdag, plan, name, dims, batch=1):
    """3D formals in formal order (inputs/inouts from the recipe, outputs empty),
    1D formals, scalars in formal order."""
    import torch
    import synth
    cfg, a3, a1, sc = synth.recipe(name)
    shape = (batch, *dims) if batch > 1 else tuple(dims)
    arrays3d, arrays1d, scal = [], [], []
    for kind, _, nm, role in plan.args():
        if kind == 0:
            if nm in a3:
                lo, hi = a3[nm]
                arrays3d.append(synth.uniform_torch(shape, lo, hi, cfg, nm))
            else:
                arrays3d.append(torch.empty(shape, dtype=torch.float64, device="cuda"))
        elif kind == 1:
            lo, hi = a1[nm]
            n = dims[role]
            arrays1d.append(torch.from_numpy(synth.uniform((n,), lo, hi, cfg, nm)).cuda())
        else:
            scal.append(sc[nm])
    return arrays3d, arrays1d, scal


def timed(step, steps, warmup, stream, clock_index, barrier=None):
    """K steps between CUDA events on `stream`, max-over-ranks done by the caller.
    The nvidia-smi clock sampler starts first (it needs ~0.3 s to come up); the W
    warm-up steps run after it, right before the timed region, so the GPU enters
    the region busy and at its working clocks rather than after 0.3 s idle (an
    idle GPU adds ~0.1 ms of ramp to the first timed launch: a 10-step region of
    the batched Jacobi read 0.117 ms per step, 100 steps 0.1066). Then a
    synchronize, the ranks' barrier (N > 1), a synchronize, and the K steps.
    -> (ms per step, launches per step, clocks)"""
    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(clock_index) as clk:
        for _ in range(warmup):
            step()
        torch.cuda.synchronize()
        if barrier is not None:
            barrier()
            torch.cuda.synchronize()
        l0 = sdag.launch_count()
        e0.record(stream)
        for _ in range(steps):
            step()
        e1.record(stream)
        torch.cuda.synchronize()
    return e0.elapsed_time(e1) / steps, (sdag.launch_count() - l0) / steps, clk.summary()


def roofline(info, kms, batch, peak_hbm, peak_src, fp64_peak, counters, kernel, sweeps_per_launch=1):
    """The kernel's roofline on ALGORITHMIC work per launch (DESIGN.md 6.3:
    bytes = R10, flops = R9 over the interior points one launch writes)."""
    pts = info["points"] * batch
    alg_bytes = info["bytes_per_point"] * pts
    canon = info["flops_per_point"] * pts * sweeps_per_launch
    t = kms * 1e-3
    hbm_bound = alg_bytes / (peak_hbm * 1e9)
    exe = counters.get("fp64_flops")
    F = min(canon, exe) if exe else canon
    fp_bound = F / fp64_peak if fp64_peak else 0.0
    r = {"kernel": kernel, "kernel_ms": kms, "traffic": counters.get("dram_bytes"),
         "alg_bytes_per_launch": alg_bytes, "canonical_flops_per_launch": canon,
         "executed_fp64_flops_per_launch": exe}
    if fp_bound > hbm_bound:  # FP64-pipe bound (rhs4center): "alu" per the contract, the FP64 pipe's DFMA peak
        r.update({"bound": "alu", "pipe": "fp64", "achieved": F / t / 1e12, "peak": fp64_peak / 1e12,
                  "unit": "TFLOP/s", "frac": fp_bound / t, "frac_canonical_flops": (canon / fp64_peak) / t,
                  "peak_source": "measured DFMA rate (sdag_measure_fp64_peak, all SMs, this run); "
                                 "nominal 148 SM x 64 DFMA/clk x 2 x 1.965 GHz = 37.2 TFLOP/s",
                  "F": "min(canonical, ncu-executed) flops (SURVEY 8(d))" if exe else "canonical flops"})
    else:
        r.update({"bound": "hbm", "achieved": alg_bytes / t / 1e9, "peak": peak_hbm, "unit": "GB/s",
                  "frac": hbm_bound / t, "peak_source": peak_src})
    return r


# ---------------------------------------------------------------------------
# per-config measurements (N = 1)
# ---------------------------------------------------------------------------

def measure_config(cid, steps, warmup, peak_hbm, peak_src, fp64_peak, tune=False):
    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    name, dims, batch, T = CONFIGS[cid]
    plan = sdag.Plan(sdag.spec_text(name), dims, batch=batch, tune=tune)
    info = plan.info
    arrays3d, arrays1d, scal = build_arrays(sdag, plan, name, dims, batch)
    stream = torch.cuda.current_stream()
    launch = [ln.strip() for ln in plan.describe().splitlines() if ln.strip().startswith("launch:")]
    res = {"workload": WORKLOAD[cid], "stencil": name, "grid": list(dims), "batch": batch, "sweeps_per_step": T,
           "variant": info["variant"], "flops_per_point": info["flops_per_point"],
           "bytes_per_point": info["bytes_per_point"], "tuned": bool(tune),
           "launch": launch[0] if launch else None}
    if cid == "1":
        # one 2 MB problem: latency-bound (launch + one short z-stream); L2 flushed
        # between iterations, each launch timed alone with events
        flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
        ev = []
        for it in range(warmup + steps):
            flush.fill_(it & 0xFF)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            plan.apply(arrays3d, arrays1d, scal, stream=stream)
            b.record(stream)
            ev.append((a, b))
        torch.cuda.synchronize()
        times = [a.elapsed_time(b) for a, b in ev[warmup:]]
        ms = statistics.median(times)
        res.update({"ms_per_step": ms, "us_min": min(times) * 1e3, "launches_per_step": 1,
                    "l2": "flushed (256 MB write) before every timed launch",
                    "gflops": info["flops_per_point"] * info["points"] / (ms * 1e-3) / 1e9,
                    "note": "latency, not throughput: 2 MB of traffic cannot fill 148 SMs (SURVEY 8(d) note)",
                    "kernel": plan.kernel_name(1)})
        return res
    if T > 1:
        b0, b1 = arrays3d[[r[3] for r in plan.args() if r[0] == 0].index(0)], None
        b1 = b0.clone()

        def step():
            plan.apply_iterated(b0, b1, T, scal, stream=stream)
    elif batch > 1:
        def step():
            plan.apply_batched(batch, arrays3d, arrays1d, scal, stream=stream)
    else:
        def step():
            plan.apply(arrays3d, arrays1d, scal, stream=stream)
    ms, lps, clk = timed(step, steps, warmup, stream, torch.cuda.current_device())
    kms = ms / lps
    spl = T / lps  # sweeps per launch
    if spl > 1:
        kernel = plan.kernel_name(int(round(spl))) if abs(spl - round(spl)) < 1e-9 else plan.kernel_name(2)
        variant = [ln for ln in plan.describe().splitlines() if "temporal fusion" in ln]
        variant = variant[0].split(":", 1)[1].split()[0] if variant else info["variant"]
    else:
        kernel, variant = plan.kernel_name(1), info["variant"]
    counters = load_counters(variant, dims, batch)
    pts_step = info["points"] * batch * T
    res.update({"variant": variant, "ms_per_step": ms, "launches_per_step": lps,
                "gflops": info["flops_per_point"] * pts_step / (ms * 1e-3) / 1e9,
                "hbm_gbs": info["bytes_per_point"] * pts_step / (ms * 1e-3) / 1e9,
                "roofline": roofline(info, kms, batch, peak_hbm, peak_src, fp64_peak, counters, kernel, spl),
                "clocks": clk, "l2": "inputs > 126 MB L2 (no flush needed)"})
    if spl > 1:
        # temporal fusion (NEXT-1): a launch reads and writes HBM once for spl
        # sweeps, so per sweep it can beat the unfused roofline
        res["roofline"]["sweep_equivalent"] = {"sweeps_per_launch": spl,
                                               "frac_of_unfused_roofline": res["roofline"]["frac"] * spl}
    if cid in PAPER_P100:
        res["paper_p100_context"] = PAPER_P100[cid]
    del arrays3d, arrays1d
    torch.cuda.empty_cache()
    return res


# ---------------------------------------------------------------------------
# the CPU oracle (cpu_baseline leg and the reference arm)
# ---------------------------------------------------------------------------

def oracle_lap25_throughput(A, c, seconds, groups=3):
    """The oracle as it stands on the host cores: whole 512^3 sweeps of the
    benchmark input, `groups` timed batches of ~seconds/groups each; the best
    batch is the value (min of 3)."""
    import oracle
    nz, ny, nx = A.shape
    out = np.zeros_like(A)
    oracle.lap25(A, c, out=out, krange=(4, 6))  # build + page-in
    oracle.lap25(A, c, out=out)  # warm
    rates, reps_total, t_total = [], 0, 0.0
    for _ in range(groups):
        reps, t0 = 0, time.perf_counter()
        while True:
            oracle.lap25(A, c, out=out)
            reps += 1
            if time.perf_counter() - t0 >= seconds / groups:
                break
        dt = time.perf_counter() - t0
        rates.append(reps * (nz - 8) * (ny - 8) * (nx - 8) * 29 / dt / 1e9)
        reps_total += reps
        t_total += dt
    return max(rates), reps_total, t_total


def cpu_cores():
    n = len(os.sched_getaffinity(0))
    omp = os.environ.get("OMP_NUM_THREADS")
    return min(n, int(omp)) if omp and omp.isdigit() else n


def run_reference(args):
    """--impl reference: the CPU oracle (this tier's reference arm) on the host
    cores, same metric and config; each step one full 512^3 sweep of the same
    seeded input.  Rank 0 only."""
    if int(os.environ.get("RANK", "0")) != 0:
        return 0
    import oracle
    import synth
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    ins, sc = synth.lap25_inputs((512, 512, 512), cfg="cfg2")
    A = ins["A"]
    c = [sc[k] for k in ("c0", "c1", "c2", "c3", "c4")]
    out = np.zeros_like(A)
    oracle.lap25(A, c, out=out, krange=(4, 6))
    for _ in range(args.warmup):
        oracle.lap25(A, c, out=out)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.lap25(A, c, out=out)
        times.append(time.perf_counter() - t0)
    dt = sum(times)
    pts = args.steps * 504 ** 3
    val = pts * 29 / dt / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": headline_config(world),
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": cpu_cores(), "kind": "oracle",
                             "cpu_model": cpu_model(), "best_step_gflops": 504 ** 3 * 29 / min(times) / 1e9,
                             "sample": f"{args.steps} full 512^3 sweeps of the benchmark input (all {504 ** 3} "
                                       f"interior points each), OpenMP over k"},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line))
    return 0


# ---------------------------------------------------------------------------
# multi-GPU: config 5 as z-slabs (the BASELINE weak-scaling workload)
# ---------------------------------------------------------------------------

def _red_dev(halo):
    """tensors for the timing reductions: the gloo group of the p2p path reduces on the host"""
    return "cpu" if halo == "p2p" else "cuda"


def measure_config5_slabs(tdist, rank, world, local, steps, warmup, comm, halo="nccl"):
    """Config 5 per rank: 1024^3 owned planes, T = 12, ghost depth 2 (one NCCL
    exchange per fused 2-sweep launch, overlapped with the interior launch);
    plus t_sweep(1): the same 1024^3 iteration on this GPU alone (single-GPU
    plan), so E(N) = t_sweep(1) / t_sweep(N) comes from one run."""
    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    import synth
    n, T, tt = 1024, 12, 2
    spec = sdag.spec_text("smooth27")
    cfg, a3, _, sc = synth.recipe("smooth27")
    scal = [sc[k] for k in ("w0", "w1", "w2", "w3", "nu")]
    stream = torch.cuda.current_stream()
    # single-GPU reference time on this rank's device (no communication)
    plan1 = sdag.Plan(spec, (n, n, n))
    b0 = synth.uniform_torch((n, n, n), -1.0, 1.0, cfg, "A")
    b1 = b0.clone()
    ms1, _, _ = timed(lambda: plan1.apply_iterated(b0, b1, T, scal, stream=stream), steps, warmup, stream, local)
    del b0, b1, plan1
    torch.cuda.empty_cache()
    gdims = (n * world, n, n)
    dd = sdag.Dist(spec, gdims, rank, world, comm=comm, time_tile=tt)
    (nza, ny, nx), g0 = dd.layout()
    part = sdag.slab_partition2(gdims[0], 1, tt, world, rank)
    x0 = synth.uniform_torch((nza, ny, nx), -1.0, 1.0, cfg + "-slab", rank)
    if halo == "p2p":
        # the boundary launches store their planes straight into the neighbours'
        # ghost planes over NVLink (CUDA IPC), flag-ordered -- no NCCL step
        p0, _ = dd.p2p_alloc()
        p0.copy_(x0)
        x0 = p0
        hs = [None] * world
        tdist.all_gather_object(hs, dd.p2p_handle())
        if rank > 0:
            dd.p2p_attach(0, hs[rank - 1])
        if rank < world - 1:
            dd.p2p_attach(1, hs[rank + 1])
        torch.cuda.synchronize()
        step = lambda: dd.p2p_apply_iterated(T, scalars=scal, stream=stream)  # noqa: E731
    else:
        x1 = x0.clone()
        cs = torch.cuda.Stream()
        step = lambda: dd.apply_iterated(x0, x1, T, scalars=scal, stream=stream, comm_stream=cs)  # noqa: E731
    msN, lps, clk = timed(step, steps, warmup, stream, local, barrier=tdist.barrier)
    t = torch.tensor([ms1, msN], dtype=torch.float64, device=_red_dev(halo))
    tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
    ms1m, msNm = float(t[0]), float(t[1])
    pts = torch.tensor([float((part["k_hi"] - part["k_lo"]) * (ny - 2) * (nx - 2) * T)], dtype=torch.float64,
                       device=_red_dev(halo))
    tdist.all_reduce(pts, op=tdist.ReduceOp.SUM)
    info = dd.plan.info
    del x0, step
    torch.cuda.empty_cache()
    return {"workload": WORKLOAD["5"], "stencil": "smooth27", "grid_per_gpu": [n, n, n], "global_grid": list(gdims),
            "decomposition": f"z-slabs x{world}",
            "halo": ("nccl send/recv" if halo == "nccl" else "p2p stores fused into the boundary kernels")
            + " (ghost depth 2: one exchange per fused 2-sweep launch)",
            "sweeps_per_step": T, "ms_per_step": msNm, "ms_per_sweep": msNm / T,
            "single_gpu_ms_per_sweep": ms1m / T, "weak_scaling_efficiency": ms1m / msNm,
            "gflops": float(pts) * info["flops_per_point"] / (msNm * 1e-3) / 1e9,
            "hbm_gbs_sweep_equivalent": float(pts) * info["bytes_per_point"] / (msNm * 1e-3) / 1e9,
            "launches_per_step": lps, "clocks": clk}


# ---------------------------------------------------------------------------
# launcher
# ---------------------------------------------------------------------------

def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(args_ns):
    """--gpus N without torchrun: run this script under torch.distributed.run."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args_ns.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="sdag", choices=["sdag", "reference"])
    ap.add_argument("--no-cpu", action="store_true", help="skip the cpu_baseline leg")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-per-config", action="store_true", help="headline only")
    ap.add_argument("--configs", default="1,1b,3,4,5", help="per_config entries at N = 1")
    ap.add_argument("--variant", default=None, help="force the headline plan's variant")
    ap.add_argument("--tune", action="store_true", help="headline: tune=1 plan (measured pick) instead of the heuristic")
    ap.add_argument("--tune-configs", action="store_true", help="per_config: tune=1 plans instead of the heuristic")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--cpu-baseline-only", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--halo", default="nccl", choices=["nccl", "p2p"], help="N > 1: config 5's slab halo path")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    env_world = os.environ.get("WORLD_SIZE")
    if args.impl == "reference":
        return run_reference(args)
    if args.cpu_baseline_only:
        import synth
        ins, _ = synth.lap25_inputs((512, 512, 512), cfg="cfg2")
        c = [synth.LAP25_COEFS[k] for k in ("c0", "c1", "c2", "c3", "c4")]
        val, reps, tt = oracle_lap25_throughput(ins["A"], c, args.cpu_seconds)
        print(json.dumps({"value": val, "unit": "GFLOP/s", "cores": cpu_cores(), "kind": "oracle",
                          "cpu_model": cpu_model(),
                          "sample": f"{reps} full 512^3 sweeps of the benchmark input in 3 timed batches "
                                    f"({tt:.1f} s); value = the best batch (min of 3); OpenMP over k, "
                                    f"separate process"}))
        return 0
    if env_world is None and args.gpus > 1:
        return relaunch(args)
    world = int(env_world or "1")
    if world != args.gpus:
        print(f"bench: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        return 2
    if world > 1:
        # NCCL communicator init lines (nranks) visible to the driver
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")

    import torch
    import paper_conf_ipps_rawatvsrps19_b200 as sdag
    import synth

    rank = int(os.environ.get("RANK", "0"))
    # SDAG_BENCH_SAME_DEVICE=1: every rank on cuda:0 (plumbing check of the N > 1
    # code path on a one-GPU box; needs --halo p2p, NCCL refuses duplicate GPUs)
    same = bool(os.environ.get("SDAG_BENCH_SAME_DEVICE"))
    local = 0 if same else int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    p2p = args.halo == "p2p"
    rdev = _red_dev(args.halo)
    tdist = None
    comm = None
    if world > 1:
        import torch.distributed as tdist
        if p2p:  # host plumbing only: IPC handles, barriers, the timing reductions
            tdist.init_process_group("gloo")
        else:
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local))
            uid = [sdag.nccl_unique_id() if rank == 0 else None]
            tdist.broadcast_object_list(uid, src=0)
            comm = sdag.nccl_comm_create(uid[0], world, rank, local)
    peak_hbm, peak_src = load_peaks()
    stream = torch.cuda.current_stream()
    spec = sdag.spec_text("lap25")
    n = 512
    c = [synth.LAP25_COEFS[k] for k in ("c0", "c1", "c2", "c3", "c4")]

    # ---- headline: config 2 ----
    if world == 1:
        plan = sdag.Plan(spec, (n, n, n), tune=args.tune, variant=args.variant)
        info = plan.info
        dA = synth.uniform_torch((n, n, n), -1.0, 1.0, "cfg2", "A")
        dB = torch.zeros((n, n, n), dtype=torch.float64, device="cuda")

        def step():
            plan.apply([dB, dA], scalars=c, stream=stream)
        ms, lps, clk = timed(step, args.steps, args.warmup, stream, local)
        kms = ms / lps
        pts_total = info["points"]
        kplan = plan
    else:
        dd = sdag.Dist(spec, (n * world, n, n), rank, world, comm=comm, tune=args.tune, variant=args.variant)
        (nza, ny, nx), g0 = dd.layout()
        part = sdag.slab_partition(n * world, 4, world, rank)
        src = synth.uniform_torch((nza, ny, nx), -1.0, 1.0, "cfg2-slab", rank)
        cs = torch.cuda.Stream()
        if p2p:
            # the sweep's boundary bands go to the neighbours' ghost planes by P2P
            # (flag-ordered, CUDA IPC); one sweep = p2p_apply_iterated with T = 1
            dA, dB = dd.p2p_alloc()
            dA.copy_(src)
            hs = [None] * world
            tdist.all_gather_object(hs, dd.p2p_handle())
            if rank > 0:
                dd.p2p_attach(0, hs[rank - 1])
            if rank < world - 1:
                dd.p2p_attach(1, hs[rank + 1])
            torch.cuda.synchronize()

            def step():
                dd.p2p_apply_iterated(1, scalars=c, stream=stream)
        else:
            dA = src
            dB = torch.zeros((nza, ny, nx), dtype=torch.float64, device="cuda")

            def step():
                dd.apply([dB, dA], scalars=c, stream=stream, comm_stream=cs)
        del src
        kplan = dd.plan
        info = kplan.info
        ms, lps, clk = timed(step, args.steps, args.warmup, stream, local, barrier=tdist.barrier)
        t = torch.tensor([ms], dtype=torch.float64, device=rdev)
        tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
        ms = float(t[0])
        p = torch.tensor([float((part["k_hi"] - part["k_lo"]) * (ny - 8) * (nx - 8))], dtype=torch.float64,
                         device=rdev)
        tdist.all_reduce(p, op=tdist.ReduceOp.SUM)
        pts_total = float(p[0])
        # the dominant kernel alone (same stream, same launch configuration)
        ka, kb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ka.record(stream)
        for _ in range(args.steps):
            kplan.apply([dB, dA], scalars=c, stream=stream)
        kb.record(stream)
        torch.cuda.synchronize()
        kms = ka.elapsed_time(kb) / args.steps
    gflops = pts_total * info["flops_per_point"] / (ms * 1e-3) / 1e9
    kernel = kplan.kernel_name(1)
    counters = load_counters(info["variant"], (n, n, n)) if world == 1 else {}
    roof = roofline(info if world == 1 else dict(info, points=(n - 8) ** 3), kms, 1, peak_hbm, peak_src, 0.0,
                    counters, kernel)

    # ---- e2e: the public call with host buffers, copies inside the timed region ----
    e2e = None
    if not args.no_e2e:
        if world == 1:
            hA = dA.cpu().pin_memory().numpy()
            hB = torch.zeros((n, n, n), dtype=torch.float64).pin_memory().numpy()
            plan.apply_host([hB, hA], scalars=c, stream=stream)  # warm workspace
            ee = []
            for _ in range(max(3, min(args.steps, 5))):
                t0 = time.perf_counter()
                up, down = plan.apply_host([hB, hA], scalars=c, stream=stream)
                ee.append(time.perf_counter() - t0)
            te = statistics.median(ee)
            e2e = {"value": info["points"] * info["flops_per_point"] / te / 1e9, "unit": "GFLOP/s",
                   "h2d_bytes_per_step": int(up), "d2h_bytes_per_step": int(down), "ms_per_step": te * 1e3,
                   "path": "sdag_apply_host (pipelined H2D / sweep / D2H over z-chunks)"}
        else:
            # owned planes host -> device (pinned), the NCCL-exchanged sweep, the
            # computed planes device -> host; wall time per step, max over ranks
            H = part["z0"] - g0
            own = slice(H, H + part["nz_own"])
            kk = slice(part["k_lo"], part["k_hi"])
            hA = dA[own].cpu().pin_memory()
            hB = torch.empty_like(dB[kk], device="cpu").pin_memory()
            ee = []
            for it in range(max(3, min(args.steps, 5)) + 1):
                tdist.barrier()
                t0 = time.perf_counter()
                dA[own].copy_(hA, non_blocking=True)
                step()
                hB.copy_(dB[kk], non_blocking=True)
                stream.synchronize()
                if it:
                    ee.append(time.perf_counter() - t0)
            t = torch.tensor([statistics.median(ee)], dtype=torch.float64, device=rdev)
            tdist.all_reduce(t, op=tdist.ReduceOp.MAX)
            te = float(t[0])
            e2e = {"value": pts_total * info["flops_per_point"] / te / 1e9, "unit": "GFLOP/s",
                   "h2d_bytes_per_step": int(hA.numel() * 8), "d2h_bytes_per_step": int(hB.numel() * 8),
                   "ms_per_step": te * 1e3, "per_rank_bytes": True,
                   "path": "owned planes H2D + the halo-exchanged sweep (" + ("P2P stores" if p2p else "NCCL")
                   + ") + computed planes D2H"}
    del dA, dB
    torch.cuda.empty_cache()

    # ---- per_config ----
    per = {}
    if not args.no_per_config:
        if world == 1:
            fp64 = sdag.fp64_peak()
            for cid in [x for x in args.configs.split(",") if x]:
                # heuristic plans by default (deterministic variants, whose ncu counters are
                # committed); --tune-configs times the plan-time measured pick instead
                per[cid] = measure_config(cid, min(args.steps, 10) if cid == "5" else args.steps, 3, peak_hbm, peak_src, fp64,
                                          tune=args.tune_configs)
            per["fp64_peak_tflops_measured"] = fp64 / 1e12
        else:
            per["5"] = measure_config5_slabs(tdist, rank, world, local, min(args.steps, 5), 3, comm, args.halo)

    # ---- cpu_baseline (rank 0, N = 1): the oracle in a fresh process (no torch /
    # CUDA threads competing with its OpenMP team: the same conditions as the
    # reference arm) ----
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu:
        r = subprocess.run([sys.executable, os.path.abspath(__file__), "--cpu-baseline-only",
                            "--cpu-seconds", str(args.cpu_seconds)], capture_output=True, text=True, timeout=600)
        cpu = json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 and r.stdout.strip() else \
            {"error": (r.stderr or "")[-300:]}

    if rank == 0:
        line = {"metric": METRIC, "value": gflops, "unit": "GFLOP/s", "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
                "vs_baseline": None, "dtype": "f64", "data": "synthetic (synth/ counter-based generator)",
                "config": headline_config(world),
                "plan": {"variant": info["variant"], "kernel": kernel, "flops_per_point": info["flops_per_point"],
                         "bytes_per_point": info["bytes_per_point"], "tuned": bool(args.tune)},
                "hbm_gbs": pts_total * info["bytes_per_point"] / (ms * 1e-3) / 1e9,
                "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": int(round(lps * args.steps)),
                "clocks": clk, "per_config": per}
        print(json.dumps(line))
    if tdist:
        tdist.barrier()
        if comm:
            sdag.nccl_comm_destroy(comm)
        tdist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
