// profile.cu -- the paper's profiling component (Section IV) on
// B200: time the plan's kernel on the caller's arrays, place it on the
// roofline of each level the library can measure itself (DRAM: algorithmic
// bytes vs measured copy bandwidth; FP64: canonical flops vs the DFMA peak),
// difference it against code-differenced twins where they are registered
// (a memory-only twin and an arithmetic-only twin), classify it
// bandwidth-, compute- or latency-bound, and emit the Section IV-A hints
// adapted to the B200 kernel family.
#include <algorithm>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "plan.hpp"
#include "sdag.h"

namespace sdag {

namespace {

struct Ev {
    cudaEvent_t a = nullptr, b = nullptr;
    Ev() {
        check_cuda(cudaEventCreate(&a), "cudaEventCreate");
        check_cuda(cudaEventCreate(&b), "cudaEventCreate");
    }
    ~Ev() {
        cudaEventDestroy(a);
        cudaEventDestroy(b);
    }
};

// median over `reps` single launches of `fn` (after one warm-up), ms
template <class F>
double time_ms(F fn, cudaStream_t st, int reps) {
    Ev e;
    fn();
    std::vector<float> t;
    for (int r = 0; r < reps; r++) {
        check_cuda(cudaEventRecord(e.a, st), "cudaEventRecord");
        fn();
        check_cuda(cudaEventRecord(e.b, st), "cudaEventRecord");
        check_cuda(cudaEventSynchronize(e.b), "cudaEventSynchronize");
        float ms = 0;
        check_cuda(cudaEventElapsedTime(&ms, e.a, e.b), "cudaEventElapsedTime");
        t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    return t[t.size() / 2];
}

// device-to-device copy bandwidth (read + write bytes / time), GB/s
double measure_hbm_gbs(cudaStream_t st) {
    const size_t n = size_t(1) << 30;
    void *a = nullptr, *b = nullptr;
    check_cuda(cudaMalloc(&a, n), "cudaMalloc(profile)");
    if (cudaMalloc(&b, n) != cudaSuccess) {
        cudaFree(a);
        check_cuda(cudaGetLastError(), "cudaMalloc(profile)");
    }
    double ms = 0;
    try {
        ms = time_ms([&] { check_cuda(cudaMemcpyAsync(b, a, n, cudaMemcpyDeviceToDevice, st), "copy"); }, st, 5);
    } catch (...) {
        cudaFree(a);
        cudaFree(b);
        throw;
    }
    cudaFree(a);
    cudaFree(b);
    return 2.0 * double(n) / (ms * 1e-3) / 1e9;
}

const KernelDesc *twin(const Plan *p, const KernelDesc &k, const char *tag) {
    // code-differenced twin of kernel k: same DAG and geometry, variant "<family>DIFF<tag>_..."
    for (const KernelDesc &c : kernel_table()) {
        if (c.dag != k.dag || c.variant.find(std::string("DIFF") + tag) == std::string::npos) continue;
        if (c.tx == k.tx && c.ty == k.ty && c.uy == k.uy && c.pf == k.pf && c.tma == k.tma) return &c;
    }
    (void)p;
    return nullptr;
}

}  // namespace

void plan_profile(Plan *p, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                  double peak_hbm_gbs, double peak_fp64_tflops, cudaStream_t st, sdag_profile *out) {
    if (!out) throw Error(SDAG_ERR_INVALID_ARG, "null profile");
    if (p->host_only) throw Error(SDAG_ERR_DEVICE, "plan was created host-only (SDAG_DEVICE_NONE)");
    plan_validate(p, a3, n3, a1, n1, s, ns, 1);
    std::memset(out, 0, sizeof *out);
    check_cuda(cudaSetDevice(p->device), "cudaSetDevice");
    const KernelDesc &k = p->kernel();
    if (k.tma) {
        bool ok = p->dims[2] % 2 == 0;
        for (int f = 0; f < n3; f++) ok = ok && reinterpret_cast<uintptr_t>(a3[f]) % 16 == 0;
        if (!ok) throw Error(SDAG_ERR_INVALID_ARG, "profile: the plan's TMA kernel needs 16-B aligned arrays, even nx");
    }
    double *const *a = a3;
    auto run = [&](const KernelDesc &kd) { plan_launch(p, kd, a, a1, s, 1, 0, p->dims[0], st); };
    out->ms = time_ms([&] { run(k); }, st, 7);
    out->flops = p->an.flops_per_point * double(p->points());
    out->bytes = p->bytes_per_point() * double(p->points());
    out->peak_hbm_gbs = peak_hbm_gbs > 0 ? peak_hbm_gbs : measure_hbm_gbs(st);
    out->peak_fp64_tflops = peak_fp64_tflops > 0 ? peak_fp64_tflops : measure_fp64_peak(st) / 1e12;
    out->oi_dram = out->bytes > 0 ? out->flops / out->bytes : 0.0;
    out->ridge = out->peak_fp64_tflops * 1e3 / out->peak_hbm_gbs;
    const double t_dram = out->bytes / (out->peak_hbm_gbs * 1e9) * 1e3;
    const double t_fp64 = out->flops / (out->peak_fp64_tflops * 1e12) * 1e3;
    out->frac_dram = t_dram / out->ms;
    out->frac_fp64 = t_fp64 / out->ms;
    if (const KernelDesc *m = twin(p, k, "mem")) out->ms_diff_mem = time_ms([&] { run(*m); }, st, 5);
    if (const KernelDesc *n = twin(p, k, "nost")) out->ms_diff_arith = time_ms([&] { run(*n); }, st, 5);

    // resources of the kernel (fission variants: the first of their kernels)
    const void *fn = k.fission ? k.fission_fns[0] : k.fn;
    if (fn) {
        cudaFuncAttributes fa;
        check_cuda(cudaFuncGetAttributes(&fa, fn), "cudaFuncGetAttributes");
        out->regs = fa.numRegs;
        out->spill_bytes = int32_t(fa.localSizeBytes);
        int blocks = 0;
        check_cuda(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&blocks, fn, k.threads, size_t(k.smem)),
                   "cudaOccupancyMaxActiveBlocksPerMultiprocessor");
        out->ctas_per_sm = blocks;
        out->warps_per_sm = blocks * ((k.threads + 31) / 32);
    }

    // classification: bandwidth-bound at DRAM when the DRAM
    // roofline time is most of the run (or the memory-only twin takes as long
    // as the kernel); compute-bound when the FP64 roofline time is; otherwise
    // latency-bound -- neither level saturated (on B200 typically shared-memory
    // latency at the occupancy the registers allow)
    const double hi = 0.75;
    if (out->frac_dram >= hi || (out->ms_diff_mem > 0 && out->ms_diff_mem >= 0.9 * out->ms))
        out->bound = SDAG_BOUND_DRAM;
    else if (out->frac_fp64 >= hi)
        out->bound = SDAG_BOUND_COMPUTE;
    else
        out->bound = SDAG_BOUND_LATENCY;

    // hints (Section IV-A), adapted
    std::string h;
    auto add = [&](const std::string &x) { h += (h.empty() ? "" : "\n") + x; };
    const bool iterative = p->n3() == 2 && p->an.n_in == 1 && p->an.n_out == 1 && p->n1() == 0;
    if (out->bound == SDAG_BOUND_COMPUTE)
        add("compute-bound: more ILP (unrolling) or staging will not help; reduce the flops "
            "(computation folding, CSE of the coefficient products)");
    if (out->regs >= 224 || out->spill_bytes > 0) {
        std::string fis;
        for (const KernelDesc *c : p->cands)
            if (c->fission) fis += (fis.empty() ? "" : ", ") + c->variant;
        add("register pressure (" + std::to_string(out->regs) + " registers, " + std::to_string(out->spill_bytes) +
            " B spilled, " + std::to_string(out->warps_per_sm) + " warps/SM): keep unrolling off; " +
            (fis.empty() ? std::string("no fission variant is registered for this DAG")
                         : "fission variants: " + fis));
    }
    if (out->bound == SDAG_BOUND_DRAM && iterative) {
        std::string fu;
        for (const KernelDesc *f : p->fused) fu += (fu.empty() ? "" : ", ") + f->variant;
        add(fu.empty() ? std::string("DRAM-bound iterative stencil: no fused multi-sweep kernel is registered")
                       : "DRAM-bound iterative stencil: raise the fusion degree (apply_iterated, time_tile): " + fu);
    }
    if (out->bound == SDAG_BOUND_DRAM && !iterative)
        add("DRAM-bound spatial stencil at " + std::to_string(int(100 * out->frac_dram + 0.5)) +
            "% of the copy bandwidth: only fewer bytes help (lower order, fewer arrays, fusion with the producer)");
    if (out->bound == SDAG_BOUND_LATENCY) {
        if (out->ms_diff_arith > 0 && out->ms_diff_arith >= 0.9 * out->ms)
            add("latency-bound in the arithmetic path (the arithmetic-only twin takes as long as the kernel): "
                "register-level reuse (retiming, folding) and more warps per SM");
        else
            add("latency-bound: neither DRAM (" + std::to_string(int(100 * out->frac_dram + 0.5)) +
                "%) nor FP64 (" + std::to_string(int(100 * out->frac_fp64 + 0.5)) +
                "%) saturated at " + std::to_string(out->warps_per_sm) +
                " warps/SM: register-level optimisations (retiming/folding) to cut shared-memory traffic, "
                "or a variant with more resident warps");
    }
    if (out->oi_dram < out->ridge && out->bound != SDAG_BOUND_DRAM)
        add("OI " + std::to_string(out->oi_dram).substr(0, 5) + " flop/B is below the ridge " +
            std::to_string(out->ridge).substr(0, 5) + ": the DRAM roofline is the attainable bound");
    std::snprintf(out->hints, sizeof out->hints, "%s", h.c_str());
    std::snprintf(out->variant, sizeof out->variant, "%s", k.variant.c_str());
}

}  // namespace sdag
