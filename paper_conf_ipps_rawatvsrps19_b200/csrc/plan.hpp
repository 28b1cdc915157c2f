// plan.hpp -- an immutable plan (a1-a3 results) plus its small mutable caches.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <tuple>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "ir.hpp"
#include "kernels.hpp"
#include "registry.hpp"
#include "sdag.h"

namespace sdag {

struct Launch {
    const KernelDesc *k = nullptr;
    int nchunk = 1, zchunk = 1;
    int tiles_x = 1, tiles_y = 1;
};

struct Plan {
    Stencil st;
    Analysis an;
    const RegEntry *reg = nullptr;
    std::vector<double> extra_scalars;  // plan-time kernel scalars (shift offsets)
    int64_t dims[3] = {1, 1, 1};        // nz, ny, nx (one problem)
    int64_t lo[3] = {0, 0, 0}, hi[3] = {0, 0, 0};
    int device = -1;
    bool host_only = false;
    int sm_count = 148;
    int batch_hint = 1;
    int tune = 0;
    bool tune_cached = false;  // tune=1 result restored from $SDAG_TUNE_CACHE
    std::string force_variant;
    std::string spec_text;      // the spec this plan was created from (empty for program stages)
    sdag_plan_opts opts_copy{};  // the options it was created with (force_variant -> the string above)

    // ABI mapping (per 3D formal kind_index): staged-input slot / output slot / inout slot
    std::vector<int> in_slot, out_slot, io_slot;
    int jit_maxrreg = 0;
    bool jit_strict = false;
    std::string jit_star_src;  // generated star-kernel body when the DAG is in star form (jit.cu)
    std::vector<std::string> box_w;  // box form: class weights w0..w3 as expressions of a.s[] (jit.cu)  // force_variant "jit_strict": generated kernels without FMA contraction
    int zchunk_tuned = 0;   // z-chunk length chosen by tune=1 (0 = the occupancy model's)
    int tuned_timed = 0;    // candidates timed by the hierarchical tuner  // --maxrregcount of the generated kernels (occupancy t), 0 = none
    int n_staged = 0;  // inputs staged in shared memory: slots [0, n_staged); generated kernels
                       // read the rest (#assign gmem) through L1/L2
    std::vector<const KernelDesc *> cands;  // candidate kernels (TMA first)
    std::vector<const KernelDesc *> fused;  // multi-sweep kernels for apply_iterated (tsteps > 1)
    double fcost[8] = {0};                  // f(x): relative cost of an x-sweep launch (deep tuning)
    bool fusion = true;                     // use fused kernels in apply_iterated
    std::vector<std::unique_ptr<KernelDesc>> jit_descs;  // NVRTC kernels of an unregistered DAG (NEXT-4)
    std::string jit_source;                 // their generated source (sdag_plan_describe shows the body)
    int chosen = -1;                        // index into cands
    std::string describe_text;

    // mutable caches
    std::mutex mu;
    std::map<std::tuple<const void *, int64_t, int64_t, int64_t, int, int>, CUtensorMap> tmaps;
    std::vector<void *> ws;  // sdag_apply_host workspace (device buffers)
    std::vector<size_t> ws_bytes;
    struct IterGraph {  // apply_iterated replays (CUDA graphs): key = buffers, T, scalars
        std::string key;
        cudaGraphExec_t exec = nullptr;
        int launches = 0;
    };
    std::vector<IterGraph> graphs;  // guarded by graph_mu (not mu: capture enqueues launches, which take mu)
    std::mutex graph_mu;
    cudaStream_t cap_stream = nullptr;  // graph capture stream
    std::mutex host_mu;              // sdag_apply_host calls on one plan are serialised (shared workspace)
    cudaStream_t hs_up = nullptr;    // sdag_apply_host copy streams (H2D, D2H), created on first use
    cudaStream_t hs_down = nullptr;
    std::map<int, std::string> kname;  // sdag_plan_kernel_name results (guarded by mu)

    ~Plan();
    const KernelDesc &kernel() const { return *cands[chosen]; }
    int n3() const { return st.n_of(ArgKind::Array3D); }
    int n1() const { return st.n_of(ArgKind::Array1D); }
    int ns() const { return st.n_of(ArgKind::Scalar); }
    int64_t points() const { return (hi[0] - lo[0]) * (hi[1] - lo[1]) * (hi[2] - lo[2]); }
    double bytes_per_point() const;
};

// planner (runtime.cu)
Plan *plan_create(const std::string &spec, const int64_t dims[3], const sdag_plan_opts &o);
Plan *plan_create_from(Stencil st, const int64_t dims[3], const sdag_plan_opts &o);

// A multi-stencil program (Fig 3c): one plan per call, run in call order on
// one stream (program.cpp).  Arguments are the program's declared arrays and
// scalars in declaration order; stage s's formal q is program argument map[s][q].
struct Program {
    ProgramIR ir;
    std::vector<std::unique_ptr<Plan>> stages;
    std::vector<sdag_plan_s *> handles;  // borrowed per-stage handles (sdag_program_stage)
    int n_of(ArgKind k) const {
        int n = 0;
        for (auto &a : ir.args) n += (a.kind == k);
        return n;
    }
    const ProgramArg &arg(ArgKind k, int idx) const;
    ~Program();
};
Program *program_create(const std::string &spec, const int64_t dims[3], const sdag_plan_opts &o);
void program_apply(Program *g, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                   int batch, cudaStream_t stream);
void plan_fill_info(Plan *p, sdag_plan_info *info);
// the fusion forest's measured pick (program.cpp, Section VI-B)
void program_forest_tune(const std::string &text, const int64_t dims[3], const sdag_plan_opts &o, double *const *a3,
                         int n3, const double *const *a1, int n1, const double *s, int ns, cudaStream_t stream,
                         int max_candidates, double *ms, int *n_candidates, int *best);

// Peer-memory halo of one launch (dist p2p path): output planes [klo[s], khi[s])
// are also stored into neighbour s's buffer `peer[s]` at element offset
// `off[s]` (same layout); launches KernelDesc::fn_mirror.
struct Mirror {
    double *peer[2] = {nullptr, nullptr};
    int64_t off[2] = {0, 0};
    int32_t klo[2] = {0, 0}, khi[2] = {0, 0};
};

// sweep launch over output planes [klo, khi) of each problem (clipped to the
// interior); all arrays are per-problem [batch][nz][ny][nx].
void plan_launch(Plan *p, const KernelDesc &k, double *const *arrays3d, const double *const *arrays1d,
                 const double *scalars, int batch, int64_t klo, int64_t khi, cudaStream_t stream,
                 const int64_t *dims_override = nullptr, const int64_t *zr = nullptr, const Mirror *mir = nullptr);

// dist p2p synchronisation (p2p.cu): wait until flags[s] - need[s] >= 0 (mod 2^32)
// for the sides with has[s]; then signal: store v into f0 / f1 (non-null) with
// system-scope release after the stream's previous work.
void p2p_wait(const uint32_t *flags, const uint32_t need[2], const int has[2], cudaStream_t stream);
void p2p_signal(uint32_t *f0, uint32_t *f1, uint32_t v, cudaStream_t stream);
void p2p_preload();
void plan_profile(Plan *p, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                  double peak_hbm_gbs, double peak_fp64_tflops, cudaStream_t st, sdag_profile *out);
void apply(Plan *p, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns, int batch,
           cudaStream_t stream);
// the argument checks of apply (counts, nulls, output aliasing), nothing enqueued
void plan_validate(Plan *p, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                   int batch);
std::vector<int> fusion_schedule(const double *f, int maxdeg, int T);
void apply_iterated(Plan *p, double *b0, double *b1, int T, const double *s, int ns, cudaStream_t stream);
void apply_host(Plan *p, double *const *h3, int n3, const double *const *h1, int n1, const double *s, int ns,
                cudaStream_t stream, int64_t *h2d, int64_t *d2h,
                const int64_t *krange = nullptr);
void check_cuda(cudaError_t e, const char *what);
// binds the plan's device for the duration of an entry point and restores the
// caller's current device on exit (also on a throw)
struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(const Plan *p) {
        if (p->host_only) throw Error(SDAG_ERR_DEVICE, "plan was created host-only (SDAG_DEVICE_NONE)");
        check_cuda(cudaGetDevice(&prev), "cudaGetDevice");
        if (prev != p->device) check_cuda(cudaSetDevice(p->device), "cudaSetDevice");
    }
    ~DeviceGuard() {
        if (prev >= 0) cudaSetDevice(prev);
    }
};
// NVTX range around a host entry point (tracing): the range
// appears on the CPU timeline of nsys / ncu --nvtx so a trace names which
// sdag call enqueued which kernels.  nvtx3 is header-only; with no tool
// attached a push/pop is a null-pointer check.
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    explicit NvtxRange(const std::string &name) { nvtxRangePushA(name.c_str()); }
    ~NvtxRange() { nvtxRangePop(); }
    NvtxRange(const NvtxRange &) = delete;
    NvtxRange &operator=(const NvtxRange &) = delete;
};
bool log_enabled();
void log_plan(const Plan *p, const char *what);
// jit.cu (NEXT-4)
std::string jit_body_source(const Plan &p, const std::string &sname, int rzr);
void jit_build_candidates(Plan *p);
// box form (jit.cu): evaluate a weight expression over the call's scalars
double jit_eval_coef(const std::string &e, const double *s, int ns);
void jit_launch(const KernelDesc &k, dim3 grid, void **args, cudaStream_t stream);
int jit_occupancy(const KernelDesc &k);

// process-wide launch counter
void count_launch();
int64_t launch_count();
double measure_fp64_peak(cudaStream_t stream);

}  // namespace sdag

// the opaque C handles (include/sdag.h) wrap a Plan / a Program
struct sdag_plan_s {
    sdag::Plan *p;
};
struct sdag_program_s {
    sdag::Program *g;
};
