// capi.cpp -- the extern "C" boundary (include/sdag.h): argument checks,
// exception -> sdag_status translation, thread-local error text.
#include <cuda_runtime.h>

#include <cxxabi.h>

#include <cstdlib>
#include <cstring>
#include <new>
#include <string>

#include "dist.hpp"
#include "plan.hpp"
#include "sdag.h"

namespace {

thread_local std::string g_err;

template <class F>
sdag_status guard(F &&f) {
    g_err.clear();
    try {
        f();
        return SDAG_OK;
    } catch (const sdag::Error &e) {
        g_err = e.what();
        return static_cast<sdag_status>(e.status);
    } catch (const std::bad_alloc &) {
        g_err = "out of host memory";
        return SDAG_ERR_NOMEM;
    } catch (const std::exception &e) {
        g_err = std::string("internal error: ") + e.what();
        return SDAG_ERR_INVALID_ARG;
    }
}

sdag::Plan *P(sdag_plan p) {
    if (!p || !p->p) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null plan");
    return p->p;
}

}  // namespace

extern "C" {

void sdag_plan_opts_init(sdag_plan_opts *o) {
    if (!o) return;
    o->order = -1;
    o->device = SDAG_DEVICE_CURRENT;
    o->tune = 0;
    o->batch = 1;
    o->force_variant = nullptr;
    o->fusion = 1;
    o->time_tile = 1;
}

sdag_status sdag_plan_create(const char *spec, const int64_t dims[3], const sdag_plan_opts *opts, sdag_plan *out) {
    return guard([&] {
        if (!spec || !dims || !out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        *out = nullptr;
        sdag_plan_opts o;
        sdag_plan_opts_init(&o);
        if (opts) o = *opts;
        sdag::Plan *p = sdag::plan_create(spec, dims, o);
        *out = new sdag_plan_s{p};
    });
}

sdag_status sdag_plan_info_get(sdag_plan plan, sdag_plan_info *out) {
    return guard([&] {
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null info");
        sdag::plan_fill_info(P(plan), out);
    });
}

sdag_status sdag_plan_arg(sdag_plan plan, int32_t kind, int32_t idx, const char **name, int32_t *role) {
    return guard([&] {
        sdag::Plan *p = P(plan);
        if (kind < 0 || kind > 2) throw sdag::Error(SDAG_ERR_INVALID_ARG, "kind must be 0, 1 or 2");
        const auto k = static_cast<sdag::ArgKind>(kind);
        if (idx < 0 || idx >= p->st.n_of(k)) throw sdag::Error(SDAG_ERR_INVALID_ARG, "index out of range");
        const sdag::Formal &f = p->st.formal(k, idx);
        if (name) *name = f.name.c_str();
        if (role)
            *role = (k == sdag::ArgKind::Array3D) ? int32_t(f.role)
                    : (k == sdag::ArgKind::Array1D ? (f.role == sdag::Role::Unused ? -1 : f.axis) : -1);
    });
}

sdag_status sdag_plan_variant_name(sdag_plan plan, int32_t idx, const char **name) {
    return guard([&] {
        sdag::Plan *p = P(plan);
        if (idx < 0 || idx >= int(p->cands.size())) throw sdag::Error(SDAG_ERR_INVALID_ARG, "index out of range");
        if (name) *name = p->cands[idx]->variant.c_str();
    });
}

sdag_status sdag_plan_kernel_name(sdag_plan plan, int32_t sweeps, const char **name) {
    return guard([&] {
        sdag::Plan *p = P(plan);
        if (!name) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null name");
        const sdag::KernelDesc *k = nullptr;
        if (sweeps == 1) {
            k = &p->kernel();
        } else {
            for (const sdag::KernelDesc *f : p->fused)
                if (f->tsteps == sweeps) {
                    k = f;
                    break;
                }
        }
        if (!k) throw sdag::Error(SDAG_ERR_INVALID_ARG, "the plan has no " + std::to_string(sweeps) + "-sweep kernel");
        std::lock_guard<std::mutex> lk(p->mu);
        auto it = p->kname.find(sweeps);
        if (it == p->kname.end()) {
            std::string s = "nvrtc:" + k->variant;  // generated (NEXT-4) kernels
            const char *mangled = nullptr;
            if (k->fn && cudaFuncGetName(&mangled, k->fn) == cudaSuccess && mangled) {
                int st = 0;
                char *dm = abi::__cxa_demangle(mangled, nullptr, nullptr, &st);
                s = (st == 0 && dm) ? dm : mangled;
                std::free(dm);
            }
            cudaGetLastError();
            it = p->kname.emplace(sweeps, s).first;
        }
        *name = it->second.c_str();
    });
}

const char *sdag_plan_describe(sdag_plan plan) {
    if (!plan || !plan->p) return "";
    return plan->p->describe_text.c_str();
}

void sdag_plan_destroy(sdag_plan plan) {
    if (!plan) return;
    delete plan->p;
    delete plan;
}

// ---- multi-stencil programs (Fig 3c) ----

static sdag::Program *G(sdag_program g) {
    if (!g || !g->g) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null program");
    return g->g;
}

sdag_status sdag_program_create(const char *spec, const int64_t dims[3], const sdag_plan_opts *opts,
                                sdag_program *out) {
    return guard([&] {
        if (!spec || !dims || !out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        *out = nullptr;
        sdag_plan_opts o;
        sdag_plan_opts_init(&o);
        if (opts) o = *opts;
        sdag::Program *g = sdag::program_create(spec, dims, o);
        *out = new sdag_program_s{g};
    });
}

sdag_status sdag_program_info(sdag_program prog, int32_t *n_stages, int32_t *n3d, int32_t *n1d, int32_t *nscalars) {
    return guard([&] {
        sdag::Program *g = G(prog);
        if (n_stages) *n_stages = int32_t(g->stages.size());
        if (n3d) *n3d = g->n_of(sdag::ArgKind::Array3D);
        if (n1d) *n1d = g->n_of(sdag::ArgKind::Array1D);
        if (nscalars) *nscalars = g->n_of(sdag::ArgKind::Scalar);
    });
}

sdag_status sdag_program_arg(sdag_program prog, int32_t kind, int32_t idx, const char **name, int32_t *role) {
    return guard([&] {
        sdag::Program *g = G(prog);
        if (kind < 0 || kind > 2) throw sdag::Error(SDAG_ERR_INVALID_ARG, "kind must be 0, 1 or 2");
        const auto k = static_cast<sdag::ArgKind>(kind);
        if (idx < 0 || idx >= g->n_of(k)) throw sdag::Error(SDAG_ERR_INVALID_ARG, "index out of range");
        const sdag::ProgramArg &a = g->arg(k, idx);
        if (name) *name = a.name.c_str();
        if (role) *role = (k == sdag::ArgKind::Array3D) ? int32_t(a.role) : (k == sdag::ArgKind::Array1D ? a.axis : -1);
    });
}

sdag_status sdag_program_stage(sdag_program prog, int32_t s, sdag_plan *out) {
    return guard([&] {
        sdag::Program *g = G(prog);
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        if (s < 0 || s >= int32_t(g->stages.size())) throw sdag::Error(SDAG_ERR_INVALID_ARG, "stage out of range");
        *out = g->handles[s];
    });
}

sdag_status sdag_program_apply(sdag_program prog, int32_t batch, double *const *a3, int32_t n3,
                               const double *const *a1, int32_t n1, const double *s, int32_t ns, sdag_stream stream) {
    return guard([&] {
        sdag::program_apply(G(prog), a3, n3, a1, n1, s, ns, batch, reinterpret_cast<cudaStream_t>(stream));
    });
}

void sdag_program_destroy(sdag_program prog) {
    if (!prog) return;
    delete prog->g;
    delete prog;
}

sdag_status sdag_apply(sdag_plan plan, double *const *a3, int32_t n3, const double *const *a1, int32_t n1,
                       const double *s, int32_t ns, sdag_stream stream) {
    return guard([&] { sdag::apply(P(plan), a3, n3, a1, n1, s, ns, 1, reinterpret_cast<cudaStream_t>(stream)); });
}

sdag_status sdag_apply_batched(sdag_plan plan, int32_t batch, double *const *a3, int32_t n3,
                               const double *const *a1, int32_t n1, const double *s, int32_t ns,
                               sdag_stream stream) {
    return guard(
        [&] { sdag::apply(P(plan), a3, n3, a1, n1, s, ns, batch, reinterpret_cast<cudaStream_t>(stream)); });
}

sdag_status sdag_apply_iterated(sdag_plan plan, double *b0, double *b1, int32_t T, const double *s, int32_t ns,
                                sdag_stream stream) {
    return guard(
        [&] { sdag::apply_iterated(P(plan), b0, b1, T, s, ns, reinterpret_cast<cudaStream_t>(stream)); });
}

sdag_status sdag_apply_host(sdag_plan plan, double *const *h3, int32_t n3, const double *const *h1, int32_t n1,
                            const double *s, int32_t ns, sdag_stream stream, int64_t *h2d, int64_t *d2h) {
    return guard([&] {
        sdag::apply_host(P(plan), h3, n3, h1, n1, s, ns, reinterpret_cast<cudaStream_t>(stream), h2d, d2h);
    });
}

sdag_status sdag_fusion_schedule(const double *f, int32_t maxdeg, int32_t T, int32_t *seq, int32_t cap, int32_t *n,
                                 double *cost) {
    return guard([&] {
        if (!f || !seq || !n || !cost) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null pointer");
        if (maxdeg < 1 || maxdeg > 7 || T < 0) throw sdag::Error(SDAG_ERR_INVALID_ARG, "maxdeg in 1..7, T >= 0");
        if (!(f[1] > 0.0)) throw sdag::Error(SDAG_ERR_INVALID_ARG, "f[1] must be > 0");
        const std::vector<int> s = sdag::fusion_schedule(f, maxdeg, T);
        if (int64_t(s.size()) > cap) throw sdag::Error(SDAG_ERR_INVALID_ARG, "seq capacity too small");
        double c = 0.0;
        for (size_t q = 0; q < s.size(); q++) {
            seq[q] = s[q];
            c += f[s[q]];
        }
        *n = int32_t(s.size());
        *cost = c;
    });
}

// ---- distributed ------------------------------------------------------------

sdag_status sdag_slab_partition(int64_t global_nz, int32_t rz, int32_t nranks, int32_t rank, int64_t out[7]) {
    return guard([&] {
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        sdag::Slab s = sdag::slab_partition(global_nz, rz, nranks, rank);
        out[0] = s.z0;
        out[1] = s.nz_own;
        out[2] = s.nz_alloc;
        out[3] = s.k_lo;
        out[4] = s.k_hi;
        out[5] = s.has_lower;
        out[6] = s.has_upper;
    });
}

sdag_status sdag_slab_halo(int64_t global_nz, int32_t rz, int32_t nranks, int32_t rank, int64_t out[5]) {
    return guard([&] {
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        sdag::Halo h = sdag::halo_schedule(sdag::slab_partition(global_nz, rz, nranks, rank), rz);
        out[0] = h.lo_send;
        out[1] = h.lo_recv;
        out[2] = h.up_send;
        out[3] = h.up_recv;
        out[4] = h.planes;
    });
}

sdag_status sdag_slab_partition2(int64_t global_nz, int32_t rz, int32_t time_tile, int32_t nranks, int32_t rank,
                                 int64_t out[8]) {
    return guard([&] {
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        sdag::Slab s = sdag::slab_partition(global_nz, rz, nranks, rank, time_tile);
        out[0] = s.z0;
        out[1] = s.nz_own;
        out[2] = s.nz_alloc;
        out[3] = s.k_lo;
        out[4] = s.k_hi;
        out[5] = s.has_lower;
        out[6] = s.has_upper;
        out[7] = s.halo;
    });
}

sdag_status sdag_slab_halo2(int64_t global_nz, int32_t rz, int32_t time_tile, int32_t nranks, int32_t rank,
                            int32_t planes, int64_t out[5]) {
    return guard([&] {
        if (!out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        sdag::Halo h = sdag::halo_schedule(sdag::slab_partition(global_nz, rz, nranks, rank, time_tile), planes);
        out[0] = h.lo_send;
        out[1] = h.lo_recv;
        out[2] = h.up_send;
        out[3] = h.up_recv;
        out[4] = h.planes;
    });
}

sdag_status sdag_nccl_get_unique_id(uint8_t id[128]) {
    return guard([&] { sdag::nccl_unique_id(id); });
}

sdag_status sdag_nccl_comm_create(const uint8_t id[128], int32_t nranks, int32_t rank, int32_t device, void **comm) {
    return guard([&] { *comm = sdag::nccl_comm_create(id, nranks, rank, device); });
}

void sdag_nccl_comm_destroy(void *comm) { sdag::nccl_comm_destroy(comm); }

sdag_status sdag_nccl_sendrecv(void *comm, int32_t peer, const double *send, double *recv, int64_t count,
                               void *stream) {
    return guard([&] { sdag::nccl_sendrecv(comm, peer, send, recv, count, reinterpret_cast<cudaStream_t>(stream)); });
}

sdag_status sdag_dist_create(const char *spec, const int64_t global_dims[3], const sdag_plan_opts *opts,
                             int32_t rank, int32_t nranks, void *nccl_comm, sdag_dist *out) {
    return guard([&] {
        if (!spec || !global_dims || !out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        sdag_plan_opts o;
        sdag_plan_opts_init(&o);
        if (opts) o = *opts;
        *out = reinterpret_cast<sdag_dist>(sdag::dist_create(spec, global_dims, o, rank, nranks, nccl_comm));
    });
}

sdag_status sdag_dist_create_local(sdag_plan local, int32_t rank, int32_t nranks, void *nccl_comm, int32_t time_tile,
                                   sdag_dist *out) {
    return guard([&] {
        if (!local || !local->p || !out) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        *out = reinterpret_cast<sdag_dist>(sdag::dist_create_local(local->p, rank, nranks, nccl_comm, time_tile));
    });
}

sdag_status sdag_dist_layout(sdag_dist d, int64_t local_dims[3], int64_t *gz0) {
    return guard([&] {
        auto *D = reinterpret_cast<sdag::Dist *>(d);
        if (!D) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null dist");
        for (int a = 0; a < 3; a++) local_dims[a] = D->local->dims[a];
        if (gz0) *gz0 = D->slab.z0 - D->slab.halo;
    });
}

sdag_status sdag_dist_alloc_dims(sdag_dist d, int64_t alloc_dims[3], int64_t *global_z0) {
    return sdag_dist_layout(d, alloc_dims, global_z0);
}

sdag_plan sdag_dist_local_plan(sdag_dist d) {
    auto *D = reinterpret_cast<sdag::Dist *>(d);
    return D ? reinterpret_cast<sdag_plan>(&D->handle) : nullptr;
}

sdag_status sdag_dist_apply(sdag_dist d, double *const *a3, int32_t n3, const double *const *a1, int32_t n1,
                            const double *s, int32_t ns, sdag_stream compute, sdag_stream comm) {
    return guard([&] {
        sdag::dist_apply(reinterpret_cast<sdag::Dist *>(d), a3, n3, a1, n1, s, ns,
                         reinterpret_cast<cudaStream_t>(compute), reinterpret_cast<cudaStream_t>(comm));
    });
}

sdag_status sdag_dist_apply_iterated(sdag_dist d, double *b0, double *b1, int32_t T, const double *s, int32_t ns,
                                     sdag_stream compute, sdag_stream comm) {
    return guard([&] {
        sdag::dist_apply_iterated(reinterpret_cast<sdag::Dist *>(d), b0, b1, T, s, ns,
                                  reinterpret_cast<cudaStream_t>(compute), reinterpret_cast<cudaStream_t>(comm));
    });
}

sdag_status sdag_dist_apply_iterated_loopback(sdag_dist *dists, int32_t nranks, double *const *b0,
                                              double *const *b1, int32_t T, const double *s, int32_t ns,
                                              sdag_stream stream) {
    return guard([&] {
        sdag::dist_apply_iterated_loopback(reinterpret_cast<sdag::Dist **>(dists), nranks, b0, b1, T, s, ns,
                                           reinterpret_cast<cudaStream_t>(stream));
    });
}

void sdag_dist_destroy(sdag_dist d) { delete reinterpret_cast<sdag::Dist *>(d); }

sdag_status sdag_dist_apply_host(sdag_dist d, double *const *h3, int32_t n3, const double *const *h1, int32_t n1,
                                 const double *s, int32_t ns, sdag_stream stream, int64_t *h2d, int64_t *d2h) {
    return guard([&] {
        sdag::dist_apply_host(reinterpret_cast<sdag::Dist *>(d), h3, n3, h1, n1, s, ns,
                              reinterpret_cast<cudaStream_t>(stream), h2d, d2h);
    });
}

sdag_status sdag_spec_fission(const char *spec, int32_t kind, char *buf, int64_t cap, int64_t *len) {
    return guard([&] {
        if (!spec || !len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        const std::string t = sdag::emit_fission(spec, kind);
        *len = int64_t(t.size());
        if (buf) {
            if (cap <= *len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "buffer too small");
            std::memcpy(buf, t.c_str(), t.size() + 1);
        }
    });
}

sdag_status sdag_program_fuse(const char *program, int32_t keep, char *buf, int64_t cap, int64_t *len) {
    return guard([&] {
        if (!program || !len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        const std::string t = sdag::fuse_program(program, keep);
        *len = int64_t(t.size());
        if (buf) {
            if (cap <= *len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "buffer too small");
            std::memcpy(buf, t.c_str(), t.size() + 1);
        }
    });
}

sdag_status sdag_program_version(const char *program, int32_t kind, int32_t *sizes, int32_t n_sizes, char *buf,
                                 int64_t cap, int64_t *len) {
    return guard([&] {
        if (!program || !len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        std::string t;
        const sdag::ProgramIR ir = sdag::parse_program(program);
        const int nst = int(ir.stages.size());
        if (kind == SDAG_VERSION_MAXFUSE) {
            t = sdag::fuse_groups(program, std::vector<int>{nst});
        } else if (kind == SDAG_VERSION_STAGED) {
            t = sdag::fuse_groups(program, std::vector<int>(nst, 1));
        } else if (kind == SDAG_VERSION_RECOMPUTE) {
            std::vector<int> g;
            t = sdag::recompute_fission(program, &g);
            if (sizes)
                for (int q = 0; q < n_sizes; q++) sizes[q] = q < int(g.size()) ? g[q] : 0;
        } else if (kind == SDAG_VERSION_GROUPS) {
            if (!sizes || n_sizes < 1) throw sdag::Error(SDAG_ERR_INVALID_ARG, "group sizes needed");
            t = sdag::fuse_groups(program, std::vector<int>(sizes, sizes + n_sizes));
        } else {
            throw sdag::Error(SDAG_ERR_INVALID_ARG, "unknown version kind");
        }
        *len = int64_t(t.size());
        if (buf) {
            if (cap <= *len) throw sdag::Error(SDAG_ERR_INVALID_ARG, "buffer too small");
            std::memcpy(buf, t.c_str(), t.size() + 1);
        }
    });
}

sdag_status sdag_program_forest(const char *program, int32_t max_candidates, int32_t *n_groups, int32_t *sizes,
                                int32_t *n_candidates) {
    return guard([&] {
        if (!program || !n_candidates || max_candidates < 1) throw sdag::Error(SDAG_ERR_INVALID_ARG, "bad argument");
        const auto c = sdag::forest_partitions(program, max_candidates);
        *n_candidates = int32_t(c.size());
        for (size_t q = 0; q < c.size(); q++) {
            if (n_groups) n_groups[q] = int32_t(c[q].size());
            if (sizes)
                for (int g = 0; g < 16; g++) sizes[q * 16 + g] = g < int(c[q].size()) ? c[q][g] : 0;
        }
    });
}

sdag_status sdag_program_forest_tune(const char *program, const int64_t dims[3], const sdag_plan_opts *opts,
                                     void *const *a3, int32_t n3, const double *const *a1, int32_t n1,
                                     const double *s, int32_t ns, sdag_stream stream, int32_t max_candidates,
                                     double *ms, int32_t *n_candidates, int32_t *best) {
    return guard([&] {
        if (!program || !dims || !n_candidates || !best || max_candidates < 1)
            throw sdag::Error(SDAG_ERR_INVALID_ARG, "bad argument");
        sdag_plan_opts o;
        sdag_plan_opts_init(&o);
        if (opts) o = *opts;
        sdag::program_forest_tune(program, dims, o, reinterpret_cast<double *const *>(a3), n3, a1, n1, s, ns,
                                  reinterpret_cast<cudaStream_t>(stream), max_candidates, ms, n_candidates, best);
    });
}

sdag_status sdag_plan_profile(sdag_plan plan, void *const *a3, int32_t n3, const double *const *a1, int32_t n1,
                              const double *s, int32_t ns, double peak_hbm_gbs, double peak_fp64_tflops,
                              sdag_stream stream, sdag_profile *out) {
    return guard([&] {
        if (!plan || !plan->p) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null plan");
        sdag::plan_profile(plan->p, reinterpret_cast<double *const *>(a3), n3, a1, n1, s, ns, peak_hbm_gbs,
                           peak_fp64_tflops, reinterpret_cast<cudaStream_t>(stream), out);
    });
}

sdag_status sdag_dist_p2p_alloc(sdag_dist d, double **buf0, double **buf1) {
    return guard([&] { sdag::dist_p2p_alloc(reinterpret_cast<sdag::Dist *>(d), buf0, buf1); });
}

sdag_status sdag_dist_p2p_handle(sdag_dist d, uint8_t handle[64]) {
    return guard([&] {
        if (!handle) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null handle");
        sdag::dist_p2p_handle(reinterpret_cast<sdag::Dist *>(d), handle);
    });
}

sdag_status sdag_dist_p2p_attach(sdag_dist d, int32_t side, const uint8_t handle[64]) {
    return guard([&] {
        if (!d || !handle) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null argument");
        sdag::dist_p2p_attach(reinterpret_cast<sdag::Dist *>(d), side, handle);
    });
}

sdag_status sdag_dist_p2p_attach_local(sdag_dist d, int32_t side, sdag_dist peer) {
    return guard([&] {
        if (side != 0 && side != 1) throw sdag::Error(SDAG_ERR_INVALID_ARG, "side must be 0 or 1");
        sdag::dist_p2p_attach_local(reinterpret_cast<sdag::Dist *>(d), side, reinterpret_cast<sdag::Dist *>(peer));
    });
}

sdag_status sdag_dist_p2p_apply_iterated(sdag_dist d, int32_t T, const double *s, int32_t ns, sdag_stream stream) {
    return guard([&] {
        sdag::dist_p2p_apply_iterated(reinterpret_cast<sdag::Dist *>(d), T, s, ns,
                                      reinterpret_cast<cudaStream_t>(stream));
    });
}

// ---- diagnostics ------------------------------------------------------------

const char *sdag_last_error(void) { return g_err.c_str(); }

const char *sdag_version(void) { return "sdag 0.1 (sm_100a)"; }

int64_t sdag_launch_count(void) { return sdag::launch_count(); }

sdag_status sdag_measure_fp64_peak(double *flops, sdag_stream stream) {
    return guard([&] {
        if (!flops) throw sdag::Error(SDAG_ERR_INVALID_ARG, "null out");
        *flops = sdag::measure_fp64_peak(reinterpret_cast<cudaStream_t>(stream));
    });
}

int32_t sdag_registry_count(void) { return int32_t(sdag::registry().size()); }

sdag_status sdag_registry_get(int32_t idx, const char **name, const char **text) {
    return guard([&] {
        const auto &r = sdag::registry();
        if (idx < 0 || idx >= int(r.size())) throw sdag::Error(SDAG_ERR_INVALID_ARG, "index out of range");
        if (name) *name = r[idx].name.c_str();
        if (text) *text = r[idx].text.c_str();
    });
}

}  // extern "C"
