// dist.cpp -- a7: z-slab decomposition (north-star addition; the paper is
// single-GPU).  Rank p owns a contiguous range of global z-planes;
// its local allocation adds R_z ghost planes below and above.  Every sweep:
//   comm stream:    ncclGroupStart; send my R_z lowest/highest owned planes of
//                   each z-read input to rank-1/rank+1; recv their planes into
//                   my ghosts; ncclGroupEnd              (no packing: C-order
//                   z-planes are contiguous)
//   compute stream: concurrently, the sweep kernel over owned planes that read
//                   no ghost; then (event join) the same kernel over the
//                   R_z planes next to each ghost layer.
// Interior and boundary launches run the same kernel instantiation, so the
// result is bit-identical to a single-GPU sweep of the global grid.
#include "dist.hpp"

#include <dlfcn.h>

#include <cstdlib>
#include <cstring>

#include "sdag.h"

namespace sdag {

// ---------------------------------------------------------------------------
// host logic
// ---------------------------------------------------------------------------

Slab slab_partition(int64_t gnz, int rz, int nranks, int rank, int time_tile) {
    if (nranks < 1 || rank < 0 || rank >= nranks) throw Error(SDAG_ERR_INVALID_ARG, "bad rank / nranks");
    if (rz < 0) throw Error(SDAG_ERR_INVALID_ARG, "negative radius");
    if (time_tile < 1 || time_tile > 7) throw Error(SDAG_ERR_INVALID_ARG, "time_tile must be in 1..7");
    const int64_t H = int64_t(rz) * time_tile;
    if (gnz < 2 * int64_t(rz) + 1) throw Error(SDAG_ERR_DOMAIN, "global z extent has no interior");
    Slab s;
    const int64_t base = gnz / nranks, rem = gnz % nranks;
    s.nz_own = base + (rank < rem ? 1 : 0);
    s.z0 = int64_t(rank) * base + std::min<int64_t>(rank, rem);
    if (base < std::max<int64_t>(H, 1))
        throw Error(SDAG_ERR_DOMAIN, "every rank must own at least max(R_z*time_tile,1) = " +
                                         std::to_string(std::max<int64_t>(H, 1)) + " planes (global nz " +
                                         std::to_string(gnz) + ", " + std::to_string(nranks) + " ranks)");
    s.halo = H;
    s.nz_alloc = s.nz_own + 2 * H;
    const int64_t g_of_l0 = s.z0 - H;  // global plane of local plane 0
    const int64_t glo = std::max<int64_t>(s.z0, rz), ghi = std::min<int64_t>(s.z0 + s.nz_own, gnz - rz);
    s.k_lo = glo - g_of_l0;
    s.k_hi = std::max(ghi - g_of_l0, s.k_lo);
    s.has_lower = rank > 0;
    s.has_upper = rank < nranks - 1;
    return s;
}

Halo halo_schedule(const Slab &s, int planes) {
    Halo h;
    if (planes < 0 || planes > s.halo) throw Error(SDAG_ERR_INVALID_ARG, "halo planes must be in 0..H");
    h.planes = planes;
    if (planes == 0) return h;
    const int64_t H = s.halo;
    if (s.has_lower) {
        h.lo_send = H;           // my lowest `planes` owned planes
        h.lo_recv = H - planes;  // the ghosts right below them
    }
    if (s.has_upper) {
        h.up_send = H + s.nz_own - planes;  // my highest `planes` owned planes
        h.up_recv = H + s.nz_own;           // the ghosts right above them
    }
    return h;
}

// ---------------------------------------------------------------------------
// NCCL, loaded from the libnccl.so.2 the process already uses (torch's)
// ---------------------------------------------------------------------------

namespace {

typedef int ncclResult_t;
typedef struct ncclComm *ncclComm_t;
struct ncclUniqueId {
    char internal[128];
};
constexpr int ncclFloat64 = 8;

struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId *) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t *, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    ncclResult_t (*Send)(const void *, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*Recv)(void *, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*GroupStart)() = nullptr;
    ncclResult_t (*GroupEnd)() = nullptr;
    ncclResult_t (*CommGetAsyncError)(ncclComm_t, ncclResult_t *) = nullptr;
    const char *(*GetErrorString)(ncclResult_t) = nullptr;
    std::string err;
};

const NcclApi &nccl() {
    static NcclApi a = [] {
        NcclApi x;
        const char *cands[] = {std::getenv("SDAG_NCCL_LIB"), "libnccl.so.2", "libnccl.so"};
        void *h = nullptr;
        for (const char *c : cands)
            if (c && (h = dlopen(c, RTLD_NOW | RTLD_GLOBAL))) break;
        if (!h) {
            x.err = "cannot dlopen libnccl.so.2 (import torch first, or set SDAG_NCCL_LIB)";
            return x;
        }
        auto sym = [&](const char *n) { return dlsym(h, n); };
        x.GetUniqueId = reinterpret_cast<decltype(x.GetUniqueId)>(sym("ncclGetUniqueId"));
        x.CommInitRank = reinterpret_cast<decltype(x.CommInitRank)>(sym("ncclCommInitRank"));
        x.CommDestroy = reinterpret_cast<decltype(x.CommDestroy)>(sym("ncclCommDestroy"));
        x.Send = reinterpret_cast<decltype(x.Send)>(sym("ncclSend"));
        x.Recv = reinterpret_cast<decltype(x.Recv)>(sym("ncclRecv"));
        x.GroupStart = reinterpret_cast<decltype(x.GroupStart)>(sym("ncclGroupStart"));
        x.GroupEnd = reinterpret_cast<decltype(x.GroupEnd)>(sym("ncclGroupEnd"));
        x.GetErrorString = reinterpret_cast<decltype(x.GetErrorString)>(sym("ncclGetErrorString"));
        x.CommGetAsyncError = reinterpret_cast<decltype(x.CommGetAsyncError)>(sym("ncclCommGetAsyncError"));
        if (!x.GetUniqueId || !x.CommInitRank || !x.Send || !x.Recv || !x.GroupStart || !x.GroupEnd)
            x.err = "libnccl.so.2 lacks the point-to-point API";
        return x;
    }();
    if (!a.err.empty()) throw Error(SDAG_ERR_NCCL, a.err);
    return a;
}

void nck(ncclResult_t r, const char *what) {
    if (r != 0) {
        const NcclApi &a = nccl();
        throw Error(SDAG_ERR_NCCL, std::string(what) + ": " + (a.GetErrorString ? a.GetErrorString(r) : "error"));
    }
}

}  // namespace

void nccl_unique_id(uint8_t id[128]) {
    ncclUniqueId u;
    nck(nccl().GetUniqueId(&u), "ncclGetUniqueId");
    std::memcpy(id, u.internal, 128);
}

void *nccl_comm_create(const uint8_t id[128], int nranks, int rank, int device) {
    ncclUniqueId u;
    std::memcpy(u.internal, id, 128);
    int prev = -1;
    check_cuda(cudaGetDevice(&prev), "cudaGetDevice");
    if (device >= 0) check_cuda(cudaSetDevice(device), "cudaSetDevice");
    ncclComm_t c = nullptr;
    const ncclResult_t r = nccl().CommInitRank(&c, nranks, u, rank);
    if (prev >= 0) cudaSetDevice(prev);  // the caller's current device is left as it was
    nck(r, "ncclCommInitRank");
    return c;
}

void nccl_comm_destroy(void *c) {
    if (c) {
        try {
            nccl().CommDestroy(static_cast<ncclComm_t>(c));
        } catch (...) {
        }
    }
}

// ---------------------------------------------------------------------------
// dist plan
// ---------------------------------------------------------------------------

Dist::~Dist() {
    for (void *m : peer_ipc)
        if (m) cudaIpcCloseMemHandle(m);
    if (p2p_base) cudaFree(p2p_base);
    if (own_comm) cudaStreamDestroy(own_comm);
    if (ev_ready) cudaEventDestroy(ev_ready);
    if (ev_halo) cudaEventDestroy(ev_halo);
    delete local;
}

Dist *dist_create(const std::string &spec, const int64_t gdims[3], const sdag_plan_opts &o, int rank, int nranks,
                  void *comm) {
    // analyse once on the global grid to get R_z (host-only)
    sdag_plan_opts ho = o;
    ho.device = SDAG_DEVICE_NONE;
    ho.tune = 0;
    std::unique_ptr<Plan> g(plan_create(spec, gdims, ho));
    const int rz = g->an.radius[0];
    std::unique_ptr<Dist> d(new Dist());
    d->time_tile = std::max(1, int(o.time_tile));
    d->slab = slab_partition(gdims[0], rz, nranks, rank, d->time_tile);
    d->rz = rz;
    d->gnz = gdims[0];
    d->rank = rank;
    d->nranks = nranks;
    d->comm = comm;
    const int64_t ldims[3] = {d->slab.nz_alloc, gdims[1], gdims[2]};
    d->local = plan_create(spec, ldims, o);
    d->handle.p = d->local;
    if (!d->local->host_only) {
        check_cuda(cudaEventCreateWithFlags(&d->ev_ready, cudaEventDisableTiming), "cudaEventCreate");
        check_cuda(cudaEventCreateWithFlags(&d->ev_halo, cudaEventDisableTiming), "cudaEventCreate");
    }
    return d.release();
}

Dist *dist_create_local(const Plan *local, int rank, int nranks, void *comm, int time_tile) {
    if (!local) throw Error(SDAG_ERR_INVALID_ARG, "null plan");
    if (local->spec_text.empty())
        throw Error(SDAG_ERR_UNSUPPORTED, "the plan was not created from spec text (a program stage)");
    if (nranks < 1) throw Error(SDAG_ERR_INVALID_ARG, "nranks must be >= 1");
    const int64_t g[3] = {local->dims[0] * nranks, local->dims[1], local->dims[2]};
    sdag_plan_opts o = local->opts_copy;
    o.force_variant = local->force_variant.empty() ? nullptr : local->force_variant.c_str();
    o.time_tile = time_tile < 1 ? 1 : time_tile;
    if (local->host_only) o.device = SDAG_DEVICE_NONE;
    else o.device = local->device;
    return dist_create(local->spec_text, g, o, rank, nranks, comm);
}

namespace {

struct Ranges {
    bool split = true;  // interior/boundary overlap possible
    int64_t in_lo = 0, in_hi = 0;
    int64_t b_lo[2] = {0, 0}, b_hi[2] = {0, 0};  // lower / upper boundary bands
};

// Output planes of one launch whose inputs reach `depth` planes in z (R_z for
// a sweep, x R_z for an x-sweep fused launch): the interior range reads no
// ghost plane and can overlap the exchange; the two bands next to the ghost
// layers run after it.
Ranges ranges_of(const Dist *d, int64_t depth) {
    const Slab &s = d->slab;
    const int64_t H = s.halo;
    Ranges r;
    if (depth == 0 || s.nz_own < 2 * depth) {  // nothing to overlap: one launch after the exchange
        r.split = false;
        r.b_lo[0] = s.k_lo;
        r.b_hi[0] = s.k_hi;
        return r;
    }
    r.in_lo = s.has_lower ? H + depth : s.k_lo;
    r.in_hi = s.has_upper ? H + s.nz_own - depth : s.k_hi;
    r.in_lo = std::max(r.in_lo, s.k_lo);
    r.in_hi = std::min(r.in_hi, s.k_hi);
    if (s.has_lower) {
        r.b_lo[0] = std::max<int64_t>(H, s.k_lo);
        r.b_hi[0] = std::min<int64_t>(H + depth, s.k_hi);
    }
    if (s.has_upper) {
        r.b_lo[1] = std::max<int64_t>(H + s.nz_own - depth, s.k_lo);
        r.b_hi[1] = std::min<int64_t>(H + s.nz_own, s.k_hi);
    }
    return r;
}

// z-read inputs that need ghost planes
std::vector<int> halo_arrays(const Dist *d) {
    std::vector<int> v;
    const Plan *p = d->local;
    for (int f = 0; f < p->n3(); f++) {
        const Formal &fo = p->st.formal(ArgKind::Array3D, f);
        if (fo.role == Role::In && p->an.arr_radius[f][0] > 0) v.push_back(f);
    }
    return v;
}

// One NCCL group of point-to-point transfers (send[i] -> peer[i], recv[i] <- peer[i]).
// Every Send/Recv between GroupStart and GroupEnd is made even after a failure,
// and GroupEnd always runs: an open group would corrupt every later call on the
// communicator.  The first error is reported after the group is closed.
struct Xfer {
    const double *send;
    double *recv;
    size_t count;
    int peer;
};
void nccl_group(void *comm, const std::vector<Xfer> &xs, cudaStream_t st) {
    const NcclApi &N = nccl();
    auto c = static_cast<ncclComm_t>(comm);
    ncclResult_t first = 0;
    const char *first_what = nullptr;
    auto call = [&](ncclResult_t r, const char *what) {
        if (r != 0 && first == 0) {
            first = r;
            first_what = what;
        }
    };
    nck(N.GroupStart(), "ncclGroupStart");
    for (const Xfer &x : xs) {
        call(N.Send(x.send, x.count, ncclFloat64, x.peer, c, st), "ncclSend");
        call(N.Recv(x.recv, x.count, ncclFloat64, x.peer, c, st), "ncclRecv");
    }
    const ncclResult_t ge = N.GroupEnd();
    if (first != 0) nck(first, first_what);
    nck(ge, "ncclGroupEnd");
    // SDAG_NCCL_CHECK=1 (debug): poll the communicator's asynchronous error
    // after every group (failure detection)
    static const bool async_check = std::getenv("SDAG_NCCL_CHECK") && std::getenv("SDAG_NCCL_CHECK")[0] == '1';
    if (async_check && N.CommGetAsyncError) {
        ncclResult_t ae = 0;
        nck(N.CommGetAsyncError(c, &ae), "ncclCommGetAsyncError");
        nck(ae, "NCCL asynchronous error");
    }
}

}  // namespace

void nccl_sendrecv(void *comm, int peer, const double *send, double *recv, int64_t count, cudaStream_t st) {
    if (!comm) throw Error(SDAG_ERR_INVALID_ARG, "null communicator");
    if (count < 0 || (count > 0 && (!send || !recv))) throw Error(SDAG_ERR_INVALID_ARG, "bad buffers");
    nccl_group(comm, {Xfer{send, recv, size_t(count), peer}}, st);
}

namespace {

void exchange_nccl(Dist *d, double *const *a3, cudaStream_t comm, int planes) {
    if (planes == 0 || d->nranks == 1) return;
    if (!d->comm) throw Error(SDAG_ERR_INVALID_ARG, "multi-rank dist without an NCCL communicator");
    const Plan *p = d->local;
    const size_t plane = size_t(p->dims[1] * p->dims[2]);
    const size_t cnt = plane * size_t(planes);
    const Halo h = halo_schedule(d->slab, planes);
    NvtxRange nr("sdag_halo_exchange_nccl");
    // to the lower neighbour: my lowest `planes` owned planes, its planes into my
    // ghosts below; likewise above (halo_schedule, tested bitwise via loopback)
    std::vector<Xfer> xs;
    for (int f : halo_arrays(d)) {
        double *a = a3[f];
        if (h.lo_send >= 0) xs.push_back({a + size_t(h.lo_send) * plane, a + size_t(h.lo_recv) * plane, cnt, d->rank - 1});
        if (h.up_send >= 0) xs.push_back({a + size_t(h.up_send) * plane, a + size_t(h.up_recv) * plane, cnt, d->rank + 1});
    }
    nccl_group(d->comm, xs, comm);
}

// local planes of the global z-interior (multi-sweep kernels keep the rest fixed)
void global_interior(const Dist *d, int64_t zr[2]) {
    const Slab &s = d->slab;
    const int64_t g_of_l0 = s.z0 - s.halo;
    const int64_t gnz = d->gnz;
    zr[0] = d->rz - g_of_l0;
    zr[1] = gnz - d->rz - g_of_l0;
}

// One launch of kernel `k` (x = k.tsteps sweeps) with its exchange of x R_z planes.
void sweep_split(Dist *d, const KernelDesc &k, double *const *a3, const double *const *a1, const double *s,
                 cudaStream_t compute, cudaStream_t comm, bool do_exchange) {
    Plan *p = d->local;
    const int64_t depth = int64_t(d->rz) * k.tsteps;
    const Ranges r = ranges_of(d, depth);
    const bool xchg = do_exchange && depth > 0 && d->nranks > 1;
    int64_t zr[2];
    global_interior(d, zr);
    if (xchg) {
        check_cuda(cudaEventRecord(d->ev_ready, compute), "cudaEventRecord");
        check_cuda(cudaStreamWaitEvent(comm, d->ev_ready, 0), "cudaStreamWaitEvent");
        exchange_nccl(d, a3, comm, int(depth));
        check_cuda(cudaEventRecord(d->ev_halo, comm), "cudaEventRecord");
    }
    double *const *a = const_cast<double *const *>(a3);
    if (r.split && r.in_hi > r.in_lo) plan_launch(p, k, a, a1, s, 1, r.in_lo, r.in_hi, compute, nullptr, zr);
    if (xchg) check_cuda(cudaStreamWaitEvent(compute, d->ev_halo, 0), "cudaStreamWaitEvent");
    for (int q = 0; q < 2; q++)
        if (r.b_hi[q] > r.b_lo[q]) plan_launch(p, k, a, a1, s, 1, r.b_lo[q], r.b_hi[q], compute, nullptr, zr);
}

cudaStream_t comm_stream(Dist *d, cudaStream_t comm) {
    if (comm) return comm;
    if (!d->own_comm) check_cuda(cudaStreamCreateWithFlags(&d->own_comm, cudaStreamNonBlocking), "cudaStreamCreate");
    return d->own_comm;
}

// the launch schedule of T sweeps on this slab: fused kernels of up to
// time_tile sweeps (their exchange depth fits the ghost layer), deep-tuning DP
std::vector<const KernelDesc *> iter_schedule(Dist *d, double *b0, double *b1, int T) {
    Plan *p = d->local;
    const KernelDesc *fk[8] = {nullptr};
    int maxdeg = 1;
    const bool aligned = (reinterpret_cast<uintptr_t>(b0) % 16) == 0 && (reinterpret_cast<uintptr_t>(b1) % 16) == 0;
    if (p->fusion && aligned && p->dims[2] % 2 == 0)
        for (const KernelDesc *f : p->fused)
            if (f->tsteps <= d->time_tile && !fk[f->tsteps]) {
                fk[f->tsteps] = f;
                maxdeg = std::max(maxdeg, f->tsteps);
            }
    double f[8];
    for (int x = 0; x < 8; x++) f[x] = (x == 1 || (x > 1 && x <= maxdeg && fk[x])) ? p->fcost[x] : 0.0;
    std::vector<const KernelDesc *> seq;
    for (int x : fusion_schedule(f, maxdeg, T)) {
        if (x == 1) {
            seq.push_back(nullptr);  // the plan's single-sweep kernel (picked per launch for alignment)
        } else {
            seq.push_back(fk[x]);
        }
    }
    return seq;
}

const KernelDesc &single_kernel(Plan *p, double *in) {
    const KernelDesc &k = p->kernel();
    if (!k.tma || (reinterpret_cast<uintptr_t>(in) % 16 == 0 && p->dims[2] % 2 == 0)) return k;
    for (const KernelDesc *c : p->cands)
        if (!c->tma && c->tx == k.tx && c->ty == k.ty && c->ux == k.ux && c->uy == k.uy && c->pf == k.pf) return *c;
    throw Error(SDAG_ERR_INVALID_ARG, "arrays are not 16-byte aligned and no LSU variant exists");
}

}  // namespace

void dist_apply(Dist *d, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                cudaStream_t compute, cudaStream_t comm) {
    if (!d) throw Error(SDAG_ERR_INVALID_ARG, "null dist");
    Plan *p = d->local;
    if (p->host_only) throw Error(SDAG_ERR_DEVICE, "host-only dist plan");
    // counts, null pointers, null scalars, output aliasing: nothing enqueued on a bad call
    plan_validate(p, a3, n3, a1, n1, s, ns, 1);
    if (p->kernel().tma)
        for (int f = 0; f < n3; f++)
            if (reinterpret_cast<uintptr_t>(a3[f]) % 16) throw Error(SDAG_ERR_INVALID_ARG, "grid arrays must be 16-B aligned");
    DeviceGuard dg(p);  // libsdag's runtime: bind the plan's device, restore the caller's
    NvtxRange nr("sdag_dist_apply " + p->st.name);
    sweep_split(d, p->kernel(), a3, a1, s, compute, comm_stream(d, comm), true);
}

void dist_apply_iterated(Dist *d, double *b0, double *b1, int T, const double *s, int ns, cudaStream_t compute,
                         cudaStream_t comm) {
    if (!d) throw Error(SDAG_ERR_INVALID_ARG, "null dist");
    Plan *p = d->local;
    if (p->host_only) throw Error(SDAG_ERR_DEVICE, "host-only dist plan");
    if (p->n3() != 2 || p->an.n_in != 1 || p->an.n_out != 1 || p->n1() != 0)
        throw Error(SDAG_ERR_INVALID_ARG, "iterated dist apply needs a 1-input 1-output plan");
    if (ns != p->ns() || (ns > 0 && !s) || !b0 || !b1 || b0 == b1 || T < 0) throw Error(SDAG_ERR_INVALID_ARG, "bad arguments");
    int fin = -1, fout = -1;
    for (int f = 0; f < 2; f++) (p->st.formal(ArgKind::Array3D, f).role == Role::In ? fin : fout) = f;
    DeviceGuard dg(p);
    NvtxRange nr("sdag_dist_apply_iterated " + p->st.name + " T=" + std::to_string(T));
    cudaStream_t cs = comm_stream(d, comm);
    double *bufs[2] = {b0, b1};
    int cur = 0;
    for (const KernelDesc *k : iter_schedule(d, b0, b1, T)) {
        double *a3[2];
        a3[fin] = bufs[cur];
        a3[fout] = bufs[1 - cur];
        sweep_split(d, k ? *k : single_kernel(p, bufs[cur]), a3, nullptr, s, compute, cs, true);
        cur = 1 - cur;
    }
}

void dist_apply_iterated_loopback(Dist **ds, int n, double *const *b0, double *const *b1, int T, const double *s,
                                  int ns, cudaStream_t stream) {
    if (!ds || n < 1) throw Error(SDAG_ERR_INVALID_ARG, "bad dist list");
    NvtxRange nr("sdag_dist_apply_iterated_loopback T=" + std::to_string(T));
    for (int r = 0; r < n; r++) {
        if (!ds[r] || ds[r]->rank != r || ds[r]->nranks != n) throw Error(SDAG_ERR_INVALID_ARG, "dists must be ranks 0..n-1");
        if (ds[r]->local->host_only) throw Error(SDAG_ERR_DEVICE, "host-only dist plan");
        if (ds[r]->time_tile != ds[0]->time_tile) throw Error(SDAG_ERR_INVALID_ARG, "dists must share time_tile");
    }
    Plan *p0 = ds[0]->local;
    if (p0->n3() != 2 || p0->an.n_in != 1 || p0->an.n_out != 1 || p0->n1() != 0 || ns != p0->ns() || (ns > 0 && !s) || T < 0)
        throw Error(SDAG_ERR_INVALID_ARG, "iterated loopback needs a 1-input 1-output plan");
    int fin = -1, fout = -1;
    for (int f = 0; f < 2; f++) (p0->st.formal(ArgKind::Array3D, f).role == Role::In ? fin : fout) = f;
    DeviceGuard dg(p0);
    const int64_t rz = ds[0]->rz;
    const size_t plane = size_t(p0->dims[1] * p0->dims[2]);
    // every rank follows rank 0's schedule (same plan, same buffers' alignment class)
    const std::vector<const KernelDesc *> sched = iter_schedule(ds[0], b0[0], b1[0], T);
    int t = 0;
    for (const KernelDesc *k0 : sched) {
        auto in = [&](int r) { return (t & 1) ? b1[r] : b0[r]; };
        auto out = [&](int r) { return (t & 1) ? b0[r] : b1[r]; };
        const int x = k0 ? k0->tsteps : 1;
        const int planes = int(rz) * x;
        if (planes > 0) {
            for (int r = 0; r < n; r++) {  // the same schedule the NCCL path sends/receives
                const Halo h = halo_schedule(ds[r]->slab, planes);
                if (h.lo_recv >= 0) {  // from the lower neighbour's upper send band
                    const Halo hl = halo_schedule(ds[r - 1]->slab, planes);
                    check_cuda(cudaMemcpyAsync(in(r) + size_t(h.lo_recv) * plane, in(r - 1) + size_t(hl.up_send) * plane,
                                               size_t(planes) * plane * 8, cudaMemcpyDeviceToDevice, stream),
                               "loopback halo");
                }
                if (h.up_recv >= 0) {  // from the upper neighbour's lower send band
                    const Halo hu = halo_schedule(ds[r + 1]->slab, planes);
                    check_cuda(cudaMemcpyAsync(in(r) + size_t(h.up_recv) * plane, in(r + 1) + size_t(hu.lo_send) * plane,
                                               size_t(planes) * plane * 8, cudaMemcpyDeviceToDevice, stream),
                               "loopback halo");
                }
            }
        }
        for (int r = 0; r < n; r++) {
            double *a3[2];
            a3[fin] = in(r);
            a3[fout] = out(r);
            sweep_split(ds[r], k0 ? *k0 : single_kernel(ds[r]->local, in(r)), a3, nullptr, s, stream, stream, false);
        }
        t++;
    }
}



// ---------------------------------------------------------------------------
// peer-memory halo path (p2p)
//
// Launch t of a call reads buf[t&1] (input) and writes buf[(t+1)&1].  Its
// boundary bands -- owned planes [H, 2H) and [nz_own, nz_own + H), the planes
// the neighbours hold as ghosts -- are stored by the sweep kernel itself both
// locally and into the neighbour's buf[(t+1)&1] ghost planes (Mirror), after
// this rank's stream has waited for the neighbours' flag >= e_t = base + t:
//  * the neighbour finished launch t-1, so its stores into MY buf[t&1] ghosts
//    (read now) have landed, and
//  * it finished reading ITS buf[(t+1)&1] (= its input of launch t-1), into
//    whose ghosts these stores go.
// After the boundary launch the rank signals e_t + 1.  The interior planes
// [2H, nz_own) read and write no ghost plane: they run first, with no wait.
// Before launch 0 the input bands of buf0 are pushed (cudaMemcpyAsync over
// P2P) after the neighbours' previous call ended, and `base` is signalled.
// Kernels without a KernelDesc::fn_mirror instantiation push their output
// bands the same way.
// ---------------------------------------------------------------------------

namespace {

size_t p2p_buf_bytes(int64_t nz_alloc, int64_t ny, int64_t nx) {
    const size_t b = size_t(nz_alloc) * size_t(ny) * size_t(nx) * 8;
    return (b + 4095) / 4096 * 4096;
}

void p2p_map_peer(Dist *d, int side, void *base) {
    if (side != 0 && side != 1) throw Error(SDAG_ERR_INVALID_ARG, "side must be 0 (lower) or 1 (upper)");
    const int nr = d->rank + (side == 0 ? -1 : 1);
    if (nr < 0 || nr >= d->nranks) throw Error(SDAG_ERR_INVALID_ARG, "no neighbour on that side");
    const Slab ns = slab_partition(d->gnz, d->rz, d->nranks, nr, d->time_tile);
    const size_t bb = p2p_buf_bytes(ns.nz_alloc, d->local->dims[1], d->local->dims[2]);
    char *b = static_cast<char *>(base);
    d->peer_buf[side][0] = reinterpret_cast<double *>(b);
    d->peer_buf[side][1] = reinterpret_cast<double *>(b + bb);
    uint32_t *pf = reinterpret_cast<uint32_t *>(b + 2 * bb);
    d->peer_flag[side] = pf + (side == 0 ? 1 : 0);  // I am my lower neighbour's upper side
    // global g = z0 - H + k (mine) = z0' - H + k' (neighbour's)
    d->peer_shift[side] = d->slab.z0 - ns.z0;
}

}  // namespace

void dist_apply_host(Dist *d, double *const *h3, int n3, const double *const *h1, int n1, const double *s, int ns,
                     cudaStream_t stream, int64_t *h2d, int64_t *d2h) {
    if (!d) throw Error(SDAG_ERR_INVALID_ARG, "null dist");
    if (d->local->host_only) throw Error(SDAG_ERR_DEVICE, "host-only dist plan");
    const int64_t kr[2] = {d->slab.k_lo, d->slab.k_hi};
    apply_host(d->local, h3, n3, h1, n1, s, ns, stream, h2d, d2h, kr);
}

void dist_p2p_alloc(Dist *d, double **buf0, double **buf1) {
    if (!d) throw Error(SDAG_ERR_INVALID_ARG, "null dist");
    if (d->local->host_only) throw Error(SDAG_ERR_DEVICE, "host-only dist plan");
    DeviceGuard dg(d->local);
    if (!d->p2p_base) {
        const int64_t *dims = d->local->dims;
        d->p2p_buf_bytes = p2p_buf_bytes(dims[0], dims[1], dims[2]);
        const size_t total = 2 * d->p2p_buf_bytes + 4096;
        check_cuda(cudaMalloc(&d->p2p_base, total), "cudaMalloc(p2p slab buffers)");
        char *b = static_cast<char *>(d->p2p_base);
        d->p2p_buf[0] = reinterpret_cast<double *>(b);
        d->p2p_buf[1] = reinterpret_cast<double *>(b + d->p2p_buf_bytes);
        d->p2p_flags = reinterpret_cast<uint32_t *>(b + 2 * d->p2p_buf_bytes);
        check_cuda(cudaMemset(d->p2p_base, 0, total), "cudaMemset(p2p)");
        check_cuda(cudaDeviceSynchronize(), "cudaDeviceSynchronize");
        d->epoch = 0;
        d->p2p_synced = false;
    }
    if (buf0) *buf0 = d->p2p_buf[0];
    if (buf1) *buf1 = d->p2p_buf[1];
}

void dist_p2p_handle(Dist *d, uint8_t handle[64]) {
    if (!d || !d->p2p_base) throw Error(SDAG_ERR_INVALID_ARG, "call sdag_dist_p2p_alloc first");
    static_assert(sizeof(cudaIpcMemHandle_t) == 64, "IPC handle size");
    cudaIpcMemHandle_t h;
    check_cuda(cudaIpcGetMemHandle(&h, d->p2p_base), "cudaIpcGetMemHandle");
    std::memcpy(handle, &h, 64);
}

void dist_p2p_attach(Dist *d, int side, const uint8_t handle[64]) {
    if (!d || !d->p2p_base) throw Error(SDAG_ERR_INVALID_ARG, "call sdag_dist_p2p_alloc first");
    if (side != 0 && side != 1) throw Error(SDAG_ERR_INVALID_ARG, "side must be 0 (lower) or 1 (upper)");
    DeviceGuard dg(d->local);
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, 64);
    void *m = nullptr;
    check_cuda(cudaIpcOpenMemHandle(&m, h, cudaIpcMemLazyEnablePeerAccess), "cudaIpcOpenMemHandle");
    if (d->peer_ipc[side]) cudaIpcCloseMemHandle(d->peer_ipc[side]);
    d->peer_ipc[side] = m;
    p2p_map_peer(d, side, m);
}

void dist_p2p_attach_local(Dist *d, int side, Dist *peer) {
    if (!d || !d->p2p_base || !peer || !peer->p2p_base)
        throw Error(SDAG_ERR_INVALID_ARG, "both dists need sdag_dist_p2p_alloc first");
    if (peer->nranks != d->nranks || peer->rank != d->rank + (side == 0 ? -1 : 1))
        throw Error(SDAG_ERR_INVALID_ARG, "peer is not this rank's neighbour on that side");
    if (peer->local->device != d->local->device) {
        int ok = 0;
        check_cuda(cudaDeviceCanAccessPeer(&ok, d->local->device, peer->local->device), "cudaDeviceCanAccessPeer");
        if (!ok) throw Error(SDAG_ERR_DEVICE, "devices cannot access each other's memory");
        DeviceGuard dg(d->local);
        const cudaError_t e = cudaDeviceEnablePeerAccess(peer->local->device, 0);
        if (e != cudaSuccess && e != cudaErrorPeerAccessAlreadyEnabled) check_cuda(e, "cudaDeviceEnablePeerAccess");
        cudaGetLastError();
    }
    p2p_map_peer(d, side, peer->p2p_base);
}

void dist_p2p_apply_iterated(Dist *d, int T, const double *s, int ns, cudaStream_t st) {
    if (!d || !d->p2p_base) throw Error(SDAG_ERR_INVALID_ARG, "call sdag_dist_p2p_alloc first");
    Plan *p = d->local;
    if (p->n3() != 2 || p->an.n_in != 1 || p->an.n_out != 1 || p->n1() != 0)
        throw Error(SDAG_ERR_INVALID_ARG, "iterated dist apply needs a 1-input 1-output plan");
    if (ns != p->ns() || (ns > 0 && !s) || T < 0) throw Error(SDAG_ERR_INVALID_ARG, "bad arguments");
    const Slab &S = d->slab;
    const int has[2] = {S.has_lower, S.has_upper};
    for (int q = 0; q < 2; q++)
        if (has[q] && !d->peer_buf[q][0])
            throw Error(SDAG_ERR_INVALID_ARG, std::string("no ") + (q ? "upper" : "lower") +
                                                  " neighbour attached (sdag_dist_p2p_attach)");
    int fin = -1, fout = -1;
    for (int f = 0; f < 2; f++) (p->st.formal(ArgKind::Array3D, f).role == Role::In ? fin : fout) = f;
    DeviceGuard dg(p);
    if (T == 0) return;
    NvtxRange nr("sdag_dist_p2p_apply_iterated " + p->st.name + " T=" + std::to_string(T));

    const int64_t H = S.halo;
    const size_t plane = size_t(p->dims[1] * p->dims[2]);
    const size_t band = size_t(H) * plane * 8;
    double **buf = d->p2p_buf;
    // bands, in my local planes: [H, 2H) goes to the lower neighbour, [nz_own, nz_own+H) to the upper
    const int64_t band_lo[2] = {H, S.nz_own};
    auto push_to = [&](int b, int pb) {  // my bands of buffer b -> the neighbours' ghost planes of their buffer pb
        for (int q = 0; q < 2; q++)
            if (has[q])
                check_cuda(cudaMemcpyAsync(d->peer_buf[q][pb] + size_t(band_lo[q] + d->peer_shift[q]) * plane,
                                           buf[b] + size_t(band_lo[q]) * plane, band, cudaMemcpyDefault, st),
                           "p2p band push");
    };
    auto push = [&](int b) { push_to(b, b); };
    auto signal = [&](uint32_t v) {
        p2p_signal(has[0] ? d->peer_flag[0] : nullptr, has[1] ? d->peer_flag[1] : nullptr, v, st);
        d->epoch = v;
    };
    auto wait = [&](uint32_t v) {
        const uint32_t need[2] = {v, v};
        p2p_wait(d->p2p_flags, need, has, st);
    };

    // every kernel this call launches is loaded before the first flag wait is
    // enqueued (lazy loading of a kernel can block behind a spinning wait)
    const std::vector<const KernelDesc *> sched = iter_schedule(d, buf[0], buf[1], T);
    p2p_preload();
    for (const KernelDesc *k0 : sched) {
        const KernelDesc &k = k0 ? *k0 : single_kernel(p, buf[0]);
        cudaFuncAttributes fa;
        for (const void *fn : {k.fn, k.fn_mirror})
            if (fn) check_cuda(cudaFuncGetAttributes(&fa, fn), "cudaFuncGetAttributes");
    }

    wait(d->epoch);  // the neighbours' previous call is over (first call: 0)
    if (!d->p2p_synced) {
        // First call after sdag_dist_p2p_alloc: the caller filled buf0's owned
        // planes.  buf1's owned planes get buf0's (its x/y ring and the global
        // z-ring planes are never written by a sweep), and my bands of buf0
        // go into the neighbours' buf1 ghost planes too (their x/y ring is
        // never written by the neighbours' mirrored stores, which cover the
        // interior only).  All of it precedes signal(base), which gates every
        // neighbour access to those planes, and nobody else writes my owned
        // planes: race-free.
        check_cuda(cudaMemcpyAsync(buf[1] + size_t(H) * plane, buf[0] + size_t(H) * plane,
                                   size_t(S.nz_own) * plane * 8, cudaMemcpyDeviceToDevice, st), "p2p buf1 init");
        push_to(0, 1);
        d->p2p_synced = true;
    }
    push(0);
    const uint32_t base = d->epoch + 1;
    signal(base);

    int64_t zr[2];
    global_interior(d, zr);
    const Ranges r = ranges_of(d, H);  // bands of full ghost depth: every plane a neighbour reads
    int cur = 0;
    uint32_t t = 0;
    for (const KernelDesc *k0 : sched) {
        const KernelDesc &k = k0 ? *k0 : single_kernel(p, buf[cur]);
        double *a3[2];
        a3[fin] = buf[cur];
        a3[fout] = buf[1 - cur];
        if (r.split && r.in_hi > r.in_lo) plan_launch(p, k, a3, nullptr, s, 1, r.in_lo, r.in_hi, st, nullptr, zr);
        wait(base + t);
        Mirror m;
        if (k.fn_mirror)
            for (int q = 0; q < 2; q++)
                if (has[q]) {
                    m.peer[q] = d->peer_buf[q][1 - cur];
                    m.off[q] = d->peer_shift[q] * int64_t(plane);
                    m.klo[q] = int32_t(band_lo[q]);
                    m.khi[q] = int32_t(band_lo[q] + H);
                }
        for (int q = 0; q < 2; q++)
            if (r.b_hi[q] > r.b_lo[q])
                plan_launch(p, k, a3, nullptr, s, 1, r.b_lo[q], r.b_hi[q], st, nullptr, zr, k.fn_mirror ? &m : nullptr);
        if (!k.fn_mirror) push(1 - cur);
        signal(base + t + 1);
        cur = 1 - cur;
        t++;
    }
}

}  // namespace sdag
