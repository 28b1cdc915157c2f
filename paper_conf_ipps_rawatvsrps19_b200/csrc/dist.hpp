// dist.hpp -- a7: z-slab domain decomposition with per-sweep halo exchange.
#pragma once

#include <cuda_runtime.h>

#include "plan.hpp"

namespace sdag {

// Pure host logic (testable without a device): which global planes a rank
// owns, its local allocation, the local plane range it computes.
struct Slab {
    int64_t z0 = 0;        // first owned global plane
    int64_t nz_own = 0;    // owned planes
    int64_t halo = 0;      // ghost planes per side H = R_z x time tile
    int64_t nz_alloc = 0;  // owned + 2 H (ghosts below and above)
    int64_t k_lo = 0, k_hi = 0;  // local planes computed (global interior only)
    int has_lower = 0, has_upper = 0;
};
// time_tile t >= 1: ghost depth H = R_z t, so t sweeps can run between
// exchanges (communication-avoiding temporal fusion).
Slab slab_partition(int64_t global_nz, int rz, int nranks, int rank, int time_tile = 1);

// Halo schedule of one exchange of `planes` (<= H) planes per side, in LOCAL
// plane indices: to the lower neighbour send [lo_send, lo_send+planes) and
// receive into [lo_recv, lo_recv+planes); likewise for the upper neighbour.
// -1 = no neighbour.
struct Halo {
    int64_t lo_send = -1, lo_recv = -1, up_send = -1, up_recv = -1, planes = 0;
};
Halo halo_schedule(const Slab &s, int planes);

struct Dist {
    Plan *local = nullptr;  // plan over the local allocation (nz_alloc, ny, nx)
    sdag_plan_s handle{nullptr};
    Slab slab;
    int rz = 0;
    int time_tile = 1;      // sweeps a fused launch may take between exchanges (H = rz * time_tile)
    int64_t gnz = 0;        // global z extent
    int rank = 0, nranks = 1;
    void *comm = nullptr;   // ncclComm_t (not owned)
    cudaStream_t own_comm = nullptr;
    cudaEvent_t ev_ready = nullptr, ev_halo = nullptr;
    // peer-memory halo path (p2p): one allocation buf0 | buf1 | flags owned here,
    // the neighbours' allocations mapped (CUDA IPC, or same-process pointers)
    void *p2p_base = nullptr;
    size_t p2p_buf_bytes = 0;
    double *p2p_buf[2] = {nullptr, nullptr};
    uint32_t *p2p_flags = nullptr;        // [0] written by the lower neighbour, [1] by the upper
    double *peer_buf[2][2] = {};          // [side][buffer] of the neighbours (0 lower, 1 upper)
    uint32_t *peer_flag[2] = {};          // the neighbour's word this rank writes
    int64_t peer_shift[2] = {0, 0};       // my local plane k is the neighbour's plane k + shift
    void *peer_ipc[2] = {};               // opened IPC mappings (closed in ~Dist)
    uint32_t epoch = 0;                   // last flag value this rank signalled
    bool p2p_synced = false;              // buf1 initialised from buf0 (first p2p call)
    ~Dist();
};

// a dist from a local plan of the rank's OWNED slab (nz_own, ny, nx), every
// rank owning nz_own planes (weak scaling): global nz = nz_own * nranks
Dist *dist_create_local(const Plan *local, int rank, int nranks, void *comm, int time_tile);
Dist *dist_create(const std::string &spec, const int64_t gdims[3], const sdag_plan_opts &o, int rank, int nranks,
                  void *comm);
void dist_apply(Dist *d, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                cudaStream_t compute, cudaStream_t comm);
void dist_apply_iterated(Dist *d, double *b0, double *b1, int T, const double *s, int ns, cudaStream_t compute,
                         cudaStream_t comm);
void dist_apply_iterated_loopback(Dist **d, int n, double *const *b0, double *const *b1, int T, const double *s,
                                  int ns, cudaStream_t stream);

// peer-memory halo path (SURVEY 8(e) B200-native alternative): the launches
// that compute a slab's boundary planes also store them into the neighbours'
// ghost planes (NVLink P2P), ordered by per-neighbour flag words; no NCCL.
// one sweep end to end with host buffers: the rank's host slab (local layout,
// ghost planes included -- the host holds them) is pipelined H2D / sweep / D2H
// like sdag_apply_host; only the rank's planes of the global interior are
// computed and returned; no exchange is needed
void dist_apply_host(Dist *d, double *const *h3, int n3, const double *const *h1, int n1, const double *s, int ns,
                     cudaStream_t stream, int64_t *h2d, int64_t *d2h);
void dist_p2p_alloc(Dist *d, double **buf0, double **buf1);
void dist_p2p_handle(Dist *d, uint8_t handle[64]);
void dist_p2p_attach(Dist *d, int side, const uint8_t handle[64]);
void dist_p2p_attach_local(Dist *d, int side, Dist *peer);
void dist_p2p_apply_iterated(Dist *d, int T, const double *s, int ns, cudaStream_t stream);

void nccl_unique_id(uint8_t id[128]);
void *nccl_comm_create(const uint8_t id[128], int nranks, int rank, int device);
void nccl_comm_destroy(void *comm);
// one grouped ncclSend + ncclRecv with `peer` (the halo exchange's code path; peer may be this rank)
void nccl_sendrecv(void *comm, int peer, const double *send, double *recv, int64_t count, cudaStream_t st);

}  // namespace sdag
