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
    ~Dist();
};

Dist *dist_create(const std::string &spec, const int64_t gdims[3], const sdag_plan_opts &o, int rank, int nranks,
                  void *comm);
void dist_apply(Dist *d, double *const *a3, int n3, const double *const *a1, int n1, const double *s, int ns,
                cudaStream_t compute, cudaStream_t comm);
void dist_apply_iterated(Dist *d, double *b0, double *b1, int T, const double *s, int ns, cudaStream_t compute,
                         cudaStream_t comm);
void dist_apply_iterated_loopback(Dist **d, int n, double *const *b0, double *const *b1, int T, const double *s,
                                  int ns, cudaStream_t stream);

void nccl_unique_id(uint8_t id[128]);
void *nccl_comm_create(const uint8_t id[128], int nranks, int rank, int device);
void nccl_comm_destroy(void *comm);

}  // namespace sdag
