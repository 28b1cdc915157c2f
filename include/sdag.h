/*
 * sdag.h -- C ABI of the B200-native FP64 stencil-DAG library ("sdag").
 *
 * Problem statement (Rawat et al., IPDPS 2019, /root/reference/PAPER.md,
 * cited P:<line> <section>): a stencil computation "sweeps a computational
 * grid, and updates the value at each point by reading a fixed neighborhood
 * around it" (section I); the user declares arrays, scalars and
 * iterators and writes the stencil function in a restricted C subset whose
 * index expressions are iterator +- constant (section II); the
 * declared arrays and scalars "will be passed as arguments to the generated
 * host function" (Listing 1).  sdag plans such a DAG
 * over N input and M output grids once (parse, analyse, choose a kernel
 * variant) and applies it asynchronously on a CUDA stream.
 *
 * Conventions common to every entry point
 * ---------------------------------------
 *  - Status: every function returning sdag_status returns SDAG_OK (0) on
 *    success.  On failure nothing has been enqueued, and sdag_last_error()
 *    returns a thread-local message (parse errors carry "line:col").
 *  - Grids: FP64, C order [nz][ny][nx] with x (iterator i, the innermost
 *    iterator) contiguous; device pointers, 8-byte aligned
 *    (16-byte aligned + nx even enables the TMA loader; otherwise the LSU
 *    loader is used).  1D arrays are device pointers of the
 *    length of the axis their iterator indexes.  Scalars are a HOST array of
 *    doubles copied into kernel parameters at enqueue time.
 *  - Argument order: 3D arrays, 1D arrays and scalars are each passed in the
 *    order they appear among the stencil function's formal parameters
 *    ("stencil jacobi (B, A, h2inv, a, b)"); sdag_plan_arg() reports
 *    names and roles.
 *  - Semantics (reading R1): out-of-place; only the interior
 *    [R_a, n_a - R_a) of each axis a is written, R_a the maximal |offset|
 *    read along a; every other element of every output is left
 *    bit-identical.  An output may not alias an input (SDAG_ERR_INVALID_ARG).
 *    "inout" arrays (read at offset 0 before being written, e.g. SW4's
 *    uacc = a1*uacc + cof*r) are updated in place.
 *  - Ownership: the caller owns all grid / 1D / scalar memory; a plan owns
 *    only immutable metadata, a TMA-descriptor cache and (for
 *    sdag_apply_host) a device workspace, all released by sdag_plan_destroy.
 *  - Synchronicity: sdag_apply* enqueue on `stream` and never synchronise
 *    (except sdag_apply_host, which is synchronous).  Device faults surface
 *    at the caller's next synchronisation.
 *  - No CPU fallback: a device that is not sm_100 returns SDAG_ERR_DEVICE.
 *  - Tracing: every enqueueing entry point opens an NVTX range named after
 *    the call ("sdag_apply <stencil> <variant>", "sdag_apply_iterated ... T=",
 *    "sdag_dist_apply*", "sdag_halo_exchange_nccl", "sdag_program_apply",
 *    "sdag_plan_create"), visible to nsys / ncu --nvtx.
 *  - Environment: SDAG_LOG=1 prints each plan's sdag_plan_describe() text
 *    (and each program stage's) to stderr at creation; SDAG_TUNE_CACHE,
 *    SDAG_GRAPHS and SDAG_NCCL_CHECK are described where they act.
 */
#ifndef SDAG_H
#define SDAG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SDAG_VERSION_MAJOR 0
#define SDAG_VERSION_MINOR 1

typedef enum sdag_status {
    SDAG_OK = 0,
    SDAG_ERR_INVALID_ARG = 1, /* null / wrong count / misaligned / aliasing / bad dims   */
    SDAG_ERR_PARSE = 2,       /* spec text does not parse (message has line:col)          */
    SDAG_ERR_SEMANTIC = 3,    /* parses but is ill-formed (undeclared name, bad index...) */
    SDAG_ERR_UNSUPPORTED = 4, /* valid DAG outside the hot path (e.g. shifted writes)     */
    SDAG_ERR_DOMAIN = 5,      /* dims too small for the radius, or order exceeded         */
    SDAG_ERR_DEVICE = 6,      /* no CUDA device / not sm_100 / host-only plan applied     */
    SDAG_ERR_CUDA = 7,        /* CUDA runtime / driver error (message has the CUDA text)  */
    SDAG_ERR_NCCL = 8,        /* NCCL error or NCCL library not loadable                  */
    SDAG_ERR_NOMEM = 9
} sdag_status;

typedef struct sdag_plan_s *sdag_plan;
typedef struct sdag_program_s *sdag_program;
typedef struct sdag_dist_s *sdag_dist;
typedef struct CUstream_st *sdag_stream; /* == cudaStream_t; NULL = legacy default stream */

/* Device selector values for sdag_plan_opts.device */
#define SDAG_DEVICE_CURRENT (-1)
#define SDAG_DEVICE_NONE (-2) /* host-only plan: parse+analyse+plan, apply -> SDAG_ERR_DEVICE */

typedef struct sdag_plan_opts {
    int32_t order;             /* declared max radius (stencil order); -1 = infer.
                                  Error SDAG_ERR_DOMAIN if any access exceeds it.          */
    int32_t device;            /* CUDA ordinal, SDAG_DEVICE_CURRENT or SDAG_DEVICE_NONE    */
    int32_t tune;              /* 0 = heuristic variant choice; 1 = time the candidates at
                                  plan time on scratch buffers (hierarchical autotuning,
                                  P:1202-1271) -- synchronises the device.  With the
                                  environment variable SDAG_TUNE_CACHE naming a file, the
                                  choice (variant, measured f(x), fused-kernel order) is
                                  appended there per (version, device, DAG, dims, batch,
                                  fusion) and later tune=1 plans of that shape restore it
                                  without timing; an unreadable/unwritable file is ignored */
    int32_t batch;             /* independent problems per apply (sdag_apply_batched); >= 1 */
    const char *force_variant; /* NULL, or a variant name from sdag_plan_variant_name()    */
    int32_t fusion;            /* sdag_apply_iterated: 1 = fuse sweeps where a fused kernel
                                  exists (temporal fusion), 0 = one launch
                                  per sweep                                               */
    int32_t time_tile;         /* sdag_dist_*: ghost depth H = R_z x time_tile (1..7), so a
                                  fused launch of up to time_tile sweeps runs between two
                                  halo exchanges (communication-avoiding temporal fusion,
                                  SURVEY 8(f) NEXT-1); 1 = exchange every sweep         */
} sdag_plan_opts;

/* Fills `o` with the defaults {order=-1, device=CURRENT, tune=0, batch=1, NULL, fusion=1,
 * time_tile=1}. */
void sdag_plan_opts_init(sdag_plan_opts *o);

typedef struct sdag_plan_info {
    int32_t n_arrays3d, n_arrays1d, n_scalars; /* formal parameters by kind           */
    int32_t n_in, n_out, n_inout;              /* roles of the 3D arrays             */
    int32_t n_statements, n_temporaries;
    int32_t radius[3];                         /* z, y, x (per-axis order)            */
    int64_t dims[3];                           /* nz, ny, nx                         */
    int64_t lo[3], hi[3];                      /* interior [lo, hi) per axis          */
    int64_t points;                            /* interior points per apply (1 problem) */
    double flops_per_point;                    /* canonical count (R9)      */
    double bytes_per_point;                    /* algorithmic HBM bytes / written pt   */
    double oi_paper;                           /* flops / (8 * #IO arrays), Table III  */
    int32_t n_kernels;                         /* launches per apply                   */
    int32_t n_variants;                        /* candidate variants considered        */
    const char *dag;                           /* registry DAG matched ("jacobi7", ...) */
    const char *variant;                       /* chosen variant name                  */
} sdag_plan_info;

/*
 * a1-a3: parse `spec` (the Listing-1 DSL, plus 1D arrays,
 * #pragma and #assign, P:461-471 / P:513-533), analyse it (radius, roles,
 * canonical flops/bytes; Table I) and choose a kernel
 * variant for grids of `dims` = {nz, ny, nx} (for 1- or 2-iterator specs the
 * missing leading extents must be 1).  `opts` may be NULL.  On success *out
 * owns the plan.  Errors: PARSE, SEMANTIC, UNSUPPORTED, DOMAIN, DEVICE
 * (device requested but unusable), INVALID_ARG.
 */
sdag_status sdag_plan_create(const char *spec, const int64_t dims[3], const sdag_plan_opts *opts,
                             sdag_plan *out);
sdag_status sdag_plan_info_get(sdag_plan plan, sdag_plan_info *out);
/* kind: 0 = 3D array, 1 = 1D array, 2 = scalar; role (3D only): 0 in, 1 out, 2 inout.
 * For 1D arrays *role is the axis (0 = z, 1 = y, 2 = x) of the iterator indexing it,
 * or -1 if the stencil never reads it (any length is accepted).  Strings live as long as the plan. */
sdag_status sdag_plan_arg(sdag_plan plan, int32_t kind, int32_t idx, const char **name, int32_t *role);
/* Candidate variants of this plan, 0 <= idx < info.n_variants. */
sdag_status sdag_plan_variant_name(sdag_plan plan, int32_t idx, const char **name);
/* The symbol of the kernel a sweep launches (demangled, as ncu lists it):
 * sweeps = 1 -> the plan's single-sweep kernel (sdag_apply); sweeps = x > 1 ->
 * the x-sweep temporally fused kernel sdag_apply_iterated uses (NEXT-1);
 * INVALID_ARG if the plan has none.  Generated kernels read "nvrtc:<variant>".
 * The string lives as long as the plan. */
sdag_status sdag_plan_kernel_name(sdag_plan plan, int32_t sweeps, const char **name);
/* Human-readable plan report (analysis counts, variant, launch geometry). */
const char *sdag_plan_describe(sdag_plan plan);
void sdag_plan_destroy(sdag_plan plan);

/*
 * a4-a5: one sweep.  arrays3d[n3d] device pointers (every 3D formal, in
 * formal order, inputs and outputs alike), arrays1d[n1d] device pointers,
 * scalars[nscalars] host doubles.  Enqueued on `stream`.
 */
sdag_status sdag_apply(sdag_plan plan, double *const *arrays3d, int32_t n3d, const double *const *arrays1d,
                       int32_t n1d, const double *scalars, int32_t nscalars, sdag_stream stream);

/* `batch` independent problems in ONE launch; every 3D array is [batch][nz][ny][nx]
 * contiguous and every 1D array [batch][len].  batch <= opts.batch is not required. */
sdag_status sdag_apply_batched(sdag_plan plan, int32_t batch, double *const *arrays3d, int32_t n3d,
                               const double *const *arrays1d, int32_t n1d, const double *scalars,
                               int32_t nscalars, sdag_stream stream);

/*
 * Multi-stencil programs (Fig 3c): a spec
 * with several `stencil` definitions and calls in sequence.  Each call is one
 * stage, planned like sdag_plan_create (registered kernel or NVRTC-generated
 * one); sdag_program_apply enqueues the stages in call order on `stream`, each
 * a full sweep over its own interior that sees the arrays as the earlier
 * stages left them (a later stage may read an earlier stage's output at any
 * offset).  sdag_plan_create rejects such specs with SDAG_ERR_UNSUPPORTED.
 *
 * Arguments are the program's DECLARED arrays and scalars that some call
 * binds, in declaration order (the generated host function's parameters,
 * P:439-441) -- not a stencil's formal order.  Roles (sdag_program_arg, 3D):
 * 0 in (read before any stage writes it), 1 out (first touched by a write;
 * intermediates read by later stages are out and caller-owned), 2 inout
 * (read, then written by a later stage).  Strings live as long as the program.
 * sdag_program_stage returns a BORROWED plan handle for stage s (info,
 * describe, variants, args); never pass it to sdag_plan_destroy.
 * sdag_program_apply validates every stage (counts, nulls, output aliasing
 * within a stage) before enqueuing anything; errors as sdag_apply.
 */
sdag_status sdag_program_create(const char *spec, const int64_t dims[3], const sdag_plan_opts *opts,
                                sdag_program *out);
sdag_status sdag_program_info(sdag_program prog, int32_t *n_stages, int32_t *n3d, int32_t *n1d, int32_t *nscalars);
sdag_status sdag_program_arg(sdag_program prog, int32_t kind, int32_t idx, const char **name, int32_t *role);
sdag_status sdag_program_stage(sdag_program prog, int32_t s, sdag_plan *out);
sdag_status sdag_program_apply(sdag_program prog, int32_t batch, double *const *arrays3d, int32_t n3d,
                               const double *const *arrays1d, int32_t n1d, const double *scalars, int32_t nscalars,
                               sdag_stream stream);
/* releases the program and its stage plans (their borrowed handles become invalid); NULL is a no-op */
void sdag_program_destroy(sdag_program prog);

/*
 * a6: T sweeps ping-pong (Fig 1a; time loop P:380-381) of a plan
 * with exactly one 3D input and one 3D output (and no 1D arrays):
 * sweep t reads buf[t&1] and writes the interior of buf[(t+1)&1].  Both
 * buffers must hold identical boundary rings on entry (fixed Dirichlet
 * ring).  Result in buf[T&1].  Sweeps may be fused per launch (temporal
 * fusion, deep-tuning DP).  Launch-bound cases (<= 4 Mi interior points,
 * T >= 4) are recorded as a CUDA graph on the second call with the same
 * buffers, T and scalars and replayed afterwards (SDAG_GRAPHS=0 disables);
 * the plan then holds the graph until it is destroyed.
 */
sdag_status sdag_apply_iterated(sdag_plan plan, double *buf0, double *buf1, int32_t T, const double *scalars,
                                int32_t nscalars, sdag_stream stream);

/*
 * End-to-end call with HOST buffers (pageable or pinned; pinned overlaps):
 * copies every 3D input/inout and 1D array host->device into a plan-owned
 * workspace, runs one sweep, copies the interior of every output/inout
 * device->host (the host ring is not written), and synchronises `stream`.
 * Pipelined over z-chunks of the output (<= 64 chunks of >= max(10, 2R_z)
 * planes): the H2D of chunk c+1 (plan-owned copy stream), the sweep of chunk c
 * (`stream`) and the D2H of chunk c-1 (second copy stream) overlap; every
 * input plane crosses the link once.  Calls on one plan are serialised.
 * h2d_bytes / d2h_bytes (nullable) receive the bytes moved.
 * Errors: INVALID_ARG (counts, null pointers), DEVICE, CUDA, NOMEM.
 */
sdag_status sdag_apply_host(sdag_plan plan, double *const *host3d, int32_t n3d, const double *const *host1d,
                            int32_t n1d, const double *scalars, int32_t nscalars, sdag_stream stream,
                            int64_t *h2d_bytes, int64_t *d2h_bytes);

/* Pure host logic, no device: the temporal-fusion schedule apply_iterated
 * uses (NEXT-1; deep tuning's dynamic program, P:1416-1440,
 * opt(T) = min_x f(x) + opt(T - x)).  f[x], x = 1..maxdeg (f[0] unused), is
 * the cost of one launch fusing x sweeps; f[x] <= 0 means "no such kernel";
 * f[1] must be > 0.  Every launch flips a ping-pong pair, so the schedule has
 * a number of launches with the parity of T (the result lands in buf[T & 1]).
 * On success seq[0..*n) holds the sweeps per launch in launch order and
 * *cost their summed f.  Errors: INVALID_ARG for null pointers, maxdeg
 * outside 1..7, T < 0, f[1] <= 0, or cap < the schedule length. */
sdag_status sdag_fusion_schedule(const double *f, int32_t maxdeg, int32_t T, int32_t *seq, int32_t cap, int32_t *n,
                                 double *cost);

/* ------------------------------------------------------------------------
 * a7: z-slab domain decomposition with per-sweep halo exchange
 * (north-star addition; the paper is single-GPU).
 * Rank p owns global interior-capable planes [z0_p, z0_p + nz_p); its local
 * allocation is (R_z + nz_p + R_z) planes: R_z ghost planes below and above.
 * ------------------------------------------------------------------------ */

/* Pure host logic, no device: partition of `global_nz` planes over `nranks`
 * for radius `rz`.  out[0] = first owned global plane, out[1] = owned planes,
 * out[2] = local allocation planes (owned + 2 rz), out[3] = first local plane
 * this rank computes, out[4] = one past the last, out[5] = 1 if the rank has
 * a lower neighbour, out[6] = 1 if it has an upper neighbour.  Remainder
 * planes go to the lowest ranks.  Error DOMAIN if some rank would own < rz. */
sdag_status sdag_slab_partition(int64_t global_nz, int32_t rz, int32_t nranks, int32_t rank, int64_t out[7]);

/* Pure host logic: the per-sweep halo schedule of that rank, in LOCAL plane
 * indices (rz planes each).  out[0] = first plane sent to the lower
 * neighbour, out[1] = first ghost plane received from it, out[2] / out[3] the
 * same for the upper neighbour (-1 = no such neighbour), out[4] = rz. */
sdag_status sdag_slab_halo(int64_t global_nz, int32_t rz, int32_t nranks, int32_t rank, int64_t out[5]);

/* As sdag_slab_partition / sdag_slab_halo for a ghost depth H = rz * time_tile:
 * out[7] = H; local plane 0 is global plane out[0] - H.  The halo schedule of
 * one exchange of `planes` (0..H) planes: ranks send their `planes` owned
 * planes next to each neighbour and receive the same number into the ghost
 * planes adjacent to their owned range.  Error DOMAIN if a rank would own < H. */
sdag_status sdag_slab_partition2(int64_t global_nz, int32_t rz, int32_t time_tile, int32_t nranks, int32_t rank,
                                 int64_t out[8]);
sdag_status sdag_slab_halo2(int64_t global_nz, int32_t rz, int32_t time_tile, int32_t nranks, int32_t rank,
                            int32_t planes, int64_t out[5]);

/* NCCL bootstrap through the same libnccl.so.2 torch loads (dlopen).
 * unique id: 128 bytes, broadcast by the caller (e.g. torch.distributed). */
sdag_status sdag_nccl_get_unique_id(uint8_t id[128]);
sdag_status sdag_nccl_comm_create(const uint8_t id[128], int32_t nranks, int32_t rank, int32_t device,
                                  void **comm);
void sdag_nccl_comm_destroy(void *comm);
/* Diagnostic: one NCCL group { ncclSend(send -> peer), ncclRecv(recv <- peer) }
 * of `count` doubles on `stream`, through the same grouped call the z-slab halo
 * exchange makes (error handling included).  `peer` may be this rank (a 1-rank
 * communicator sends to itself), which lets a single GPU exercise the exact
 * NCCL entry points, datatype and counts the exchange uses.  Device buffers,
 * caller-owned; enqueued asynchronously. */
sdag_status sdag_nccl_sendrecv(void *comm, int32_t peer, const double *send, double *recv, int64_t count,
                               void *stream);

/* SURVEY 8(b)'s form: this rank's slab from a LOCAL plan of its owned planes
 * (dims = nz_own, ny, nx), every rank owning nz_own planes (weak scaling:
 * global nz = nz_own * nranks).  The plan must come from sdag_plan_create (its
 * spec text and options are reused; the dist plans its own local layout with
 * ghost planes, sdag_dist_layout); the caller keeps ownership of `local`.
 * time_tile as opts.time_tile.  UNSUPPORTED for program stages. */
sdag_status sdag_dist_create_local(sdag_plan local, int32_t rank, int32_t nranks, void *nccl_comm, int32_t time_tile,
                                   sdag_dist *out);
/* Create this rank's slab of a `global_dims` problem.  `nccl_comm` is an
 * ncclComm_t from sdag_nccl_comm_create (or NULL when nranks == 1). */
sdag_status sdag_dist_create(const char *spec, const int64_t global_dims[3], const sdag_plan_opts *opts,
                             int32_t rank, int32_t nranks, void *nccl_comm, sdag_dist *out);
/* local_dims = {nz_alloc, ny, nx}; global_z_of_local0 = global plane index of local plane 0 */
sdag_status sdag_dist_layout(sdag_dist d, int64_t local_dims[3], int64_t *global_z_of_local0);
/* The same, under the name of the SURVEY 8(b) boundary sketch: alloc_dims =
 * {nz_owned + 2H, ny, nx}, *global_z0 = global plane of local plane 0. */
sdag_status sdag_dist_alloc_dims(sdag_dist d, int64_t alloc_dims[3], int64_t *global_z0);
sdag_plan sdag_dist_local_plan(sdag_dist d);

/* One sweep of a slab: exchange the R_z boundary planes of every z-staged
 * input with the neighbours (NCCL send/recv on `comm`, or an internal stream
 * if NULL), compute owned planes that need no ghosts on `compute`
 * concurrently, then the ghost-dependent planes.  1D z-arrays span the local
 * allocation.  Ordered on `compute` on return. */
sdag_status sdag_dist_apply(sdag_dist d, double *const *arrays3d, int32_t n3d, const double *const *arrays1d,
                            int32_t n1d, const double *scalars, int32_t nscalars, sdag_stream compute,
                            sdag_stream comm);
/* T sweeps, ping-pong (1 in -> 1 out plans), result in buf[T&1].  With
 * opts.time_tile = t > 1 and a fused kernel (opts.fusion), the sweeps are
 * scheduled as fused launches of up to t sweeps (the apply_iterated DP), each
 * preceded by ONE exchange of x R_z planes (x = its sweeps): 1/x of the
 * exchanges; planes next to the ghosts are recomputed redundantly inside the
 * launch.  Bit-identical to the single-GPU sdag_apply_iterated schedule. */
sdag_status sdag_dist_apply_iterated(sdag_dist d, double *buf0, double *buf1, int32_t T, const double *scalars,
                                     int32_t nscalars, sdag_stream compute, sdag_stream comm);
void sdag_dist_destroy(sdag_dist d);
/* One sweep of this rank's slab end to end with HOST buffers (local layout of
 * sdag_dist_layout, ghost planes included: the host holds them, so no
 * exchange is needed): pipelined H2D / sweep / D2H as sdag_apply_host; only
 * the slab's planes of the global interior are computed and copied back (the
 * rest of every output is not written).  Synchronous on `stream`. */
sdag_status sdag_dist_apply_host(sdag_dist d, double *const *host3d, int32_t n3d, const double *const *host1d,
                                 int32_t n1d, const double *scalars, int32_t nscalars, sdag_stream stream,
                                 int64_t *h2d_bytes, int64_t *d2h_bytes);

/* Loopback exchanger (all slabs in one process on one device; halos moved
 * with cudaMemcpyAsync): same index bookkeeping as the NCCL path, for
 * bit-exact single-GPU tests.  dists[r] from sdag_dist_create(..., r, n, NULL). */
sdag_status sdag_dist_apply_iterated_loopback(sdag_dist *dists, int32_t nranks, double *const *buf0,
                                              double *const *buf1, int32_t T, const double *scalars,
                                              int32_t nscalars, sdag_stream stream);

/* Peer-memory halo path for iterated slabs ("B200-native
 * alternative"; NEXT-4).  Instead of an NCCL send/recv step, the sweep kernel
 * that computes a slab's boundary planes stores each of them twice: into its
 * own output and, over NVLink P2P, into the ghost planes of the neighbour that
 * reads them next sweep (store-side fusion, tile by tile).  The ordering is a
 * 32-bit flag word per neighbour in each rank's HBM, written by the neighbour
 * with a system-scope release after its boundary launch and waited on (acquire)
 * by this rank's stream before the launch that reads the ghosts.
 *
 * Usage (every rank, same spec/dims/opts/T; opts.tune = 0 so all ranks derive
 * the same launch schedule):
 *   sdag_dist_create(..., rank, nranks, NULL, &d);   (no NCCL communicator)
 *   sdag_dist_p2p_alloc(d, &buf0, &buf1);
 *   exchange handles: sdag_dist_p2p_handle(d, h) -> all-gather on the host ->
 *   sdag_dist_p2p_attach(d, 0, h_of(rank-1)), sdag_dist_p2p_attach(d, 1, h_of(rank+1))
 *   (or sdag_dist_p2p_attach_local(d, side, peer) for slabs of one process);
 *   fill the OWNED planes of buf0 (local planes [H, H + nz_own) of the layout of
 *   sdag_dist_layout; ghost planes and buf1 need no filling), then
 *   sdag_dist_p2p_apply_iterated(d, T, scalars, n, stream)  -> result in buf[T&1].
 *
 * sdag_dist_p2p_alloc: the library allocates ONE device region holding buf0,
 *   buf1 (each nz_alloc*ny*nx doubles, C order, 4 KiB-aligned) and the flag
 *   words, zero-filled; it is owned by the dist (freed by sdag_dist_destroy).
 *   Repeated calls return the same buffers.
 * sdag_dist_p2p_handle: the cudaIpcMemHandle_t (64 bytes) of that region.
 * sdag_dist_p2p_attach: side 0 = rank-1, 1 = rank+1; opens the neighbour's
 *   handle (another process; cudaIpcOpenMemHandle with lazy peer access).
 *   INVALID_ARG if there is no neighbour on that side or alloc was not called.
 * sdag_dist_p2p_attach_local: same for a neighbour dist of this process
 *   (its region is used directly; peer access is enabled if on another device).
 * sdag_dist_p2p_apply_iterated: T sweeps of a 1-in/1-out plan over buf0/buf1
 *   (fused launches as sdag_dist_apply_iterated), enqueued on `stream` only;
 *   bit-identical to the single-GPU schedule.  The FIRST call after
 *   sdag_dist_p2p_alloc initialises buf1 from buf0 (owned planes locally, ghost
 *   planes from the neighbours' bands), so the boundary ring (the x/y ring of
 *   every plane, the global z-ring planes) is taken from buf0 at that call and
 *   is never written afterwards.  Each call starts from buf0.  Consecutive calls on a rank are
 *   ordered against the neighbours' previous calls by the same flags.  A wait
 *   that does not complete within SDAG_P2P_TIMEOUT_S seconds (default 60)
 *   traps the kernel (the error surfaces at the next synchronisation). */
sdag_status sdag_dist_p2p_alloc(sdag_dist d, double **buf0, double **buf1);
sdag_status sdag_dist_p2p_handle(sdag_dist d, uint8_t handle[64]);
sdag_status sdag_dist_p2p_attach(sdag_dist d, int32_t side, const uint8_t handle[64]);
sdag_status sdag_dist_p2p_attach_local(sdag_dist d, int32_t side, sdag_dist peer);
sdag_status sdag_dist_p2p_apply_iterated(sdag_dist d, int32_t T, const double *scalars, int32_t nscalars,
                                         sdag_stream stream);

/* ------------------------------------------------------------------------
 * Fission (paper Section VI-B): split versions written out as DSL
 * ------------------------------------------------------------------------ */
enum { SDAG_FISSION_MAXFUSE = 0, SDAG_FISSION_TRIVIAL = 1 };
/* From a single-stage spec, the DSL text of a split version, accepted by
 * sdag_program_create with the same arguments (declaration order = the
 * stencil's formal order):
 *   SDAG_FISSION_MAXFUSE: the stencil re-printed from the IR (one stage);
 *   SDAG_FISSION_TRIVIAL: one stencil function per output array with the
 *     statements it needs (temporaries replicated, Fig 3b/3c), called in an
 *     order that preserves every value a statement reads; UNSUPPORTED if no
 *     such order exists.
 * Statements are selected, not rewritten (parenthesised trees, exact
 * literals), so each output is computed by the same operations.  *len = text
 * length (without the NUL); the text is copied into buf when cap > *len, and
 * INVALID_ARG is returned when buf is non-null and too small.  Parse and
 * semantic errors as sdag_plan_create.  Host only. */
sdag_status sdag_spec_fission(const char *spec, int32_t kind, char *buf, int64_t cap, int64_t *len);
/* The reverse direction for a multi-stencil program (Fig 3c form): maxfuse with
 * recomputation -- ONE stencil in which every read of an array an earlier stage
 * wrote is replaced by that stage's expression at the read's offset
 * (temporaries inlined), so intermediates never go through memory.  The fused
 * stencil's radius is the composed one; on its interior every written value is
 * computed by the same operations as in the staged program.  Its formals are
 * the program's declared arguments (declaration order).  keep_intermediates = 0:
 * arrays read by a later stage are not written (only the sinks).  UNSUPPORTED
 * when a written array is also read at an offset before any stage writes it.
 * Buffer convention as sdag_spec_fission.  Host only. */
/* Section VI-B versions of a multi-stencil program, as DSL text
 * with the program's arguments unchanged (declaration order):
 *   SDAG_VERSION_MAXFUSE    all calls fused into one stencil with recomputation
 *                           (intermediates only read inside are not written);
 *   SDAG_VERSION_STAGED     every call its own stencil (the program re-printed);
 *   SDAG_VERSION_RECOMPUTE  recompute-fission: calls grouped in call order, each
 *                           group grown while its recomputation halo stays
 *                           <= max(4, r), r the largest order of its calls
 *                           (P:1538-1544); the group sizes are written to
 *                           sizes[] (capacity n_sizes) if non-null;
 *   SDAG_VERSION_GROUPS     the calls grouped as sizes[0..n_sizes) (sum = number
 *                           of calls), each group fused.
 * A fused group writes the arrays later groups read and the program's results
 * on ITS composed interior, where every value is computed by the operations of
 * the staged program (reading R24).  Buffer convention as sdag_spec_fission.
 * UNSUPPORTED when a group would read an array it writes at an offset.  Host only. */
enum { SDAG_VERSION_MAXFUSE = 0, SDAG_VERSION_STAGED = 1, SDAG_VERSION_RECOMPUTE = 2, SDAG_VERSION_GROUPS = 3 };
sdag_status sdag_program_version(const char *program, int32_t kind, int32_t *sizes, int32_t n_sizes, char *buf,
                                 int64_t cap, int64_t *len);
/* The fusion forest: every partition of the calls into contiguous
 * groups whose recomputation halo is <= max(4, r) and which recompute at most 4
 * RAW intermediates -- the staged program first, maxfuse last when allowed.
 * Candidate c has n_groups[c] groups of sizes sizes[c * 16 + g].  At most
 * max_candidates are returned (*n_candidates); programs of > 16 calls are
 * UNSUPPORTED.  Host only. */
sdag_status sdag_program_forest(const char *program, int32_t max_candidates, int32_t *n_groups, int32_t *sizes,
                                int32_t *n_candidates);
/* The measured pick among the forest's candidates (ARTEMIS's tuning of the
 * fission versions): each candidate is planned (opts as
 * sdag_program_create) and timed on the caller's arrays (device pointers,
 * program argument order; outputs are overwritten) with CUDA events, median of
 * 5 runs after 2 warm-ups; ms[c] receives candidate c's time (capacity
 * max_candidates) and *best the fastest.  Synchronous. */
sdag_status sdag_program_forest_tune(const char *program, const int64_t dims[3], const sdag_plan_opts *opts,
                                     void *const *arrays3d, int32_t n3d, const double *const *arrays1d,
                                     int32_t n1d, const double *scalars, int32_t nscalars, sdag_stream stream,
                                     int32_t max_candidates, double *ms, int32_t *n_candidates, int32_t *best);
sdag_status sdag_program_fuse(const char *program, int32_t keep_intermediates, char *buf, int64_t cap,
                              int64_t *len);

/* ------------------------------------------------------------------------
 * Profile-guided classification (paper Section IV)
 * ------------------------------------------------------------------------ */
enum { SDAG_BOUND_DRAM = 0, SDAG_BOUND_COMPUTE = 1, SDAG_BOUND_LATENCY = 2 };
typedef struct {
    char variant[96];          /* the plan's kernel */
    double ms;                 /* median of 7 timed launches on the caller's arrays */
    double flops, bytes;       /* canonical flops, algorithmic bytes of one apply (R9, R10) */
    double oi_dram, ridge;     /* flops/bytes; peak_fp64 / peak_hbm (flop/B) */
    double peak_hbm_gbs, peak_fp64_tflops;  /* as passed, or measured (copy, DFMA) when 0 */
    double frac_dram, frac_fp64;            /* roofline time of each level / ms */
    double ms_diff_mem, ms_diff_arith;      /* code-differenced twins, 0 if none */
    int32_t regs, spill_bytes, ctas_per_sm, warps_per_sm;
    int32_t bound;             /* SDAG_BOUND_* */
    char hints[1024];          /* Section IV-A guidelines applied to this plan, '\n'-separated */
} sdag_profile;
/* Runs the plan's kernel on the caller's arrays (same arguments as sdag_apply;
 * the outputs are overwritten several times) and classifies it.  Synchronous
 * on `stream`.  peak_* <= 0: measured here (a 1 GiB device copy, the DFMA
 * micro-benchmark).  Errors as sdag_apply. */
sdag_status sdag_plan_profile(sdag_plan plan, void *const *arrays3d, int32_t n3d, const double *const *arrays1d,
                              int32_t n1d, const double *scalars, int32_t nscalars, double peak_hbm_gbs,
                              double peak_fp64_tflops, sdag_stream stream, sdag_profile *out);

/* ------------------------------------------------------------------------
 * Diagnostics
 * ------------------------------------------------------------------------ */
const char *sdag_last_error(void); /* thread-local; valid until the next sdag_* call on this thread */
const char *sdag_version(void);
/* Number of sweep-kernel launches this process has enqueued (all plans). */
int64_t sdag_launch_count(void);
/* FP64 peak micro-benchmark (dependent-chain-free DFMA over all SMs) on the
 * current device; returns achieved FLOP/s in *flops (synchronous). */
sdag_status sdag_measure_fp64_peak(double *flops, sdag_stream stream);

/* Registered DAGs with hand-written sm_100a bodies: name and canonical spec
 * text (a spec whose canonical form equals one of these, up to renaming, is
 * accepted by sdag_plan_create).  Strings live for the process. */
int32_t sdag_registry_count(void);
sdag_status sdag_registry_get(int32_t idx, const char **name, const char **text);

#ifdef __cplusplus
}
#endif
#endif /* SDAG_H */
