/* csx.h — C-ABI of the B200-native ConvStencil hot path (libcsx.so).
 *
 * The operation: explicit FP64 stencil time stepping (PAPER.md P.146-149 §1, P.277-287 §2.1):
 *     u_{t+1}[p] = sum_{o in {-r..r}^d} w[o] * u_t[p + o]
 * computed as matrix multiplication on FP64 tensor cores (DMMA.8x8x4) by ConvStencil's
 * stencil2row layout (Eq 5/6, P.731-785), dual tessellation (P.900-959, P.1304-1336), lookup
 * table + dirty-bits padding (P.1711-1773) and kernel fusion (P.1466-1482).
 *
 * Conventions shared by every entry point
 *   - extents[0] is the SLOWEST axis (C / torch order); grids are dense row-major float64.
 *   - weights: dense (2r+1)^ndim doubles, row-major over offsets -r..r on every axis; entry
 *     [i0][i1]... multiplies u[p0 + i0 - r][p1 + i1 - r]... (correlation; the output sits at the
 *     window centre — Fig 3 and P.1326-1330; readings A2/A3).  STAR shapes must have
 *     zeros off the axes.
 *   - Boundary (paper silent, reading A1): CSX_BC_FIXED holds every point within r of
 *     a face at its initial value; CSX_BC_PERIODIC wraps.
 *   - timesteps count BASE steps (Eq 16's T, reading A5).
 *   - All device pointers are plain CUDA device pointers on the current device; the caller
 *     owns them.  Streams are cudaStream_t passed as void* (NULL = legacy default stream).
 *
 * Errors: every function returns csx_status.  Argument checks are synchronous
 * (CSX_ERR_INVALID_ARGUMENT / CSX_ERR_UNSUPPORTED); launch failures return CSX_ERR_CUDA with
 * detail in csx_last_error() (thread-local); asynchronous device faults surface at the
 * caller's next synchronisation.  No function falls back to the CPU.
 */
#ifndef CSX_H_
#define CSX_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  CSX_OK = 0,
  CSX_ERR_INVALID_ARGUMENT = 1,
  CSX_ERR_UNSUPPORTED = 2,
  CSX_ERR_OUT_OF_MEMORY = 3,
  CSX_ERR_CUDA = 4,
  CSX_ERR_NCCL = 5,
  CSX_ERR_INTERNAL = 6
} csx_status;

/* Stencil shapes, P.277-287: star = axial neighbours only, box = full (2r+1)^d cube. */
typedef enum { CSX_SHAPE_STAR = 0, CSX_SHAPE_BOX = 1 } csx_shape;

typedef enum { CSX_BC_FIXED = 0, CSX_BC_PERIODIC = 1 } csx_boundary;

/* Which engine runs the fused passes.
 *   TC_S2R : the paper's design — implicit stencil2row in shared memory through the lookup
 *            table with dirty-bits padding, dual tessellation 8 x (nk+1) per DMMA chain.
 *   TC_TILE: B200 variant of the same stencil-as-GEMM on DMMA: 4x2 output blocks per MMA
 *            column group, A fragments read straight from the staged input tile.
 *   DIRECT : CUDA-core direct weighted sum with temporal blocking (the comparator, N2).
 *   AUTO   : TC_TILE where supported, else TC_S2R. */
typedef enum {
  CSX_ENGINE_AUTO = 0,
  CSX_ENGINE_TC_S2R = 1,
  CSX_ENGINE_TC_TILE = 2,
  CSX_ENGINE_DIRECT = 3
} csx_engine;

typedef struct csx_plan_s* csx_plan_t;
typedef struct csx_comm_s* csx_comm_t;

/* Build a plan (host-only work: fusion depth, composed weights W^(Tf) (P.1466-1482), weight
 * matrices W_A/W_B (P.961-975), the lookup table (P.1711-1721) and tile geometry).  Device
 * buffers (weight fragments, LUT, two padded ping-pong grids) are allocated and uploaded at
 * the first csx_run on the then-current device.
 *   ndim 1..3; extents[ndim] >= 2*r*Tf+1 each; radius 1..3; fuse_steps 0 = automatic
 *   (composed window nk = 2*r*Tf+1: 1D nk <= 31 (TC_S2R: <= 15), 2D nk <= 13 (TC_S2R: <= 7),
 *   3D Tf = 1)
 *   (DESIGN.md "Fusion depth"), else Tf >= 1.  *out receives the plan (caller frees with
 *   csx_plan_destroy).  Errors: INVALID_ARGUMENT (null pointers, bad ndim/radius/extents,
 *   off-axis star weights, non-finite weights), UNSUPPORTED (a combination no engine covers). */
csx_status csx_plan(int ndim, const int64_t* extents, csx_shape shape, int radius,
                    const double* weights, csx_boundary bc, int fuse_steps, csx_plan_t* out);

/* The fusion depth csx_plan picks for fuse_steps = 0 (reading A4), for a plan that
 * will run on `engine` (AUTO = the depth csx_plan itself uses; TC_S2R 1D keeps the paper's
 * nk + 1 <= 16).  Returns Tf >= 1, or 0 for ndim / radius / engine out of range.  Host-only. */
int csx_auto_fuse_steps(int ndim, int radius, csx_engine engine);

/* Select the engine for subsequent runs (default AUTO).  UNSUPPORTED if the engine cannot run
 * this plan's (ndim, radius, Tf). */
csx_status csx_plan_set_engine(csx_plan_t plan, csx_engine engine);

/* CUDA-graph replay of csx_run (default off).  With on != 0, csx_run captures the pass sequence
 * of a (d_in, d_out, timesteps) triple into a CUDA graph (after running it eagerly once) and
 * replays later calls with the same triple as one cudaGraphLaunch on the caller's stream; a
 * different triple re-captures.  Same results as eager runs; the plan must not be used on two
 * streams at once (as for eager runs).  Ignored while csx_profile_enable is active.  Errors:
 * INVALID_ARGUMENT (NULL plan); capture / instantiate failures surface as CUDA from csx_run. */
csx_status csx_plan_set_graph(csx_plan_t plan, int on);

/* Cap the persistent grids of every kernel the plan launches (TC_TILE, TC_S2R, DIRECT) at
 * max_ctas CTAs (0 = the default: occupancy x SMs).  Results do not depend on it; it exists so
 * that tests can drive each persistent CTA around its shared-memory ring many times on small
 * grids (slot reuse, mbarrier phase flips, empty-slot waits), and for tuning.  Invalidates a
 * captured graph.  Errors: INVALID_ARGUMENT (NULL plan, max_ctas < 0). */
csx_status csx_plan_set_max_ctas(csx_plan_t plan, int max_ctas);

/* TC_S2R breakdown variants (Fig 6, P.1865-1950), 2D only: padding = 0 uses the bare
 * stencil2row pitch nk*rr (Fig 5's conflicting 266) instead of the conflict-free one (268);
 * dirty_bits = 0 replaces the dirty-bits padding by conditional stores in the LUT copy loop.
 * (1, 1) is the paper's full design (the default); (0, 0) = variant III, (1, 0) = IV;
 * padding = 2 selects variant II (same tiles, the tessellation GEMM on CUDA cores / DFMA);
 * padding = 3 selects variant I (explicit stencil2row: A and B materialised in global memory
 * by an Eq 5/6 div/mod transform kernel, then the tessellation on CUDA cores reading them back;
 * the plan allocates ~2 nk/(nk+1) x the grid of scratch at the first run).
 * INVALID_ARGUMENT for padding outside 0..3; UNSUPPORTED for non-default variants in 1D/3D. */
csx_status csx_plan_set_s2r_variant(csx_plan_t plan, int padding, int dirty_bits);

/* Advance d_in by `timesteps` base steps into d_out (both prod(extents) doubles, device,
 * 8-byte aligned; d_in == d_out allowed, any other overlap is INVALID_ARGUMENT; d_in is never
 * written).  Enqueues floor(T/Tf) fused passes plus a remainder pass on `stream` with no host
 * synchronisation; T == 0 copies.  The plan owns one set of scratch buffers, so a plan must not
 * be run on two streams concurrently. */
csx_status csx_run(csx_plan_t plan, const double* d_in, double* d_out, int64_t timesteps,
                   void* stream);

/* Same as csx_run, but d_in / d_out are HOST buffers (pageable or pinned): copies in, runs,
 * copies out, synchronises `stream` before returning.  The end-to-end call used by bench.py's
 * e2e leg.  With pinned, non-overlapping buffers and a grid of >= 8 (T + 1) r rows and >= 16M
 * points, the call pipelines up to 8 ghost-zone chunks of its slowest axis (each chunk's rows plus (T + 1) r
 * ghost rows per side, advanced by a sub-plan of the same stencil; the H2D copy of the next
 * chunk, the run of this one and the D2H copy of the previous one overlap on three streams);
 * results equal the whole-grid run up to rounding order.  Otherwise (pageable or overlapping
 * buffers, short grids, CSX_HOST_CHUNKS=0) one copy in, one run, one copy out.  The plan owns
 * the chunk sub-plans and two device slots, freed by csx_plan_destroy.  h_in is never written. */
csx_status csx_run_host(csx_plan_t plan, const double* h_in, double* h_out, int64_t timesteps,
                        void* stream);

/* What the last csx_run_host on this plan did: chunks run (1 = serial path, 0 = none yet) and
 * the bytes it copied host -> device (ghost rows included) and device -> host. */
csx_status csx_host_last(const csx_plan_t plan, int* chunks, int64_t* h2d_bytes, int64_t* d2h_bytes);

/* Multi-GPU (one process per GPU).  nccl_unique_id points to an ncclUniqueId
 * (NCCL_UNIQUE_ID_BYTES = 128 bytes) created by rank 0 and broadcast by the caller. */
csx_status csx_comm_create(const void* nccl_unique_id, int rank, int nranks, csx_comm_t* out);
csx_status csx_comm_destroy(csx_comm_t comm);

/* ncclGetUniqueId into out128 (128 bytes), for rank 0 to broadcast. */
csx_status csx_nccl_unique_id(void* out128);

/* Rows [lo, hi) of the slowest axis owned by `rank`: lo = floor(rank*N0/nranks). */
csx_status csx_shard_rows(const csx_plan_t plan, int rank, int nranks, int64_t* lo, int64_t* hi);

/* The halo-exchange schedule csx_run_sharded posts before every pass (host logic, no GPU).
 * Writes up to 4 ops of 4 int64 each into ops: {kind (0 send, 1 recv), peer rank, first slab
 * row (local interior index; negative = top ghost rows, >= local rows = bottom ghost rows),
 * number of rows (= r*Tf)} in posting order (send down, recv up, send up, recv down), and
 * their count into *nops.  PERIODIC closes the ring; FIXED end ranks skip the missing side. */
csx_status csx_halo_schedule(const csx_plan_t plan, int rank, int nranks, int64_t* ops, int* nops);

/* Slab-sharded run: the plan describes the GLOBAL grid; d_in_local / d_out_local hold this
 * rank's rows [lo, hi) (csx_shard_rows) x the other extents.  Halos of depth r*Tf are exchanged
 * with NCCL send/recv every pass (ring for PERIODIC).  Every rank must call with equal plan
 * parameters and T.  UNSUPPORTED if a rank owns fewer than r*Tf rows. */
csx_status csx_run_sharded(csx_plan_t plan, csx_comm_t comm, const double* d_in_local,
                           double* d_out_local, int64_t timesteps, void* stream);

/* ----- Pencil (block) decomposition (not in the paper) -------------
 * The two slowest stencil axes are split over a p0 x p1 process grid (p0 * p1 = nranks):
 * 3D (z, y) — every rank owns a pencil running the full x extent; 2D (rows, cols) — blocks.
 * rank = i0 * p1 + i1 owns [floor(i0 N_a / p0), floor((i0+1) N_a / p0)) along the first split
 * axis and the same with (i1, p1, N_b) along the second.  Halos of depth r*Tf are exchanged in
 * two phases per pass (second split axis first, packed strided faces; then the first split axis
 * with full padded rows, which carry the corners / edges).  Not overlapped with compute.
 *
 * csx_shard_box: lo[ndim], hi[ndim] of rank's block in the user's axis order.
 * csx_pencil_schedule: up to 8 ops of 5 int64 {phase (0 second split axis, 1 first), kind
 *   (0 send, 1 recv), peer rank, first row along the phase's axis (local index; negative = low
 *   ghosts, >= local extent = high ghosts), rows (= r*Tf)} in posting order; *nops = count.
 * csx_run_sharded_pencil: d_in_local / d_out_local hold rank's block (dense, C order); every
 *   rank calls with equal plan parameters, p0, p1 and T.  INVALID_ARGUMENT if p0*p1 differs
 *   from the communicator size; UNSUPPORTED for ndim = 1 or a block thinner than r*Tf. */
csx_status csx_shard_box(const csx_plan_t plan, int rank, int p0, int p1, int64_t* lo, int64_t* hi);
csx_status csx_pencil_schedule(const csx_plan_t plan, int rank, int p0, int p1, int64_t* ops,
                               int* nops);
csx_status csx_run_sharded_pencil(csx_plan_t plan, csx_comm_t comm, int p0, int p1,
                                  const double* d_in_local, double* d_out_local, int64_t timesteps,
                                  void* stream);

/* ----- Slab halo exchange over NVLink peer memory (no NCCL on the data path) -----------
 * The same slab decomposition and results as csx_run_sharded, but after every pass the
 * boundary slab rows are copied by SM peer stores straight into the neighbours' ghost rows
 * (CUDA IPC mappings of their plan-owned slab buffers over NVLink / NVSwitch), and readiness is
 * signalled by 64-bit epoch flags in peer memory (fence + st.release.sys / ld.acquire.sys).
 * Bootstrap, once per plan, collectively:
 *   1. every rank calls csx_peer_export(plan, rank, nranks, desc) — allocates this rank's slab
 *      buffers and flag block (fixed from then on) and writes CSX_PEER_DESC_BYTES of IPC handles
 *      and geometry into desc;
 *   2. the caller all-gathers the descriptors in rank order (e.g. torch.distributed
 *      all_gather_object) and every rank calls csx_peer_connect(plan, descs) with the
 *      nranks * CSX_PEER_DESC_BYTES array — it maps the up / down neighbours (a rank that is its
 *      own neighbour, 1-rank PERIODIC, uses its own buffers).
 * Then csx_run_sharded_peer(plan, d_in_local, d_out_local, T, stream) on every rank with equal T.
 * Errors: INVALID_ARGUMENT (bad rank, export twice, connect before export, descriptors from a
 * different plan or out of rank order), UNSUPPORTED (fewer than r*Tf rows per rank), CUDA (IPC
 * failures).  Ranks spin on device flags: every rank must make progress (one process per GPU,
 * or time-sliced processes sharing a GPU in tests). */
#define CSX_PEER_DESC_BYTES 512
csx_status csx_peer_export(csx_plan_t plan, int rank, int nranks, void* desc);
csx_status csx_peer_connect(csx_plan_t plan, const void* descs);
csx_status csx_run_sharded_peer(csx_plan_t plan, const double* d_in_local, double* d_out_local,
                                int64_t timesteps, void* stream);

csx_status csx_plan_destroy(csx_plan_t plan);

const char* csx_status_string(csx_status s);
const char* csx_last_error(void);

/* ----- Introspection (host-only, valid without a GPU) --------------------------------- */

typedef struct {
  int ndim;
  int radius;
  int fuse_steps;        /* Tf of the main passes */
  int nk;                /* composed window edge 2*r*Tf + 1 */
  int remainder_steps;   /* reserved (per-run remainder is T mod Tf) */
  int engine;            /* csx_engine actually used by csx_run */
  int tile_m, tile_n;    /* CTA output tile (rows x cols of the two fastest axes) */
  int s2r_pitch;         /* stencil2row smem pitch in doubles (P.1736-1757) */
  int64_t mma_per_pass;  /* DMMA.8x8x4 instructions one main pass executes (Eq 13, A7) */
  double tc_flops_per_point_step;  /* 512 * mma_per_pass / (points * Tf) */
  double useful_flops_per_point_step; /* 2 * nnz(w) */
} csx_plan_info_t;

csx_status csx_plan_info(const csx_plan_t plan, csx_plan_info_t* info);

/* ----- Measurement hooks (bench.py) -----------------------------------------------------
 * csx_profile_enable(plan, n): n = 0 disables; n >= 1 brackets every n-th main-pass TC kernel
 * launch (the dominant kernel) with CUDA events recorded on the launching stream (n = 1: all
 * of them; events between launches defeat programmatic dependent launch, so a period > 1
 * keeps most passes chained), and counts every kernel the library launches.  n < 0 ->
 * CSX_ERR_INVALID_ARGUMENT.  csx_profile_read synchronises on the recorded events and returns
 * the mean timed TC kernel duration x the number of main-pass TC launches (ms; = the summed
 * time when n = 1) and the launch counts since the last reset. */
csx_status csx_profile_enable(csx_plan_t plan, int enable);
csx_status csx_profile_read(csx_plan_t plan, double* tc_kernel_ms, int64_t* tc_launches,
                            int64_t* total_launches, int reset);

/* Composed weights W^(Tf) = w * w * ... (Tf-fold discrete convolution of the offset-indexed
 * arrays), shape (2*r*Tf+1)^ndim; applying w Tf times equals applying W^(Tf) once on a torus
 * (Fig 4, P.1466-1482). */
csx_status csx_compose_weights(int ndim, int radius, const double* weights, int fuse_steps,
                               double* out);

/* The paper's weight matrices (P.961-975, Fig 3) for an nk x nk window w (row-major):
 *   W_A[nk*i + j][c] = w[i][j-c] for j >= c, else 0;  W_B[nk*i + j][c] = w[i][j+nk-c] for j < c.
 * Written as (nk*nk) x (nk+1) row-major arrays.  For 1D pass ndim1 = 1 and an nk-vector. */
csx_status csx_weight_matrices(int nk, int ndim1, const double* w, double* wa, double* wb);

/* Eq 5 / Eq 6: where input element (x, y) of an m x n grid lands in stencil2row matrix A
 * (which = 0) or B (which = 1).  Returns 1 and (*row, *col) if it lands, 0 if the element is
 * not part of that matrix (it is then a "dirty bit", P.1759-1773). */
int csx_stencil2row_index(int nk, int which, int64_t x, int64_t y, int64_t* row, int64_t* col);

/* Shared-memory conflict degree of one FP64 m8n8k4 A-fragment load (two 4x4 requests,
 * P.1736-1757) from a stencil2row tile of pitch `pitch` doubles at column offset `col`:
 * the max number of distinct 8-byte words one 4-byte bank must serve per request. */
int csx_fragment_bank_conflicts(int pitch, int col);

/* Copy the plan's lookup table: per element of the CTA input region (row-major,
 * region_rows x region_cols) the smem offsets in A and B (dirty slots included).  With lut
 * NULL, only *count is returned. */
csx_status csx_plan_lut(const csx_plan_t plan, int32_t* lut_a, int32_t* lut_b, int64_t* count,
                        int* region_rows, int* region_cols);

#ifdef __cplusplus
}
#endif
#endif /* CSX_H_ */
