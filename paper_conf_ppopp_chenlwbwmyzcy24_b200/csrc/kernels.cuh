// kernels.cuh — device-side argument blocks and launcher declarations (product code).
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

namespace csx {

// A grid view: pointer at the interior origin plus strides of axes 0 and 1 (axis 2 stride 1).
struct View {
  double* p;
  int64_t s0, s1;
};
struct CView {
  const double* p;
  int64_t s0, s1;
  // allocation geometry of a padded grid (for TMA tensor maps): interior origin inside the
  // allocation and the number of allocated planes (rows = s0 / s1, row pitch = s1).
  // n0 == 0: unknown (kernels fall back to per-row bulk copies).
  int64_t o0 = 0, o1 = 0, o2 = 0, n0 = 0;
};

struct S2RArgs {
  CView src;            // padded source (halo >= r*Tf readable around the interior)
  View dst;             // destination (padded scratch or the user's dense d_out)
  int64_t E0, E1, E2;   // interior extents (normalised, E0 slowest)
  int tiles_x, tiles_y; // CTA tiles over (E2, E1) [2D: rows E1, cols E2]
  int64_t ntiles;
  const int2* lut;      // per region element {source offset, a | b << 16}
  const double* frags;  // per-lane B fragments
  const double* wc;     // composed weights (3D CUDA-core planes)
  // TC_TILE fused FIXED band fix-up (0 = none): edge CTAs recompute the points within
  // fix_band = r*Tf of a GLOBAL face by Tf plain steps on CUDA cores from the staged tile.
  int tc_mask = 0;                // 3D: bit dz set = z offset dz runs on tensor cores
  // slab-axis tile subset (sharded overlap): part 0 = all, 1 = interior (no ghost reads),
  // 2 = edge (the first / last slab tiles, whose halo reaches the exchanged ghost rows)
  int part = 0;
  int max_ctas = 0;               // cap on the persistent grid (0 = all SMs)
  int dst_aligned = 0;            // dst rows are 16-B aligned (unguarded double2 stores)
  int64_t ra0 = 0, ra1 = 0, rb0 = 0, rb1 = 0;  // slab-tile ranges, filled by the launcher
  int s2r_variant = 3;            // TC_S2R 2D: bit 0 padding, bit 1 dirty bits (breakdown)
  int fix_band = 0;
  int pdl = 1;                    // TC_TILE: launch with programmatic dependent launch
  int hold_frame = 0;             // write held (frame) values from the staged tile (Tf = 1)
  int use_tma = 0;                // TC_TILE 2D/3D: stage tiles with one TMA tensor copy
  int l2hint = 0;                 // TMA loads' L2 eviction priority: 0 normal, 1 last, 2 first
  int64_t tma_x0 = 0, tma_y0 = 0, tma_z0 = 0;  // interior origin in tensor-map coordinates
  int lockstep = 0;               // 3D experiment: producers sync grid-wide every k planes
  int r = 0;
  const double* wbase = nullptr;  // base weights (2r+1)^2
  int64_t gorg0 = 0, gorg1 = 0, gorg2 = 0;  // local origin in global coordinates
  int64_t GE0 = 0, GE1 = 0, GE2 = 0;        // global extents
};

struct DirectArgs {
  CView src;
  View dst;
  int64_t E[3];         // local interior extents
  int64_t gorg[3];      // local origin in global coordinates (slab offset; 0 single-GPU)
  int64_t GE[3];        // global extents (FIXED frame and band are global)
  int real[3];          // 1 if the axis is a real (stencil) axis
  int r, tf, fixed_bc;
  int band;             // 0: write every point; >0: write only points within `band` of a face
  int B[3];             // tile extents (outputs)
  int tiles[3];
  int64_t ntiles;
  const int32_t* tile_list;  // band mode: linear tile ids; nullptr = all tiles
  const int64_t* tile_org;   // band strips: explicit tile origins (3 per tile), or nullptr
  const double* w;      // base weights (2r+1)^ndim dense
  int ndim;
  int max_ctas = 0;     // cap on the persistent grid (0 = all SMs; csx_plan_set_max_ctas)
};

// NVLink peer-memory halo push (kernels_peer.cu)
struct PeerPushArgs {
  const double* src_first = nullptr;  // this rank's first h slab rows (full padded rows)
  const double* src_last = nullptr;   // this rank's last h slab rows
  double* dst_up = nullptr;           // up neighbour's bottom ghost rows (peer memory) or null
  double* dst_down = nullptr;         // down neighbour's top ghost rows (peer memory) or null
  int64_t n = 0;                      // doubles per side
  int vec2 = 0;                       // all four pointers 16-B aligned
  const unsigned long long* freed_up = nullptr;    // local: up has finished reading ghosts
  const unsigned long long* freed_down = nullptr;  // local: down has finished reading ghosts
  unsigned long long wait_v = 0;
  unsigned long long* ready_up_remote = nullptr;    // up's READY_BOTTOM
  unsigned long long* ready_down_remote = nullptr;  // down's READY_TOP
  unsigned long long* freed_up_remote = nullptr;    // up's FREED_BY_DOWN
  unsigned long long* freed_down_remote = nullptr;  // down's FREED_BY_UP
  unsigned long long ready_v = 0, freed_v = 0;      // 0 = do not publish
  unsigned int* counter = nullptr;                  // local last-CTA counter
};
cudaError_t launch_peer_push(const PeerPushArgs& a, cudaStream_t st);
cudaError_t launch_peer_wait(const unsigned long long* ready_top, const unsigned long long* ready_bottom,
                             unsigned long long v, cudaStream_t st);

// launchers (return cudaError_t of the launch)
cudaError_t launch_pack(const double* in, View dst, const int64_t* E, cudaStream_t st);
cudaError_t launch_ghost_fill(View buf, const int64_t* E, const int* real, const int* fill, int H,
                              cudaStream_t st);
cudaError_t launch_s2r(int ndim, int nk, int nf, const S2RArgs& a, int tc_mask, cudaStream_t st);
// TC_TILE pass of `tf` fused steps of a base radius `radius` stencil (nk = 2 radius tf + 1)
cudaError_t launch_tile(int ndim, int radius, int tf, const S2RArgs& a, cudaStream_t st);
cudaError_t launch_direct(const DirectArgs& a, cudaStream_t st);
// 2D comparator kernel (kernels_direct2d.cu): compile-time (r, Tf), weights by value.
bool direct2d_exists(int r, int tf);
// register-wavefront 2D comparator (kernels_direct2d_wf.cu): R = 1 (Tf <= 4), 2 (Tf <= 2), 3 (Tf = 1)
bool direct2d_wf_exists(int r, int tf, const double* w_host);
cudaError_t launch_direct2d_wf(const DirectArgs& a, const double* w_host, cudaStream_t st);
cudaError_t launch_direct2d(const DirectArgs& a, const double* w_host, cudaStream_t st);
// 1D / 3D comparator kernels (kernels_direct13.cu): compile-time r, weights by value.
bool direct1d_exists(int r, int tf);
cudaError_t launch_direct1d(const DirectArgs& a, const double* w_host, cudaStream_t st);
bool direct3d_exists(int r, int tf);
cudaError_t launch_direct3d(const DirectArgs& a, const double* w_host, cudaStream_t st);
// FIXED band fix-up after a fused pass of Tf > 1 steps (kernels_band.cu), 1D and 2D.
cudaError_t launch_band(int ndim, int r, int tf, CView src, View dst, const int64_t* E,
                        const int64_t* gorg, const int64_t* GE, const double* w_host,
                        cudaStream_t st, int* launched);
// FIXED frame (points within r of a GLOBAL face) copied src -> dst: the whole fix-up of a
// Tf = 1 pass, whose composed window is the plain stencil (no band beyond the frame).
cudaError_t launch_frame_copy(CView src, View dst, const int64_t* E, const int64_t* gorg,
                              const int64_t* GE, const int* real, int r, cudaStream_t st);
int s2r_smem_bytes(int ndim, int nk, int nf);
// Breakdown variant I (kernels_s2r_explicit.cu): explicit stencil2row A/B in global memory
// (scratch of s2r_explicit_elems doubles) + dual tessellation on CUDA cores.  2D only.
int64_t s2r_explicit_elems(int nk, int64_t E1, int64_t E2);
cudaError_t launch_s2r_explicit(int nk, CView src, View dst, const int64_t* E, const double* wc,
                                double* scratch, cudaStream_t st);
int num_sms();
// persistent grid size: occupancy x SMs, capped by max_ctas (> 0) and by the work items
int64_t persistent_grid(int occ, int max_ctas, int64_t items);

}  // namespace csx
