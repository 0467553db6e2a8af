// kernels_direct2d_wf.cu — the 2D CUDA-core comparator (north_star item 2),
// register-wavefront form: the whole temporal block lives in registers, no shared memory.
//
// The question the comparator answers is how far plain FP64 FMA (DFMA) gets on the same chip as
// the tensor-core path.  On B200 DMMA and DFMA share one FP64 datapath (PEAKS_FP64.json "mixed":
// the two pipes' times add), so the answer is decided by how many FP64 operations each method
// issues per point-step and how well it feeds them.  This kernel feeds them from registers:
//
//   * a warp owns a vertical strip of 32 V input columns (V consecutive columns per lane) and
//     marches down a chunk of BH output rows;
//   * every input row is loaded once (16-B loads, coalesced; the row N = 2R+1 ahead is in flight
//     while this one is used) and extended by the 2R halo columns of the neighbouring lanes with
//     warp shuffles;
//   * level l (l = 1..TF, the fused time steps) keeps an N-row rolling window of level l-1 rows
//     in registers and produces its row i - lR as soon as level l-1 row i - (l-1)R exists: TF
//     time steps per input row, one global read and one global write per point per pass;
//   * each level loses R columns at each strip edge, so strips overlap by 2 R TF columns (the
//     overlap is read twice, mostly from L2); chunks overlap by R TF rows at each end;
//   * the row loop is unrolled by N so every window slot is a compile-time register;
//   * FIXED: points within R of a global face keep their value at every level (edge items only).
//
// Inputs come from the plan's padded grid (ghost cells of depth >= R TF and >= 128 slack rows /
// 160 slack columns), so no load is guarded; stores are guarded to the grid.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

struct WFWeights {
  double w[49];
};

template <int R, int TF, int V>
struct WFCfg {
  static constexpr int N = 2 * R + 1;
  static constexpr int H = R * TF;
  static constexpr int SH = H & 1;                    // shift so strip starts are 16-B aligned
  static constexpr int W = 32 * V;                    // input columns per strip
  static constexpr int S = (W - 2 * H - SH) & ~1;     // output columns per strip (even)
  static constexpr int E = V + 2 * R;                 // extended row per lane
  static constexpr int NT = 128;                      // 4 independent warps per CTA
  static constexpr int P = 8;                         // input rows in flight per warp (smem ring)
  static constexpr int SMEM = (NT / 32) * P * 32 * V * 8;
  static_assert(S > 0, "strip narrower than its halo");
};

__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(
                   static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int K>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;\n" ::"n"(K) : "memory");
}

// WF_EXTEND(o, lvl, s): slot s of level lvl's window <- the E-wide extended row of this lane from
// its V values o[]: the halo columns come from the lanes that own them (left: lane - ceil((R-k)/V),
// right: lane + ceil((k+1)/V)) by shuffles.  (A macro writing win[][][] in place: binding a
// reference to a slot of the register array let the compiler reorder the writes of a later
// unrolled row ahead of the reads of an earlier one.)
template <int R, int V>
__device__ __forceinline__ void wf_extend(const double* o, double* e) {
#pragma unroll
  for (int q = 0; q < V; ++q) e[R + q] = o[q];
#pragma unroll
  for (int k = 0; k < R; ++k) {
    const int rel = k - R;
    const int dl = (rel - (V - 1)) / V;  // floor(rel / V), rel < 0
    e[k] = __shfl_up_sync(0xffffffffu, o[rel - dl * V], -dl);
    const int dr = (V + k) / V;
    e[R + V + k] = __shfl_down_sync(0xffffffffu, o[V + k - dr * V], dr);
  }
}

template <int R, int TF, int V, int UNR, bool STAR, bool EDGE>
__device__ __forceinline__ void wf_item(const DirectArgs& a, const WFWeights& Wt, double* ring, int64_t r0,
                                        int64_t r1, int64_t x0, int64_t xs0, int64_t xs1, int lane) {
  using C = WFCfg<R, TF, V>;
  constexpr int N = C::N, E = C::E, P = C::P;
  const double* src = a.src.p + x0 + lane * V;
  const int64_t rin0 = r0 - C::H;
  const int64_t nin = (r1 - r0) + 2 * C::H;
  // per-lane column facts: store mask, FIXED column hold
  bool cst[V], chold[V];
#pragma unroll
  for (int q = 0; q < V; ++q) {
    const int64_t x = x0 + lane * V + q;
    cst[q] = x >= xs0 && x < xs1;
    const int64_t gx = x + a.gorg[2];
    chold[q] = EDGE && (gx < R || gx >= a.GE[2] - R);
  }
  const bool vec_ok = cst[0] && (V == 1 || cst[V - 1]);
  // input rows stream through a P-row ring in this warp's shared memory (cp.async, one group per
  // row): the loads are in flight P - 1 rows ahead without holding registers
  double* my = ring + lane * V;
#pragma unroll
  for (int p = 0; p < P - 1; ++p) {
    const double* rp = src + (rin0 + p) * a.src.s1;
#pragma unroll
    for (int q = 0; q < V; q += 2) cp_async16(my + p * 32 * V + q, rp + q);
    cp_async_commit();
  }
  // win[l][k]: the N newest rows of level l (k = N-1 newest), extended by the 2R halo columns
  // (zero-initialised: the rows read before the window fills only feed outputs that are never
  // stored, but reading an uninitialised register array lets the optimiser fold the loop-carried
  // window rotation into the newest row — it did, and the kernel returned shifted rows)
  double win[TF][N][E];
#pragma unroll
  for (int l = 0; l < TF; ++l)
#pragma unroll
    for (int k = 0; k < N; ++k)
#pragma unroll
      for (int c = 0; c < E; ++c) win[l][k][c] = 0.0;
#pragma unroll UNR
  for (int64_t i = 0; i < nin; ++i) {
    // row i + P - 1 into the slot row i - 1 used; then wait for row i
    {
      const double* rp = src + (rin0 + i + P - 1) * a.src.s1;
      double* d = my + (int)((i + P - 1) % P) * 32 * V;
#pragma unroll
      for (int q = 0; q < V; q += 2) cp_async16(d + q, rp + q);
      cp_async_commit();
    }
    cp_async_wait<P - 1>();
    double lv[V];
    {
      const double* sp = my + (int)(i % P) * 32 * V;
#pragma unroll
      for (int q = 0; q < V; q += 2) {
        const double2 v = *reinterpret_cast<const double2*>(sp + q);
        lv[q] = v.x;
        lv[q + 1] = v.y;
      }
    }
    double ext[E];
    wf_extend<R, V>(lv, ext);
#pragma unroll
    for (int k = 0; k < N - 1; ++k)
#pragma unroll
      for (int c = 0; c < E; ++c) win[0][k][c] = win[0][k + 1][c];
#pragma unroll
    for (int c = 0; c < E; ++c) win[0][N - 1][c] = ext[c];
#ifdef WF_DEBUG
    if (lane == 1 && r0 == 0 && x0 < 0 && i < 6)
      printf("i=%d lv0=%g ring=%d win0=[%g %g %g]\n", (int)i, lv[0], (int)(i % P), win[0][0][R], win[0][1][R], win[0][N - 1][R]);
#endif
    // level l computes its row i - l R from level l-1 rows i - (l+1) R .. i - (l-1) R: level l-1's
    // window before its newest row is pushed at this step for l >= 2 holds rows up to i - (l-1)R
#pragma unroll
    for (int l = 1; l <= TF; ++l) {
      double o[V];
#pragma unroll
      for (int q = 0; q < V; ++q) {
        double v0 = 0.0, v1 = 0.0;
#pragma unroll
        for (int k = 0; k < N; ++k)
#pragma unroll
          for (int b = 0; b < N; ++b) {
            if (STAR && k != R && b != R) continue;  // star footprint: axial taps only
            const double xv = win[l - 1][k][q + b];
            if ((k * N + b) & 1) v1 = fma(Wt.w[k * N + b], xv, v1);
            else v0 = fma(Wt.w[k * N + b], xv, v0);
          }
        o[q] = v0 + v1;
      }
      const int64_t y = rin0 + i - l * R;  // row of this level's output
      if (EDGE) {
        const int64_t gy = y + a.gorg[1];
        const bool rh = gy < R || gy >= a.GE[1] - R;
#pragma unroll
        for (int q = 0; q < V; ++q)
          if (rh || chold[q]) o[q] = win[l - 1][R][R + q];
      }
      if (l < TF) {
        double ex[E];
        wf_extend<R, V>(o, ex);
#pragma unroll
        for (int k = 0; k < N - 1; ++k)
#pragma unroll
          for (int c = 0; c < E; ++c) win[l][k][c] = win[l][k + 1][c];
#pragma unroll
        for (int c = 0; c < E; ++c) win[l][N - 1][c] = ex[c];
      } else if (y >= r0 && y < r1) {
        double* dp = a.dst.p + y * a.dst.s1 + x0 + lane * V;
        if (vec_ok && ((reinterpret_cast<uintptr_t>(dp) & 15) == 0)) {
#pragma unroll
          for (int q = 0; q < V; q += 2) *reinterpret_cast<double2*>(dp + q) = make_double2(o[q], o[q + 1]);
        } else {
#pragma unroll
          for (int q = 0; q < V; ++q)
            if (cst[q]) dp[q] = o[q];
        }
      }
    }
  }
  cp_async_wait<0>();
  __syncwarp();
}

template <int R, int TF, int V, int BH, int UNR, bool STAR>
__global__ void __launch_bounds__(128) k_direct2d_wf(DirectArgs a, WFWeights Wt) {
  using C = WFCfg<R, TF, V>;
  extern __shared__ __align__(16) double wf_smem[];
  const int lane = threadIdx.x & 31;
  double* ring = wf_smem + (threadIdx.x >> 5) * C::P * 32 * V;
  const int64_t gw = ((int64_t)blockIdx.x * C::NT + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * C::NT) >> 5;
  const int64_t nstrips = (a.E[2] + C::S - 1) / C::S;
  const int64_t nchunks = (a.E[1] + BH - 1) / BH;
  const int64_t nitems = nstrips * nchunks;
  for (int64_t item = gw; item < nitems; item += nwarps) {
    const int64_t chunk = item / nstrips, j = item - chunk * nstrips;
    const int64_t r0 = chunk * BH, r1 = min(r0 + BH, a.E[1]);
    const int64_t xs0 = j * C::S, xs1 = min(xs0 + C::S, a.E[2]);
    const int64_t x0 = xs0 - C::H - C::SH;
    bool edge = false;
    if (a.fixed_bc) {
      const int64_t gy0 = r0 - C::H + a.gorg[1], gy1 = r1 + C::H + a.gorg[1];
      const int64_t gx0 = x0 + a.gorg[2], gx1 = x0 + C::W + a.gorg[2];
      edge = gy0 < R || gy1 > a.GE[1] - R || gx0 < R || gx1 > a.GE[2] - R;
    }
    if (edge) wf_item<R, TF, V, UNR, STAR, true>(a, Wt, ring, r0, r1, x0, xs0, xs1, lane);
    else wf_item<R, TF, V, UNR, STAR, false>(a, Wt, ring, r0, r1, x0, xs0, xs1, lane);
  }
}

template <int R, int TF, int V, int UNR, bool STAR>
static cudaError_t launch_wf_s(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  using C = WFCfg<R, TF, V>;
  constexpr int BH = 256;
  // the row loop reads up to 2N rows past the chunk's last halo row and the strip's columns
  // [x0, x0 + 32 V): both inside the padded allocation (planner.cpp layout_padded slack)
  if (a.src.s1 % 2 != 0 || (reinterpret_cast<uintptr_t>(a.src.p) & 15) != 0) return cudaErrorNotSupported;
  WFWeights W;
  const int n = 2 * R + 1;
  for (int i = 0; i < 49; ++i) W.w[i] = i < n * n ? w_host[i] : 0.0;
  int occ = 0;
  cudaError_t e = cudaFuncSetAttribute(k_direct2d_wf<R, TF, V, BH, UNR, STAR>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct2d_wf<R, TF, V, BH, UNR, STAR>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t items = ((a.E[2] + C::S - 1) / C::S) * ((a.E[1] + BH - 1) / BH);
  const int64_t grid = persistent_grid(occ, a.max_ctas, (items + 3) / 4);
  if (grid < 1) return cudaSuccess;
  k_direct2d_wf<R, TF, V, BH, UNR, STAR><<<(unsigned)grid, C::NT, C::SMEM, st>>>(a, W);
  return cudaGetLastError();
}

// star weights (every off-axis tap zero): the kernel skips those taps at compile time
static bool wf_star(int r, const double* w) {
  const int n = 2 * r + 1;
  for (int k = 0; k < n; ++k)
    for (int b = 0; b < n; ++b)
      if (k != r && b != r && w[k * n + b] != 0.0) return false;
  return true;
}

template <int R, int TF, int V, int UNR = 1>
static cudaError_t launch_wf(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  return wf_star(R, w_host) ? launch_wf_s<R, TF, V, UNR, true>(a, w_host, st)
                            : launch_wf_s<R, TF, V, UNR, false>(a, w_host, st);
}

static int wf_v() {
  static const int v = [] {
    const char* e = getenv("CSX_DIRECT2D_V");
    return e ? atoi(e) : 2;
  }();
  return v;
}

// row-loop unroll (CSX_DIRECT2D_UNR = 1: the window rotation is register moves; 0 (default):
// unrolled by N = 2R + 1, so the rotation becomes register renaming)
static int wf_unr() {
  static const int v = [] {
    const char* e = getenv("CSX_DIRECT2D_UNR");
    return e ? atoi(e) : 0;
  }();
  return v;
}

// Where the register window is larger than the shared-memory kernels' working set (box r = 2,
// Tf = 2: 2 x 5 x 6 doubles per lane; box r = 3: 7 x 8, spilling) those kernels measured faster
// (240 vs 223, 151 vs 139 GSt/s on B200) and keep the case; star weights skip most taps here.
// (r = 3, Tf = 2 spills outright; V = 4 only up to Tf = 2)
bool direct2d_wf_exists(int r, int tf, const double* w) {
  const bool star = wf_star(r, w);
  return (r == 1 && tf >= 1 && tf <= 4) || (r == 2 && tf == 1) || (r == 2 && tf == 2 && star) ||
         (r == 3 && tf == 1 && star);
}

cudaError_t launch_direct2d_wf(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  const bool v4 = wf_v() == 4 && a.tf <= 2;
  const bool u1 = wf_unr() == 1;
  if (a.r == 1) {
    switch (a.tf) {
      case 1: return v4 ? launch_wf<1, 1, 4, 3>(a, w_host, st) : u1 ? launch_wf<1, 1, 2, 1>(a, w_host, st) : launch_wf<1, 1, 2, 3>(a, w_host, st);
      case 2: return v4 ? launch_wf<1, 2, 4, 3>(a, w_host, st) : u1 ? launch_wf<1, 2, 2, 1>(a, w_host, st) : launch_wf<1, 2, 2, 3>(a, w_host, st);
      case 3: return u1 ? launch_wf<1, 3, 2, 1>(a, w_host, st) : launch_wf<1, 3, 2, 3>(a, w_host, st);
      case 4: return u1 ? launch_wf<1, 4, 2, 1>(a, w_host, st) : launch_wf<1, 4, 2, 3>(a, w_host, st);
    }
  } else if (a.r == 2 && a.tf == 1) {
    return u1 ? launch_wf<2, 1, 2, 1>(a, w_host, st) : launch_wf<2, 1, 2, 5>(a, w_host, st);
  } else if (a.r == 2 && a.tf == 2) {
    return launch_wf<2, 2, 2, 1>(a, w_host, st);
  } else if (a.r == 3 && a.tf == 1) {
    return u1 ? launch_wf<3, 1, 2, 1>(a, w_host, st) : launch_wf<3, 1, 2, 7>(a, w_host, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
