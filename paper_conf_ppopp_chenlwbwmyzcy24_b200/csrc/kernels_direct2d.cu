// kernels_direct2d.cu — the CUDA-core comparator for 2D (north_star item 2):
// direct weighted sum in FP64 FMA with temporal blocking, register blocking and bulk-copy
// staging.  This is the "how far do CUDA cores get on the same chip" reference that the TC
// engines are compared against (DMMA and DFMA share one FP64 datapath on B200).
//
//   * CTA tile 64 x 64 outputs, TF fused steps in shared memory (ping-pong), halo R*TF;
//   * the input region arrives by cp.async.bulk (one 16-B aligned copy per row);
//   * each thread owns 4 consecutive columns of a row strip and slides a (2R+1) x (4+2R)
//     register window down the strip: per output row it loads one new row of 4+2R values
//     and issues 4 (2R+1)^2 DFMAs whose weights are kernel parameters (constant-bank operands);
//   * FIXED: points within R of a global face are held (copied) at every step.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

struct Direct2DWeights {
  double w[49];
};

template <int R, int TF>
struct D2Cfg {
  static constexpr int BY = 64, BX = 64;
  static constexpr int H = R * TF;
  static constexpr int SH = H & 1;                         // left shift for 16-B aligned rows
  static constexpr int RY = BY + 2 * H;
  static constexpr int RX = BX + 2 * H;
  static constexpr int PX = ((SH + RX + 3) / 4) * 4 + 4;   // smem row pitch (>= SH + RX, 4-aligned)
  static constexpr int NT = 256;
  static constexpr int SMEM = 2 * RY * PX * 8;
};

__device__ __forceinline__ uint32_t d2_smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

template <int R, int TF>
__global__ void __launch_bounds__(256, (R == 1 ? 2 : 1)) k_direct2d(DirectArgs a, Direct2DWeights W) {
  using C = D2Cfg<R, TF>;
  constexpr int N = 2 * R + 1;
  extern __shared__ __align__(128) double sm[];
  __shared__ __align__(8) uint64_t bar;
  double* buf[2] = {sm, sm + C::RY * C::PX};
  const int tid = threadIdx.x;
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(d2_smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  const int tiles_x = (int)((a.E[2] + C::BX - 1) / C::BX);
  uint32_t phase = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x) {
    const int ty = (int)(tile / tiles_x), tx = (int)(tile - (int64_t)ty * tiles_x);
    const int64_t oy = (int64_t)ty * C::BY - C::H, ox = (int64_t)tx * C::BX - C::H - C::SH;
    // stage the region (rows oy .. oy+RY, cols ox .. ox+PX) with bulk copies
    if (tid < 32) {
      if (tid == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(d2_smem_u32(&bar)),
                     "r"((uint32_t)(C::RY * C::PX * 8))
                     : "memory");
      __syncwarp();
      for (int r = tid; r < C::RY; r += 32) {
        const double* src = a.src.p + (oy + r) * a.src.s1 + ox;
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::
                "r"(d2_smem_u32(buf[0] + r * C::PX)),
            "l"(src), "r"((uint32_t)(C::PX * 8)), "r"(d2_smem_u32(&bar))
            : "memory");
      }
    }
    asm volatile(
        "{\n.reg .pred P1;\nWAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n}\n" ::"r"(d2_smem_u32(&bar)),
        "r"(phase)
        : "memory");
    phase ^= 1;
    int cur = 0;
#pragma unroll 1
    for (int s = 1; s <= TF; ++s) {
      const double* in = buf[cur];
      double* out = buf[cur ^ 1];
      // valid output box of this step (region coordinates, before the SH shift)
      const int lo = R * s, hy = C::RY - R * s, hx = C::RX - R * s;
      const int ncg = (hx - lo + 3) / 4;             // 4-column groups
      const int nrows = hy - lo;
      const int nstrips = C::NT / ncg;               // thread rows (strips) per column group
      const int cg = tid % ncg, strip = tid / ncg;
      if (strip < nstrips) {
        const int x0 = lo + 4 * cg;                  // first output column of this thread
        const int rows_per = (nrows + nstrips - 1) / nstrips;
        const int y0 = lo + strip * rows_per, y1 = min(hy, y0 + rows_per);
        if (y0 < y1) {
          const int64_t gx0 = a.gorg[2] + ox + C::SH + x0;  // global column of output x0
          double win[N][4 + 2 * R];
#pragma unroll
          for (int i = 0; i < N - 1; ++i)
#pragma unroll
            for (int j = 0; j < 4 + 2 * R; ++j) win[i + 1][j] = in[(y0 - R + i) * C::PX + C::SH + x0 - R + j];
          for (int y = y0; y < y1; ++y) {
#pragma unroll
            for (int i = 0; i < N - 1; ++i)
#pragma unroll
              for (int j = 0; j < 4 + 2 * R; ++j) win[i][j] = win[i + 1][j];
#pragma unroll
            for (int j = 0; j < 4 + 2 * R; ++j) win[N - 1][j] = in[(y + R) * C::PX + C::SH + x0 - R + j];
            double o[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              double v = 0.0;
#pragma unroll
              for (int i = 0; i < N; ++i)
#pragma unroll
                for (int j = 0; j < N; ++j) v = fma(W.w[i * N + j], win[i][q + j], v);
              o[q] = v;
            }
            if (a.fixed_bc) {
              const int64_t gy = a.gorg[1] + oy + y;
              const bool rowhold = gy < R || gy >= a.GE[1] - R;
#pragma unroll
              for (int q = 0; q < 4; ++q) {
                const int64_t gx = gx0 + q;
                if (rowhold || gx < R || gx >= a.GE[2] - R) o[q] = win[R][q + R];
              }
            }
            double* po = out + y * C::PX + C::SH + x0;
#pragma unroll
            for (int q = 0; q < 4; ++q)
              if (x0 + q < hx) po[q] = o[q];
          }
        }
      }
      __syncthreads();
      cur ^= 1;
    }
    // write the 64 x 64 outputs (region rows/cols H .. H+63)
    const double* fin = buf[cur];
    for (int i = tid; i < C::BY * (C::BX / 2); i += C::NT) {
      const int y = i / (C::BX / 2), x = 2 * (i % (C::BX / 2));
      const int64_t ly = (int64_t)ty * C::BY + y, lx = (int64_t)tx * C::BX + x;
      if (ly >= a.E[1] || lx >= a.E[2]) continue;
      const double* pv = fin + (C::H + y) * C::PX + C::SH + C::H + x;
      double* pd = a.dst.p + ly * a.dst.s1 + lx;
      if (lx + 1 < a.E[2] && ((reinterpret_cast<uintptr_t>(pd) & 15) == 0)) {
        *reinterpret_cast<double2*>(pd) = make_double2(pv[0], pv[1]);
      } else {
        pd[0] = pv[0];
        if (lx + 1 < a.E[2]) pd[1] = pv[1];
      }
    }
    __syncthreads();  // buffers are restaged by the next tile
  }
}

// One thread's vertical strip: outputs (y, x) for y in [y0, y1) from the shared-memory column
// `col` (input (y, x - R + j) at col[y * pitch + j]; plain loads the compiler may schedule); the (2R+1) x (2R+1)
// window slides down the strip with the row loop unrolled by 2R+1 so the rotation is register
// renaming, not moves; each output sums its taps into two partial accumulators (ILP).
template <int R, bool EDGE>
__device__ __forceinline__ void d2_strip(const double* wr, const double* col, int pitch, int y0, int y1,
                                         double* outc, int64_t opitch, int64_t gy_org, int64_t G1,
                                         bool colhold) {
  constexpr int N = 2 * R + 1;
  double win[N][N];
#pragma unroll
  for (int i = 0; i < N - 1; ++i)
#pragma unroll
    for (int j = 0; j < N; ++j) win[i][j] = col[(y0 - R + i) * pitch + j];
  int y = y0;
  for (; y + N <= y1; y += N) {
#pragma unroll
    for (int u = 0; u < N; ++u) {
#pragma unroll
      for (int j = 0; j < N; ++j) win[(u + N - 1) % N][j] = col[(y + u + R) * pitch + j];
      double v0 = 0.0, v1 = 0.0;
#pragma unroll
      for (int i = 0; i < N; ++i)
#pragma unroll
        for (int j = 0; j < N; ++j) {
          if ((i * N + j) & 1) v1 = fma(wr[i * N + j], win[(u + i) % N][j], v1);
          else v0 = fma(wr[i * N + j], win[(u + i) % N][j], v0);
        }
      double v = v0 + v1;
      if (EDGE) {
        const int64_t gy = gy_org + y + u;
        if (colhold || gy < R || gy >= G1 - R) v = win[(u + R) % N][R];
      }
      outc[(int64_t)(y + u) * opitch] = v;
    }
  }
  // tail rows (fewer than N): the window is rotated by moves
  for (; y < y1; ++y) {
#pragma unroll
    for (int j = 0; j < N; ++j) win[N - 1][j] = col[(y + R) * pitch + j];
    double v0 = 0.0, v1 = 0.0;
#pragma unroll
    for (int i = 0; i < N; ++i)
#pragma unroll
      for (int j = 0; j < N; ++j) {
        if ((i * N + j) & 1) v1 = fma(wr[i * N + j], win[i][j], v1);
        else v0 = fma(wr[i * N + j], win[i][j], v0);
      }
    double v = v0 + v1;
    if (EDGE) {
      const int64_t gy = gy_org + y;
      if (colhold || gy < R || gy >= G1 - R) v = win[R][R];
    }
    outc[(int64_t)y * opitch] = v;
#pragma unroll
    for (int i = 0; i < N - 1; ++i)
#pragma unroll
      for (int j = 0; j < N; ++j) win[i][j] = win[i + 1][j];
  }
}

// ------------------------------------------------------------------------------------------
// Warp-specialised variant: a producer warp streams the input regions of successive tiles into a
// 2-stage ring (cp.async.bulk + mbarrier full/empty) so HBM latency overlaps the DFMA work; the
// consumer warps run steps 1..TF-1 into two smem level buffers and the last step straight to
// global memory.  The stage is released as soon as step 1 has read it.
template <int R, int TF>
struct D2WCfg {
  static constexpr int BY = 48, BX = 96 - 2 * R * TF;  // region rows are 96 wide: 3 warps of lanes
  static constexpr int H = R * TF;
  static constexpr int SH = H & 1;
  static constexpr int RY = BY + 2 * H;
  static constexpr int RX = BX + 2 * H;
  static constexpr int PX = ((SH + RX + 3) / 4) * 4 + 4;
  static constexpr int STAGES = 2;
  static constexpr int NCW = 12;                              // 3 warps across x 4 strips
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int LV = TF > 1 ? 2 : 0;                   // smem level buffers
  static constexpr int SMEM = (STAGES + LV) * RY * PX * 8;
};

template <int R, int TF>
__global__ void __launch_bounds__(D2WCfg<R, TF>::NT, 1) k_direct2d_ws(DirectArgs a, Direct2DWeights W) {
  using C = D2WCfg<R, TF>;
  constexpr int N = 2 * R + 1;
  extern __shared__ __align__(128) double sm[];
  __shared__ __align__(8) uint64_t full[C::STAGES], empty[C::STAGES];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;\n" ::"r"(d2_smem_u32(&full[s])));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(d2_smem_u32(&empty[s])), "r"(C::NCW));
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  const int tiles_x = (int)((a.E[2] + C::BX - 1) / C::BX);
  if (warp == C::NCW) {  // producer
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % C::STAGES, n = it / C::STAGES;
      if (n > 0)
        asm volatile(
            "{\n.reg .pred P1;\nWAIT_%=:\n"
            "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
            "@!P1 bra WAIT_%=;\n}\n" ::"r"(d2_smem_u32(&empty[s])),
            "r"((n - 1) & 1)
            : "memory");
      const int ty = (int)(tile / tiles_x), tx = (int)(tile - (int64_t)ty * tiles_x);
      const int64_t oy = (int64_t)ty * C::BY - C::H, ox = (int64_t)tx * C::BX - C::H - C::SH;
      if (lane == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(d2_smem_u32(&full[s])),
                     "r"((uint32_t)(C::RY * C::PX * 8))
                     : "memory");
      __syncwarp();
      for (int r = lane; r < C::RY; r += 32)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::
                "r"(d2_smem_u32(sm + s * C::RY * C::PX + r * C::PX)),
            "l"(a.src.p + (oy + r) * a.src.s1 + ox), "r"((uint32_t)(C::PX * 8)), "r"(d2_smem_u32(&full[s]))
            : "memory");
    }
    return;
  }
  // offsets from the shared array itself (not pointers picked at run time), so the loads and
  // stores below stay LDS / STS instead of generic LD / ST
  const int lvo[2] = {C::STAGES * C::RY * C::PX, (C::STAGES + 1) * C::RY * C::PX};
  double wr[N * N];
#pragma unroll
  for (int i = 0; i < N * N; ++i) wr[i] = W.w[i];
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    const int st = it % C::STAGES;
    asm volatile(
        "{\n.reg .pred P1;\nWAIT_%=:\n"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
        "@!P1 bra WAIT_%=;\n}\n" ::"r"(d2_smem_u32(&full[st])),
        "r"((it / C::STAGES) & 1)
        : "memory");
    const int ty = (int)(tile / tiles_x), tx = (int)(tile - (int64_t)ty * tiles_x);
    const int64_t oy = (int64_t)ty * C::BY - C::H, ox = (int64_t)tx * C::BX - C::H - C::SH;
    int in_off = st * C::RY * C::PX;
    // edge tiles (touching a FIXED global face) check the frame per point; others skip it
    const int64_t gy_min = a.gorg[1] + oy, gy_max = gy_min + C::RY - 1;
    const int64_t gx_min = a.gorg[2] + ox + C::SH, gx_max = gx_min + C::RX - 1;
    const bool edge = a.fixed_bc && (gy_min < R || gy_max >= a.GE[1] - R || gx_min < R ||
                                     gx_max >= a.GE[2] - R);
#pragma unroll 1
    for (int s = 1; s <= TF; ++s) {
      const bool last = s == TF;
      const int out_off = last ? 0 : lvo[(s - 1) & 1];
      // one output column per lane (consecutive lanes -> consecutive addresses: conflict-free
      // LDS), a vertical strip of rows per thread with a (2R+1) x (2R+1) sliding window
      const int lo = R * s, hy = C::RY - R * s, hx = C::RX - R * s;
      const int ncol = hx - lo;                      // <= 96 - 2R
      const int nwc = (ncol + 31) / 32;              // warps across
      const int nws = C::NCW / nwc > 0 ? C::NCW / nwc : 1;  // warp rows (strips)
      const int wc = warp % nwc, wsr = warp / nwc;
      const int x = lo + wc * 32 + lane;
      const int rows_per = (hy - lo + nws - 1) / nws;
      const int y0 = lo + wsr * rows_per, y1 = min(hy, y0 + rows_per);
      if (wsr < nws && x < hx && y0 < y1) {
        const int64_t gx = a.gorg[2] + ox + C::SH + x;
        const bool colhold = gx < R || gx >= a.GE[2] - R;
        const double* col = sm + in_off + C::SH + x - R;
        if (!last) {
          double* oc = sm + out_off + C::SH + x;
          if (edge) d2_strip<R, true>(wr, col, C::PX, y0, y1, oc, C::PX, a.gorg[1] + oy, a.GE[1], colhold);
          else d2_strip<R, false>(wr, col, C::PX, y0, y1, oc, C::PX, 0, 0, false);
        } else {
          const int64_t lx = ox + C::SH + x;
          if (lx < a.E[2]) {
            const int yend = (int)min((int64_t)y1, a.E[1] - oy);  // rows beyond the grid are not stored
            double* oc = a.dst.p + oy * a.dst.s1 + lx;            // row y -> oc[y * s1]
            if (edge) d2_strip<R, true>(wr, col, C::PX, y0, yend, oc, a.dst.s1, a.gorg[1] + oy, a.GE[1], colhold);
            else d2_strip<R, false>(wr, col, C::PX, y0, yend, oc, a.dst.s1, 0, 0, false);
          }
        }
      }
      if (s == 1) {  // every consumer has read the stage
        __syncwarp();
        if (lane == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(d2_smem_u32(&empty[st])) : "memory");
      }
      asm volatile("bar.sync 1, %0;\n" ::"r"(C::NCW * 32) : "memory");
      in_off = out_off;
    }
  }
}

template <int R, int TF>
static cudaError_t launch_d2w(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  using C = D2WCfg<R, TF>;
  Direct2DWeights W;
  const int n = 2 * R + 1;
  for (int i = 0; i < 49; ++i) W.w[i] = i < n * n ? w_host[i] : 0.0;
  DirectArgs b = a;
  b.ntiles = (int64_t)((a.E[1] + C::BY - 1) / C::BY) * ((a.E[2] + C::BX - 1) / C::BX);
  cudaError_t e = cudaFuncSetAttribute(k_direct2d_ws<R, TF>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct2d_ws<R, TF>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, b.ntiles);
  k_direct2d_ws<R, TF><<<(unsigned)grid, C::NT, C::SMEM, st>>>(b, W);
  return cudaGetLastError();
}

template <int R, int TF>
static cudaError_t launch_d2(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  using C = D2Cfg<R, TF>;
  Direct2DWeights W;
  const int n = 2 * R + 1;
  for (int i = 0; i < 49; ++i) W.w[i] = i < n * n ? w_host[i] : 0.0;
  cudaError_t e;
  DirectArgs b = a;
  b.ntiles = (int64_t)((a.E[1] + C::BY - 1) / C::BY) * ((a.E[2] + C::BX - 1) / C::BX);
  e = cudaFuncSetAttribute(k_direct2d<R, TF>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct2d<R, TF>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, b.ntiles);
  k_direct2d<R, TF><<<(unsigned)grid, C::NT, C::SMEM, st>>>(b, W);
  return cudaGetLastError();
}

static int direct_ws() {
  static const int ws = [] {
    const char* e = getenv("CSX_DIRECT_WS");
    return e ? atoi(e) : 1;
  }();
  return ws;
}

// r = 3, Tf = 2 (C3 "multi-step fused", nk = 13) exists only as the warp-specialised kernel:
// with CSX_DIRECT_WS=0 it reports unsupported, so the generic direct kernel runs instead
bool direct2d_exists(int r, int tf) {
  return (r == 1 && tf >= 1 && tf <= 4) || (r == 2 && tf <= 2) || (r == 3 && tf == 1) ||
         (r == 3 && tf == 2 && direct_ws());
}

// which 2D comparator kernel: CSX_DIRECT2D=wf (default: register wavefront, where it exists) or
// smem (the shared-memory temporal-blocking kernels below; CSX_DIRECT_WS picks ws / plain)
static bool use_wf(int r, int tf, const double* w) {
  static const int smem = [] {
    const char* e = getenv("CSX_DIRECT2D");
    return e && e[0] == 's';
  }();
  return !smem && direct2d_wf_exists(r, tf, w);
}

// The base weights travel by value as kernel parameters (constant-bank DFMA operands).
cudaError_t launch_direct2d(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  if (use_wf(a.r, a.tf, w_host)) {
    const cudaError_t e = launch_direct2d_wf(a, w_host, st);
    if (e != cudaErrorNotSupported) return e;
  }
  const int ws = direct_ws();
  if (a.r == 1) {
    switch (a.tf) {
      case 1: return ws ? launch_d2w<1, 1>(a, w_host, st) : launch_d2<1, 1>(a, w_host, st);
      case 2: return ws ? launch_d2w<1, 2>(a, w_host, st) : launch_d2<1, 2>(a, w_host, st);
      case 3: return ws ? launch_d2w<1, 3>(a, w_host, st) : launch_d2<1, 3>(a, w_host, st);
      case 4: return ws ? launch_d2w<1, 4>(a, w_host, st) : launch_d2<1, 4>(a, w_host, st);
    }
  } else if (a.r == 2) {
    switch (a.tf) {
      case 1: return ws ? launch_d2w<2, 1>(a, w_host, st) : launch_d2<2, 1>(a, w_host, st);
      case 2: return ws ? launch_d2w<2, 2>(a, w_host, st) : launch_d2<2, 2>(a, w_host, st);
    }
  } else if (a.r == 3 && a.tf == 1) {
    return ws ? launch_d2w<3, 1>(a, w_host, st) : launch_d2<3, 1>(a, w_host, st);
  } else if (a.r == 3 && a.tf == 2 && ws) {  // C3 "multi-step fused" (nk = 13)
    return launch_d2w<3, 2>(a, w_host, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
