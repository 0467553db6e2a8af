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
  int64_t grid = (int64_t)(occ < 1 ? 1 : occ) * num_sms();
  if (grid > b.ntiles) grid = b.ntiles;
  k_direct2d<R, TF><<<(unsigned)grid, C::NT, C::SMEM, st>>>(b, W);
  return cudaGetLastError();
}

bool direct2d_exists(int r, int tf) {
  return (r == 1 && tf >= 1 && tf <= 4) || (r == 2 && tf <= 2) || (r == 3 && tf <= 1);
}

// The base weights travel by value as kernel parameters (constant-bank DFMA operands).
cudaError_t launch_direct2d(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  if (a.r == 1) {
    switch (a.tf) {
      case 1: return launch_d2<1, 1>(a, w_host, st);
      case 2: return launch_d2<1, 2>(a, w_host, st);
      case 3: return launch_d2<1, 3>(a, w_host, st);
      case 4: return launch_d2<1, 4>(a, w_host, st);
    }
  } else if (a.r == 2) {
    switch (a.tf) {
      case 1: return launch_d2<2, 1>(a, w_host, st);
      case 2: return launch_d2<2, 2>(a, w_host, st);
    }
  } else if (a.r == 3 && a.tf == 1) {
    return launch_d2<3, 1>(a, w_host, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
