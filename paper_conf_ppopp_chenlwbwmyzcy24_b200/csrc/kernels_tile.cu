// kernels_tile.cu — engine TC_TILE: the B200 variant of ConvStencil's stencil-as-GEMM.
//
// Same contraction as the paper's dual tessellation (8 output groups x 8 outputs x K taps on
// DMMA.8x8x4, P.900-959), but laid out for sm_100a:
//   * the 8 N columns of one DMMA hold an a x b block of outputs (4x2 for nk = 3, 7; 2x4 for
//     nk = 5) instead of 1 x (nk+1).  K = the block's (a+nk-1) x kc input region (kc = b+nk-1
//     rounded up to 4) — 24 / 48 / 80 taps per output block for nk = 3 / 5 / 7 instead of the
//     paper's 2*ceil(nk^2/4)*4 = 24 / 56 / 104, i.e. 23 % fewer DMMAs at nk = 7;
//   * every k-slice is 4 consecutive cells of ONE input row, so the M x K operand tile is a
//     strided view of the raw input tile: no stencil2row scatter, no LUT, and an A fragment
//     loaded for input row rho serves every output block whose window contains rho (register
//     reuse down the column: ~0.5 LDS.64 per DMMA instead of 1);
//   * the input tile is staged by cp.async.bulk (TMA bulk copies, one per row) into a
//     double-buffered smem ring with mbarrier completion, so the next tile streams in while the
//     DMMA pipe works on the current one (persistent CTAs, 2 per SM).
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

__device__ __forceinline__ void dmma_t(double& c0, double& c1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(c0), "+d"(c1)
      : "d"(a), "d"(b));
}

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}

// Compile-time geometry of one TC_TILE instantiation.
template <int NK_, int A_, int B_, int KC_, int G_, int WM_, int WN_, int STAGES_>
struct TileCfg {
  static constexpr int NK = NK_, A = A_, B = B_, KC = KC_, G = G_, WM = WM_, WN = WN_;
  static constexpr int STAGES = STAGES_;
  static constexpr int R = (NK - 1) / 2;
  static constexpr int ODD = R & 1;                 // smem col = region col + ODD (16-B aligned rows)
  static constexpr int KR = A + NK - 1;             // input rows per output block
  static constexpr int KS = KR * KC / 4;            // k-slices (DMMAs) per output block
  static constexpr int BM = WM * A * G;             // CTA output rows
  static constexpr int BN = WN * 8 * B;             // CTA output cols
  static constexpr int RR = BM + NK - 1;            // staged input rows
  static constexpr int TP = ((ODD + BN + KC - B) + 1) / 2 * 2;  // staged row length (even)
  static constexpr int STAGE = RR * TP;             // doubles per stage
  static constexpr int NCW = WM * WN;               // consumer (DMMA) warps
  static constexpr int NT = 32 * (NCW + 1);         // + one producer warp
  static constexpr int SMEM = STAGES * STAGE * 8;
};

template <class C>
__device__ __forceinline__ void issue_tile(const S2RArgs& a, int64_t tile, double* stage,
                                           uint64_t* bar, int lane) {
  const int ty = (int)(tile / a.tiles_x);
  const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
  const double* src = a.src.p + (int64_t)(ty * C::BM - C::R) * a.src.s1 + (tx * C::BN - C::R - C::ODD);
  if (lane == 0) mbar_expect_tx(bar, (uint32_t)(C::STAGE * 8));
  __syncwarp();
  for (int r = lane; r < C::RR; r += 32)
    bulk_g2s(stage + r * C::TP, src + (int64_t)r * a.src.s1, (uint32_t)(C::TP * 8), bar);
}

template <class C>
__device__ __forceinline__ bool tile_is_edge(const S2RArgs& a, int ty, int tx) {
  if (a.fix_band <= 0) return false;
  const int64_t gy0 = (int64_t)ty * C::BM + a.gorg1, gx0 = (int64_t)tx * C::BN + a.gorg2;
  return gy0 < a.fix_band || gy0 + C::BM > a.GE1 - a.fix_band || gx0 < a.fix_band ||
         gx0 + C::BN > a.GE2 - a.fix_band;
}

// Warp-specialised persistent kernel: warp NCW is the producer (bulk copies of the input tile
// into a STAGES-deep smem ring, full/empty mbarriers); warps 0..NCW-1 run the DMMA GEMM.
template <class C>
__global__ void __launch_bounds__(C::NT, 1) k_tile2d(S2RArgs a) {
  extern __shared__ __align__(128) double smem[];
  __shared__ __align__(8) uint64_t full[C::STAGES], empty[C::STAGES];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], C::NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == C::NCW) {
    // ---------------- producer ----------------
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % C::STAGES;
      const int n = it / C::STAGES;
      if (n > 0) mbar_wait(&empty[s], (n - 1) & 1);
      issue_tile<C>(a, tile, smem + s * C::STAGE, &full[s], lane);
    }
    return;
  }
  // ---------------- consumers ----------------
  const int wm = warp / C::WN, wn = warp - (warp / C::WN) * C::WN;
  const int g = lane >> 2, t = lane & 3;
  double wf[C::KS];
#pragma unroll
  for (int s = 0; s < C::KS; ++s) wf[s] = a.frags[s * 32 + lane];
  // output (alpha, beta) of this lane's two accumulator columns n = 2t, 2t+1
  const int alpha = (2 * t) / C::B, beta = (2 * t) % C::B;
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    const int s = it % C::STAGES;
    mbar_wait(&full[s], (it / C::STAGES) & 1);
    const int ty = (int)(tile / a.tiles_x);
    const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
    const double* base = smem + s * C::STAGE + (wm * C::A * C::G) * C::TP + wn * 8 * C::B + C::ODD +
                         C::B * g + t;
    double acc[C::G][2];
#pragma unroll
    for (int j = 0; j < C::G; ++j) acc[j][0] = acc[j][1] = 0.0;
    // Stream the warp's input rows; each A fragment (4 cells of one row) feeds every output
    // block whose window contains the row.  Consecutive DMMAs go to different accumulators.
#pragma unroll
    for (int ra = 0; ra < C::A * C::G + C::NK - 1; ++ra) {
      double f[C::KC / 4];
#pragma unroll
      for (int h = 0; h < C::KC / 4; ++h) f[h] = base[ra * C::TP + 4 * h];
#pragma unroll
      for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
        for (int j = 0; j < C::G; ++j) {
          const int rho = ra - C::A * j;
          if (rho >= 0 && rho < C::KR) dmma_t(acc[j][0], acc[j][1], f[h], wf[rho * (C::KC / 4) + h]);
        }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);  // this warp no longer reads stage s
    // FIXED: band outputs of an edge tile are written by k_band (kernels_band.cu)
    const bool edge = tile_is_edge<C>(a, ty, tx);
    // store: block j covers output rows ty*BM + wm*A*G + A*j + [0, A), cols tx*BN + wn*8B + B*g + [0, B)
    const int64_t col = (int64_t)tx * C::BN + wn * 8 * C::B + C::B * g + beta;
    const int64_t row0 = (int64_t)ty * C::BM + wm * C::A * C::G + alpha;
    const int64_t gcol = col + a.gorg2;
    const bool col_band = edge && (gcol < a.fix_band || gcol + 1 >= a.GE2 - a.fix_band);
#pragma unroll
    for (int j = 0; j < C::G; ++j) {
      const int64_t row = row0 + C::A * j;
      const int64_t grow = row + a.gorg1;
      if (edge && (col_band || grow < a.fix_band || grow >= a.GE1 - a.fix_band)) {
        // band points were written by band_fix; only a pair straddling the band edge keeps
        // its non-band half
        if (!(col_band && !(grow < a.fix_band || grow >= a.GE1 - a.fix_band))) continue;
        if (row >= a.E1) continue;
        double* p = a.dst.p + row * a.dst.s1 + col;
        if (gcol >= a.fix_band && gcol < a.GE2 - a.fix_band && col < a.E2) p[0] = acc[j][0];
        if (gcol + 1 >= a.fix_band && gcol + 1 < a.GE2 - a.fix_band && col + 1 < a.E2) p[1] = acc[j][1];
        continue;
      }
      if (row < a.E1 && col < a.E2) {
        double* p = a.dst.p + row * a.dst.s1 + col;
        if (col + 1 < a.E2 && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
          *reinterpret_cast<double2*>(p) = make_double2(acc[j][0], acc[j][1]);
        } else {
          p[0] = acc[j][0];
          if (col + 1 < a.E2) p[1] = acc[j][1];
        }
      }
    }
  }
}

// nk -> (a, b, kc); G blocks per warp column, WM x WN consumer warps, STAGES-deep ring.
// Variant 0: 12 DMMA warps, 3 stages (CTA 96 x 64).  Variant 1: 16 DMMA warps, 2 stages
// (CTA 128 x 64).  CSX_TILE_VARIANT selects (default 0).
using Tile3 = TileCfg<3, 4, 2, 4, 8, 3, 4, 3>;
using Tile5 = TileCfg<5, 2, 4, 8, 8, 6, 2, 3>;
using Tile7 = TileCfg<7, 4, 2, 8, 8, 3, 4, 3>;
using Tile3b = TileCfg<3, 4, 2, 4, 8, 4, 4, 2>;
using Tile5b = TileCfg<5, 2, 4, 8, 8, 8, 2, 2>;
using Tile7b = TileCfg<7, 4, 2, 8, 8, 4, 4, 2>;

static int tile_variant() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("CSX_TILE_VARIANT");
    v = e ? atoi(e) : 0;
  }
  return v;
}

// ------------------------------------------------------------------------------------------
// 3D (Tf = 1, P.1788-1800): out[z] = sum_dz Conv2D(in[z + dz - R], W[dz]).  The producer warp
// streams the input planes of a (y, x) tile and a z chunk through a STAGES-deep plane ring; the
// DMMA warps compute output plane zo from the NK staged planes zo-R .. zo+R (every tensor-core z
// offset is a K-slice group of the same GEMM; single-tap z offsets — the star arms, reading A9 —
// are DFMAs on the same staged planes), then release plane zo-R, which no later output needs.
template <int NK_, int G_, int WM_, int WN_, int STAGES_, int ZCH_>
struct Tile3DCfg {
  static constexpr int NK = NK_, A = 4, B = 2, KC = 4 * ((2 + NK - 1 + 3) / 4), G = G_, WM = WM_,
                       WN = WN_, STAGES = STAGES_, ZCH = ZCH_;
  static constexpr int R = (NK - 1) / 2;
  static constexpr int ODD = R & 1;
  static constexpr int KR = A + NK - 1;
  static constexpr int KS = KR * KC / 4;
  static constexpr int BM = WM * A * G;
  static constexpr int BN = WN * 8 * B;
  static constexpr int RR = BM + NK - 1;
  static constexpr int TP = ((ODD + BN + KC - B) + 1) / 2 * 2;
  static constexpr int STAGE = RR * TP;
  static constexpr int NCW = WM * WN;
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int SMEM = STAGES * STAGE * 8;
  static_assert(STAGES >= NK + 1, "plane ring must hold NK planes plus one in flight");
};

template <class C>
__device__ __forceinline__ void issue_plane(const S2RArgs& a, int ty, int tx, int64_t zi, double* stage,
                                            uint64_t* bar, int lane) {
  const double* src = a.src.p + zi * a.src.s0 + (int64_t)(ty * C::BM - C::R) * a.src.s1 +
                      (tx * C::BN - C::R - C::ODD);
  if (lane == 0) mbar_expect_tx(bar, (uint32_t)(C::STAGE * 8));
  __syncwarp();
  for (int r = lane; r < C::RR; r += 32)
    bulk_g2s(stage + r * C::TP, src + (int64_t)r * a.src.s1, (uint32_t)(C::TP * 8), bar);
}

template <class C>
__global__ void __launch_bounds__(C::NT, 2) k_tile3d(S2RArgs a, int tc_mask) {
  extern __shared__ __align__(128) double smem[];
  __shared__ __align__(8) uint64_t full[C::STAGES], empty[C::STAGES];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], C::NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  const int64_t ncol = (int64_t)a.tiles_x * a.tiles_y;
  if (warp == C::NCW) {  // producer: planes of every work item, in consumption order
    int64_t q = 0;
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int64_t zc = item / ncol, tile = item - zc * ncol;
      const int ty = (int)(tile / a.tiles_x), tx = (int)(tile - (int64_t)ty * a.tiles_x);
      const int64_t z0 = zc * C::ZCH, z1 = min(a.E0, z0 + C::ZCH);
      for (int64_t zi = z0 - C::R; zi < z1 + C::R; ++zi, ++q) {
        const int s = (int)(q % C::STAGES);
        const int64_t n = q / C::STAGES;
        if (n > 0) mbar_wait(&empty[s], (uint32_t)((n - 1) & 1));
        issue_plane<C>(a, ty, tx, zi, smem + s * C::STAGE, &full[s], lane);
      }
    }
    return;
  }
  const int wm = warp / C::WN, wn = warp - (warp / C::WN) * C::WN;
  const int g = lane >> 2, t = lane & 3;
  double wf[C::NK][C::KS];
  double wz[C::NK];
#pragma unroll
  for (int p = 0; p < C::NK; ++p) {
#pragma unroll
    for (int s = 0; s < C::KS; ++s) wf[p][s] = a.frags[(p * C::KS + s) * 32 + lane];
    wz[p] = a.wc[(p * C::NK + C::R) * C::NK + C::R];
  }
  const int alpha = (2 * t) / C::B, beta = (2 * t) % C::B;
  const bool any_cuda = tc_mask != (1 << C::NK) - 1;
  int64_t q0 = 0;  // plane sequence number of the current item's first plane
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int64_t zc = item / ncol, tile = item - zc * ncol;
    const int ty = (int)(tile / a.tiles_x), tx = (int)(tile - (int64_t)ty * a.tiles_x);
    const int64_t z0 = zc * C::ZCH, z1 = min(a.E0, z0 + C::ZCH);
    const int64_t col = (int64_t)tx * C::BN + wn * 8 * C::B + C::B * g + beta;
    const int64_t row0 = (int64_t)ty * C::BM + wm * C::A * C::G + alpha;
    // planes z0-R .. z0+R-1 are needed before the first output plane
    for (int k = 0; k < 2 * C::R; ++k) {
      const int64_t qq = q0 + k;
      mbar_wait(&full[qq % C::STAGES], (uint32_t)((qq / C::STAGES) & 1));
    }
    for (int64_t zo = z0; zo < z1; ++zo) {
      const int64_t qn = q0 + (zo - z0) + 2 * C::R;  // newest plane zo + R
      mbar_wait(&full[qn % C::STAGES], (uint32_t)((qn / C::STAGES) & 1));
      double acc[C::G][2];
#pragma unroll
      for (int j = 0; j < C::G; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
      for (int dz = 0; dz < C::NK; ++dz) {
        const int64_t qp = q0 + (zo - z0) + dz;  // plane zo - R + dz
        const double* stg = smem + (qp % C::STAGES) * C::STAGE;
        if (tc_mask & (1 << dz)) {
          const double* base = stg + (wm * C::A * C::G) * C::TP + wn * 8 * C::B + C::ODD + C::B * g + t;
#pragma unroll
          for (int ra = 0; ra < C::A * C::G + C::NK - 1; ++ra) {
            double f[C::KC / 4];
#pragma unroll
            for (int h = 0; h < C::KC / 4; ++h) f[h] = base[ra * C::TP + 4 * h];
#pragma unroll
            for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
              for (int j = 0; j < C::G; ++j) {
                const int rho = ra - C::A * j;
                if (rho >= 0 && rho < C::KR)
                  dmma_t(acc[j][0], acc[j][1], f[h], wf[dz][rho * (C::KC / 4) + h]);
              }
          }
        } else if (any_cuda && wz[dz] != 0.0) {
#pragma unroll
          for (int j = 0; j < C::G; ++j) {
            const int lr = wm * C::A * C::G + C::A * j + alpha + C::R;
            const int lc = wn * 8 * C::B + C::B * g + beta + C::R + C::ODD;
            const double2 v = *reinterpret_cast<const double2*>(stg + lr * C::TP + lc);
            acc[j][0] = fma(wz[dz], v.x, acc[j][0]);
            acc[j][1] = fma(wz[dz], v.y, acc[j][1]);
          }
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[(q0 + (zo - z0)) % C::STAGES]);  // plane zo-R is done
      double* plane = a.dst.p + zo * a.dst.s0;
#pragma unroll
      for (int j = 0; j < C::G; ++j) {
        const int64_t row = row0 + C::A * j;
        if (row < a.E1 && col < a.E2) {
          double* p = plane + row * a.dst.s1 + col;
          if (col + 1 < a.E2 && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
            *reinterpret_cast<double2*>(p) = make_double2(acc[j][0], acc[j][1]);
          } else {
            p[0] = acc[j][0];
            if (col + 1 < a.E2) p[1] = acc[j][1];
          }
        }
      }
    }
    // release the last 2R planes of the item (not released by an output plane)
    __syncwarp();
    if (lane == 0)
      for (int k = 0; k < 2 * C::R; ++k) mbar_arrive(&empty[(q0 + (z1 - z0) + k) % C::STAGES]);
    q0 += (z1 - z0) + 2 * C::R;
  }
}

using Tile3D3 = Tile3DCfg<3, 8, 2, 2, 4, 32>;  // CTA 64 x 32 outputs, 4-plane ring, 32 planes per item


bool tile_kernel_exists(int ndim, int nk) {
  return (ndim == 2 && (nk == 3 || nk == 5 || nk == 7)) || (ndim == 3 && nk == 3);
}

template <class C>
static cudaError_t launch_tile_cfg(S2RArgs a, cudaStream_t st) {
  a.tiles_x = (int)((a.E2 + C::BN - 1) / C::BN);
  a.tiles_y = (int)((a.E1 + C::BM - 1) / C::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y;
  cudaError_t e = cudaFuncSetAttribute(k_tile2d<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile2d<C>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  int64_t grid = (int64_t)(occ < 1 ? 1 : occ) * num_sms();
  if (grid > a.ntiles) grid = a.ntiles;
  k_tile2d<C><<<(unsigned)grid, C::NT, C::SMEM, st>>>(a);
  return cudaGetLastError();
}

template <class C>
static cudaError_t launch_tile3d_cfg(S2RArgs a, int tc_mask, cudaStream_t st) {
  a.tiles_x = (int)((a.E2 + C::BN - 1) / C::BN);
  a.tiles_y = (int)((a.E1 + C::BM - 1) / C::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y * ((a.E0 + C::ZCH - 1) / C::ZCH);
  cudaError_t e = cudaFuncSetAttribute(k_tile3d<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile3d<C>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  int64_t grid = (int64_t)(occ < 1 ? 1 : occ) * num_sms();
  if (grid > a.ntiles) grid = a.ntiles;
  k_tile3d<C><<<(unsigned)grid, C::NT, C::SMEM, st>>>(a, tc_mask);
  return cudaGetLastError();
}

cudaError_t launch_tile(int ndim, int nk, const S2RArgs& a, cudaStream_t st) {
  if (ndim == 3) {
    if (nk == 3) return launch_tile3d_cfg<Tile3D3>(a, a.tc_mask, st);
    return cudaErrorNotSupported;
  }
  if (ndim != 2) return cudaErrorNotSupported;
  const int v = tile_variant();
  switch (nk) {
    case 3: return v ? launch_tile_cfg<Tile3b>(a, st) : launch_tile_cfg<Tile3>(a, st);
    case 5: return v ? launch_tile_cfg<Tile5b>(a, st) : launch_tile_cfg<Tile5>(a, st);
    case 7: return v ? launch_tile_cfg<Tile7b>(a, st) : launch_tile_cfg<Tile7>(a, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
