// kernels_s2r.cu — the paper's design on sm_100a DMMA (engine TC_S2R).
//
// Per CTA tile (persistent CTAs, one LUT load per CTA):
//   a4  implicit stencil2row: the input region is read once from HBM (coalesced along rows)
//       and scattered through the lookup table into the stencil2row tiles A and B in shared
//       memory; elements belonging to neither land in the dirty row — no branches
//       (P.787-797, P.1711-1773, Fig 5).
//   a5  dual tessellation: for each output row, acc(8x8) = Tile_A . W_A + Tile_B . W_B as one
//       chain of 2*ceil(K/4) DMMA.8x8x4 (mma.sync m8n8k4 f64), vitrolite B accumulated onto A
//       (P.900-959, P.1332-1336, P.1449-1461).  W_A/W_B fragments live in registers.
//   a6  store: lane (g, t) holds outputs (x, g*(nk+1) + 2t + {0,1}) — the window centre
//       (P.1326-1331): one warp writes 8*(nk+1) contiguous doubles.
//   a8  1D: stencil2row rows of length nk, same dual tessellation, N fragments when nk+1 > 8.
//   a9  3D: sum over z offsets of 2D ConvStencils with per-plane weights; single-tap planes
//       (star arms) on CUDA cores in the same kernel (P.1788-1800).
#include <cuda_runtime.h>

#include <cstdlib>

#include "kernels.cuh"
#include "s2r_geom.h"

namespace csx {

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
      : "+d"(c0), "+d"(c1)
      : "d"(a), "d"(b));
}

// Store the two accumulator values of one lane (columns col, col+1 of one output row).
__device__ __forceinline__ void store_pair(double* row_ptr, int64_t col, int64_t ncols, bool v0,
                                           bool v1, double c0, double c1) {
  double* p = row_ptr + col;
  if (v0 && v1 && col + 1 < ncols && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
    *reinterpret_cast<double2*>(p) = make_double2(c0, c1);
  } else {
    if (v0 && col < ncols) p[0] = c0;
    if (v1 && col + 1 < ncols) p[1] = c1;
  }
}

// ------------------------------------------------------------------------------------------
// 2D.  Persistent CTAs: warp NCW is a producer that streams each tile's raw input region into a
// 2-stage smem ring with cp.async.bulk (mbarrier full/empty); the 8 consumer warps run the
// paper's pipeline per tile: LUT scatter (smem raw -> stencil2row A/B, dirty row absorbs the
// unused elements), then dual tessellation on DMMA, then the centre store.
__device__ __forceinline__ uint32_t s2r_smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void s2r_mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(s2r_smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void s2r_mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred P1;\nWAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n}\n" ::"r"(s2r_smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void s2r_mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(s2r_smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void s2r_issue_rows(const double* src, int64_t pitch, double* dst, int rows,
                                               int tp, uint64_t* bar, int lane) {
  if (lane == 0)
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(s2r_smem_u32(bar)),
                 "r"((uint32_t)(rows * tp * 8))
                 : "memory");
  __syncwarp();
  for (int r = lane; r < rows; r += 32)
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::
            "r"(s2r_smem_u32(dst + r * tp)),
        "l"(src + (int64_t)r * pitch), "r"((uint32_t)(tp * 8)), "r"(s2r_smem_u32(bar))
        : "memory");
}

// FMA = true is breakdown variant II (Fig 6): the same implicit stencil2row tiles, the dual
// tessellation computed on CUDA cores (DFMA) from weight matrices staged in shared memory.
template <int NK, bool PAD, bool DIRTY, bool FMA = false>
__global__ void __launch_bounds__(S2R2D<NK>::NT, 2) k_s2r2d(S2RArgs a) {
  using G = S2R2D<NK, PAD>;
  extern __shared__ __align__(128) double smem[];
  __shared__ double sW[FMA ? 2 * G::KS * 4 * 8 : 1];  // [A|B][k][c] for the FMA variant
  __shared__ __align__(8) uint64_t full[G::RAW_STAGES], empty[G::RAW_STAGES];
  double* raw = smem;                                           // RAW_STAGES x RAW
  double* sAB = raw + G::RAW_STAGES * G::RAW;                   // AB_BUFS x (A | B)
  uint32_t* sL = reinterpret_cast<uint32_t*>(sAB + G::AB_BUFS * G::AB);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr int NC = G::NCW * 32;
  // Zero the tiles once so that the K-padding and pad slots are finite (0 * weight 0 = 0);
  // the LUT packs the A and B offsets of each region element (P.1711-1721).
  for (int i = tid; i < G::AB_BUFS * G::AB; i += G::NT) sAB[i] = 0.0;
  for (int i = tid; i < G::NE; i += G::NT) sL[i] = (uint32_t)a.lut[i].y;
  if (FMA)  // W[k][c] from the per-lane fragments: lane l of slice s holds W[4s + l%4][l/4]
    for (int i = tid; i < 2 * G::KS * 32; i += G::NT) {
      const int m = i / (G::KS * 32), r = i - m * G::KS * 32, k = r / 8, c = r % 8;
      sW[i] = a.frags[(m * G::KS + k / 4) * 32 + (k % 4) + 4 * c];
    }
  if (tid == 0) {
    for (int s = 0; s < G::RAW_STAGES; ++s) {
      s2r_mbar_init(&full[s], 1);
      s2r_mbar_init(&empty[s], G::NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == G::NCW) {  // producer
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % G::RAW_STAGES, n = it / G::RAW_STAGES;
      if (n > 0) s2r_mbar_wait(&empty[s], (n - 1) & 1);
      const int ty = (int)(tile / a.tiles_x);
      const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
      const double* src = a.src.p + (int64_t)(ty * G::BM - G::R) * a.src.s1 + (tx * G::BN - G::R - G::ODD);
      s2r_issue_rows(src, a.src.s1, raw + s * G::RAW, G::RR, G::TPR, &full[s], lane);
    }
    return;
  }
  double wa[G::KS], wb[G::KS];
#pragma unroll
  for (int s = 0; s < G::KS; ++s) {
    wa[s] = a.frags[s * 32 + lane];
    wb[s] = a.frags[(G::KS + s) * 32 + lane];
  }
  const int g = lane >> 2, t = lane & 3;
  const bool v0 = 2 * t < G::SW, v1 = 2 * t + 1 < G::SW;
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    const int s = it % G::RAW_STAGES;
    const int ty = (int)(tile / a.tiles_x);
    const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
    s2r_mbar_wait(&full[s], (it / G::RAW_STAGES) & 1);
    // A/B buffer of this tile: last read by tile it-2's tessellation, which every warp finished
    // before it passed tile it-1's "A/B complete" barrier — no barrier needed here
    double* sA = sAB + (it % G::AB_BUFS) * G::AB;
    double* sB = sA + (G::STRIPS + 1) * G::PITCH;
    // implicit stencil2row: scatter the staged region through the LUT (branch-free)
    const double* rs = raw + s * G::RAW + G::ODD;
    for (int x = warp; x < G::RR; x += G::NCW) {
      const double* rrow = rs + x * G::TPR;
      const uint32_t* lrow = sL + x * G::RC;
      for (int y = lane; y < G::RC; y += 32) {
        const double v = rrow[y];
        const uint32_t l = lrow[y];
        if (DIRTY) {  // dirty bits absorb the unused elements: no branch (P.1759-1773)
          sA[l & 0xffffu] = v;
          sB[l >> 16] = v;
        } else {      // breakdown variants III/IV: conditional stores
          if ((l & 0xffffu) != 0xffffu) sA[l & 0xffffu] = v;
          if ((l >> 16) != 0xffffu) sB[l >> 16] = v;
        }
      }
    }
    __syncwarp();
    if (lane == 0) s2r_mbar_arrive(&empty[s]);  // raw stage consumed
    asm volatile("bar.sync 1, %0;\n" ::"r"(NC) : "memory");  // A/B complete
    const int64_t col = (int64_t)tx * G::BN + g * G::SW + 2 * t;
    // the warp's BM/NCW = 4 output rows as 4 independent accumulation chains (vitrolite B
    // accumulated onto A, P.1332-1336)
    constexpr int RW = G::BM / G::NCW;
    const int xr0 = warp * RW;
    const double* pa = sA + g * G::PITCH + G::NKV * xr0 + t;
    const double* pb = sB + g * G::PITCH + G::NKV * xr0 + t;
    double c[RW][2];
#pragma unroll
    for (int q = 0; q < RW; ++q) c[q][0] = c[q][1] = 0.0;
    if (!FMA) {
#pragma unroll
      for (int s2 = 0; s2 < G::KS; ++s2)
#pragma unroll
        for (int q = 0; q < RW; ++q) dmma(c[q][0], c[q][1], pa[4 * s2 + q * G::NKV], wa[s2]);
#pragma unroll
      for (int s2 = 0; s2 < G::KS; ++s2)
#pragma unroll
        for (int q = 0; q < RW; ++q) dmma(c[q][0], c[q][1], pb[4 * s2 + q * G::NKV], wb[s2]);
    } else {
      // lane (g, t) owns C[g][2t], C[g][2t+1]: sum over k of tile[g][k] * W[k][c]
      const double* qa = sA + g * G::PITCH + G::NKV * xr0;
      const double* qb = sB + g * G::PITCH + G::NKV * xr0;
#pragma unroll 4
      for (int k = 0; k < G::NKV * G::NKV; ++k) {
        const double2 wA = *reinterpret_cast<const double2*>(&sW[k * 8 + 2 * t]);
        const double2 wB = *reinterpret_cast<const double2*>(&sW[G::KS * 32 + k * 8 + 2 * t]);
#pragma unroll
        for (int q = 0; q < RW; ++q) {
          const double xa = qa[k + q * G::NKV], xb = qb[k + q * G::NKV];
          c[q][0] = fma(xa, wA.x, fma(xb, wB.x, c[q][0]));
          c[q][1] = fma(xa, wA.y, fma(xb, wB.y, c[q][1]));
        }
      }
    }
#pragma unroll
    for (int q = 0; q < RW; ++q) {
      const int64_t row = (int64_t)ty * G::BM + xr0 + q;
      if (row < a.E1) store_pair(a.dst.p + row * a.dst.s1, col, a.E2, v0, v1, c[q][0], c[q][1]);
    }
  }
}

// ------------------------------------------------------------------------------------------
// 2D, warp-specialised (the default for the DMMA variants III / IV / V): the LUT scatter and the
// dual tessellation run on DIFFERENT warps, so the DMMA warps never wait for a scatter.
//   warp NCW + NSW      producer: raw input regions -> RAW_STAGES ring (cp.async.bulk rows)
//   warps NCW .. +NSW   scatter: raw stage -> stencil2row A/B buffer it % 2 through the LUT
//   warps 0 .. NCW-1    dual tessellation on DMMA from A/B buffer it % 2, centre store
// Buffer hand-offs are mbarriers: raw full/empty, ab_full (scatter warps arrive) and ab_empty
// (DMMA warps arrive), so tile k+1 is scattered while tile k is tessellated.
#ifndef S2R_NG7
#define S2R_NG7 2
#endif
template <int NK, bool PAD = true>
struct S2R2DWS {
  using G = S2R2D<NK, PAD>;
  // nk = 7 keeps 26 weight fragments per DMMA lane: at 2 CTAs / SM two scatter warps make the
  // DMMA warps spill (80 registers: 0.646 of the DMMA roof) and one cannot keep up (0.447), so
  // nk = 7 runs one CTA per SM with four scatter warps and a 2-stage raw ring; nk <= 5 runs two
  // CTAs per SM with two scatter warps
  static constexpr int MINB = NK >= 7 ? 1 : 2;
  static constexpr int NSW = NK >= 7 ? 4 : 2;
  // nk = 7 (one CTA per SM): two groups of 8 DMMA warps tessellate alternate tiles, four A/B
  // buffers in flight (16 DMMA warps per SM as at two CTAs, without the second LUT and ring)
  static constexpr int NG = NK >= 7 ? S2R_NG7 : 1;
  static constexpr int NB = 2 * NG;                    // A/B buffers
  static constexpr int RAW_STAGES = 2;
  static constexpr int NT = 32 * (NG * G::NCW + NSW + 1);
  static constexpr int SMEM = RAW_STAGES * G::RAW * 8 + NB * G::AB * 8 + G::NE * 4;
};

template <int NK, bool PAD, bool DIRTY>
__global__ void __launch_bounds__(S2R2DWS<NK>::NT, S2R2DWS<NK>::MINB) k_s2r2d_ws(S2RArgs a) {
  using G = S2R2D<NK, PAD>;
  using W = S2R2DWS<NK, PAD>;
  constexpr int NSW = W::NSW, NB = W::NB, NCW = W::NG * G::NCW;
  extern __shared__ __align__(128) double smem[];
  __shared__ __align__(8) uint64_t full[W::RAW_STAGES], empty[W::RAW_STAGES], ab_full[NB], ab_empty[NB];
  double* raw = smem;                                           // RAW_STAGES x RAW
  double* sAB = raw + W::RAW_STAGES * G::RAW;                   // NB x (A | B)
  uint32_t* sL = reinterpret_cast<uint32_t*>(sAB + NB * G::AB);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < NB * G::AB; i += W::NT) sAB[i] = 0.0;
  for (int i = tid; i < G::NE; i += W::NT) sL[i] = (uint32_t)a.lut[i].y;
  if (tid == 0) {
    for (int s = 0; s < W::RAW_STAGES; ++s) {
      s2r_mbar_init(&full[s], 1);
      s2r_mbar_init(&empty[s], NSW);
    }
    for (int b = 0; b < NB; ++b) {
      s2r_mbar_init(&ab_full[b], NSW);
      s2r_mbar_init(&ab_empty[b], G::NCW);  // one DMMA group
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == NCW + NSW) {  // producer
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % W::RAW_STAGES, n = it / W::RAW_STAGES;
      if (n > 0) s2r_mbar_wait(&empty[s], (n - 1) & 1);
      const int ty = (int)(tile / a.tiles_x);
      const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
      const double* src = a.src.p + (int64_t)(ty * G::BM - G::R) * a.src.s1 + (tx * G::BN - G::R - G::ODD);
      s2r_issue_rows(src, a.src.s1, raw + s * G::RAW, G::RR, G::TPR, &full[s], lane);
    }
    return;
  }
  if (warp >= NCW) {  // scatter warps: implicit stencil2row through the LUT (branch-free)
    const int sw = warp - NCW;
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % W::RAW_STAGES, b = it % NB;
      if (it >= NB) s2r_mbar_wait(&ab_empty[b], ((it / NB) - 1) & 1);  // tile it-NB tessellated
      s2r_mbar_wait(&full[s], (it / W::RAW_STAGES) & 1);
      double* sA = sAB + b * G::AB;
      double* sB = sA + (G::STRIPS + 1) * G::PITCH;
      const double* rs = raw + s * G::RAW + G::ODD;
      for (int x = sw; x < G::RR; x += NSW) {
        const double* rrow = rs + x * G::TPR;
        const uint32_t* lrow = sL + x * G::RC;
        for (int y = lane; y < G::RC; y += 32) {
          const double v = rrow[y];
          const uint32_t l = lrow[y];
          if (DIRTY) {  // dirty bits absorb the unused elements: no branch (P.1759-1773)
            sA[l & 0xffffu] = v;
            sB[l >> 16] = v;
          } else {      // breakdown variants III / IV: conditional stores
            if ((l & 0xffffu) != 0xffffu) sA[l & 0xffffu] = v;
            if ((l >> 16) != 0xffffu) sB[l >> 16] = v;
          }
        }
      }
      __syncwarp();
      if (lane == 0) {
        s2r_mbar_arrive(&empty[s]);    // raw stage consumed
        s2r_mbar_arrive(&ab_full[b]);  // this warp's share of A/B written
      }
    }
    return;
  }
  // DMMA warps
  double wa[G::KS], wb[G::KS];
#pragma unroll
  for (int s = 0; s < G::KS; ++s) {
    wa[s] = a.frags[s * 32 + lane];
    wb[s] = a.frags[(G::KS + s) * 32 + lane];
  }
  const int g = lane >> 2, t = lane & 3;
  const bool v0 = 2 * t < G::SW, v1 = 2 * t + 1 < G::SW;
  constexpr int RW = G::BM / G::NCW;
  const int grp = warp / G::NCW;              // DMMA group: tiles it with it % NG == grp
  const int xr0 = (warp - grp * G::NCW) * RW;
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    if (it % W::NG != grp) continue;
    const int b = it % NB;
    const int ty = (int)(tile / a.tiles_x);
    const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
    s2r_mbar_wait(&ab_full[b], (it / NB) & 1);
    const double* sA = sAB + b * G::AB;
    const double* sB = sA + (G::STRIPS + 1) * G::PITCH;
    const double* pa = sA + g * G::PITCH + G::NKV * xr0 + t;
    const double* pb = sB + g * G::PITCH + G::NKV * xr0 + t;
    double c[RW][2];
#pragma unroll
    for (int q = 0; q < RW; ++q) c[q][0] = c[q][1] = 0.0;
    // the warp's RW output rows as RW independent chains, vitrolite B accumulated onto A
    // (P.1332-1336)
#pragma unroll
    for (int s2 = 0; s2 < G::KS; ++s2)
#pragma unroll
      for (int q = 0; q < RW; ++q) dmma(c[q][0], c[q][1], pa[4 * s2 + q * G::NKV], wa[s2]);
#pragma unroll
    for (int s2 = 0; s2 < G::KS; ++s2)
#pragma unroll
      for (int q = 0; q < RW; ++q) dmma(c[q][0], c[q][1], pb[4 * s2 + q * G::NKV], wb[s2]);
    __syncwarp();
    if (lane == 0) s2r_mbar_arrive(&ab_empty[b]);  // A/B buffer b no longer read by this warp
    const int64_t col = (int64_t)tx * G::BN + g * G::SW + 2 * t;
#pragma unroll
    for (int q = 0; q < RW; ++q) {
      const int64_t row = (int64_t)ty * G::BM + xr0 + q;
      if (row < a.E1) store_pair(a.dst.p + row * a.dst.s1, col, a.E2, v0, v1, c[q][0], c[q][1]);
    }
  }
}

// ------------------------------------------------------------------------------------------
// 1D (P.1779-1786): stencil2row rows k hold X[k(nk+1) .. k(nk+1)+nk); one dual tessellation
// covers 8 rows = 8 (nk+1) outputs; N fragments f cover output columns 8f .. 8f+7.
template <int NK>
__global__ void __launch_bounds__(128, 4) k_s2r1d(S2RArgs a) {
  using G = S2R1D<NK>;
  constexpr int NF = G::NF, KS = G::KS;
  extern __shared__ __align__(16) double smem[];
  double* sA = smem;
  double* sB = smem + (G::STRIPS + 1) * G::PITCH;
  int2* sL = reinterpret_cast<int2*>(smem + 2 * (G::STRIPS + 1) * G::PITCH);
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < 2 * (G::STRIPS + 1) * G::PITCH; i += G::NT) smem[i] = 0.0;
  for (int i = tid; i < G::NE; i += G::NT) sL[i] = a.lut[i];
  double wa[NF][KS], wb[NF][KS];
#pragma unroll
  for (int f = 0; f < NF; ++f)
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      wa[f][s] = a.frags[((0 * NF + f) * KS + s) * 32 + lane];
      wb[f][s] = a.frags[((1 * NF + f) * KS + s) * 32 + lane];
    }
  const int g = lane >> 2, t = lane & 3;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x) {
    const double* base = a.src.p + tile * G::BN - G::R;
    __syncthreads();
#pragma unroll 4
    for (int e = tid; e < G::NE; e += G::NT) {
      const int2 l = sL[e];
      const double v = __ldg(base + l.x);
      sA[l.y & 0xffff] = v;
      sB[((unsigned)l.y) >> 16] = v;
    }
    __syncthreads();
#pragma unroll 1
    for (int d = warp; d < G::NDT; d += 4) {
      const double* pa = sA + (8 * d + g) * G::PITCH + t;
      const double* pb = sB + (8 * d + g) * G::PITCH + t;
      double c[NF][2];
#pragma unroll
      for (int f = 0; f < NF; ++f) c[f][0] = c[f][1] = 0.0;
#pragma unroll
      for (int s = 0; s < KS; ++s) {
        const double x = pa[4 * s];
#pragma unroll
        for (int f = 0; f < NF; ++f) dmma(c[f][0], c[f][1], x, wa[f][s]);
      }
#pragma unroll
      for (int s = 0; s < KS; ++s) {
        const double x = pb[4 * s];
#pragma unroll
        for (int f = 0; f < NF; ++f) dmma(c[f][0], c[f][1], x, wb[f][s]);
      }
      const int64_t o = tile * G::BN + (int64_t)(8 * d + g) * G::SW;
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        const int cc = 8 * f + 2 * t;
        store_pair(a.dst.p, o + cc, a.E2, cc < G::SW, cc + 1 < G::SW, c[f][0], c[f][1]);
      }
    }
  }
}

// ------------------------------------------------------------------------------------------
// 1D, warp-specialised (default): the tile's input run (contiguous in 1D) arrives by ONE bulk
// copy into a 2-stage raw ring, dedicated scatter warps run the LUT scatter smem -> smem into
// one of two A/B buffers while the DMMA warps tessellate the other (round 1 gathered every LUT
// element with its own __ldg from global memory, synchronously, between two CTA barriers).
template <int NK>
struct S2R1DWS {
  using G = S2R1D<NK>;
  static constexpr int ODD = G::R & 1;                       // 16-B aligned copy start
  static constexpr int RAWN = (ODD + G::RC + 1) / 2 * 2;     // staged doubles (16-B multiple)
  static constexpr int RAW_A = (RAWN + 15) / 16 * 16;        // 128-B aligned ring slots
  // DMMA warps, scatter warps (the scatter is the heavier role in 1D: 2 / 4 / 8 scatter warps
  // measured 1320 / 1704 / 1792 GSt/s on Heat-1D 10.24M at Tf = 7)
  static constexpr int NCW = 8, NSW = 8;
  static constexpr int NT = 32 * (NCW + NSW + 1);
  static constexpr int AB = 2 * (G::STRIPS + 1) * G::PITCH;  // doubles per A/B buffer
  static constexpr int SMEM = 2 * RAW_A * 8 + 2 * AB * 8 + G::NE * 4 + 128;
};

template <int NK>
__global__ void __launch_bounds__(S2R1DWS<NK>::NT, 1) k_s2r1d_ws(S2RArgs a) {
  using G = S2R1D<NK>;
  using W = S2R1DWS<NK>;
  constexpr int NF = G::NF, KS = G::KS;
  extern __shared__ __align__(128) double smem_raw1[];
  double* raw = smem_raw1 + ((128u - (s2r_smem_u32(smem_raw1) & 127u)) & 127u) / 8u;  // 2 x RAW_A
  double* sAB = raw + 2 * W::RAW_A;                                                   // 2 x AB
  uint32_t* sL = reinterpret_cast<uint32_t*>(sAB + 2 * W::AB);
  __shared__ __align__(8) uint64_t full[2], empty[2], ab_full[2], ab_empty[2];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < 2 * W::AB; i += W::NT) sAB[i] = 0.0;
  for (int i = tid; i < G::NE; i += W::NT) sL[i] = (uint32_t)a.lut[i].y;
  if (tid == 0) {
    for (int s = 0; s < 2; ++s) {
      s2r_mbar_init(&full[s], 1);
      s2r_mbar_init(&empty[s], W::NSW);
      s2r_mbar_init(&ab_full[s], W::NSW);
      s2r_mbar_init(&ab_empty[s], W::NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  if (warp == W::NCW + W::NSW) {  // producer: one bulk copy per tile
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it & 1, n = it >> 1;
      if (n > 0) s2r_mbar_wait(&empty[s], (n - 1) & 1);
      if (lane == 0) {
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(s2r_smem_u32(&full[s])),
                     "r"((uint32_t)(W::RAWN * 8))
                     : "memory");
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                s2r_smem_u32(raw + s * W::RAW_A)),
            "l"(a.src.p + tile * G::BN - G::R - W::ODD), "r"((uint32_t)(W::RAWN * 8)), "r"(s2r_smem_u32(&full[s]))
            : "memory");
      }
    }
    return;
  }
  if (warp >= W::NCW) {  // scatter warps: implicit stencil2row through the LUT (branch-free)
    const int sw = warp - W::NCW;
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it & 1, b = it & 1;
      if (it >= 2) s2r_mbar_wait(&ab_empty[b], ((it >> 1) - 1) & 1);
      s2r_mbar_wait(&full[s], (it >> 1) & 1);
      double* sA = sAB + b * W::AB;
      double* sB = sA + (G::STRIPS + 1) * G::PITCH;
      const double* rs = raw + s * W::RAW_A + W::ODD;
#pragma unroll 4
      for (int e = sw * 32 + lane; e < G::NE; e += 32 * W::NSW) {
        const double v = rs[e];
        const uint32_t l = sL[e];
        sA[l & 0xffffu] = v;
        sB[l >> 16] = v;
      }
      __syncwarp();
      if (lane == 0) {
        s2r_mbar_arrive(&empty[s]);
        s2r_mbar_arrive(&ab_full[b]);
      }
    }
    return;
  }
  double wa[NF][KS], wb[NF][KS];
#pragma unroll
  for (int f = 0; f < NF; ++f)
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      wa[f][s] = a.frags[((0 * NF + f) * KS + s) * 32 + lane];
      wb[f][s] = a.frags[((1 * NF + f) * KS + s) * 32 + lane];
    }
  const int g = lane >> 2, t = lane & 3;
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    const int b = it & 1;
    s2r_mbar_wait(&ab_full[b], (it >> 1) & 1);
    const double* sA = sAB + b * W::AB;
    const double* sB = sA + (G::STRIPS + 1) * G::PITCH;
    double c[G::NDT / W::NCW][NF][2];
#pragma unroll
    for (int u = 0; u < G::NDT / W::NCW; ++u) {
      const int d = warp + u * W::NCW;
      const double* pa = sA + (8 * d + g) * G::PITCH + t;
      const double* pb = sB + (8 * d + g) * G::PITCH + t;
#pragma unroll
      for (int f = 0; f < NF; ++f) c[u][f][0] = c[u][f][1] = 0.0;
#pragma unroll
      for (int s = 0; s < KS; ++s) {
        const double x = pa[4 * s];
#pragma unroll
        for (int f = 0; f < NF; ++f) dmma(c[u][f][0], c[u][f][1], x, wa[f][s]);
      }
#pragma unroll
      for (int s = 0; s < KS; ++s) {
        const double x = pb[4 * s];
#pragma unroll
        for (int f = 0; f < NF; ++f) dmma(c[u][f][0], c[u][f][1], x, wb[f][s]);
      }
    }
    __syncwarp();
    if (lane == 0) s2r_mbar_arrive(&ab_empty[b]);
#pragma unroll
    for (int u = 0; u < G::NDT / W::NCW; ++u) {
      const int d = warp + u * W::NCW;
      const int64_t o = tile * G::BN + (int64_t)(8 * d + g) * G::SW;
#pragma unroll
      for (int f = 0; f < NF; ++f) {
        const int cc = 8 * f + 2 * t;
        store_pair(a.dst.p, o + cc, a.E2, cc < G::SW, cc + 1 < G::SW, c[u][f][0], c[u][f][1]);
      }
    }
  }
}

// ------------------------------------------------------------------------------------------
// 3D (Tf = 1): stream input planes along z; input plane zi contributes to output planes
// zo = zi - R + j with the 2D weights of z offset dz = NK-1-j (P.1788-1800).  Accumulators of
// the NK live output planes rotate in registers.  Planes whose weights are a single centre tap
// (star arms) are applied with DFMA on CUDA cores from a raw copy of the region.
template <int NK>
__global__ void __launch_bounds__(128, 3) k_s2r3d(S2RArgs a, int tc_mask) {
  using G = S2R3D<NK>;
  constexpr int KS = G::KS, R = G::R;
  extern __shared__ __align__(16) double smem[];
  double* sA = smem;
  double* sB = smem + (G::STRIPS + 1) * G::PITCH;
  int2* sL = reinterpret_cast<int2*>(smem + 2 * (G::STRIPS + 1) * G::PITCH);
  double* sX = reinterpret_cast<double*>(sL + G::NE);  // raw region (CUDA-core planes)
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < 2 * (G::STRIPS + 1) * G::PITCH; i += G::NT) smem[i] = 0.0;
  for (int i = tid; i < G::NE; i += G::NT) sL[i] = a.lut[i];
  double wa[NK][KS], wb[NK][KS], wz[NK];
#pragma unroll
  for (int p = 0; p < NK; ++p) {
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      wa[p][s] = a.frags[((p * 2 + 0) * KS + s) * 32 + lane];
      wb[p][s] = a.frags[((p * 2 + 1) * KS + s) * 32 + lane];
    }
    wz[p] = a.wc[(p * NK + R) * NK + R];
  }
  const int g = lane >> 2, t = lane & 3;
  const bool v0 = 2 * t < G::SW, v1 = 2 * t + 1 < G::SW;
  const bool need_raw = tc_mask != (1 << NK) - 1;
  const int64_t nz = (a.E0 + G::ZCHUNK - 1) / G::ZCHUNK;
  const int64_t ncol = (int64_t)a.tiles_x * a.tiles_y;
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int64_t zc = item / ncol;
    const int64_t tile = item - zc * ncol;
    const int ty = (int)(tile / a.tiles_x);
    const int tx = (int)(tile - (int64_t)ty * a.tiles_x);
    const int64_t z0 = zc * G::ZCHUNK;
    const int64_t z1 = min(a.E0, z0 + G::ZCHUNK);
    (void)nz;
    const double* base2 = a.src.p + (int64_t)(ty * G::BM - R) * a.src.s1 + (tx * G::BN - R);
    constexpr int RW = G::BM / 4;  // output rows per warp (4 compute warps)
    double acc[NK][RW][2];
#pragma unroll
    for (int j = 0; j < NK; ++j)
#pragma unroll
      for (int h = 0; h < RW; ++h) acc[j][h][0] = acc[j][h][1] = 0.0;
    const int xr = warp * RW;
    const int64_t col = (int64_t)tx * G::BN + g * G::SW + 2 * t;
    for (int64_t zi = z0 - R; zi < z1 + R; ++zi) {
      const double* base = base2 + zi * a.src.s0;
      __syncthreads();
#pragma unroll 4
      for (int e = tid; e < G::NE; e += G::NT) {
        const int2 l = sL[e];
        const double v = __ldg(base + l.x);
        sA[l.y & 0xffff] = v;
        sB[((unsigned)l.y) >> 16] = v;
        if (need_raw) sX[e] = v;
      }
      __syncthreads();
      const double* pa = sA + g * G::PITCH + NK * xr + t;
      const double* pb = sB + g * G::PITCH + NK * xr + t;
#pragma unroll
      for (int j = 0; j < NK; ++j) {
        const int dz = NK - 1 - j;
        if (tc_mask & (1 << dz)) {
#pragma unroll
          for (int s = 0; s < KS; ++s) {
#pragma unroll
            for (int h = 0; h < RW; ++h) dmma(acc[j][h][0], acc[j][h][1], pa[4 * s + h * NK], wa[dz][s]);
          }
#pragma unroll
          for (int s = 0; s < KS; ++s) {
#pragma unroll
            for (int h = 0; h < RW; ++h) dmma(acc[j][h][0], acc[j][h][1], pb[4 * s + h * NK], wb[dz][s]);
          }
        } else if (wz[dz] != 0.0) {
          // centre tap of output (xr + h, g*SW + 2t + e) is region (xr + h + R, g*SW + 2t + e + R)
#pragma unroll
          for (int h = 0; h < RW; ++h) {
            const double* px = sX + (xr + h + R) * G::RC + g * G::SW + 2 * t + R;
            acc[j][h][0] = fma(wz[dz], px[0], acc[j][h][0]);
            acc[j][h][1] = fma(wz[dz], px[1], acc[j][h][1]);
          }
        }
      }
      const int64_t zo = zi - R;
      if (zo >= z0) {
        double* plane = a.dst.p + zo * a.dst.s0;
        const int64_t row = (int64_t)ty * G::BM + xr;
#pragma unroll
        for (int h = 0; h < RW; ++h)
          if (row + h < a.E1)
            store_pair(plane + (row + h) * a.dst.s1, col, a.E2, v0, v1, acc[0][h][0], acc[0][h][1]);
      }
#pragma unroll
      for (int j = 0; j + 1 < NK; ++j) {
#pragma unroll
        for (int h = 0; h < RW; ++h) {
          acc[j][h][0] = acc[j + 1][h][0];
          acc[j][h][1] = acc[j + 1][h][1];
        }
      }
#pragma unroll
      for (int h = 0; h < RW; ++h) acc[NK - 1][h][0] = acc[NK - 1][h][1] = 0.0;
    }
  }
}

// ------------------------------------------------------------------------------------------
// 3D with a staged plane ring (default; CSX_S2R_WS=0 = the kernel above): a producer warp
// streams each input plane's raw region (RR rows, one cp.async.bulk per row) into a STAGES-deep
// ring, so the plane loads are in flight while earlier planes are scattered and tessellated
// (k_s2r3d gathers every LUT element from global memory between two CTA barriers, exposing the
// load latency once per plane).  The 4 compute warps scatter plane k through the LUT into A/B
// buffer k & 1 (smem -> smem), meet at one named barrier, and run the dual tessellations of the
// NK accumulating output planes; the single-tap planes read the staged raw region directly.
template <int NK>
struct S2R3DWS {
  using G = S2R3D<NK>;
  static constexpr int ODD = G::R & 1;
  static constexpr int TP = (ODD + G::RC + 1) / 2 * 2;   // staged row length (16-B multiple)
  static constexpr int RAW = G::RR * TP;
  static constexpr int RAW_A = (RAW + 15) / 16 * 16;
  static constexpr int STAGES = 4;
  static constexpr int NCW = 4;
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int AB = 2 * (G::STRIPS + 1) * G::PITCH;
  static constexpr int SMEM = STAGES * RAW_A * 8 + 2 * AB * 8 + G::NE * 4 + 128;
};

template <int NK>
__global__ void __launch_bounds__(S2R3DWS<NK>::NT, 3) k_s2r3d_ws(S2RArgs a, int tc_mask) {
  using G = S2R3D<NK>;
  using W = S2R3DWS<NK>;
  constexpr int KS = G::KS, R = G::R;
  extern __shared__ __align__(128) double smem_raw3[];
  double* raw = smem_raw3 + ((128u - (s2r_smem_u32(smem_raw3) & 127u)) & 127u) / 8u;  // STAGES x RAW_A
  double* sAB = raw + W::STAGES * W::RAW_A;                                            // 2 x AB
  uint32_t* sL = reinterpret_cast<uint32_t*>(sAB + 2 * W::AB);
  __shared__ __align__(8) uint64_t full[W::STAGES], empty[W::STAGES];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < 2 * W::AB; i += W::NT) sAB[i] = 0.0;
  for (int i = tid; i < G::NE; i += W::NT) sL[i] = (uint32_t)a.lut[i].y;
  if (tid == 0) {
    for (int s = 0; s < W::STAGES; ++s) {
      s2r_mbar_init(&full[s], 1);
      s2r_mbar_init(&empty[s], W::NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  const int64_t ncol = (int64_t)a.tiles_x * a.tiles_y;
  if (warp == W::NCW) {  // producer: raw regions of planes z0-R .. z1+R-1 of every item
    int q = 0;
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int64_t zc = item / ncol, tile = item - zc * ncol;
      const int ty = (int)(tile / a.tiles_x), tx = (int)(tile - (int64_t)ty * a.tiles_x);
      const int64_t z0 = zc * G::ZCHUNK, z1 = min(a.E0, z0 + G::ZCHUNK);
      const double* base2 = a.src.p + (int64_t)(ty * G::BM - R) * a.src.s1 + (tx * G::BN - R - W::ODD);
      for (int64_t zi = z0 - R; zi < z1 + R; ++zi, ++q) {
        const int s = q % W::STAGES, n = q / W::STAGES;
        if (n > 0) s2r_mbar_wait(&empty[s], (n - 1) & 1);
        s2r_issue_rows(base2 + zi * a.src.s0, a.src.s1, raw + s * W::RAW_A, G::RR, W::TP, &full[s], lane);
      }
    }
    return;
  }
  double wa[NK][KS], wb[NK][KS], wz[NK];
#pragma unroll
  for (int p = 0; p < NK; ++p) {
#pragma unroll
    for (int s = 0; s < KS; ++s) {
      wa[p][s] = a.frags[((p * 2 + 0) * KS + s) * 32 + lane];
      wb[p][s] = a.frags[((p * 2 + 1) * KS + s) * 32 + lane];
    }
    wz[p] = a.wc[(p * NK + R) * NK + R];
  }
  const int g = lane >> 2, t = lane & 3;
  const bool v0 = 2 * t < G::SW, v1 = 2 * t + 1 < G::SW;
  int q = 0;  // input plane sequence number (producer order)
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int64_t zc = item / ncol, tile = item - zc * ncol;
    const int ty = (int)(tile / a.tiles_x), tx = (int)(tile - (int64_t)ty * a.tiles_x);
    const int64_t z0 = zc * G::ZCHUNK, z1 = min(a.E0, z0 + G::ZCHUNK);
    constexpr int RW = G::BM / 4;  // output rows per warp (4 compute warps)
    double acc[NK][RW][2];
#pragma unroll
    for (int j = 0; j < NK; ++j)
#pragma unroll
      for (int h = 0; h < RW; ++h) acc[j][h][0] = acc[j][h][1] = 0.0;
    const int xr = warp * RW;
    const int64_t col = (int64_t)tx * G::BN + g * G::SW + 2 * t;
    for (int64_t zi = z0 - R; zi < z1 + R; ++zi, ++q) {
      const int s = q % W::STAGES;
      s2r_mbar_wait(&full[s], (q / W::STAGES) & 1);
      const double* rs = raw + s * W::RAW_A + W::ODD;
      double* sA = sAB + (q & 1) * W::AB;
      double* sB = sA + (G::STRIPS + 1) * G::PITCH;
      // implicit stencil2row of this plane (A/B buffer q & 1: last read two planes ago, before
      // every warp passed the previous plane's barrier)
      for (int e = tid; e < G::NE; e += W::NCW * 32) {
        const int x = e / G::RC, y = e - (e / G::RC) * G::RC;
        const double v = rs[x * W::TP + y];
        const uint32_t l = sL[e];
        sA[l & 0xffffu] = v;
        sB[l >> 16] = v;
      }
      asm volatile("bar.sync 1, %0;\n" ::"n"(W::NCW * 32) : "memory");
      const double* pa = sA + g * G::PITCH + NK * xr + t;
      const double* pb = sB + g * G::PITCH + NK * xr + t;
#pragma unroll
      for (int j = 0; j < NK; ++j) {
        const int dz = NK - 1 - j;
        if (tc_mask & (1 << dz)) {
#pragma unroll
          for (int s2 = 0; s2 < KS; ++s2) {
#pragma unroll
            for (int h = 0; h < RW; ++h) dmma(acc[j][h][0], acc[j][h][1], pa[4 * s2 + h * NK], wa[dz][s2]);
          }
#pragma unroll
          for (int s2 = 0; s2 < KS; ++s2) {
#pragma unroll
            for (int h = 0; h < RW; ++h) dmma(acc[j][h][0], acc[j][h][1], pb[4 * s2 + h * NK], wb[dz][s2]);
          }
        } else if (wz[dz] != 0.0) {
          // centre tap of output (xr + h, g*SW + 2t + e) is region (xr + h + R, g*SW + 2t + e + R)
#pragma unroll
          for (int h = 0; h < RW; ++h) {
            const double* px = rs + (xr + h + R) * W::TP + g * G::SW + 2 * t + R;
            acc[j][h][0] = fma(wz[dz], px[0], acc[j][h][0]);
            acc[j][h][1] = fma(wz[dz], px[1], acc[j][h][1]);
          }
        }
      }
      __syncwarp();
      if (lane == 0) s2r_mbar_arrive(&empty[s]);  // raw plane no longer read by this warp
      const int64_t zo = zi - R;
      if (zo >= z0) {
        double* plane = a.dst.p + zo * a.dst.s0;
        const int64_t row = (int64_t)ty * G::BM + xr;
#pragma unroll
        for (int h = 0; h < RW; ++h)
          if (row + h < a.E1)
            store_pair(plane + (row + h) * a.dst.s1, col, a.E2, v0, v1, acc[0][h][0], acc[0][h][1]);
      }
#pragma unroll
      for (int j = 0; j + 1 < NK; ++j) {
#pragma unroll
        for (int h = 0; h < RW; ++h) {
          acc[j][h][0] = acc[j + 1][h][0];
          acc[j][h][1] = acc[j + 1][h][1];
        }
      }
#pragma unroll
      for (int h = 0; h < RW; ++h) acc[NK - 1][h][0] = acc[NK - 1][h][1] = 0.0;
    }
  }
}

// ------------------------------------------------------------------------------------------
int64_t persistent_grid(int occ, int max_ctas, int64_t items) {
  int64_t grid = (int64_t)(occ < 1 ? 1 : occ) * num_sms();
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;
  if (grid > items) grid = items;
  return grid;
}

int num_sms() {
  static int n = 0;
  if (n == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <class K>
static cudaError_t launch_persistent(K kernel, int smem, int nthreads, int64_t items, cudaStream_t st,
                                     const S2RArgs& a) {
  cudaError_t e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kernel, nthreads, smem);
  if (e != cudaSuccess) return e;
  if (occ < 1) return cudaErrorInvalidConfiguration;
  int64_t grid = persistent_grid(occ, a.max_ctas, items);
  if (grid < 1) grid = 1;
  kernel<<<(unsigned)grid, nthreads, smem, st>>>(a);
  return cudaGetLastError();
}

// CSX_S2R_WS=0 selects the round-1 kernel (scatter and tessellation on the same 8 warps)
static bool s2r_ws() {
  static const int v = [] {
    const char* e = getenv("CSX_S2R_WS");
    return e ? atoi(e) : 1;
  }();
  return v != 0;
}

template <int NK>
static cudaError_t launch_s2r2d_var(const S2RArgs& a, int variant, cudaStream_t st) {
  // variant bit 0 = padding, bit 1 = dirty bits (default 3 = the paper's full design),
  // bit 2 = CUDA-core tessellation (breakdown II, with padding and dirty bits)
  if (variant & 4)
    return launch_persistent(k_s2r2d<NK, true, true, true>, S2R2D<NK, true>::SMEM, S2R2D<NK>::NT, a.ntiles, st, a);
  if (s2r_ws()) {  // warp-specialised scatter / tessellation (default)
    constexpr int NT = S2R2DWS<NK>::NT;
    switch (variant) {
      case 3: return launch_persistent(k_s2r2d_ws<NK, true, true>, S2R2DWS<NK, true>::SMEM, NT, a.ntiles, st, a);
      case 1: return launch_persistent(k_s2r2d_ws<NK, true, false>, S2R2DWS<NK, true>::SMEM, NT, a.ntiles, st, a);
      case 2: return launch_persistent(k_s2r2d_ws<NK, false, true>, S2R2DWS<NK, false>::SMEM, NT, a.ntiles, st, a);
      default: return launch_persistent(k_s2r2d_ws<NK, false, false>, S2R2DWS<NK, false>::SMEM, NT, a.ntiles, st, a);
    }
  }
  switch (variant) {
    case 3: return launch_persistent(k_s2r2d<NK, true, true>, S2R2D<NK, true>::SMEM, S2R2D<NK>::NT, a.ntiles, st, a);
    case 1: return launch_persistent(k_s2r2d<NK, true, false>, S2R2D<NK, true>::SMEM, S2R2D<NK>::NT, a.ntiles, st, a);
    case 2: return launch_persistent(k_s2r2d<NK, false, true>, S2R2D<NK, false>::SMEM, S2R2D<NK>::NT, a.ntiles, st, a);
    default: return launch_persistent(k_s2r2d<NK, false, false>, S2R2D<NK, false>::SMEM, S2R2D<NK>::NT, a.ntiles, st, a);
  }
}

int s2r_smem_bytes(int ndim, int nk, int nf) {
  (void)nf;
  if (ndim == 1) {
    switch (nk) {
      case 3: return S2R1D<3>::SMEM;
      case 5: return S2R1D<5>::SMEM;
      case 7: return S2R1D<7>::SMEM;
      case 9: return S2R1D<9>::SMEM;
      case 11: return S2R1D<11>::SMEM;
      case 13: return S2R1D<13>::SMEM;
      case 15: return S2R1D<15>::SMEM;
    }
  } else if (ndim == 2) {
    switch (nk) {
      case 3: return S2R2D<3>::SMEM;
      case 5: return S2R2D<5>::SMEM;
      case 7: return S2R2D<7>::SMEM;
    }
  } else if (nk == 3) {
    return S2R3D<3>::SMEM;
  }
  return -1;
}

cudaError_t launch_s2r(int ndim, int nk, int nf, const S2RArgs& a, int tc_mask, cudaStream_t st) {
  (void)nf;
  const int smem = s2r_smem_bytes(ndim, nk, nf);
  if (smem < 0) return cudaErrorInvalidValue;
  if (ndim == 1 && s2r_ws()) {
    switch (nk) {
      case 3: return launch_persistent(k_s2r1d_ws<3>, S2R1DWS<3>::SMEM, S2R1DWS<3>::NT, a.ntiles, st, a);
      case 5: return launch_persistent(k_s2r1d_ws<5>, S2R1DWS<5>::SMEM, S2R1DWS<5>::NT, a.ntiles, st, a);
      case 7: return launch_persistent(k_s2r1d_ws<7>, S2R1DWS<7>::SMEM, S2R1DWS<7>::NT, a.ntiles, st, a);
      case 9: return launch_persistent(k_s2r1d_ws<9>, S2R1DWS<9>::SMEM, S2R1DWS<9>::NT, a.ntiles, st, a);
      case 11: return launch_persistent(k_s2r1d_ws<11>, S2R1DWS<11>::SMEM, S2R1DWS<11>::NT, a.ntiles, st, a);
      case 13: return launch_persistent(k_s2r1d_ws<13>, S2R1DWS<13>::SMEM, S2R1DWS<13>::NT, a.ntiles, st, a);
      case 15: return launch_persistent(k_s2r1d_ws<15>, S2R1DWS<15>::SMEM, S2R1DWS<15>::NT, a.ntiles, st, a);
    }
  }
  if (ndim == 1) {
    switch (nk) {
      case 3: return launch_persistent(k_s2r1d<3>, smem, 128, a.ntiles, st, a);
      case 5: return launch_persistent(k_s2r1d<5>, smem, 128, a.ntiles, st, a);
      case 7: return launch_persistent(k_s2r1d<7>, smem, 128, a.ntiles, st, a);
      case 9: return launch_persistent(k_s2r1d<9>, smem, 128, a.ntiles, st, a);
      case 11: return launch_persistent(k_s2r1d<11>, smem, 128, a.ntiles, st, a);
      case 13: return launch_persistent(k_s2r1d<13>, smem, 128, a.ntiles, st, a);
      case 15: return launch_persistent(k_s2r1d<15>, smem, 128, a.ntiles, st, a);
    }
  } else if (ndim == 2) {
    switch (nk) {
      case 3: return launch_s2r2d_var<3>(a, a.s2r_variant, st);
      case 5: return launch_s2r2d_var<5>(a, a.s2r_variant, st);
      case 7: return launch_s2r2d_var<7>(a, a.s2r_variant, st);
    }
  } else if (nk == 3 && s2r_ws()) {
    using W = S2R3DWS<3>;
    auto kern = k_s2r3d_ws<3>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, W::SMEM);
    if (e != cudaSuccess) return e;
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, W::NT, W::SMEM);
    if (e != cudaSuccess) return e;
    const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
    kern<<<(unsigned)grid, W::NT, W::SMEM, st>>>(a, tc_mask);
    return cudaGetLastError();
  } else if (nk == 3) {
    auto kern = k_s2r3d<3>;
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    int occ = 0;
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 128, smem);
    if (e != cudaSuccess) return e;
    const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
    kern<<<(unsigned)grid, 128, smem, st>>>(a, tc_mask);
    return cudaGetLastError();
  }
  return cudaErrorInvalidValue;
}

}  // namespace csx
