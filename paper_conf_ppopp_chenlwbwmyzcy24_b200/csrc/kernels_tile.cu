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
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstring>
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

// TMA tensor copy of one box {x, y, z} (elements, innermost first) of the padded source grid
// into smem, completing on `bar` (expect_tx set by the caller).  One instruction per staged
// tile / plane instead of one bulk copy per row (the per-row loop was the 3D producer's
// bottleneck: ~66 serialised UBLKCP per plane).
__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar, int x,
                                            int y, int z) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4}], [%5];\n" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar))
      : "memory");
}

// the same with an L2 eviction-priority hint (hint 1: evict_last, 2: evict_first)
__device__ __forceinline__ void tma_load_3d_hint(void* dst, const CUtensorMap* map, uint64_t* bar, int x,
                                                 int y, int z, int hint) {
  uint64_t pol;
  if (hint == 1)
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(pol));
  else
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(pol));
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3, %4}], [%5], %6;\n" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

// 16-B output store; with `hinted` the line gets L2 evict_first priority (`pol`), so streamed
// outputs leave the L2 to the input planes whose halos neighbouring tiles re-read
__device__ __forceinline__ void st_out(double* p, double v0, double v1, bool hinted, uint64_t pol) {
  if (hinted)
    asm volatile("st.global.L2::cache_hint.v2.f64 [%0], {%1, %2}, %3;\n" ::"l"(p), "d"(v0), "d"(v1), "l"(pol)
                 : "memory");
  else
    *reinterpret_cast<double2*>(p) = make_double2(v0, v1);
}

// 8-B output store (same hint)
__device__ __forceinline__ void st_out1(double* p, double v, bool hinted, uint64_t pol) {
  if (hinted)
    asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;\n" ::"l"(p), "d"(v), "l"(pol) : "memory");
  else
    *p = v;
}

__device__ __forceinline__ void bulk_g2s_hint(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                              uint64_t pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;\n" ::
          "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}

__device__ __forceinline__ void tma_prefetch_desc(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];\n" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}

// 128-B aligned base of the dynamic smem ring (TMA tensor destinations need 128 B alignment)
// (offset arithmetic on the __shared__ array itself, so the compiler keeps LDS addressing)
__device__ __forceinline__ double* ring_base(double* raw) {
  return raw + ((128u - (smem_u32(raw) & 127u)) & 127u) / 8u;
}

static CUtensorMapL2promotion tma_promotion() {
  static const int v = [] {
    const char* e = getenv("CSX_TMA_PROMO");
    return e ? atoi(e) : 0;
  }();
  switch (v) {
    case 64: return CU_TENSOR_MAP_L2_PROMOTION_L2_64B;
    case 128: return CU_TENSOR_MAP_L2_PROMOTION_L2_128B;
    case 256: return CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  }
  return CU_TENSOR_MAP_L2_PROMOTION_NONE;
}

// Host: a rank-3 tensor map over the whole allocation of a padded grid (FP64, no swizzle, box
// {bx, by, 1}); fills the interior origin in tensor-map coordinates.  Returns false (caller
// falls back to per-row bulk copies) if the geometry is unknown or the driver entry point is
// missing.
static bool make_tmap(S2RArgs& a, int bx, int by, CUtensorMap* map) {
  static PFN_cuTensorMapEncodeTiled_v12000 encode = [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return (PFN_cuTensorMapEncodeTiled_v12000) nullptr;
    }
    return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  }();
  const char* e = getenv("CSX_TMA");
  if (e && e[0] == '0') return false;
  const CView& v = a.src;
  if (!encode || v.n0 <= 0 || v.s1 <= 0 || v.s0 % v.s1 != 0) return false;
  const double* base = v.p - (v.o0 * v.s0 + v.o1 * v.s1 + v.o2);
  if ((reinterpret_cast<uintptr_t>(base) & 15) != 0 || (v.s1 * 8) % 16 != 0) return false;
  cuuint64_t dims[3] = {(cuuint64_t)v.s1, (cuuint64_t)(v.s0 / v.s1), (cuuint64_t)v.n0};
  cuuint64_t strides[2] = {(cuuint64_t)v.s1 * 8, (cuuint64_t)v.s0 * 8};
  cuuint32_t box[3] = {(cuuint32_t)bx, (cuuint32_t)by, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = encode(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 3, const_cast<double*>(base), dims,
                      strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                      tma_promotion(), CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return false;
  a.use_tma = 1;
  a.tma_x0 = v.o2;
  a.tma_y0 = v.o1;
  a.tma_z0 = v.o0;
  return true;
}

// Host: can the TC_TILE 2D / 3D kernels stage their tiles straight from a DENSE grid (the user's
// d_in: no ghost cells, row pitch E2)?  The TMA tensor map zero-fills the halo boxes that fall
// outside the grid, which only the held FIXED frame and the band recomputed by k_band could see.
// Decided by a trial encode of the dense geometry (the kernels' boxes are <= 256 x 256, which
// the encoder accepts whenever it accepts the geometry), so a rejected map falls back to the
// pack instead of failing the pass.
bool tile_reads_dense(const double* p, const int64_t* E) {
  const char* e = getenv("CSX_TMA");
  if (e && e[0] == '0') return false;
  const char* d = getenv("CSX_DENSE_SRC");
  if (d && d[0] == '0') return false;
  if ((reinterpret_cast<uintptr_t>(p) & 15) != 0 || E[2] % 2 != 0) return false;
  S2RArgs a;
  a.src = CView{p, E[1] * E[2], E[2], 0, 0, 0, E[0]};
  CUtensorMap map;
  return make_tmap(a, 8, 8, &map);
}

// Programmatic dependent launch (sm_90+): the kernels below are launched with programmatic
// stream serialisation (launch_pdl), so pass p+1's CTAs are scheduled onto SMs as pass p's CTAs
// retire.  Everything before pdl_begin() touches only smem and the plan's constant tables;
// griddepcontrol.wait then blocks until the previous grid has completed and its writes are
// visible, so no global read of src (or write of dst, which the previous pass read) precedes it.
__device__ __forceinline__ void pdl_begin() {
  asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory");
  asm volatile("griddepcontrol.wait;\n" ::: "memory");
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(bar)) : "memory");
}

// slab tile k of this launch -> slab tile index (ranges A then B, see S2RArgs::part)
__device__ __forceinline__ int64_t slab_map(const S2RArgs& a, int64_t k) {
  const int64_t na = a.ra1 - a.ra0;
  return k < na ? a.ra0 + k : a.rb0 + (k - na);
}

// host: fill the slab-tile ranges for part (0 all, 1 interior, 2 edge); n slab tiles of `size`
// outputs along the slab axis of local length El, halo R.  Returns the number of slab tiles.
static int64_t set_ranges(S2RArgs& a, int64_t n, int64_t size, int64_t El, int R) {
  int64_t e1 = n;  // first tile of the trailing edge run
  while (e1 > 0 && e1 * size + R > El) --e1;
  // tile k is "edge" if k == 0 or k >= e1 (k*size - R < 0 or (k+1)*size + R > El)
  a.ra0 = a.ra1 = a.rb0 = a.rb1 = 0;
  if (a.part == 0 || e1 <= 1) {
    if (a.part == 1) return 0;  // no interior
    a.ra0 = 0;
    a.ra1 = n;
  } else if (a.part == 1) {
    a.ra0 = 1;
    a.ra1 = e1;
  } else {
    a.ra0 = 0;
    a.ra1 = 1;
    a.rb0 = e1;
    a.rb1 = n;
  }
  return (a.ra1 - a.ra0) + (a.rb1 - a.rb0);
}

static bool pdl_enabled() {
  static const int v = [] {
    const char* e = getenv("CSX_PDL");
    return e ? atoi(e) : 1;
  }();
  return v != 0;
}

// launch with programmatic stream serialisation (see pdl_begin)
template <class... KArgs, class... Args>
static cudaError_t launch_pdl(bool pdl, void (*k)(KArgs...), int64_t grid, int nt, int smem,
                              cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3((unsigned)nt);
  cfg.dynamicSmemBytes = (size_t)smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl && pdl_enabled() ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, k, args...);
}


constexpr int s2r_pitch_dev(int min_pitch) {
  int p = min_pitch;
  while (p % 16 != 4 && p % 16 != 12) ++p;
  return p;
}

// Compile-time geometry of one TC_TILE instantiation.
template <int NK_, int A_, int B_, int KC_, int G_, int WM_, int WN_, int STAGES_, int CG_ = 1,
          int MINB_ = 1, int KO_ = 0>
struct TileCfg {
  static constexpr int NK = NK_, A = A_, B = B_, KC = KC_, G = G_, WM = WM_, WN = WN_;
  static constexpr int KO = KO_;                    // 1: k-slice-outer DMMA order (Tile3DCfg)
  static constexpr int MINB = MINB_;                // CTAs per SM the registers are sized for
  static constexpr int STAGES = STAGES_;
  static constexpr int CG = CG_;                    // 8-block column groups per warp
  static constexpr int R = (NK - 1) / 2;
  static constexpr int ODD = R & 1;                 // smem col = region col + ODD (16-B aligned rows)
  static constexpr int KR = A + NK - 1;             // input rows per output block
  static constexpr int KS = KR * KC / 4;            // k-slices (DMMAs) per output block
  static constexpr int BM = WM * A * G;             // CTA output rows
  static constexpr int WC = CG * 8 * B;             // output cols per warp
  static constexpr int BN = WN * WC;                // CTA output cols
  static constexpr int RR = BM + NK - 1;            // staged input rows
  static constexpr int TP = ((ODD + BN + KC - B) + 1) / 2 * 2;  // staged row length (even)
  static constexpr int STAGE = RR * TP;             // doubles staged per tile
  static constexpr int STAGE_A = (STAGE + 15) / 16 * 16;  // ring slot (128-B aligned)
  static constexpr int NCW = WM * WN;               // consumer (DMMA) warps
  static constexpr int NT = 32 * (NCW + 1);         // + one producer warp
  static constexpr int SMEM = STAGES * STAGE_A * 8 + 128;
  static_assert(TP <= 256 && RR <= 256, "TMA box dimensions");
};

template <class C>
__device__ __forceinline__ void issue_tile(const S2RArgs& a, const CUtensorMap* tmap, int64_t tile,
                                           double* stage, uint64_t* bar, int lane) {
  const int64_t tyl = tile / a.tiles_x;
  const int tx = (int)(tile - tyl * a.tiles_x);
  const int ty = (int)slab_map(a, tyl);
  if (a.use_tma) {
    if (lane == 0) {
      mbar_expect_tx(bar, (uint32_t)(C::STAGE * 8));
      tma_load_3d(stage, tmap, bar, (int)(a.tma_x0 + tx * C::BN - C::R - C::ODD),
                  (int)(a.tma_y0 + (int64_t)ty * C::BM - C::R), (int)a.tma_z0);
    }
    return;
  }
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
__global__ void __launch_bounds__(C::NT, C::MINB)
    k_tile2d(S2RArgs a, const __grid_constant__ CUtensorMap tmap) {
  extern __shared__ __align__(128) double smem_raw[];
  double* smem = ring_base(smem_raw);
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
  pdl_begin();  // PDL: let the next pass launch; wait for the previous pass's writes
  if (warp == C::NCW) {
    // ---------------- producer ----------------
    int it = 0;
    if (a.use_tma && lane == 0) tma_prefetch_desc(&tmap);
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % C::STAGES;
      const int n = it / C::STAGES;
      if (n > 0) mbar_wait(&empty[s], (n - 1) & 1);
      issue_tile<C>(a, &tmap, tile, smem + s * C::STAGE_A, &full[s], lane);
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
    const int64_t tyl = tile / a.tiles_x;
    const int tx = (int)(tile - tyl * a.tiles_x);
    const int ty = (int)slab_map(a, tyl);
    const double* base = smem + s * C::STAGE_A + (wm * C::A * C::G) * C::TP + wn * C::WC + C::ODD +
                         C::B * g + t;
    double acc[C::CG][C::G][2];
#pragma unroll
    for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
      for (int j = 0; j < C::G; ++j) acc[cg][j][0] = acc[cg][j][1] = 0.0;
    // FIXED: band outputs of an edge tile are written by k_band (kernels_band.cu) after a pass
    // of Tf > 1 steps; for Tf = 1 the band is the held frame, written here from the staged tile.
    const bool edge = tile_is_edge<C>(a, ty, tx);
    // block j of column group cg covers output rows ty*BM + wm*A*G + A*j + [0, A),
    // cols tx*BN + wn*WC + cg*8B + B*g + [0, B)
    const int64_t row0 = (int64_t)ty * C::BM + wm * C::A * C::G + alpha;
    const int64_t col0 = (int64_t)tx * C::BN + wn * C::WC + C::B * g + beta;
    const bool full_tile = a.dst_aligned && (int64_t)(ty + 1) * C::BM <= a.E1 &&
                           (int64_t)(tx + 1) * C::BN <= a.E2;
    // Stream the warp's input rows; each A fragment (4 cells of one row) feeds every output
    // block whose window contains the row.  Block j is complete after input row A*j + KR - 1 and
    // (interior tiles) is stored right there, so the epilogue interleaves with the DMMA stream.
    if (C::KO == 1) {
#pragma unroll
      for (int rho = 0; rho < C::KR; ++rho)
#pragma unroll
        for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
          for (int j = 0; j < C::G; ++j)
#pragma unroll
            for (int cg = 0; cg < C::CG; ++cg)
              dmma_t(acc[cg][j][0], acc[cg][j][1], base[(C::A * j + rho) * C::TP + cg * 8 * C::B + 4 * h],
                     wf[rho * (C::KC / 4) + h]);
    }
#pragma unroll
    for (int ra = (C::KO == 1 ? C::KR - 1 : 0); ra < C::A * C::G + C::NK - 1; ++ra) {
      double f[C::CG][C::KC / 4];
#pragma unroll
      for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
        for (int h = 0; h < C::KC / 4; ++h)
          if (C::KO == 0) f[cg][h] = base[ra * C::TP + cg * 8 * C::B + 4 * h];
#pragma unroll
      for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
        for (int j = 0; j < C::G; ++j) {
          const int rho = ra - C::A * j;
          if (C::KO == 0 && rho >= 0 && rho < C::KR)
#pragma unroll
            for (int cg = 0; cg < C::CG; ++cg)
              dmma_t(acc[cg][j][0], acc[cg][j][1], f[cg][h], wf[rho * (C::KC / 4) + h]);
        }
      if (!edge && ra >= C::KR - 1 && (ra - (C::KR - 1)) % C::A == 0) {
        const int j = (ra - (C::KR - 1)) / C::A;
        const int64_t row = row0 + C::A * j;
#pragma unroll
        for (int cg = 0; cg < C::CG; ++cg) {
          const int64_t col = col0 + cg * 8 * C::B;
          if (full_tile) {  // whole tile inside the grid, 16-B aligned rows: unguarded stores
            *reinterpret_cast<double2*>(a.dst.p + row * a.dst.s1 + col) =
                make_double2(acc[cg][j][0], acc[cg][j][1]);
          } else if (row < a.E1 && col < a.E2) {
            double* p = a.dst.p + row * a.dst.s1 + col;
            if (col + 1 < a.E2 && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
              *reinterpret_cast<double2*>(p) = make_double2(acc[cg][j][0], acc[cg][j][1]);
            } else {
              p[0] = acc[cg][j][0];
              if (col + 1 < a.E2) p[1] = acc[cg][j][1];
            }
          }
        }
      }
    }
    if (!edge) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);  // this warp no longer reads stage s
    }
#pragma unroll
    for (int cg = 0; cg < C::CG; ++cg) {
      const int64_t col = col0 + cg * 8 * C::B;
#pragma unroll
      for (int j = 0; j < C::G; ++j) {
        const int64_t row = row0 + C::A * j;
        if (!edge) {
          // stored inside the DMMA loop
        } else if (row < a.E1) {
          const int64_t grow = row + a.gorg1;
          const bool rowband = grow < a.fix_band || grow >= a.GE1 - a.fix_band;
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int64_t c = col + e;
            if (c >= a.E2) continue;
            const int64_t gc = c + a.gorg2;
            double v = acc[cg][j][e];
            if (rowband || gc < a.fix_band || gc >= a.GE2 - a.fix_band) {
              if (!a.hold_frame) continue;
              v = smem[s * C::STAGE_A + (int)(row - (int64_t)ty * C::BM + C::R) * C::TP +
                       (int)(c - (int64_t)tx * C::BN) + C::R + C::ODD];
            }
            a.dst.p[row * a.dst.s1 + c] = v;
          }
        }
      }
    }
    if (edge) {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
  }
}

// nk -> (a, b, kc); G blocks per warp column, WM x WN consumer warps, STAGES-deep ring.
// Variant 0: 12 DMMA warps, 3 stages (CTA 96 x 64).  Variant 1: 16 DMMA warps, 2 stages
// (CTA 128 x 64).  Variant 2: 12 warps of 2 column groups x 4 block rows (CTA 96 x 64) — twice
// the independent accumulator chains per input row.  CSX_TILE_VARIANT selects (default 1,
// the fastest measured: 0.875 of the DMMA peak vs 0.83 for variant 0 on Box-2D9P).
using Tile3 = TileCfg<3, 4, 2, 4, 8, 3, 4, 3>;
using Tile5 = TileCfg<5, 2, 4, 8, 8, 6, 2, 3>;
using Tile7 = TileCfg<7, 4, 2, 8, 8, 3, 4, 3>;
using Tile3b = TileCfg<3, 4, 2, 4, 8, 4, 4, 2>;
using Tile5b = TileCfg<5, 2, 4, 8, 8, 8, 2, 2>;
using Tile7b = TileCfg<7, 4, 2, 8, 8, 4, 4, 2>;
using Tile3c = TileCfg<3, 4, 2, 4, 4, 6, 2, 3, 2>;
using Tile5c = TileCfg<5, 2, 4, 8, 4, 12, 1, 3, 2>;
// nk = 5: Tile5b with the k-slice-outer DMMA order (the default); experiments (CSX_TILE_VARIANT
// 7 / 8): 2 CTAs / SM of 8 DMMA warps (64 x 64), row-outer and k-slice-outer (both slower)
using Tile5bk = TileCfg<5, 2, 4, 8, 8, 8, 2, 2, 1, 1, 1>;
using Tile5d = TileCfg<5, 2, 4, 8, 8, 4, 2, 3, 1, 2, 0>;
using Tile5dk = TileCfg<5, 2, 4, 8, 8, 4, 2, 3, 1, 2, 1>;
using Tile7c = TileCfg<7, 4, 2, 8, 4, 6, 2, 3, 2>;
using Tile7d = TileCfg<7, 4, 2, 8, 8, 2, 3, 3, 1, 2>;  // variant 3: 2 CTAs/SM of 6 DMMA warps (64 x 48)
using Tile7e = TileCfg<7, 4, 2, 8, 8, 2, 4, 2, 1, 2>;  // variant 4: 2 CTAs/SM of 8 DMMA warps (64 x 64)
using Tile7k = TileCfg<7, 4, 2, 8, 8, 4, 4, 2, 1, 1, 1>;  // variant 5: Tile7b, k-slice-outer DMMA order

// fused windows beyond the paper's one N fragment (reading A7): 8 DMMA warps, CTA 64 x 64,
// 3-stage ring; the K/4 weight fragments (30 / 42 / 56) stay in registers
using Tile9 = TileCfg<9, 2, 4, 12, 8, 4, 2, 3>;
using Tile11 = TileCfg<11, 4, 2, 12, 8, 2, 4, 3>;
using Tile13 = TileCfg<13, 2, 4, 16, 8, 4, 2, 3>;

static int tile_variant() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("CSX_TILE_VARIANT");
    v = e ? atoi(e) : 1;
  }
  return v;
}

// ------------------------------------------------------------------------------------------
// 3D (Tf = 1, P.1788-1800): out[z] = sum_dz Conv2D(in[z + dz - R], W[dz]).  The producer warp
// streams the input planes of a (y, x) tile and a z chunk through a STAGES-deep plane ring; the
// DMMA warps compute output plane zo from the NK staged planes zo-R .. zo+R (every tensor-core z
// offset is a K-slice group of the same GEMM; single-tap z offsets — the star arms, reading A9 —
// are DFMAs on the same staged planes), then release plane zo-R, which no later output needs.
//
// Radius 2 / 3 (nk = 5 / 7, §8(f)#2) use the same kernel with the planner's block shape for the
// window (2x4 for nk = 5, 4x2 for nk = 7: the smaller K, as in 2D) and, where NK x KS weight
// fragments would not fit the register file (WREG = 0, nk = 7: 7 x 20), each TC plane's KS
// fragments loaded from L1 just before its GEMM (KS loads per G*KS DMMAs).
// TPX: extra staged columns (a row pitch whose bank offset keeps the star planes' DFMA loads
// conflict-free); CM: column-major numbering of the a x b output block in the DMMA N dimension
// (n -> alpha = n % a, beta = n / a, only a = 2), so a lane's two accumulators are vertically
// adjacent and the DFMA planes load them as two conflict-free LDS.64 rows instead of one
// 2-way-conflicted LDS.128 (round 2: 36 M smem load conflicts per Star-3D13P launch).
template <int NK_, int G_, int WM_, int WN_, int STAGES_, int ZCH_, int CG_ = 1, int KO_ = 0,
          int A_ = 4, int B_ = 2, int WREG_ = 1, int TPX_ = 0, int CM_ = 0, int MINB_ = 0>
struct Tile3DCfg {
  // resident CTAs per SM the register budget is sized for (0: 1 above 4 DMMA warps, else 2)
  static constexpr int MINB = MINB_ ? MINB_ : (WM_ * WN_ > 4 ? 1 : 2);
  static constexpr int NK = NK_, A = A_, B = B_, KC = 4 * ((B_ + NK - 1 + 3) / 4), G = G_, WM = WM_,
                       WN = WN_, STAGES = STAGES_, ZCH = ZCH_, CG = CG_;
  static constexpr int WREG = WREG_;  // 1: all planes' weight fragments live in registers
  // DMMA issue order inside a TC plane: 0 = by input row (an A fragment feeds every block whose
  // window holds the row; consecutive DMMAs often hit the same accumulator chain), 1 = k-slice
  // outer, blocks inner (G independent chains between dependent DMMAs; one LDS per DMMA)
  static constexpr int KO = KO_;
  static constexpr int R = (NK - 1) / 2;
  static constexpr int ODD = R & 1;  // staged col = region col + ODD (16-B aligned rows)
  static constexpr int KR = A + NK - 1;
  static constexpr int KS = KR * KC / 4;
  static constexpr int BM = WM * A * G;
  static constexpr int WC = CG * 8 * B;             // output cols per warp (CG column groups)
  static constexpr int BN = WN * WC;
  static constexpr int RR = BM + NK - 1;
  static constexpr int TP = ((ODD + BN + KC - B) + 1) / 2 * 2 + TPX_;
  static constexpr int CM = CM_;
  static_assert(!CM || (A == 2 && CG == 1), "column-major block numbering: a = 2 only");
  static constexpr int STAGE = RR * TP;
  static constexpr int STAGE_A = (STAGE + 15) / 16 * 16;  // ring slot (128-B aligned)
  static constexpr int NCW = WM * WN;
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int SMEM = STAGES * STAGE_A * 8 + 128;
  static_assert(STAGES >= NK + 1, "plane ring must hold NK planes plus one in flight");
  static_assert(TP <= 256 && RR <= 256, "TMA box dimensions");
};

__device__ unsigned long long g_lock_ctr[1];  // CSX_LOCKSTEP experiment counter

template <class C>
__device__ __forceinline__ void issue_plane(const S2RArgs& a, const CUtensorMap* tmap, int ty, int tx,
                                            int64_t zi, double* stage, uint64_t* bar, int lane) {
  if (lane == 0) {
    mbar_expect_tx(bar, (uint32_t)(C::STAGE * 8));
    if (a.l2hint)
      tma_load_3d_hint(stage, tmap, bar, (int)(a.tma_x0 + tx * C::BN - C::R - C::ODD),
                       (int)(a.tma_y0 + (int64_t)ty * C::BM - C::R), (int)(a.tma_z0 + zi),
                       a.l2hint == 2 ? 2 : 1);
    else
      tma_load_3d(stage, tmap, bar, (int)(a.tma_x0 + tx * C::BN - C::R - C::ODD),
                  (int)(a.tma_y0 + (int64_t)ty * C::BM - C::R), (int)(a.tma_z0 + zi));
  }
}

__device__ __forceinline__ int ring_next(int s, int n) { return s + 1 == n ? 0 : s + 1; }

template <class C, bool ONE = false>  // ONE: a single TC plane (star shapes)
__global__ void __launch_bounds__(C::NT, C::MINB)
    k_tile3d(S2RArgs a, int tc_mask, const __grid_constant__ CUtensorMap tmap) {
  extern __shared__ __align__(128) double smem_raw[];
  double* smem = ring_base(smem_raw);
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
  pdl_begin();  // PDL: let the next pass launch; wait for the previous pass's writes
  const int ncol = a.tiles_x * a.tiles_y;
  if (warp == C::NCW) {  // producer: planes of every work item, in consumption order
    if (lane == 0) tma_prefetch_desc(&tmap);
    int s = 0, round = 0;  // ring slot and how many times the ring has been filled
    // CSX_LOCKSTEP=k (experiment): producers of all CTAs meet every k plane slots so that
    // neighbouring tiles' halo planes are fetched while they are still in L2.  Every CTA walks the
    // same schedule of (item round, plane slot) pairs, arriving also for the slots it has no
    // plane for (last round, short last z chunk), so the counts match.
    const int64_t rounds = (a.ntiles + gridDim.x - 1) / gridDim.x;
    unsigned long long q = 0;
    for (int64_t rr = 0; rr < rounds; ++rr) {
      const int64_t item = blockIdx.x + rr * gridDim.x;
      const bool has = item < a.ntiles;
      int ty = 0, tx = 0;
      int64_t z0 = 0, z1 = 0;
      if (has) {
        const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
        const int64_t zc = slab_map(a, zcl);
        ty = tile / a.tiles_x;
        tx = tile - ty * a.tiles_x;
        z0 = zc * C::ZCH;
        z1 = min(a.E0, z0 + C::ZCH);
      }
      const int64_t nsl = a.lockstep > 0 ? (int64_t)C::ZCH + 2 * C::R : (has ? z1 - z0 + 2 * C::R : 0);
      for (int64_t p = 0; p < nsl; ++p) {
        const int64_t zi = z0 - C::R + p;
        const bool real = has && zi < z1 + C::R;
        if (a.lockstep > 0 && (++q % a.lockstep) == 0) {
          if (lane == 0) {
            atomicAdd(g_lock_ctr, 1ull);
            const unsigned long long target = (q / a.lockstep) * gridDim.x;
            unsigned long long v;
            do {
              asm volatile("ld.acquire.gpu.global.u64 %0, [%1];\n" : "=l"(v) : "l"(g_lock_ctr) : "memory");
            } while (v < target);
          }
          __syncwarp();
        }
        if (!real) continue;
        if (round > 0) mbar_wait(&empty[s], (uint32_t)((round - 1) & 1));
        issue_plane<C>(a, &tmap, ty, tx, zi, smem + s * C::STAGE_A, &full[s], lane);
        if (++s == C::STAGES) {
          s = 0;
          ++round;
        }
      }
    }
    return;
  }
  const int wm = warp / C::WN, wn = warp - (warp / C::WN) * C::WN;
  const int g = lane >> 2, t = lane & 3;
  double wf[C::WREG ? C::NK : 1][C::KS];
  double wz[C::NK];
#pragma unroll
  for (int p = 0; p < C::NK; ++p) {
    if (C::WREG)
#pragma unroll
      for (int k = 0; k < C::KS; ++k) wf[C::WREG ? p : 0][k] = a.frags[(p * C::KS + k) * 32 + lane];
    wz[p] = a.wc[(p * C::NK + C::R) * C::NK + C::R];
  }
  // star shapes have one TC plane (the centre): its fragments stay in registers for the launch
  constexpr bool single_tc = ONE;
  if (!C::WREG && single_tc) {
    const int dz1 = __ffs(tc_mask) - 1;
#pragma unroll
    for (int k = 0; k < C::KS; ++k) wf[0][k] = __ldg(a.frags + (dz1 * C::KS + k) * 32 + lane);
  }
  // CM: B-fragment lane (k = lane % 4, n' = lane / 4) takes the planner's column n = alpha * b +
  // beta of its output (alpha, beta) = (n' % 2, n' / 2)
  const int cm_src = (lane & 3) + 4 * (((lane >> 2) & 1) * C::B + (lane >> 3));
  if (C::CM) {
    if (C::WREG) {
#pragma unroll
      for (int p = 0; p < C::NK; ++p)
#pragma unroll
        for (int k = 0; k < C::KS; ++k) wf[C::WREG ? p : 0][k] = __shfl_sync(0xffffffffu, wf[C::WREG ? p : 0][k], cm_src);
    } else if (single_tc) {
#pragma unroll
      for (int k = 0; k < C::KS; ++k) wf[0][k] = __shfl_sync(0xffffffffu, wf[0][k], cm_src);
    }
  }
  // this lane's accumulator e sits at block position (alpha + e * CM, beta + e * (1 - CM))
  const int alpha = C::CM ? 0 : (2 * t) / C::B, beta = C::CM ? t : (2 * t) % C::B;
  const bool any_cuda = tc_mask != (1 << C::NK) - 1;
  uint64_t spol = 0;
  if (a.l2hint == 3) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(spol));
  const bool aligned = a.dst_aligned != 0;
  // ring position / phase of the next plane this warp consumes (planes are consumed in issue
  // order, so slot = sequence number mod STAGES and phase = (sequence / STAGES) & 1)
  int cs = 0;
  uint32_t cph = 0;
  // lane-invariant offsets inside a staged plane
  const int lane_off = (wm * C::A * C::G) * C::TP + wn * C::WC + C::ODD + C::B * g + t;
  const int frame_off = (wm * C::A * C::G + alpha + C::R) * C::TP + wn * C::WC + C::B * g + beta +
                        C::R + C::ODD;
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
    const int64_t zc = slab_map(a, zcl);
    const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
    const int64_t z0 = zc * C::ZCH, z1 = min(a.E0, z0 + C::ZCH);
    const int64_t col0 = (int64_t)tx * C::BN + wn * C::WC + C::B * g + beta;
    const int64_t row0 = (int64_t)ty * C::BM + wm * C::A * C::G + alpha;
    const bool full_tile = aligned && (int64_t)(ty + 1) * C::BM <= a.E1 && (int64_t)(tx + 1) * C::BN <= a.E2;
    const bool tile_edge = a.hold_frame &&
                           ((int64_t)ty * C::BM + a.gorg1 < C::R || (int64_t)(ty + 1) * C::BM + a.gorg1 > a.GE1 - C::R ||
                            (int64_t)tx * C::BN + a.gorg2 < C::R || (int64_t)(tx + 1) * C::BN + a.gorg2 > a.GE2 - C::R);
    // slots of the NK planes zo-R .. zo+R of the current output plane
    int slot[C::NK];
    uint32_t sph[C::NK];
    slot[0] = cs;
    sph[0] = cph;
#pragma unroll
    for (int k = 1; k < C::NK; ++k) {
      slot[k] = ring_next(slot[k - 1], C::STAGES);
      sph[k] = slot[k] == 0 ? sph[k - 1] ^ 1 : sph[k - 1];
    }
#pragma unroll
    for (int k = 0; k < C::NK - 1; ++k) mbar_wait(&full[slot[k]], sph[k]);
    for (int64_t zo = z0; zo < z1; ++zo) {
      mbar_wait(&full[slot[C::NK - 1]], sph[C::NK - 1]);  // newest plane zo + R
      double acc[C::CG][C::G][2];
#pragma unroll
      for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
        for (int j = 0; j < C::G; ++j) acc[cg][j][0] = acc[cg][j][1] = 0.0;
      if constexpr (C::KO == 2) {
        // KO = 2 (box shapes, every plane on the tensor cores, weights in registers): input
        // rows outer as in KO = 0 (one A fragment per plane and row feeds every block whose
        // window holds the row), but the NK planes interleaved with one accumulator set each,
        // so consecutive DMMAs belong to NK independent chains instead of one (the KO = 0
        // schedule issued up to 5 dependent DMMAs back to back); summed at the end
        double accz[C::NK][C::CG][C::G][2];
#pragma unroll
        for (int dz = 0; dz < C::NK; ++dz)
#pragma unroll
          for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
            for (int j = 0; j < C::G; ++j) accz[dz][cg][j][0] = accz[dz][cg][j][1] = 0.0;
#pragma unroll
        for (int ra = 0; ra < C::A * C::G + C::NK - 1; ++ra) {
          double f[C::NK][C::CG][C::KC / 4];
#pragma unroll
          for (int dz = 0; dz < C::NK; ++dz)
#pragma unroll
            for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
              for (int h = 0; h < C::KC / 4; ++h)
                f[dz][cg][h] = smem[slot[dz] * C::STAGE_A + lane_off + ra * C::TP + cg * 8 * C::B + 4 * h];
#pragma unroll
          for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
            for (int j = 0; j < C::G; ++j) {
              const int rho = ra - C::A * j;
              if (rho >= 0 && rho < C::KR)
#pragma unroll
                for (int dz = 0; dz < C::NK; ++dz)
#pragma unroll
                  for (int cg = 0; cg < C::CG; ++cg)
                    dmma_t(accz[dz][cg][j][0], accz[dz][cg][j][1], f[dz][cg][h],
                           wf[C::WREG ? dz : 0][rho * (C::KC / 4) + h]);
            }
        }
#pragma unroll
        for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
          for (int j = 0; j < C::G; ++j)
#pragma unroll
            for (int e = 0; e < 2; ++e) {
              double v = accz[0][cg][j][e];
#pragma unroll
              for (int dz = 1; dz < C::NK; ++dz) v += accz[dz][cg][j][e];
              acc[cg][j][e] = v;
            }
      }
#pragma unroll
      for (int dz = 0; dz < (C::KO == 2 ? 0 : C::NK); ++dz) {
        const double* stg = smem + slot[dz] * C::STAGE_A;
        if (!C::WREG && !single_tc && (tc_mask & (1 << dz))) {  // this plane's fragments, from L1
#pragma unroll
          for (int k = 0; k < C::KS; ++k) {
            wf[0][k] = __ldg(a.frags + (dz * C::KS + k) * 32 + lane);
            if (C::CM) wf[0][k] = __shfl_sync(0xffffffffu, wf[0][k], cm_src);
          }
        }
        const int wp = C::WREG ? dz : 0;
        if ((tc_mask & (1 << dz)) && C::KO == 1) {
          const double* base = stg + lane_off;
#pragma unroll
          for (int rho = 0; rho < C::KR; ++rho)
#pragma unroll
            for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
              for (int j = 0; j < C::G; ++j)
#pragma unroll
                for (int cg = 0; cg < C::CG; ++cg)
                  dmma_t(acc[cg][j][0], acc[cg][j][1],
                         base[(C::A * j + rho) * C::TP + cg * 8 * C::B + 4 * h],
                         wf[wp][rho * (C::KC / 4) + h]);
        } else if (tc_mask & (1 << dz)) {
          const double* base = stg + lane_off;
#pragma unroll
          for (int ra = 0; ra < C::A * C::G + C::NK - 1; ++ra) {
            double f[C::CG][C::KC / 4];
#pragma unroll
            for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
              for (int h = 0; h < C::KC / 4; ++h) f[cg][h] = base[ra * C::TP + cg * 8 * C::B + 4 * h];
#pragma unroll
            for (int h = 0; h < C::KC / 4; ++h)
#pragma unroll
              for (int j = 0; j < C::G; ++j) {
                const int rho = ra - C::A * j;
                if (rho >= 0 && rho < C::KR)
#pragma unroll
                  for (int cg = 0; cg < C::CG; ++cg)
                    dmma_t(acc[cg][j][0], acc[cg][j][1], f[cg][h], wf[wp][rho * (C::KC / 4) + h]);
              }
          }
        } else if (any_cuda && wz[dz] != 0.0) {
#pragma unroll
          for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
            for (int j = 0; j < C::G; ++j) {
              if (C::CM) {  // vertically adjacent pair: two conflict-free row loads
                const double* q = stg + frame_off + C::A * j * C::TP;
                acc[cg][j][0] = fma(wz[dz], q[0], acc[cg][j][0]);
                acc[cg][j][1] = fma(wz[dz], q[C::TP], acc[cg][j][1]);
              } else {
                const double2 v = *reinterpret_cast<const double2*>(stg + frame_off + C::A * j * C::TP + cg * 8 * C::B);
                acc[cg][j][0] = fma(wz[dz], v.x, acc[cg][j][0]);
                acc[cg][j][1] = fma(wz[dz], v.y, acc[cg][j][1]);
              }
            }
        }
      }
      // FIXED frame (held points) of this output plane: the staged plane zo (dz = R) holds them
      const int64_t gzo = zo + a.gorg0;
      const bool plane_frame = a.hold_frame && (gzo < C::R || gzo >= a.GE0 - C::R);
      double* plane = a.dst.p + zo * a.dst.s0;
      if (full_tile && !tile_edge && !plane_frame) {  // interior: unguarded 16-B stores
        double* p0 = plane + row0 * a.dst.s1 + col0;
#pragma unroll
        for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
          for (int j = 0; j < C::G; ++j) {
            if (C::CM) {  // rows row0 + A j and + 1: each warp store covers 32 consecutive columns
              st_out1(p0 + (int64_t)(C::A * j) * a.dst.s1, acc[cg][j][0], a.l2hint == 3, spol);
              st_out1(p0 + (int64_t)(C::A * j + 1) * a.dst.s1, acc[cg][j][1], a.l2hint == 3, spol);
            } else {
              st_out(p0 + (int64_t)(C::A * j) * a.dst.s1 + cg * 8 * C::B, acc[cg][j][0], acc[cg][j][1],
                     a.l2hint == 3, spol);
            }
          }
      } else {
        const double* cstg = smem + slot[C::R] * C::STAGE_A;
        const bool edge = tile_edge || plane_frame;
#pragma unroll
        for (int cg = 0; cg < C::CG; ++cg)
#pragma unroll
          for (int j = 0; j < C::G; ++j) {
            if constexpr (C::CM) {  // accumulator e at row + e, same column
#pragma unroll
              for (int e = 0; e < 2; ++e) {
                const int64_t row = row0 + C::A * j + e;
                const int64_t c = col0 + cg * 8 * C::B, gc = c + a.gorg2;
                if (row >= a.E1 || c >= a.E2) continue;
                const int64_t grow = row + a.gorg1;
                const bool rf = plane_frame || grow < C::R || grow >= a.GE1 - C::R;
                double v = acc[cg][j][e];
                if (edge && (rf || gc < C::R || gc >= a.GE2 - C::R))
                  v = cstg[frame_off + (C::A * j + e) * C::TP + cg * 8 * C::B];
                plane[row * a.dst.s1 + c] = v;
              }
            } else {
              const int64_t row = row0 + C::A * j, col = col0 + cg * 8 * C::B;
              if (row >= a.E1 || col >= a.E2) continue;
              double* p = plane + row * a.dst.s1 + col;
              const int64_t grow = row + a.gorg1;
              const bool rf = plane_frame || grow < C::R || grow >= a.GE1 - C::R;
#pragma unroll
              for (int e = 0; e < 2; ++e) {
                const int64_t c = col + e, gc = c + a.gorg2;
                if (c >= a.E2) continue;
                double v = acc[cg][j][e];
                if (edge && (rf || gc < C::R || gc >= a.GE2 - C::R))
                  v = cstg[frame_off + C::A * j * C::TP + cg * 8 * C::B + e];
                p[e] = v;
              }
            }
          }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot[0]]);  // plane zo-R is done
      // advance the window by one plane
#pragma unroll
      for (int k = 0; k < C::NK - 1; ++k) {
        slot[k] = slot[k + 1];
        sph[k] = sph[k + 1];
      }
      slot[C::NK - 1] = ring_next(slot[C::NK - 2], C::STAGES);
      sph[C::NK - 1] = slot[C::NK - 1] == 0 ? sph[C::NK - 2] ^ 1 : sph[C::NK - 2];
    }
    // release the last 2R planes of the item (not released by an output plane)
    __syncwarp();
    if (lane == 0)
#pragma unroll
      for (int k = 0; k < C::NK - 1; ++k) mbar_arrive(&empty[slot[k]]);
    cs = slot[C::NK - 1];
    cph = sph[C::NK - 1];
  }
}

// ------------------------------------------------------------------------------------------
// 3D, two fused time steps by temporal blocking in shared memory (Tf = 2, base radius 1).
// Composing W twice (the 2D path's kernel fusion, P.1466-1482) would turn the single-tap z arms
// of a star stencil into 5-tap planes that need the tensor cores (3 TC planes of nk = 5: 3x the
// DMMAs of Tf = 1 per step).  Instead each pass streams the input planes once and runs the BASE
// stencil twice: level 1 computes step-1 planes on the tile grown by one cell (its own GEMM
// tiling, 36 x 80 for a 32 x 64 output tile) into a 3-plane shared-memory ring, level 2 computes
// the outputs from that ring — the same per-plane GEMM (4x2 output blocks on DMMA.8x8x4,
// single-tap planes as DFMA) at both levels.  HBM traffic per step halves; DMMAs per step grow
// by the recomputed halo (~1.2x).  FIXED: both levels hold the frame, so no band fix-up.
struct Tile3DTB {
  static constexpr int NK = 3, R = 1, A = 4, B = 2, KC = 4, KR = 6, KS = 6;
  static constexpr int WM = 2, WN = 4, NCW = 8, NT = 32 * (NCW + 1);
  static constexpr int G2 = 4;                  // level-2 blocks per warp (column)
  static constexpr int BM = WM * A * G2;        // 32 output rows
  static constexpr int BN = WN * 8 * B;         // 64 output cols
  static constexpr int G1 = 3;                  // level-1 blocks per unit
  static constexpr int U1R = 3, U1C = 5;        // level-1 units: 3 block-row groups x 5 col groups
  static constexpr int BM1 = U1R * A * G1;      // 36 >= BM + 2 step-1 rows
  static constexpr int BN1 = U1C * 8 * B;       // 80 >= BN + 3 step-1 cols
  static constexpr int TP = 84;                 // plane pitch (input and step-1), even
  static constexpr int RIN = BM1 + 2;           // staged input rows (38)
  static constexpr int SIN = RIN * TP;          // doubles per input plane
  static constexpr int SIN_A = (SIN + 15) / 16 * 16;
  static constexpr int SL1 = BM1 * TP;          // doubles per step-1 plane
  static constexpr int SL1_A = (SL1 + 15) / 16 * 16;
  static constexpr int STAGES = 4;              // input ring
  static constexpr int L1S = 4;                 // step-1 plane ring
  static constexpr int ZCH = 32;
  static constexpr int H = 2;                   // halo of the pass (R * Tf)
  static constexpr int SMEM = (STAGES * SIN_A + L1S * SL1_A) * 8 + 128;
  static_assert(TP >= 8 * B * U1C + 4 && TP <= 256 && RIN <= 256, "plane geometry");
};

// One z-window GEMM of G output blocks (4 x 2 each) for a warp: out rows r0 + 4j + alpha, cols
// c0 + 2g + beta (+e) of the destination grid whose staged planes `pl[dz]` hold its inputs at
// (row + dy, col + 1 + dx) (level 1: input planes; level 2: step-1 planes).  TC planes on DMMA,
// single-tap planes (star z arms) as DFMA on the centre cell.
template <int G>
__device__ __forceinline__ void tb_window(double (&acc)[G][2], const double* const (&pl)[3], int r0, int c0,
                                          int tc_mask, const double (&wf)[3][Tile3DTB::KS],
                                          const double (&wz)[3], int lane) {
  using C = Tile3DTB;
  const int g = lane >> 2, t = lane & 3;
  const int alpha = (2 * t) / C::B, beta = (2 * t) % C::B;
#pragma unroll
  for (int j = 0; j < G; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
  for (int dz = 0; dz < 3; ++dz) {
    if (tc_mask & (1 << dz)) {
      const double* base = pl[dz] + r0 * C::TP + c0 + 1 + C::B * g + t;
#pragma unroll
      for (int rho = 0; rho < C::KR; ++rho)
#pragma unroll
        for (int j = 0; j < G; ++j)
          dmma_t(acc[j][0], acc[j][1], base[(C::A * j + rho) * C::TP], wf[dz][rho]);
    } else if (wz[dz] != 0.0) {
#pragma unroll
      for (int j = 0; j < G; ++j) {
        const double2 v = *reinterpret_cast<const double2*>(
            pl[dz] + (r0 + C::A * j + alpha + C::R) * C::TP + c0 + C::B * g + beta + C::R + 1);
        acc[j][0] = fma(wz[dz], v.x, acc[j][0]);
        acc[j][1] = fma(wz[dz], v.y, acc[j][1]);
      }
    }
  }
}

__global__ void __launch_bounds__(Tile3DTB::NT, 1)
    k_tile3d_tb(S2RArgs a, int tc_mask, const __grid_constant__ CUtensorMap tmap) {
  using C = Tile3DTB;
  extern __shared__ __align__(128) double smem_raw[];
  double* smem = ring_base(smem_raw);
  double* l1 = smem + C::STAGES * C::SIN_A;  // L1S step-1 planes
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
  pdl_begin();
  const int ncol = a.tiles_x * a.tiles_y;
  if (warp == C::NCW) {  // producer: input planes z0-2 .. z1+1 of every work item
    if (lane == 0) tma_prefetch_desc(&tmap);
    int q = 0;
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
      const int64_t zc = slab_map(a, zcl);
      const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
      const int64_t z0 = zc * C::ZCH, z1 = min(a.E0, z0 + C::ZCH);
      for (int64_t zi = z0 - C::H; zi < z1 + C::H; ++zi, ++q) {
        const int s = q % C::STAGES, n = q / C::STAGES;
        if (n > 0) mbar_wait(&empty[s], (uint32_t)((n - 1) & 1));
        if (lane == 0) {
          mbar_expect_tx(&full[s], (uint32_t)(C::SIN * 8));
          tma_load_3d(smem + s * C::SIN_A, &tmap, &full[s], (int)(a.tma_x0 + (int64_t)tx * C::BN - 4),
                      (int)(a.tma_y0 + (int64_t)ty * C::BM - 2), (int)(a.tma_z0 + zi));
        }
      }
    }
    return;
  }
  double wf[3][C::KS], wz[3];
#pragma unroll
  for (int p = 0; p < 3; ++p) {
#pragma unroll
    for (int k = 0; k < C::KS; ++k) wf[p][k] = a.frags[(p * C::KS + k) * 32 + lane];
    wz[p] = a.wc[(p * 3 + 1) * 3 + 1];
  }
  const int g = lane >> 2, t = lane & 3;
  const int alpha = (2 * t) / C::B, beta = (2 * t) % C::B;
  const bool fixed = a.hold_frame != 0;
  // level-2 unit of this warp: block rows wm*G2.., column group wn
  const int wm = warp / C::WN, wn = warp - (warp / C::WN) * C::WN;
  int q = 0;  // sequence number of the next input plane (producer order)
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
    const int64_t zc = slab_map(a, zcl);
    const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
    const int64_t z0 = zc * C::ZCH, z1 = min(a.E0, z0 + C::ZCH);
    const int64_t y0 = (int64_t)ty * C::BM, x0 = (int64_t)tx * C::BN;
    // global origin of the tile (FIXED holds use global coordinates)
    const int64_t gy0 = y0 + a.gorg1, gx0 = x0 + a.gorg2;
    const bool tile_edge = fixed && (gy0 < 2 || gy0 + C::BM + 1 > a.GE1 - 1 || gx0 < 2 ||
                                     gx0 + C::BN + 1 > a.GE2 - 1);
    // input planes zl-1, zl, zl+1 for step-1 plane zl: sequence numbers q0 + (zl - (z0-2)) ...
    const int q0 = q;
    auto in_plane = [&](int64_t zi) -> const double* {
      return smem + ((q0 + (int)(zi - (z0 - C::H))) % C::STAGES) * C::SIN_A;
    };
    auto wait_in = [&](int64_t zi) {
      const int qq = q0 + (int)(zi - (z0 - C::H));
      mbar_wait(&full[qq % C::STAGES], (uint32_t)((qq / C::STAGES) & 1));
    };
    auto release_in = [&]() {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[q % C::STAGES]);
      ++q;
    };
    wait_in(z0 - 2);
    wait_in(z0 - 1);
    auto l1_plane = [&](int64_t zl) { return l1 + (int)((zl - (z0 - 1)) % C::L1S) * C::SL1_A; };
    // Phase k: level 1 writes step-1 plane k (inputs k-1..k+1), level 2 writes output plane k-2
    // (step-1 planes k-3..k-1, finished in earlier phases); the 4-plane step-1 ring keeps the
    // two apart, so one barrier per phase orders everything.
    for (int64_t k = z0 - 1; k <= z1 + 1; ++k) {
      if (k <= z1) {
        wait_in(k + 1);
        // ---- level 1: step-1 plane k on the grown tile (rows y0-1 .., cols x0-2 ..) ----
        const double* pin[3] = {in_plane(k - 1), in_plane(k), in_plane(k + 1)};
        double* dl1 = l1_plane(k);
        const int64_t gz1 = k + a.gorg0;
        const bool zf1 = fixed && (gz1 < 1 || gz1 >= a.GE0 - 1);
        for (int u = warp; u < C::U1R * C::U1C; u += C::NCW) {
          const int ur = u / C::U1C, uc = u - (u / C::U1C) * C::U1C;
          const int r0 = ur * C::A * C::G1, c0 = uc * 8 * C::B;
          double acc[C::G1][2];
          tb_window<C::G1>(acc, pin, r0, c0, tc_mask, wf, wz, lane);
#pragma unroll
          for (int j = 0; j < C::G1; ++j) {
            const int r = r0 + C::A * j + alpha, c = c0 + C::B * g + beta;  // step-1 plane coords
            double v0 = acc[j][0], v1 = acc[j][1];
            if (fixed && (zf1 || tile_edge)) {  // held frame points keep the input value
              const int64_t gy = gy0 - 1 + r, gx = gx0 - 2 + c;
              const double* ctr = pin[1] + (r + 1) * C::TP + c + 2;
              const bool yf = zf1 || gy < 1 || gy >= a.GE1 - 1;
              if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
              if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
            }
            *reinterpret_cast<double2*>(dl1 + r * C::TP + c) = make_double2(v0, v1);
          }
        }
        release_in();  // input plane k-1 is not read again
      }
      // ---- level 2: output plane zo = k-2 from step-1 planes k-3, k-2, k-1 ----
      const int64_t zo = k - 2;
      if (zo >= z0) {
        const double* p1[3] = {l1_plane(k - 3), l1_plane(k - 2), l1_plane(k - 1)};
        const int r0 = wm * C::A * C::G2, c0 = wn * 8 * C::B;
        double acc[C::G2][2];
        tb_window<C::G2>(acc, p1, r0, c0, tc_mask, wf, wz, lane);
        const int64_t gzo = zo + a.gorg0;
        const bool zf = fixed && (gzo < 1 || gzo >= a.GE0 - 1);
        double* plane = a.dst.p + zo * a.dst.s0;
#pragma unroll
        for (int j = 0; j < C::G2; ++j) {
          const int r = r0 + C::A * j + alpha, c = c0 + C::B * g + beta;  // output tile coords
          const int64_t row = y0 + r, col = x0 + c;
          if (row >= a.E1 || col >= a.E2) continue;
          double v0 = acc[j][0], v1 = acc[j][1];
          if (fixed && (zf || tile_edge)) {
            const double* ctr = p1[1] + (r + 1) * C::TP + c + 2;
            const int64_t gy = gy0 + r, gx = gx0 + c;
            const bool yf = zf || gy < 1 || gy >= a.GE1 - 1;
            if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
            if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
          }
          double* p = plane + row * a.dst.s1 + col;
          if (col + 1 < a.E2 && a.dst_aligned) {
            *reinterpret_cast<double2*>(p) = make_double2(v0, v1);
          } else {
            p[0] = v0;
            if (col + 1 < a.E2) p[1] = v1;
          }
        }
      }
      asm volatile("bar.sync 1, %0;\n" ::"n"(C::NCW * 32) : "memory");  // phase k complete
    }
    release_in();  // input planes z1, z1+1
    release_in();
  }
}

template <class C>
static cudaError_t launch_tile3d_tb(S2RArgs a, int tc_mask, cudaStream_t st) {
  a.dst_aligned = ((reinterpret_cast<uintptr_t>(a.dst.p) & 15) == 0) && (a.dst.s1 % 2 == 0) &&
                  (a.dst.s0 % 2 == 0);
  a.tiles_x = (int)((a.E2 + C::BN - 1) / C::BN);
  a.tiles_y = (int)((a.E1 + C::BM - 1) / C::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y * set_ranges(a, (a.E0 + C::ZCH - 1) / C::ZCH, C::ZCH, a.E0, C::H);
  if (a.ntiles == 0) return cudaSuccess;
  CUtensorMap tmap;
  if (!make_tmap(a, C::TP, C::RIN, &tmap)) return cudaErrorNotSupported;
  cudaError_t e = cudaFuncSetAttribute(k_tile3d_tb, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile3d_tb, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, k_tile3d_tb, grid, C::NT, C::SMEM, st, a, tc_mask, tmap);
}

// ------------------------------------------------------------------------------------------
// 3D Tf = 2 by temporal blocking, decoupled levels (round 2, k_tile3d_tb2; the default depth of
// 3D r = 1 stars): the same two-level computation as k_tile3d_tb, but level 1 and level 2 run on
// DIFFERENT warps that hand planes over through mbarriers instead of meeting at one CTA barrier
// per plane, so a slow warp of one level no longer stalls the other:
//   warp 17            producer: input planes -> IN-slot ring (TMA tensor copies)
//   warps 8 .. 16      level 1: step-1 plane k (one row of W1 DMMA tiles of 4 x 16 per warp) from
//                      input planes k-1 .. k+1 -> L1S-slot step-1 ring
//   warps 0 .. 7       level 2: output plane k-1 (one row of 4 tiles per warp) from step-1 planes
//                      k-2 .. k, stored to global memory
// Heat-3D 512^3: 313 GSt/s (round-1 k_tile3d_tb 215, Tf = 1 k_tile3d 293).  FIXED: both levels
// hold the frame (no band fix-up).
// BM: output tile rows (a multiple of 4).  BM = 28: 7 level-2 + 8 level-1 warps + the producer =
// 16 warps, 4 per SM sub-partition with equal DMMA work on each (BM = 32: 18 warps, the
// sub-partition holding warps 0, 4, 8, 12, 16 carries 138 DMMAs per plane against 108 on the
// others), and the smaller planes leave room for a 5-deep input ring.
// BAL (BM = 32 only): warp roles spread so the four SM sub-partitions (warp w runs on w mod 4)
// carry equal DMMA work: sub-partition 0's five warps 0, 4, 8, 12, 16 and warps 1, 2, 3 are the
// level-2 warps (24 DMMAs per plane each), warps 5-7, 9-11, 13-15 level 1 (30 each), warp 17
// the producer: 120 / 114 / 114 / 114 DMMAs per plane instead of 138 / 108 / 108 / 108.
template <int IN_ = 4, int L1S_ = 5, int WIDE_ = 1, int BM_ = 32, int BAL_ = 0>
struct Tile3DTB2 {
  static constexpr int BAL = BAL_;
  // BM = 16: two CTAs per SM (two independent level-1 / level-2 pipelines per SM)
  static constexpr int MINB = BM_ <= 16 ? 2 : 1;
  static constexpr int R = 1, A = 4, B = 2, KR = 6, KS = 6, H = 2, ZCH = 32;
  // WIDE = 1: 32 x 64 output tile, step-1 plane 36 x 80 (level-1 warps: 5 DMMA tiles each),
  //           inputs of output (row, col) at staged (row + dy, col + 1 + dx)   [OFF = 1]
  // WIDE = 0: 32 x 62 output tile, step-1 plane 36 x 64 (4 tiles each: both levels equal work),
  //           inputs at staged (row + dy, col + dx)                             [OFF = 0]
  // (measured: WIDE = 1 312.7 GSt/s on Heat-3D, WIDE = 0 281 despite 9 % fewer DMMAs per output)
  static constexpr int WIDE = WIDE_, OFF = WIDE_;
  static constexpr int BM = BM_, BN = WIDE_ ? 64 : 62;  // output tile (stored)
  static_assert(BM % 4 == 0, "output tile rows");
  static constexpr int W1 = WIDE_ ? 5 : 4;               // level-1 DMMA tiles per warp
  static constexpr int NL2 = BM / 4, NL1 = BM / 4 + 1;   // level-2 / level-1 warps
  static constexpr int NT = 32 * (NL2 + NL1 + 1);
  static constexpr int TP = WIDE_ ? 84 : 68;             // plane pitch (input and step-1)
  static constexpr int RIN = BM + 6, R1 = BM + 4;        // staged input rows, step-1 rows
  static constexpr int SIN = RIN * TP, SIN_A = (SIN + 15) / 16 * 16;
  static constexpr int SL1 = R1 * TP, SL1_A = (SL1 + 15) / 16 * 16;
  // ring slots: input (3 read + IN - 3 in flight) and step-1 (3 read + 1 written + slack);
  // measured: the step-1 slack matters, deeper input rings do not
  static constexpr int IN = IN_, L1S = L1S_;
  static constexpr int SMEM = (IN * SIN_A + L1S * SL1_A) * 8 + 128;
  static_assert(SMEM <= 227 * 1024, "shared memory");
};

// G DMMA tiles of 4 x 16 outputs side by side (columns c0 + 16 j) of a plane window whose staged
// planes pl[dz] hold the inputs of output (row, col) at (row + dy, col + OFF + dx), dy, dx in 0..2:
// TC planes on DMMA (4x2 output blocks, K = 24), single-tap planes as DFMA on the centre cell.
template <class C, int G, bool ONE>
__device__ __forceinline__ void tb_hwindow(double (&acc)[G][2], const double* const (&pl)[3], int r0, int c0,
                                           int tc_mask, const double (&wf)[ONE ? 1 : 3][6],
                                           const double (&wz)[3], int lane) {
  const int g = lane >> 2, t = lane & 3;
  const int alpha = (2 * t) / C::B, beta = (2 * t) % C::B;
#pragma unroll
  for (int j = 0; j < G; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
  for (int dz = 0; dz < 3; ++dz) {
    if (tc_mask & (1 << dz)) {
      const double* base = pl[dz] + r0 * C::TP + c0 + C::OFF + C::B * g + t;
#pragma unroll
      for (int rho = 0; rho < C::KR; ++rho)
#pragma unroll
        for (int j = 0; j < G; ++j) dmma_t(acc[j][0], acc[j][1], base[rho * C::TP + 16 * j], wf[ONE ? 0 : dz][rho]);
    } else if (wz[dz] != 0.0) {  // (an integer mask test here measured 12 % slower: code layout)
#pragma unroll
      for (int j = 0; j < G; ++j) {
        const double* v = pl[dz] + (r0 + alpha + C::R) * C::TP + c0 + 16 * j + C::B * g + beta + C::R + C::OFF;
        double v0, v1;
        if (C::OFF) {  // even centre column: one 16-B load
          const double2 w2 = *reinterpret_cast<const double2*>(v);
          v0 = w2.x;
          v1 = w2.y;
        } else {
          v0 = v[0];
          v1 = v[1];
        }
        acc[j][0] = fma(wz[dz], v0, acc[j][0]);
        acc[j][1] = fma(wz[dz], v1, acc[j][1]);
      }
    }
  }
}

template <bool ONE, class D>  // ONE: a single TC plane (star shapes): only its fragments in registers
__global__ void __launch_bounds__(D::NT, D::MINB)
    k_tile3d_tb2(S2RArgs a, int tc_mask, const __grid_constant__ CUtensorMap tmap) {
  extern __shared__ __align__(128) double smem_raw[];
  double* smem = ring_base(smem_raw);
  double* l1 = smem + D::IN * D::SIN_A;  // L1S step-1 planes
  __shared__ __align__(8) uint64_t in_full[D::IN], in_empty[D::IN], l1_full[D::L1S], l1_empty[D::L1S];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  // step-1 columns 64 .. TP-1 are read (by level 2's last DMMA tile, for outputs 62, 63, which
  // are not stored) but never written: keep them finite
  for (int i = tid; i < D::L1S * D::R1; i += D::NT) {
    double* row = l1 + (i / D::R1) * D::SL1_A + (i % D::R1) * D::TP;
    for (int c = 16 * D::W1; c < D::TP; ++c) row[c] = 0.0;
  }
  if (tid == 0) {
    for (int s = 0; s < D::IN; ++s) {
      mbar_init(&in_full[s], 1);
      mbar_init(&in_empty[s], D::NL1);
    }
    for (int s = 0; s < D::L1S; ++s) {
      mbar_init(&l1_full[s], D::NL1);
      mbar_init(&l1_empty[s], D::NL2);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  pdl_begin();
  const int ncol = a.tiles_x * a.tiles_y;
  // role: 0 level 2, 1 level 1, 2 producer; rb = the warp's row block within its level
  int role, rb;
  if constexpr (D::BAL) {
    static_assert(!D::BAL || (D::NL2 == 8 && D::NL1 == 9), "balanced roles: 18 warps");
    if (warp == 17) { role = 2; rb = 0; }
    else if ((warp & 3) == 0) { role = 0; rb = warp >> 2; }     // 0, 4, 8, 12, 16 -> 0 .. 4
    else if (warp < 4) { role = 0; rb = 4 + warp; }             // 1, 2, 3 -> 5, 6, 7
    else { role = 1; rb = warp - 5 - (warp - 5) / 4; }         // 5-7, 9-11, 13-15 -> 0 .. 8
  } else {
    role = warp == D::NL2 + D::NL1 ? 2 : warp >= D::NL2 ? 1 : 0;
    rb = role == 1 ? warp - D::NL2 : warp;
  }
  if (role == 2) {  // producer: input planes z0-2 .. z1+1 of every item
    if (lane == 0) tma_prefetch_desc(&tmap);
    int q = 0;
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
      const int64_t zc = slab_map(a, zcl);
      const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
      const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
      for (int64_t zi = z0 - D::H; zi < z1 + D::H; ++zi, ++q) {
        const int s = q % D::IN, n = q / D::IN;
        if (n > 0) mbar_wait(&in_empty[s], (uint32_t)((n - 1) & 1));
        if (lane == 0) {
          mbar_expect_tx(&in_full[s], (uint32_t)(D::SIN * 8));
          tma_load_3d(smem + s * D::SIN_A, &tmap, &in_full[s], (int)(a.tma_x0 + (int64_t)tx * D::BN - 2 - 2 * D::OFF),
                      (int)(a.tma_y0 + (int64_t)ty * D::BM - 2), (int)(a.tma_z0 + zi));
        }
      }
    }
    return;
  }
  double wf[ONE ? 1 : 3][D::KS], wz[3];
  const int dz1 = __ffs(tc_mask) - 1;
#pragma unroll
  for (int p = 0; p < (ONE ? 1 : 3); ++p)
#pragma unroll
    for (int k = 0; k < D::KS; ++k) wf[p][k] = a.frags[((ONE ? dz1 : p) * D::KS + k) * 32 + lane];
#pragma unroll
  for (int p = 0; p < 3; ++p) wz[p] = a.wc[(p * 3 + 1) * 3 + 1];
  const int g = lane >> 2, t = lane & 3;
  const int alpha = (2 * t) / D::B, beta = (2 * t) % D::B;
  const bool fixed = a.hold_frame != 0;
  if (role == 1) {
    // ---------------- level 1: step-1 planes ----------------
    // rb: step-1 rows 4 rb .. 4 rb + 3, cols 0 .. 16 W1 - 1
    int q = 0, p = 0;              // input / step-1 plane sequence numbers
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
      const int64_t zc = slab_map(a, zcl);
      const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
      const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
      // global origin of the step-1 plane: (y0 - 1, x0 - 1 - OFF)
      const int64_t sy0 = (int64_t)ty * D::BM + a.gorg1 - 1, sx0 = (int64_t)tx * D::BN + a.gorg2 - 1 - D::OFF;
      const bool tile_edge =
          fixed && (sy0 < 1 || sy0 + D::R1 > a.GE1 - 1 || sx0 < 1 || sx0 + 16 * D::W1 > a.GE2 - 1);
      const int q0 = q;  // input plane z0-2 of this item
      auto in_slot = [&](int qq) { return smem + (qq % D::IN) * D::SIN_A; };
      mbar_wait(&in_full[q0 % D::IN], (uint32_t)((q0 / D::IN) & 1));
      mbar_wait(&in_full[(q0 + 1) % D::IN], (uint32_t)(((q0 + 1) / D::IN) & 1));
      // step-1 plane k (k = z0-1 .. z1) from input planes k-1, k, k+1 (sequence q0 + j, +1, +2)
      for (int64_t k = z0 - 1; k <= z1; ++k, ++p) {
        const int j = (int)(k - (z0 - 1));
        mbar_wait(&in_full[(q0 + j + 2) % D::IN], (uint32_t)(((q0 + j + 2) / D::IN) & 1));
        const int sl = p % D::L1S, nl = p / D::L1S;
        if (nl > 0) mbar_wait(&l1_empty[sl], (uint32_t)((nl - 1) & 1));
        const double* pin[3] = {in_slot(q0 + j), in_slot(q0 + j + 1), in_slot(q0 + j + 2)};
        double* dl1 = l1 + sl * D::SL1_A;
        double acc[D::W1][2];
        tb_hwindow<D, D::W1, ONE>(acc, pin, 4 * rb, 0, tc_mask, wf, wz, lane);
        const int64_t gz1 = k + a.gorg0;
        const bool zf1 = fixed && (gz1 < 1 || gz1 >= a.GE0 - 1);
#pragma unroll
        for (int jj = 0; jj < D::W1; ++jj) {
          const int r = 4 * rb + alpha, c = 16 * jj + D::B * g + beta;  // step-1 plane coords
          double v0 = acc[jj][0], v1 = acc[jj][1];
          if (fixed && (zf1 || tile_edge)) {  // held frame points keep the input value
            const int64_t gy = sy0 + r, gx = sx0 + c;
            const double* ctr = pin[1] + (r + 1) * D::TP + c + 1 + D::OFF;
            const bool yf = zf1 || gy < 1 || gy >= a.GE1 - 1;
            if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
            if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
          }
          *reinterpret_cast<double2*>(dl1 + r * D::TP + c) = make_double2(v0, v1);
        }
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&l1_full[sl]);                    // this warp's rows of plane k written
          mbar_arrive(&in_empty[(q0 + j) % D::IN]);     // input plane k-1 no longer read
        }
      }
      __syncwarp();
      if (lane == 0) {  // input planes z1, z1+1 (read by the last step-1 plane only)
        mbar_arrive(&in_empty[(q0 + (int)(z1 - z0) + 2) % D::IN]);
        mbar_arrive(&in_empty[(q0 + (int)(z1 - z0) + 3) % D::IN]);
      }
      q = q0 + (int)(z1 - z0) + 4;
    }
    return;
  }
  // ---------------- level 2: output planes ----------------
  // rb: output rows 4 rb .. 4 rb + 3, cols 0 .. 63 (BN stored)
  int p = 0;            // step-1 plane sequence number
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
    const int64_t zc = slab_map(a, zcl);
    const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
    const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
    const int64_t y0 = (int64_t)ty * D::BM, x0 = (int64_t)tx * D::BN;
    const int64_t gy0 = y0 + a.gorg1, gx0 = x0 + a.gorg2;
    const bool tile_edge = fixed && (gy0 < 1 || gy0 + D::BM > a.GE1 - 1 || gx0 < 1 || gx0 + D::BN > a.GE2 - 1);
    const int p0 = p;  // step-1 plane z0-1 of this item
    auto l1_slot = [&](int pp) { return l1 + (pp % D::L1S) * D::SL1_A; };
    auto l1_wait = [&](int pp) { mbar_wait(&l1_full[pp % D::L1S], (uint32_t)((pp / D::L1S) & 1)); };
    l1_wait(p0);
    l1_wait(p0 + 1);
    for (int64_t zo = z0; zo < z1; ++zo) {
      const int j = (int)(zo - z0);
      l1_wait(p0 + j + 2);
      const double* p1[3] = {l1_slot(p0 + j), l1_slot(p0 + j + 1), l1_slot(p0 + j + 2)};
      double acc[4][2];
      tb_hwindow<D, 4, ONE>(acc, p1, 4 * rb, 0, tc_mask, wf, wz, lane);
      const int64_t gzo = zo + a.gorg0;
      const bool zf = fixed && (gzo < 1 || gzo >= a.GE0 - 1);
      double* plane = a.dst.p + zo * a.dst.s0;
#pragma unroll
      for (int jj = 0; jj < 4; ++jj) {
        const int r = 4 * rb + alpha, c = 16 * jj + D::B * g + beta;  // output tile coords
        if (c >= D::BN) continue;  // columns 62, 63 are the neighbour tile's
        const int64_t row = y0 + r, col = x0 + c;
        double v0 = acc[jj][0], v1 = acc[jj][1];
        if (fixed && (zf || tile_edge)) {
          const double* ctr = p1[1] + (r + 1) * D::TP + c + 1 + D::OFF;
          const int64_t gy = gy0 + r, gx = gx0 + c;
          const bool yf = zf || gy < 1 || gy >= a.GE1 - 1;
          if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
          if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
        }
        if (row >= a.E1 || col >= a.E2) continue;
        double* pp = plane + row * a.dst.s1 + col;
        if (col + 1 < a.E2 && a.dst_aligned) {
          *reinterpret_cast<double2*>(pp) = make_double2(v0, v1);
        } else {
          pp[0] = v0;
          if (col + 1 < a.E2) pp[1] = v1;
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&l1_empty[(p0 + j) % D::L1S]);  // step-1 plane zo-1 done
    }
    __syncwarp();
    if (lane == 0) {  // step-1 planes z1-1, z1 (read by the last output plane only)
      mbar_arrive(&l1_empty[(p0 + (int)(z1 - z0)) % D::L1S]);
      mbar_arrive(&l1_empty[(p0 + (int)(z1 - z0) + 1) % D::L1S]);
    }
    p = p0 + (int)(z1 - z0) + 2;
  }
}

template <class D>
static cudaError_t launch_tile3d_tb2(S2RArgs a, int tc_mask, cudaStream_t st) {
  a.dst_aligned = ((reinterpret_cast<uintptr_t>(a.dst.p) & 15) == 0) && (a.dst.s1 % 2 == 0) &&
                  (a.dst.s0 % 2 == 0);
  a.tiles_x = (int)((a.E2 + D::BN - 1) / D::BN);
  a.tiles_y = (int)((a.E1 + D::BM - 1) / D::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y * set_ranges(a, (a.E0 + D::ZCH - 1) / D::ZCH, D::ZCH, a.E0, D::H);
  if (a.ntiles == 0) return cudaSuccess;
  CUtensorMap tmap;
  if (!make_tmap(a, D::TP, D::RIN, &tmap)) return cudaErrorNotSupported;
  auto kern = __builtin_popcount((unsigned)tc_mask) == 1 ? k_tile3d_tb2<true, D> : k_tile3d_tb2<false, D>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, D::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, D::NT, D::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, kern, grid, D::NT, D::SMEM, st, a, tc_mask, tmap);
}

// ------------------------------------------------------------------------------------------
// 3D Tf = 2, k_tile3d_tb3: k_tile3d_tb2's decoupled levels with the level-1 over-computation cut.
// tb2's level 1 covers the 34 x 66 step-1 cells a 32 x 64 output tile needs with 45 DMMA tiles of
// 4 x 16 (a 36 x 80 plane: 28 % of its DMMAs are wasted columns 67-79).  Here level 1 computes
// step-1 columns 0-63 with 36 such tiles and columns 64-67 with 3 "strip" tiles whose 8 blocks
// (4 x 2 each) sit one above the other (lane group g <-> row block g: every lane addresses its own
// block, so a DMMA tile need not be a row of blocks): 39 tiles instead of 45, 420 DMMAs per plane
// and TC plane instead of 462.  8 level-1 warps (tiles li, li + 8, ...: 5 / 5 / ... / 4), 8
// level-2 warps and a producer = 17 warps, two level-1 and two level-2 warps per SM sub-partition
// (DMMAs per plane 108 / 108 / 108 / 102 against tb2's best 120 / 114 / 114 / 114).  Input planes
// are staged with a 76-column pitch (reads reach column 70; 2 x 76 = 24 banks mod 32 keeps the
// single-tap plane loads conflict-free), step-1 planes with 68.
// Measured (CSX_TB_GEOM a / b / c = ring depths 5+5 / 4+6 / 6+4): Heat-3D 294.5 / 301.4 / 281.0
// GSt/s against tb2's 319.3 — 9 % fewer DMMAs and balanced sub-partitions do not pay: the
// two-level pipeline is bound by its plane hand-offs, not by the DMMA pipe (52 % active) or the
// smem wavefronts (~50 %).  Kept as a parity-tested variant, not the default.
template <int IN_ = 5, int L1S_ = 5>
struct Tile3DTB3 {
  static constexpr int R = 1, A = 4, B = 2, KR = 6, KS = 6, H = 2, ZCH = 32;
  static constexpr int BM = 32, BN = 64;
  static constexpr int NL2 = 8, NL1 = 8, NTL1 = 39;  // warps per level, level-1 DMMA tiles
  static constexpr int NT = 32 * (NL2 + NL1 + 1);
  static constexpr int TPI = 76, TP1 = 68;          // input / step-1 plane pitch
  static constexpr int C1 = 68;                     // step-1 columns computed (0 .. 67)
  static constexpr int RIN = 38, R1 = 36;
  static constexpr int SIN = RIN * TPI, SIN_A = (SIN + 15) / 16 * 16;
  static constexpr int SL1 = R1 * TP1, SL1_A = (SL1 + 15) / 16 * 16;
  static constexpr int IN = IN_, L1S = L1S_;
  static constexpr int SMEM = (IN * SIN_A + L1S * SL1_A) * 8 + 128;
  static_assert(SMEM <= 227 * 1024, "shared memory");
};

// block origin (row, col) of lane group g in level-1 tile tt (step-1 plane coordinates); `st`:
// the lane group's block is a real one (tile 38 carries 2 blocks, its other groups repeat them)
__device__ __forceinline__ void tb3_block(int tt, int g, int& row, int& col, bool& st) {
  st = true;
  if (tt < 36) {
    row = 4 * (tt >> 2);
    col = 16 * (tt & 3) + 2 * g;
  } else if (tt < 38) {
    row = 4 * g;
    col = tt == 36 ? 64 : 66;
  } else {
    row = 32;
    col = (g & 1) ? 66 : 64;
    st = g < 2;
  }
}

// G DMMA tiles, lane group g's block of tile j at staged-plane offset boff[j] (row * TPS + col):
// the inputs of output (row, col) sit at (row + dy, col + 1 + dx) of the planes pl[dz] (pitch TPS)
template <int G, int TPS, bool ONE>
__device__ __forceinline__ void tb3_tiles(double (&acc)[G][2], const double* const (&pl)[3], const int (&boff)[G],
                                          int tc_mask, const double (&wf)[ONE ? 1 : 3][6],
                                          const double (&wz)[3], int t) {
#pragma unroll
  for (int j = 0; j < G; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
  for (int dz = 0; dz < 3; ++dz) {
    if (tc_mask & (1 << dz)) {
#pragma unroll
      for (int rho = 0; rho < 6; ++rho)
#pragma unroll
        for (int j = 0; j < G; ++j)
          dmma_t(acc[j][0], acc[j][1], pl[dz][boff[j] + rho * TPS + 1 + t], wf[ONE ? 0 : dz][rho]);
    } else if (wz[dz] != 0.0) {
#pragma unroll
      for (int j = 0; j < G; ++j) {
        const double2 v = *reinterpret_cast<const double2*>(pl[dz] + boff[j] + (t + 1) * TPS + 2);
        acc[j][0] = fma(wz[dz], v.x, acc[j][0]);
        acc[j][1] = fma(wz[dz], v.y, acc[j][1]);
      }
    }
  }
}

// one level-1 step-1 plane for a warp's G tiles (tile li + 8 i): DMMA, FIXED frame, store
template <int G, bool ONE, class D>
__device__ __forceinline__ void tb3_level1(const double* const (&pin)[3], double* dl1, int li, int tc_mask,
                                           const double (&wf)[ONE ? 1 : 3][6], const double (&wz)[3],
                                           int g, int t, bool frame, bool zf1, int64_t sy0, int64_t sx0,
                                           const S2RArgs& a) {
  int boff[G];
#pragma unroll
  for (int i = 0; i < G; ++i) {
    int r0, c0;
    bool s0;
    tb3_block(li + 8 * i, g, r0, c0, s0);
    boff[i] = r0 * D::TPI + c0;
  }
  double acc[G][2];
  tb3_tiles<G, D::TPI, ONE>(acc, pin, boff, tc_mask, wf, wz, t);
#pragma unroll
  for (int i = 0; i < G; ++i) {
    int r0, c, s0;
    bool st;
    tb3_block(li + 8 * i, g, r0, c, st);
    (void)s0;
    const int r = r0 + t;  // this lane's two step-1 cells (r, c), (r, c + 1)
    double v0 = acc[i][0], v1 = acc[i][1];
    if (frame) {  // held frame points keep the input value
      const int64_t gy = sy0 + r, gx = sx0 + c;
      const double* ctr = pin[1] + (r + 1) * D::TPI + c + 2;
      const bool yf = zf1 || gy < 1 || gy >= a.GE1 - 1;
      if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
      if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
    }
    if (st) *reinterpret_cast<double2*>(dl1 + r * D::TP1 + c) = make_double2(v0, v1);
  }
}

template <bool ONE, class D>  // (17 warps: one SM sub-partition holds 5, so <= 96 registers)
__global__ void __launch_bounds__(D::NT, 1)
    k_tile3d_tb3(S2RArgs a, int tc_mask, const __grid_constant__ CUtensorMap tmap) {
  extern __shared__ __align__(128) double smem_raw[];
  double* smem = ring_base(smem_raw);
  double* l1 = smem + D::IN * D::SIN_A;  // L1S step-1 planes
  __shared__ __align__(8) uint64_t in_full[D::IN], in_empty[D::IN], l1_full[D::L1S], l1_empty[D::L1S];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) {
    for (int s = 0; s < D::IN; ++s) {
      mbar_init(&in_full[s], 1);
      mbar_init(&in_empty[s], D::NL1);
    }
    for (int s = 0; s < D::L1S; ++s) {
      mbar_init(&l1_full[s], D::NL1);
      mbar_init(&l1_empty[s], D::NL2);
    }
    asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
  }
  __syncthreads();
  pdl_begin();
  const int ncol = a.tiles_x * a.tiles_y;
  // warps 0-7 level 2 (output row block = warp), 8-15 level 1 (li = warp - 8), 16 producer
  if (warp == D::NL2 + D::NL1) {  // producer: input planes z0-2 .. z1+1 of every item
    if (lane == 0) tma_prefetch_desc(&tmap);
    int q = 0;
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
      const int64_t zc = slab_map(a, zcl);
      const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
      const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
      for (int64_t zi = z0 - D::H; zi < z1 + D::H; ++zi, ++q) {
        const int s = q % D::IN, n = q / D::IN;
        if (n > 0) mbar_wait(&in_empty[s], (uint32_t)((n - 1) & 1));
        if (lane == 0) {
          mbar_expect_tx(&in_full[s], (uint32_t)(D::SIN * 8));
          tma_load_3d(smem + s * D::SIN_A, &tmap, &in_full[s], (int)(a.tma_x0 + (int64_t)tx * D::BN - 4),
                      (int)(a.tma_y0 + (int64_t)ty * D::BM - 2), (int)(a.tma_z0 + zi));
        }
      }
    }
    return;
  }
  double wf[ONE ? 1 : 3][D::KS], wz[3];
  const int dz1 = __ffs(tc_mask) - 1;
#pragma unroll
  for (int p = 0; p < (ONE ? 1 : 3); ++p)
#pragma unroll
    for (int k = 0; k < D::KS; ++k) wf[p][k] = a.frags[((ONE ? dz1 : p) * D::KS + k) * 32 + lane];
#pragma unroll
  for (int p = 0; p < 3; ++p) wz[p] = a.wc[(p * 3 + 1) * 3 + 1];
  const int g = lane >> 2, t = lane & 3;
  const bool fixed = a.hold_frame != 0;
  if (warp >= D::NL2) {
    // ---------------- level 1: step-1 planes (cols 0 .. 67; col c <-> x0 - 2 + c) ----------------
    const int li = warp - D::NL2;
    int q = 0, p = 0;  // input / step-1 plane sequence numbers
    for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
      const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
      const int64_t zc = slab_map(a, zcl);
      const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
      const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
      const int64_t sy0 = (int64_t)ty * D::BM + a.gorg1 - 1, sx0 = (int64_t)tx * D::BN + a.gorg2 - 2;
      const bool tile_edge = fixed && (sy0 < 1 || sy0 + D::R1 > a.GE1 - 1 || sx0 < 1 || sx0 + D::C1 > a.GE2 - 1);
      const int q0 = q;  // input plane z0-2 of this item
      auto in_slot = [&](int qq) { return smem + (qq % D::IN) * D::SIN_A; };
      mbar_wait(&in_full[q0 % D::IN], (uint32_t)((q0 / D::IN) & 1));
      mbar_wait(&in_full[(q0 + 1) % D::IN], (uint32_t)(((q0 + 1) / D::IN) & 1));
      for (int64_t k = z0 - 1; k <= z1; ++k, ++p) {
        const int j = (int)(k - (z0 - 1));
        mbar_wait(&in_full[(q0 + j + 2) % D::IN], (uint32_t)(((q0 + j + 2) / D::IN) & 1));
        const int sl = p % D::L1S, nl = p / D::L1S;
        if (nl > 0) mbar_wait(&l1_empty[sl], (uint32_t)((nl - 1) & 1));
        const double* pin[3] = {in_slot(q0 + j), in_slot(q0 + j + 1), in_slot(q0 + j + 2)};
        double* dl1 = l1 + sl * D::SL1_A;
        const int64_t gz1 = k + a.gorg0;
        const bool zf1 = fixed && (gz1 < 1 || gz1 >= a.GE0 - 1);
        const bool frame = fixed && (zf1 || tile_edge);
        if (li + 32 < D::NTL1)
          tb3_level1<5, ONE, D>(pin, dl1, li, tc_mask, wf, wz, g, t, frame, zf1, sy0, sx0, a);
        else
          tb3_level1<4, ONE, D>(pin, dl1, li, tc_mask, wf, wz, g, t, frame, zf1, sy0, sx0, a);
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&l1_full[sl]);                 // this warp's cells of plane k written
          mbar_arrive(&in_empty[(q0 + j) % D::IN]);  // input plane k-1 no longer read
        }
      }
      __syncwarp();
      if (lane == 0) {  // input planes z1, z1+1 (read by the last step-1 plane only)
        mbar_arrive(&in_empty[(q0 + (int)(z1 - z0) + 2) % D::IN]);
        mbar_arrive(&in_empty[(q0 + (int)(z1 - z0) + 3) % D::IN]);
      }
      q = q0 + (int)(z1 - z0) + 4;
    }
    return;
  }
  // ---------------- level 2: output planes ----------------
  const int rb = warp;  // output rows 4 rb .. 4 rb + 3, cols 0 .. 63
  int boff[4];
#pragma unroll
  for (int jj = 0; jj < 4; ++jj) boff[jj] = 4 * rb * D::TP1 + 16 * jj + 2 * g;
  int p = 0;  // step-1 plane sequence number
  for (int64_t item = blockIdx.x; item < a.ntiles; item += gridDim.x) {
    const int zcl = (int)(item / ncol), tile = (int)(item - (int64_t)zcl * ncol);
    const int64_t zc = slab_map(a, zcl);
    const int ty = tile / a.tiles_x, tx = tile - ty * a.tiles_x;
    const int64_t z0 = zc * D::ZCH, z1 = min(a.E0, z0 + D::ZCH);
    const int64_t y0 = (int64_t)ty * D::BM, x0 = (int64_t)tx * D::BN;
    const int64_t gy0 = y0 + a.gorg1, gx0 = x0 + a.gorg2;
    const bool tile_edge = fixed && (gy0 < 1 || gy0 + D::BM > a.GE1 - 1 || gx0 < 1 || gx0 + D::BN > a.GE2 - 1);
    const int p0 = p;  // step-1 plane z0-1 of this item
    auto l1_slot = [&](int pp) { return l1 + (pp % D::L1S) * D::SL1_A; };
    auto l1_wait = [&](int pp) { mbar_wait(&l1_full[pp % D::L1S], (uint32_t)((pp / D::L1S) & 1)); };
    l1_wait(p0);
    l1_wait(p0 + 1);
    for (int64_t zo = z0; zo < z1; ++zo) {
      const int j = (int)(zo - z0);
      l1_wait(p0 + j + 2);
      const double* p1[3] = {l1_slot(p0 + j), l1_slot(p0 + j + 1), l1_slot(p0 + j + 2)};
      double acc[4][2];
      tb3_tiles<4, D::TP1, ONE>(acc, p1, boff, tc_mask, wf, wz, t);
      const int64_t gzo = zo + a.gorg0;
      const bool zf = fixed && (gzo < 1 || gzo >= a.GE0 - 1);
      double* plane = a.dst.p + zo * a.dst.s0;
#pragma unroll
      for (int jj = 0; jj < 4; ++jj) {
        const int r = 4 * rb + t, c = 16 * jj + 2 * g;  // output tile coords
        const int64_t row = y0 + r, col = x0 + c;
        double v0 = acc[jj][0], v1 = acc[jj][1];
        if (fixed && (zf || tile_edge)) {
          const double* ctr = p1[1] + (r + 1) * D::TP1 + c + 2;
          const int64_t gy = gy0 + r, gx = gx0 + c;
          const bool yf = zf || gy < 1 || gy >= a.GE1 - 1;
          if (yf || gx < 1 || gx >= a.GE2 - 1) v0 = ctr[0];
          if (yf || gx + 1 < 1 || gx + 1 >= a.GE2 - 1) v1 = ctr[1];
        }
        if (row >= a.E1 || col >= a.E2) continue;
        double* pp = plane + row * a.dst.s1 + col;
        if (col + 1 < a.E2 && a.dst_aligned) {
          *reinterpret_cast<double2*>(pp) = make_double2(v0, v1);
        } else {
          pp[0] = v0;
          if (col + 1 < a.E2) pp[1] = v1;
        }
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&l1_empty[(p0 + j) % D::L1S]);  // step-1 plane zo-1 done
    }
    __syncwarp();
    if (lane == 0) {  // step-1 planes z1-1, z1 (read by the last output plane only)
      mbar_arrive(&l1_empty[(p0 + (int)(z1 - z0)) % D::L1S]);
      mbar_arrive(&l1_empty[(p0 + (int)(z1 - z0) + 1) % D::L1S]);
    }
    p = p0 + (int)(z1 - z0) + 2;
  }
}

template <class D>
static cudaError_t launch_tile3d_tb3(S2RArgs a, int tc_mask, cudaStream_t st) {
  a.dst_aligned = ((reinterpret_cast<uintptr_t>(a.dst.p) & 15) == 0) && (a.dst.s1 % 2 == 0) &&
                  (a.dst.s0 % 2 == 0);
  a.tiles_x = (int)((a.E2 + D::BN - 1) / D::BN);
  a.tiles_y = (int)((a.E1 + D::BM - 1) / D::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y * set_ranges(a, (a.E0 + D::ZCH - 1) / D::ZCH, D::ZCH, a.E0, D::H);
  if (a.ntiles == 0) return cudaSuccess;
  CUtensorMap tmap;
  if (!make_tmap(a, D::TPI, D::RIN, &tmap)) return cudaErrorNotSupported;
  auto kern = __builtin_popcount((unsigned)tc_mask) == 1 ? k_tile3d_tb3<true, D> : k_tile3d_tb3<false, D>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, D::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, D::NT, D::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, kern, grid, D::NT, D::SMEM, st, a, tc_mask, tmap);
}

using Tile3D3 = Tile3DCfg<3, 8, 2, 2, 5, 32>;      // CTA 64 x 32 outputs, 4 DMMA warps, 5-plane ring, 32 planes per item
using Tile3D3b = Tile3DCfg<3, 4, 4, 1, 5, 32, 2>;  // CTA 64 x 32, 4 warps of 4 block rows x 2 column groups
using Tile3D3c = Tile3DCfg<3, 8, 2, 4, 6, 32>;     // CTA 64 x 64 outputs, 8 DMMA warps, 6-plane ring
using Tile3D3d = Tile3DCfg<3, 2, 8, 1, 5, 32, 2>;  // CTA 64 x 32, 8 warps of 2 block rows x 2 column groups
using Tile3D3k = Tile3DCfg<3, 8, 2, 2, 5, 32, 1, 1>;  // Tile3D3, k-slice-outer DMMA order
using Tile3D3ck = Tile3DCfg<3, 8, 2, 4, 6, 32, 1, 1>;  // Tile3D3c, k-slice-outer DMMA order
// Tile3D3 with the plane-interleaved row-outer order (KO = 2, box shapes only)
using Tile3D3i = Tile3DCfg<3, 8, 2, 2, 5, 32, 1, 2>;
using Tile3D3ci = Tile3DCfg<3, 8, 2, 4, 6, 32, 1, 2>;
// wide tiles (the lateral x halo costs a 64-B DRAM granule on each side of every staged row:
// 25 % extra reads at 64 columns, 12.5 % at 128; the TMA box is <= 256 wide): CTA 32 x 128
// (8 warps of 2 column groups), 6-plane ring, 32- or 64-plane z chunks
using Tile3D3w = Tile3DCfg<3, 4, 2, 4, 6, 32, 2, 1>;
using Tile3D3y = Tile3DCfg<3, 4, 2, 4, 6, 64, 2, 1>;
// long z runs (the z-chunk halo planes are re-read from DRAM: 2 / ZCH extra): 64 x 64 tiles with
// 128-plane chunks (1 CTA / SM), 64 x 32 tiles with 256-plane chunks (2 CTAs / SM)
using Tile3D3z = Tile3DCfg<3, 8, 2, 4, 6, 128, 1, 1>;
using Tile3D3l = Tile3DCfg<3, 8, 2, 2, 5, 256, 1, 1>;
// one item per (y, x) tile column: 64 x 64 (1 CTA / SM) or 64 x 32 (2 CTAs / SM) tiles over the
// whole z extent (no z-chunk halo re-reads; neighbouring columns advance in step)
using Tile3D3za = Tile3DCfg<3, 8, 2, 4, 6, 1 << 20, 1, 1>;
using Tile3D3zb = Tile3DCfg<3, 8, 2, 2, 5, 1 << 20, 1, 1>;
// radius 2: 2x4 blocks (K = 6 x 8), 8 DMMA warps, CTA 32 x 64, 9-plane ring (4 planes in flight), weights per plane
using Tile3D5 = Tile3DCfg<5, 4, 4, 2, 9, 32, 1, 0, 2, 4, 0>;
// radius 3: 4x2 blocks (K = 10 x 8), 8 DMMA warps, CTA 32 x 64, 10-plane ring (3 in flight), weights per plane
using Tile3D7 = Tile3DCfg<7, 4, 2, 4, 10, 32, 1, 0, 4, 2, 0>;
// the same with the k-slice-outer DMMA order (G independent accumulator chains per k-slice)
using Tile3D5k = Tile3DCfg<5, 4, 4, 2, 9, 32, 1, 1, 2, 4, 0>;
using Tile3D7k = Tile3DCfg<7, 4, 2, 4, 10, 32, 1, 1, 4, 2, 0>;
// radius 2 with twice the blocks per warp (8 accumulator chains, CTA 64 x 64, 6-plane ring)
using Tile3D5g = Tile3DCfg<5, 8, 4, 2, 6, 32, 1, 1, 2, 4, 0>;
// star shapes, conflict-free DFMA planes: r = 2 with the column-major block numbering (the
// 72-column pitch would not fit the 6-plane ring), r = 3 with a 76-column pitch (2 TP = 24 banks
// mod 32: the four block rows of one 8-lane LDS.128 phase fall on disjoint banks)
using Tile3D5gc = Tile3DCfg<5, 8, 4, 2, 6, 32, 1, 1, 2, 4, 0, 0, 1>;
using Tile3D7ks = Tile3DCfg<7, 4, 2, 4, 10, 32, 1, 1, 4, 2, 0, 4>;
// 16 DMMA warps per CTA (CSX_TILE3D_W16; the 8-warp star kernels keep the DMMA pipe ~50 % busy):
// default for r = 2 stars (+4.6 %); r = 3 stars (spills at 96 registers) and Heat-3D (271 vs 295)
// measured slower
using Tile3D5w = Tile3DCfg<5, 4, 8, 2, 6, 32, 1, 1, 2, 4, 0, 0, 1>;
using Tile3D7w = Tile3DCfg<7, 2, 4, 4, 10, 32, 1, 1, 4, 2, 0, 4>;
using Tile3D3w16 = Tile3DCfg<3, 4, 4, 4, 6, 32, 1, 1>;
using Tile3D3z16 = Tile3DCfg<3, 4, 2, 8, 6, 32, 1, 1>;   // r = 1: 16 warps, CTA 32 x 128 (x halo 4 / 128)
using Tile3D3u = Tile3DCfg<3, 8, 1, 8, 6, 32, 1, 1>;     // r = 1: 8 warps, CTA 32 x 128
using Tile3D7w1 = Tile3DCfg<7, 1, 4, 4, 10, 32, 1, 1, 4, 2, 0, 4>;  // star r = 3: 16 warps of one block row, CTA 16 x 64
using Tile3D3w16r = Tile3DCfg<3, 4, 4, 4, 6, 32, 1, 0>;  // row-outer DMMA order (boxes)
using Tile3D5w16 = Tile3DCfg<5, 2, 8, 2, 9, 32, 1, 1, 2, 4, 0>;  // box r = 2, 16 warps, CTA 32 x 64
using Tile3D7w16 = Tile3DCfg<7, 2, 4, 4, 10, 32, 1, 1, 4, 2, 0>;  // box r = 3, 16 warps, CTA 32 x 64
// box r = 1: two CTAs of 8 DMMA warps per SM (CTA 64 x 32), row-outer / k-slice-outer order
using Tile3D3m2 = Tile3DCfg<3, 4, 4, 2, 5, 32, 1, 0, 4, 2, 1, 0, 0, 2>;
using Tile3D3m2k = Tile3DCfg<3, 4, 4, 2, 5, 32, 1, 1, 4, 2, 1, 0, 0, 2>;


// ------------------------------------------------------------------------------------------
// 1D (P.1779-1786) on the TC_TILE pipeline, re-laid out for DMMA.8x8x4.  The 8 M rows of a DMMA
// are 8 SEGMENTS of the tile (each L outputs, staged by cp.async.bulk with a segment pitch
// P = 4 or 12 mod 16 doubles: conflict-free fragment loads); the 8 N columns are 8 CONSECUTIVE
// outputs of a segment, so the weight operand is the banded Toeplitz matrix
// W[k][n] = w[k - n] (0 <= k - n < nk) of K = nk + 7 rounded up to 4 rows — ks = ceil((nk+7)/4)
// DMMAs per 8 x 8 outputs instead of the paper's 2 ceil(nk/4) nf per 8 x (nk+1) (6 vs 8 per 64
// outputs at nk = 15, 5 vs 9.1 at nk = 13).  Block b+1's window is block b's shifted by 8
// inputs = 2 k-slices, so an A fragment loaded from smem serves ks/2 blocks: a warp runs NB
// blocks at once over a register window of 2 NB + ks - 2 fragments (0.5 LDS.64 per DMMA at
// NB = 4, nk = 15).  The kernel streams HBM through a STAGES-deep ring.
template <int NK_, int L_, int NCW_, int STAGES_, int NB_>
struct Tile1DCfg {
  static constexpr int NK = NK_, L = L_, NCW = NCW_, STAGES = STAGES_, NB = NB_;
  static constexpr int R = (NK - 1) / 2;
  static constexpr int ODD = R & 1;                                  // 16-B aligned copies
  static constexpr int KS = (NK + 7 + 3) / 4;                        // k-slices per 8 outputs
  static constexpr int NBLK = L / 8;                                 // 8-output blocks per segment
  static constexpr int BPW = NBLK / NCW;                             // blocks per consumer warp
  static constexpr int WIN = 2 * NB + KS - 2;                        // A-fragment register window
  static constexpr int SLA = ODD + L - 8 + 4 * KS;                   // read by the GEMM
  static constexpr int SLB = ODD + L + 2 * R;                        // read by the band code
  static constexpr int SL = ((SLA > SLB ? SLA : SLB) + 1) / 2 * 2;   // staged segment length
  static constexpr int P = s2r_pitch_dev(SL);                        // segment pitch (doubles)
  static constexpr int STAGE = 8 * P;
  static constexpr int TILE = 8 * L;                                 // outputs per tile
  static constexpr int NT = 32 * (NCW + 1);
  static constexpr int SMEM = STAGES * STAGE * 8;
  static_assert(L % 8 == 0 && NBLK % NCW == 0 && BPW % NB == 0, "1D tile geometry");
};

template <class C>
__global__ void __launch_bounds__(C::NT, 2) k_tile1d(S2RArgs a) {  // 2 CTAs/SM
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
  pdl_begin();  // PDL: let the next pass launch; wait for the previous pass's writes
  // L2 residency across passes (CSX_TMA_HINT != 0): a 1D grid of <= ~60 MB per buffer fits the
  // 126 MB L2, so outputs are stored evict_last (the next pass reads them) and inputs loaded
  // evict_first (consumed once)
  uint64_t lpol = 0, spol = 0;
  if (a.l2hint) {
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;\n" : "=l"(lpol));
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(spol));
  }
  if (warp == C::NCW) {  // producer: 8 segment copies per tile
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
      const int s = it % C::STAGES, n = it / C::STAGES;
      if (n > 0) mbar_wait(&empty[s], (n - 1) & 1);
      const int64_t t0 = slab_map(a, tile) * C::TILE;
      int nseg = (int)min((int64_t)8, (a.E2 - t0 + C::L - 1) / C::L);
      if (lane == 0) mbar_expect_tx(&full[s], (uint32_t)(nseg * C::SL * 8));
      __syncwarp();
      if (lane < nseg) {
        const double* src = a.src.p + t0 + (int64_t)lane * C::L - C::R - C::ODD;
        if (a.l2hint)
          bulk_g2s_hint(smem + s * C::STAGE + lane * C::P, src, (uint32_t)(C::SL * 8), &full[s], lpol);
        else
          bulk_g2s(smem + s * C::STAGE + lane * C::P, src, (uint32_t)(C::SL * 8), &full[s]);
      }
    }
    return;
  }
  const int g = lane >> 2, t = lane & 3;
  double wt[C::KS];  // Toeplitz B fragments: lane (k = t, n = g) of slice q holds w[4q + t - g]
#pragma unroll
  for (int q = 0; q < C::KS; ++q) wt[q] = a.frags[q * 32 + lane];
  const int fb = a.fix_band;
  int it = 0;
  for (int64_t tile = blockIdx.x; tile < a.ntiles; tile += gridDim.x, ++it) {
    const int s = it % C::STAGES;
    mbar_wait(&full[s], (it / C::STAGES) & 1);
    const double* seg = smem + s * C::STAGE + g * C::P + C::ODD + t;  // this lane's segment g
    const int64_t tsl = slab_map(a, tile);
    const int64_t t0 = tsl * C::TILE + (int64_t)g * C::L;
#pragma unroll 1
    for (int grp = 0; grp < C::BPW / C::NB; ++grp) {
      const int b0 = warp * C::BPW + grp * C::NB;
      double x[C::WIN];
#pragma unroll
      for (int i = 0; i < C::WIN; ++i) x[i] = seg[8 * b0 + 4 * i];
      double acc[C::NB][2];
#pragma unroll
      for (int j = 0; j < C::NB; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
      for (int q = 0; q < C::KS; ++q)
#pragma unroll
        for (int j = 0; j < C::NB; ++j) dmma_t(acc[j][0], acc[j][1], x[2 * j + q], wt[q]);
#pragma unroll
      for (int j = 0; j < C::NB; ++j) {
        const int64_t o = t0 + 8 * (b0 + j) + 2 * t;  // outputs o, o+1 of segment g
        if (fb > 0) {  // band points are written by the band code below
          const int64_t go = o + a.gorg2;
          if (o < a.E2 && !(go < fb || go >= a.GE2 - fb)) a.dst.p[o] = acc[j][0];
          if (o + 1 < a.E2 && !(go + 1 < fb || go + 1 >= a.GE2 - fb)) a.dst.p[o + 1] = acc[j][1];
          continue;
        }
        if (o < a.E2) {
          double* p = a.dst.p + o;
          if (o + 1 < a.E2 && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
            st_out(p, acc[j][0], acc[j][1], a.l2hint != 0, spol);
          } else {
            p[0] = acc[j][0];
            if (o + 1 < a.E2) p[1] = acc[j][1];
          }
        }
      }
    }
    // FIXED: the band b = r*Tf at each global end is recomputed by Tf plain steps (reading A1)
    // by warp 0 from the staged segments, one lane per point, neighbours via shuffles, in
    // chunks of 32 - 2 r (Tf-1) points (the lanes a chunk's Tf-level cone leaves valid).
    const int64_t tg0 = tsl * C::TILE + a.gorg2;  // global index of the tile's first output
    if (fb > 0 && warp == 0 && (tg0 < fb || tg0 + C::TILE > a.GE2 - fb)) {
      const int r = a.r, tf = fb / r, D = r * (tf - 1), CH = 32 - 2 * D;
      for (int sg = 0; sg < 8; ++sg) {
        const int64_t s0 = tg0 + (int64_t)sg * C::L;  // global range of segment sg
        const double* sgm = smem + s * C::STAGE + sg * C::P + C::ODD;  // index = pos - s0 + R
        for (int side = 0; side < 2; ++side) {
          int64_t q0 = side == 0 ? 0 : a.GE2 - fb, q1 = side == 0 ? fb : a.GE2;
          q0 = max(q0, s0);
          q1 = min(q1, min(s0 + (int64_t)C::L, a.GE2));
          q1 = min(q1, a.gorg2 + a.E2);
          for (int64_t qc = q0; qc < q1; qc += CH) {
            const int64_t gp = qc - D + lane;  // lane <-> global position
            const bool hold = gp < r || gp >= a.GE2 - r;
            const int li = (int)(gp - s0) + C::R;
            double v = 0.0;
            if (li >= 0 && li < C::SL) {
              if (hold) {
                v = sgm[li];
              } else {
                for (int o = -r; o <= r; ++o)
                  if (li + o >= 0 && li + o < C::SL) v = fma(__ldg(a.wbase + o + r), sgm[li + o], v);
              }
            }
            for (int lv = 2; lv <= tf; ++lv) {
              double nv = 0.0;
              for (int o = -r; o <= r; ++o) {
                const double xv = __shfl_sync(0xffffffffu, v, (lane + o) & 31);
                nv = fma(__ldg(a.wbase + o + r), xv, nv);
              }
              v = hold ? v : nv;
            }
            if (gp >= qc && gp < min(q1, qc + CH)) a.dst.p[gp - a.gorg2] = v;
          }
        }
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
  }
}

template <class C>
static cudaError_t launch_tile1d_cfg(S2RArgs a, cudaStream_t st) {
  {
    // default on where the grid is near L2 size: +5-6 % on the 10.24M-point 1D configs (82 MB per
    // buffer); off for grids far beyond the L2 (102.4M points: 4460 vs 4355 GSt/s without hints)
    const char* h = getenv("CSX_TMA_HINT");
    a.l2hint = h ? atoi(h) : (a.E2 * (int64_t)sizeof(double) <= (int64_t(256) << 20) ? 1 : 0);
  }
  a.ntiles = set_ranges(a, (a.E2 + C::TILE - 1) / C::TILE, C::TILE, a.E2, C::R);
  if (a.ntiles == 0) return cudaSuccess;
  cudaError_t e = cudaFuncSetAttribute(k_tile1d<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile1d<C>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, k_tile1d<C>, grid, C::NT, C::SMEM, st, a);
}

static int tile1d_variant() {
  static const int v = [] {
    const char* e = getenv("CSX_TILE1D_VARIANT");
    return e ? atoi(e) : 0;
  }();
  return v;
}

template <int NK>
static cudaError_t launch_tile1d_nk(const S2RArgs& a, cudaStream_t st) {
  if constexpr (NK >= 15) {  // tuning variants (CSX_TILE1D_VARIANT)
    switch (tile1d_variant()) {
      case 1: return launch_tile1d_cfg<Tile1DCfg<NK, 512, 4, 4, 4>>(a, st);
      case 2: return launch_tile1d_cfg<Tile1DCfg<NK, 256, 4, 6, 2>>(a, st);
      case 3: return launch_tile1d_cfg<Tile1DCfg<NK, 512, 8, 3, 4>>(a, st);
      case 4: return launch_tile1d_cfg<Tile1DCfg<NK, 384, 4, 4, 4>>(a, st);
      case 5: return launch_tile1d_cfg<Tile1DCfg<NK, 128, 4, 8, 4>>(a, st);
      case 6: return launch_tile1d_cfg<Tile1DCfg<NK, 256, 8, 4, 4>>(a, st);
      case 7: return launch_tile1d_cfg<Tile1DCfg<NK, 256, 4, 6, 8>>(a, st);
      case 8: return launch_tile1d_cfg<Tile1DCfg<NK, 256, 4, 6, 4>>(a, st);
    }
  }
  // nk >= 21: 8 DMMA warps per CTA, 4-stage ring (variant 6; round-2 sweep: Heat-1D 102.4M at
  // Tf = 13 3858 -> 4358 GSt/s, 10.24M 3263 -> 3727, 1D5P Tf = 7 2086 -> 2299); below that the
  // 4-warp, 6-stage CTA (2 per SM) stays ahead (Tf = 7 / 9: 2435 / 3048 vs 2290 / 2941)
  if constexpr (NK >= 21) return launch_tile1d_cfg<Tile1DCfg<NK, 256, 8, 4, 4>>(a, st);
  return launch_tile1d_cfg<Tile1DCfg<NK, 256, 4, 6, 4>>(a, st);  // 2 CTAs/SM x 4 DMMA warps
}

static cudaError_t launch_tile1d(int nk, const S2RArgs& a, cudaStream_t st) {
  switch (nk) {
    case 3: return launch_tile1d_nk<3>(a, st);
    case 5: return launch_tile1d_nk<5>(a, st);
    case 7: return launch_tile1d_nk<7>(a, st);
    case 9: return launch_tile1d_nk<9>(a, st);
    case 11: return launch_tile1d_nk<11>(a, st);
    case 13: return launch_tile1d_nk<13>(a, st);
    case 15: return launch_tile1d_nk<15>(a, st);
    case 17: return launch_tile1d_nk<17>(a, st);
    case 19: return launch_tile1d_nk<19>(a, st);
    case 21: return launch_tile1d_nk<21>(a, st);
    case 23: return launch_tile1d_nk<23>(a, st);
    case 25: return launch_tile1d_nk<25>(a, st);
    case 27: return launch_tile1d_nk<27>(a, st);
    case 29: return launch_tile1d_nk<29>(a, st);
    case 31: return launch_tile1d_nk<31>(a, st);
  }
  return cudaErrorNotSupported;
}

// 3D Tf = 2 geometry (CSX_TB_GEOM, read per call; the planner's DMMA count follows the same
// choice): '0' tb2 32 x 62, '1' tb2 32 x 64 roles by warp index, 't' tb2 32 x 64 balanced roles,
// '3'-'5' tb2 28 x 64, '6' / '8' tb2 ring depths, 'a'-'c' tb3 strip tiles, 'h' tb2 16 x 64 at two
// CTAs per SM
#define CSX_TB_GEOM_DEFAULT 't'
static char tb_geom() {
  const char* r = getenv("CSX_TB_GEOM");
  if (r && r[0] && std::strchr("0134568abcht", r[0])) return r[0];
  return CSX_TB_GEOM_DEFAULT;  // balanced roles (Heat-3D 315.0 -> 320.0 GSt/s)
}

// DMMAs per output point and pass, per TC plane of the base window, of the Tf = 2 geometry that
// runs: (level-1 DMMA tiles x 34 / 32 planes — the z chunk's two extra step-1 planes — + level-2
// tiles) x 6 DMMAs (K = 24) per tile, over the output tile's points
double tile3d_tb_mma_per_point() {
  switch (tb_geom()) {
    case '0': return (36.0 * 34.0 / 32.0 + 32.0) * 6.0 / (32.0 * 62.0);  // step-1 36 x 64
    case '3': case '4': case '5': return (40.0 * 34.0 / 32.0 + 28.0) * 6.0 / (28.0 * 64.0);
    case 'a': case 'b': case 'c': return (39.0 * 34.0 / 32.0 + 32.0) * 6.0 / (32.0 * 64.0);
    case 'h': return (25.0 * 34.0 / 32.0 + 16.0) * 6.0 / (16.0 * 64.0);  // step-1 20 x 80
    default: return (45.0 * 34.0 / 32.0 + 32.0) * 6.0 / (32.0 * 64.0);  // step-1 36 x 80
  }
}

// (ndim, base radius, fused steps) -> is there a TC_TILE kernel for the pass?  3D: Tf = 1 runs
// the per-plane GEMM of the composed window (= the base window) for r = 1..3 (nk = 3, 5, 7);
// Tf = 2 only by the temporal blocking of the base r = 1 stencil (k_tile3d_tb).
bool tile_kernel_exists(int ndim, int radius, int tf) {
  const int nk = 2 * radius * tf + 1;
  if (ndim == 1) return nk >= 3 && nk <= 31;
  if (ndim == 2) return nk >= 3 && nk <= 13;
  if (ndim == 3) return (tf == 1 && radius >= 1 && radius <= 3) || (tf == 2 && radius == 1);
  return false;
}

template <class C>
static cudaError_t launch_tile_cfg(S2RArgs a, cudaStream_t st) {
  a.dst_aligned = ((reinterpret_cast<uintptr_t>(a.dst.p) & 15) == 0) && (a.dst.s1 % 2 == 0);
  a.tiles_x = (int)((a.E2 + C::BN - 1) / C::BN);
  a.tiles_y = (int)((a.E1 + C::BM - 1) / C::BM);
  a.ntiles = (int64_t)a.tiles_x * set_ranges(a, a.tiles_y, C::BM, a.E1, C::R);
  if (a.ntiles == 0) return cudaSuccess;
  CUtensorMap tmap;
  if (!make_tmap(a, C::TP, C::RR, &tmap)) {
    if (a.src.o2 == 0) return cudaErrorNotSupported;  // dense source: no ghost cells to overread
    a.use_tma = 0;
  }
  cudaError_t e = cudaFuncSetAttribute(k_tile2d<C>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile2d<C>, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, k_tile2d<C>, grid, C::NT, C::SMEM, st, a, tmap);
}

template <class C>
static cudaError_t launch_tile3d_cfg(S2RArgs a, int tc_mask, cudaStream_t st) {
  {
    // HBM-bound star shapes (one TC plane): input planes evict_last, outputs evict_first, so the
    // L2 keeps input lines whose halos the neighbouring tiles re-read (+0.8 % on Heat-3D);
    // DMMA-bound boxes: no hint (measured neutral).  CSX_TMA_HINT overrides (0 none, 1 loads
    // evict_last, 2 loads evict_first, 3 = 1 + outputs evict_first).
    const char* h = getenv("CSX_TMA_HINT");
    a.l2hint = h ? atoi(h) : (__builtin_popcount((unsigned)tc_mask) <= 1 ? 3 : 0);
  }
  a.dst_aligned = ((reinterpret_cast<uintptr_t>(a.dst.p) & 15) == 0) && (a.dst.s1 % 2 == 0) &&
                  (a.dst.s0 % 2 == 0);
  a.tiles_x = (int)((a.E2 + C::BN - 1) / C::BN);
  a.tiles_y = (int)((a.E1 + C::BM - 1) / C::BM);
  a.ntiles = (int64_t)a.tiles_x * a.tiles_y * set_ranges(a, (a.E0 + C::ZCH - 1) / C::ZCH, C::ZCH, a.E0, C::R);
  if (a.ntiles == 0) return cudaSuccess;
  CUtensorMap tmap;
  if (!make_tmap(a, C::TP, C::RR, &tmap)) return cudaErrorNotSupported;  // 3D stages by TMA only
  {
    const char* ls = getenv("CSX_LOCKSTEP");
    a.lockstep = ls ? atoi(ls) : 0;
    if (a.lockstep > 0) {
      void* ctr = nullptr;
      cudaGetSymbolAddress(&ctr, g_lock_ctr);
      cudaMemsetAsync(ctr, 0, 8, st);
    }
  }
  // star shapes (one TC plane) keep that plane's fragments in registers (C::WREG = 0 configs)
  auto kern = (!C::WREG && __builtin_popcount((unsigned)tc_mask) == 1) ? k_tile3d<C, true> : k_tile3d<C, false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  return launch_pdl(a.pdl != 0, kern, grid, C::NT, C::SMEM, st, a, tc_mask, tmap);
}

cudaError_t launch_tile(int ndim, int radius, int tf, const S2RArgs& a, cudaStream_t st) {
  if (!tile_kernel_exists(ndim, radius, tf)) return cudaErrorNotSupported;
  const int nk = 2 * radius * tf + 1;
  if (ndim == 1) return launch_tile1d(nk, a, st);
  if (ndim == 3) {
    if (tf == 2) {  // r = 1: temporal blocking (CSX_TB=1: the round-1 single-barrier kernel)
      const char* e = getenv("CSX_TB");
      if (e && e[0] == '1') return launch_tile3d_tb<Tile3DTB>(a, a.tc_mask, st);
      const char g = tb_geom();  // 0: the 32 x 62 tile (equal level work), ... (see tb_geom)
      if (g == '0') return launch_tile3d_tb2<Tile3DTB2<5, 6, 0>>(a, a.tc_mask, st);
      if (g == '3') return launch_tile3d_tb2<Tile3DTB2<5, 5, 1, 28>>(a, a.tc_mask, st);
      if (g == '4') return launch_tile3d_tb2<Tile3DTB2<4, 6, 1, 28>>(a, a.tc_mask, st);
      if (g == '5') return launch_tile3d_tb2<Tile3DTB2<6, 4, 1, 28>>(a, a.tc_mask, st);
      if (g == '6') return launch_tile3d_tb2<Tile3DTB2<5, 4, 1, 32>>(a, a.tc_mask, st);
      // (BM = 28, geometries 3-5: 16 warps, balanced sub-partitions, deeper rings: 281-296 GSt/s, slower)
      if (g == '1') return launch_tile3d_tb2<Tile3DTB2<4, 5, 1>>(a, a.tc_mask, st);  // unbalanced roles
      if (g == 't') return launch_tile3d_tb2<Tile3DTB2<4, 5, 1, 32, 1>>(a, a.tc_mask, st);
      if (g == 'h') return launch_tile3d_tb2<Tile3DTB2<4, 4, 1, 16>>(a, a.tc_mask, st);
      if (g == 'a') return launch_tile3d_tb3<Tile3DTB3<5, 5>>(a, a.tc_mask, st);
      if (g == 'b') return launch_tile3d_tb3<Tile3DTB3<4, 6>>(a, a.tc_mask, st);
      if (g == 'c') return launch_tile3d_tb3<Tile3DTB3<6, 4>>(a, a.tc_mask, st);
      if (g == '8') return launch_tile3d_tb2<Tile3DTB2<5, 4, 1, 32, 1>>(a, a.tc_mask, st);
      return cudaErrorNotSupported;
    }
    if (nk == 5 || nk == 7) {
      // k-slice-outer DMMA order by default (box r = 2 / 3: 56.4 -> 60.0 / 26.6 -> 27.6 GSt/s)
      const char* e = getenv("CSX_TILE3D_KO");
      const bool ko = e ? e[0] == '1' : true;
      // star (one TC plane): 8 blocks per warp (Star-3D13P 158 -> 180 GSt/s); box: 4 (the 9-plane
      // ring; Box-3D125P 59.9 vs 58.4).  CSX_TILE3D5_G8 = 0 / 1 forces either.
      const char* g8 = getenv("CSX_TILE3D5_G8");
      const bool star = __builtin_popcount((unsigned)a.tc_mask) == 1;
      // star: conflict-free DFMA plane loads (CSX_STAR_CF = 0: the round-2 layouts)
      const char* cf = getenv("CSX_STAR_CF");
      const bool scf = star && !(cf && cf[0] == '0');
      // 16 DMMA warps (CSX_TILE3D_W16): the default for r = 2 stars (Star-3D13P 190.5 -> 199.2
      // GSt/s); r = 3 stars spill at 16 warps (121.7 -> 96.4) and keep 8 unless W16 = 1
      const char* w16 = getenv("CSX_TILE3D_W16");
      const bool w16_on = w16 ? w16[0] == '1' : nk == 5;
      if (star && scf && nk == 7 && w16 && w16[0] == '2') return launch_tile3d_cfg<Tile3D7w1>(a, a.tc_mask, st);
      if (star && scf && w16_on)
        return nk == 5 ? launch_tile3d_cfg<Tile3D5w>(a, a.tc_mask, st) : launch_tile3d_cfg<Tile3D7w>(a, a.tc_mask, st);
      if (nk == 5 && (g8 ? g8[0] == '1' : star))
        return scf ? launch_tile3d_cfg<Tile3D5gc>(a, a.tc_mask, st) : launch_tile3d_cfg<Tile3D5g>(a, a.tc_mask, st);
      if (nk == 7 && scf && ko) return launch_tile3d_cfg<Tile3D7ks>(a, a.tc_mask, st);
      // boxes: 16 DMMA warps for r = 2 / 3 by default (Box-3D125P 59.8 -> 70.7 GSt/s, 0.78 ->
      // 0.92 of the DMMA roof; Box-3D343P 27.5 -> 31.3, 0.83 -> 0.95); CSX_TILE3D_W16 = 0: 8 warps
      if (nk == 5 && !star && !(w16 && w16[0] == '0')) return launch_tile3d_cfg<Tile3D5w16>(a, a.tc_mask, st);
      if (nk == 7 && !star && !(w16 && w16[0] == '0')) return launch_tile3d_cfg<Tile3D7w16>(a, a.tc_mask, st);
      if (nk == 5) return ko ? launch_tile3d_cfg<Tile3D5k>(a, a.tc_mask, st) : launch_tile3d_cfg<Tile3D5>(a, a.tc_mask, st);
      return ko ? launch_tile3d_cfg<Tile3D7k>(a, a.tc_mask, st) : launch_tile3d_cfg<Tile3D7>(a, a.tc_mask, st);
    }
    if (nk == 3) {
      const char* e = getenv("CSX_TILE3D_VARIANT");
      if (e && e[0] == '1') return launch_tile3d_cfg<Tile3D3b>(a, a.tc_mask, st);
      if (e && e[0] == '2') return launch_tile3d_cfg<Tile3D3c>(a, a.tc_mask, st);
      if (e && e[0] == '3') return launch_tile3d_cfg<Tile3D3d>(a, a.tc_mask, st);
      if (e && e[0] == '0') return launch_tile3d_cfg<Tile3D3>(a, a.tc_mask, st);
      if (e && e[0] == '8') return launch_tile3d_cfg<Tile3D3k>(a, a.tc_mask, st);
      if (e && e[0] == '9') return launch_tile3d_cfg<Tile3D3ck>(a, a.tc_mask, st);
      if (e && e[0] == '4') return launch_tile3d_cfg<Tile3D3w>(a, a.tc_mask, st);
      if (e && e[0] == '6') return launch_tile3d_cfg<Tile3D3y>(a, a.tc_mask, st);
      if (e && e[0] == '5') return launch_tile3d_cfg<Tile3D3z>(a, a.tc_mask, st);
      if (e && e[0] == '7') return launch_tile3d_cfg<Tile3D3l>(a, a.tc_mask, st);
      if (e && e[0] == 'a') return launch_tile3d_cfg<Tile3D3za>(a, a.tc_mask, st);
      if (e && e[0] == 'b') return launch_tile3d_cfg<Tile3D3zb>(a, a.tc_mask, st);
      if (e && e[0] == 'z') return launch_tile3d_cfg<Tile3D3z16>(a, a.tc_mask, st);
      if (e && e[0] == 'u') return launch_tile3d_cfg<Tile3D3u>(a, a.tc_mask, st);
      // default: star shapes (one TC plane, HBM-bound) take the 64 x 64 tile with 8 DMMA warps
      // (less halo per plane); box shapes (DMMA-bound) the 64 x 32 tile at 2 CTAs / SM
      // (measured)
      // (k-slice-outer DMMA order: 287 vs 283 GSt/s on Heat-3D, but 184 vs 196 on Box-3D27P)
      if (__builtin_popcount((unsigned)a.tc_mask) <= 1) {
        const char* w16 = getenv("CSX_TILE3D_W16");
        if (w16 && w16[0] == '1') return launch_tile3d_cfg<Tile3D3w16>(a, a.tc_mask, st);
        return launch_tile3d_cfg<Tile3D3ck>(a, a.tc_mask, st);
      }
      if (a.tc_mask == 7) {  // box: every plane on the tensor cores
        if (e && e[0] == 'w') return launch_tile3d_cfg<Tile3D3w16>(a, a.tc_mask, st);
        if (e && e[0] == 'x') return launch_tile3d_cfg<Tile3D3w16r>(a, a.tc_mask, st);
        if (e && e[0] == 'm') return launch_tile3d_cfg<Tile3D3m2>(a, a.tc_mask, st);
        if (e && e[0] == 'n') return launch_tile3d_cfg<Tile3D3m2k>(a, a.tc_mask, st);
        if (e && e[0] == 'i') return launch_tile3d_cfg<Tile3D3i>(a, a.tc_mask, st);
        if (e && e[0] == 'j') return launch_tile3d_cfg<Tile3D3ci>(a, a.tc_mask, st);
      }
      return launch_tile3d_cfg<Tile3D3>(a, a.tc_mask, st);
    }
    return cudaErrorNotSupported;
  }
  if (ndim != 2) return cudaErrorNotSupported;
  const int v = tile_variant();
  switch (nk) {
    case 3: return v == 2 ? launch_tile_cfg<Tile3c>(a, st) : v ? launch_tile_cfg<Tile3b>(a, st) : launch_tile_cfg<Tile3>(a, st);
    case 5:  // default (1): Tile5b in k-slice-outer order (Box-2D25P 311 -> 319 GSt/s); 6: Tile5b
      if (v == 1) return launch_tile_cfg<Tile5bk>(a, st);
      if (v == 6) return launch_tile_cfg<Tile5b>(a, st);
      if (v == 7) return launch_tile_cfg<Tile5d>(a, st);
      if (v == 8) return launch_tile_cfg<Tile5dk>(a, st);
      return v == 2 ? launch_tile_cfg<Tile5c>(a, st) : launch_tile_cfg<Tile5>(a, st);
    case 9: return launch_tile_cfg<Tile9>(a, st);
    case 11: return launch_tile_cfg<Tile11>(a, st);
    case 13: return launch_tile_cfg<Tile13>(a, st);
    case 7: return v == 5 ? launch_tile_cfg<Tile7k>(a, st) : v == 4 ? launch_tile_cfg<Tile7e>(a, st) : v == 3 ? launch_tile_cfg<Tile7d>(a, st) : v == 2 ? launch_tile_cfg<Tile7c>(a, st) : v ? launch_tile_cfg<Tile7b>(a, st) : launch_tile_cfg<Tile7>(a, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
