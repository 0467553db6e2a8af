// kernels_direct13.cu — the CUDA-core comparator (north_star item 2) for 1D
// and 3D, the counterparts of kernels_direct2d.cu: direct weighted sums in FP64 FMA with the
// base weights as kernel parameters (constant-bank DFMA operands), register blocking and
// coalesced 128-bit global / shared traffic.  They answer "how far do CUDA cores get on the
// same chip" for the 1D and 3D configs (DMMA and DFMA share one FP64 datapath on B200,
// DESIGN.md §7).
//
//   * k_direct1d<R, V, PF>: every warp owns a window of 32*V consecutive points (V per lane, loaded
//     with LDG.128) and runs the Tf fused steps in registers; the R neighbours across lanes come
//     from warp shuffles.  The error front of the window edges moves R points per step, so the
//     inner 32 V - 2 hp points (hp = R Tf rounded up to even) are exact and stored.
//   * k_direct3d<R> (Tf = 1): 2.5D z-march.  A CTA owns a 32 x 64 (y, x) tile and a z chunk;
//     the planes stream through a (2R+2)-slot shared-memory ring by cp.async (16 B), one plane
//     in flight while the previous output plane is computed.  A thread owns 4 rows x 2 columns
//     and reads its input rows as LDS.128 pairs (a warp covers 64 contiguous doubles:
//     conflict-free); rows / columns whose weights are all zero are skipped by uniform branches
//     (star shapes: the +-z planes read one pair per row).
//   * FIXED: points within r of a global face keep their value at every step.
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <type_traits>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

struct Direct1DW {
  double w[7];
};

template <int R, int V, bool PF>
__global__ void __launch_bounds__(128, (V <= 8 ? 8 : 1)) k_direct1d(DirectArgs a, Direct1DW W) {
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int h = R * a.tf;
  const int hp = (h + 1) & ~1;
  const int OUT = 32 * V - 2 * hp;
  const int64_t N = a.E[2];
  const int64_t nseg = (N + OUT - 1) / OUT;
  const int64_t G = a.GE[2];
  // PF: the next segment's window is loaded into registers before this one is computed, so
  // a warp's HBM latency overlaps its own Tf steps of DFMA
  double2 nxt[PF ? V / 2 : 1];
  if (PF && gw < nseg) {
    const double2* src = reinterpret_cast<const double2*>(a.src.p + gw * OUT - hp + lane * V);
#pragma unroll
    for (int i = 0; i < V / 2; ++i) nxt[i] = src[i];
  }
  for (int64_t sg = gw; sg < nseg; sg += nw) {
    const int64_t s0 = sg * OUT;
    const int64_t w0 = s0 - hp + lane * V;  // local index of x[0]
    double x[V];
    if (PF) {
#pragma unroll
      for (int i = 0; i < V / 2; ++i) {
        x[2 * i] = nxt[i].x;
        x[2 * i + 1] = nxt[i].y;
      }
      if (sg + nw < nseg) {
        const double2* src = reinterpret_cast<const double2*>(a.src.p + (sg + nw) * OUT - hp + lane * V);
#pragma unroll
        for (int i = 0; i < V / 2; ++i) nxt[i] = src[i];
      }
    } else {
      const double2* src = reinterpret_cast<const double2*>(a.src.p + w0);
#pragma unroll
      for (int i = 0; i < V / 2; ++i) {
        const double2 v = src[i];
        x[2 * i] = v.x;
        x[2 * i + 1] = v.y;
      }
    }
    const int64_t g0 = a.gorg[2] + w0;  // global index of x[0]
    // lanes whose points are all at least R from both global ends skip the per-point hold test
    const bool edge = a.fixed_bc && (g0 < R || g0 + V > G - R);
    // one step in -> out: the R neighbours across the lane boundary by shuffles; FIXED edge
    // lanes hold the frame points
    auto step = [&](const double (&in)[V], double (&out)[V], auto edge_c) {
      constexpr bool EDGE = decltype(edge_c)::value;
      double l[R], r[R];
#pragma unroll
      for (int k = 0; k < R; ++k) {
        l[k] = __shfl_up_sync(0xffffffffu, in[V - R + k], 1);
        r[k] = __shfl_down_sync(0xffffffffu, in[k], 1);
      }
#pragma unroll
      for (int i = 0; i < V; ++i) {
        double acc = 0.0;
#pragma unroll
        for (int k = 0; k <= 2 * R; ++k) {
          const int j = i + k - R;
          const double v = j < 0 ? l[j + R] : (j >= V ? r[j - V] : in[j]);
          acc = fma(W.w[k], v, acc);
        }
        if (EDGE) {
          const int64_t gi = g0 + i;
          out[i] = (gi < R || gi >= G - R) ? in[i] : acc;
        } else {
          out[i] = acc;
        }
      }
    };
    double y[V];
    int s = 0;
    if (edge) {
      for (; s < a.tf; ++s) {
        step(x, y, std::true_type{});
#pragma unroll
        for (int i = 0; i < V; ++i) x[i] = y[i];
      }
    } else {
      for (; s + 1 < a.tf; s += 2) {  // two steps per trip: x -> y -> x, no register copies
        step(x, y, std::false_type{});
        step(y, x, std::false_type{});
      }
      if (s < a.tf) {
        step(x, y, std::false_type{});
#pragma unroll
        for (int i = 0; i < V; ++i) x[i] = y[i];
      }
    }
#pragma unroll
    for (int i = 0; i < V; i += 2) {
      const int p = lane * V + i;  // window position of x[i]
      const int64_t o = s0 + p - hp;
      if (p < hp || p >= 32 * V - hp || o >= N) continue;
      if (o + 1 < N) *reinterpret_cast<double2*>(a.dst.p + o) = make_double2(x[i], x[i + 1]);
      else a.dst.p[o] = x[i];
    }
  }
}

bool direct1d_exists(int r, int tf) { return r >= 1 && r <= 3 && tf >= 1 && r * tf <= 16; }

template <int R, int V, bool PF>
static cudaError_t launch_d1v(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  Direct1DW W;
  for (int i = 0; i < 7; ++i) W.w[i] = i <= 2 * R ? w_host[i] : 0.0;
  const int hp = (R * a.tf + 1) & ~1;
  if (32 * V - 2 * hp <= 0) return cudaErrorNotSupported;
  const int64_t nseg = (a.E[2] + (32 * V - 2 * hp) - 1) / (32 * V - 2 * hp);
  int occ = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct1d<R, V, PF>, 128, 0);
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, (nseg + 3) / 4);
  if (grid < 1) return cudaSuccess;
  k_direct1d<R, V, PF><<<(unsigned)grid, 128, 0, st>>>(a, W);
  return cudaGetLastError();
}

// V points per lane: CSX_DIRECT1D_V = 4 / 8 / 16 / 32; CSX_DIRECT1D_PF = 0 / 1 (register
// prefetch of the next segment).  Default V = 8 without prefetch, measured (profiles/r01/
// direct1d_sweep.txt): Heat-1D Tf = 11 2686 GSt/s (V = 16: 1958, V = 4: 2236, V = 8 + PF: 2463),
// 1D5P Tf = 5 1323 (V = 16: 925) — 72 registers instead of 126 doubles the resident warps;
// __launch_bounds__ min 8 CTAs (64 registers) adds ~1.5 % (2727 / 1335).
template <int R>
static cudaError_t launch_d1(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  static int v = -1, pf = -1;
  if (v < 0) {
    const char* e = getenv("CSX_DIRECT1D_V");
    v = e ? atoi(e) : 8;
    const char* f = getenv("CSX_DIRECT1D_PF");
    pf = f ? atoi(f) : 0;
  }
  const int hp = (R * a.tf + 1) & ~1;
  if (v == 4 && 2 * hp < 128) return pf ? launch_d1v<R, 4, true>(a, w_host, st) : launch_d1v<R, 4, false>(a, w_host, st);
  if (v == 16) return pf ? launch_d1v<R, 16, true>(a, w_host, st) : launch_d1v<R, 16, false>(a, w_host, st);
  if (v == 32) return pf ? launch_d1v<R, 32, true>(a, w_host, st) : launch_d1v<R, 32, false>(a, w_host, st);
  if (2 * hp < 256) return pf ? launch_d1v<R, 8, true>(a, w_host, st) : launch_d1v<R, 8, false>(a, w_host, st);
  return pf ? launch_d1v<R, 16, true>(a, w_host, st) : launch_d1v<R, 16, false>(a, w_host, st);
}

cudaError_t launch_direct1d(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  switch (a.r) {
    case 1: return launch_d1<1>(a, w_host, st);
    case 2: return launch_d1<2>(a, w_host, st);
    case 3: return launch_d1<3>(a, w_host, st);
  }
  return cudaErrorNotSupported;
}

// ------------------------------------------------------------------------------------------
// 3D, Tf = 1
struct Direct3DW {
  double w[343];     // base weights, dense (2R+1)^3, row-major over (dz, dy, dx)
  int plane_nz[7];   // plane dz has a non-zero weight
  int plane_ctr[7];  // plane dz's non-zeros all lie in column dx = R (read one pair per row)
  int row_nz[7][7];  // row (dz, dy) has a non-zero weight
};

template <int R>
struct D3Cfg {
  static constexpr int BY = 32, BX = 64, NT = 256;
  static constexpr int LP = (R + 1) & ~1;  // left pad (even): staged col 0 = x0 - LP
  static constexpr int PW = BX + 2 * LP;   // staged row length (doubles, even)
  static constexpr int RY = BY + 2 * R;    // staged rows
  // planes in flight ahead of the window (2 measured slower at r = 1: 5 ring slots leave 2 CTAs
  // per SM instead of 3 -- Heat-3D 220 vs 244 GSt/s)
  static constexpr int PF = 1;
  static constexpr int NS = 2 * R + 1 + PF;  // ring slots: 2R+1 planes in use + PF in flight
  static constexpr int PLANE = RY * PW;
  static constexpr int SMEM = NS * PLANE * 8;
  static constexpr int ZC = 32;            // output planes per work item
  static constexpr int NPAIR = PW / 2;     // 16-B chunks per staged row
};

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(
                   static_cast<uint32_t>(__cvta_generic_to_shared(smem))),
               "l"(gmem)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }
template <int K>
__device__ __forceinline__ void cp_async_wait_n() { asm volatile("cp.async.wait_group %0;\n" ::"n"(K) : "memory"); }

template <int R>
__device__ __forceinline__ void d3_issue_plane(const DirectArgs& a, double* slot, int64_t zi,
                                               int64_t y0, int64_t x0) {
  using C = D3Cfg<R>;
  const double* base = a.src.p + zi * a.src.s0 + (y0 - R) * a.src.s1 + (x0 - C::LP);
  for (int c = threadIdx.x; c < C::RY * C::NPAIR; c += C::NT) {
    const int row = c / C::NPAIR, pr = c - row * C::NPAIR;
    cp_async16(slot + row * C::PW + 2 * pr, base + row * a.src.s1 + 2 * pr);
  }
  cp_async_commit();
}

// STAR (every non-zero weight on an axis through the centre): the centre plane's off-centre rows
// carry only their dx = R tap, skipped at compile time (the uniform row / plane tests above cannot
// see zeros inside a row: Star-3D13P / 19P executed 29 / 55 FMAs per point for 13 / 19 taps)
template <int R, bool STAR>
__global__ void __launch_bounds__(256) k_direct3d(DirectArgs a, const __grid_constant__ Direct3DW W) {
  using C = D3Cfg<R>;
  constexpr int N = 2 * R + 1;
  extern __shared__ __align__(16) double sm[];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int tiles_x = (int)((a.E[2] + C::BX - 1) / C::BX);
  const int tiles_y = (int)((a.E[1] + C::BY - 1) / C::BY);
  const int64_t nzc = (a.E[0] + C::ZC - 1) / C::ZC;
  const int64_t nitems = (int64_t)tiles_x * tiles_y * nzc;
  for (int64_t item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int64_t zc = item / ((int64_t)tiles_x * tiles_y);
    const int tile = (int)(item - zc * tiles_x * tiles_y);
    const int ty = tile / tiles_x, tx = tile - ty * tiles_x;
    const int64_t y0 = (int64_t)ty * C::BY, x0 = (int64_t)tx * C::BX;
    const int64_t z0 = zc * C::ZC, z1 = min(a.E[0], z0 + C::ZC);
    // prologue: planes z0-R .. z0+R+PF-1 (slots by plane index mod NS), one commit group each
    // (a group past the chunk's last plane z1+R-1 is committed empty, so that the number of
    // groups per plane stays one and wait_group<PF - 1> always means "window complete")
    for (int64_t zi = z0 - R; zi <= z0 + R + C::PF - 1; ++zi) {
      if (zi < z1 + R) d3_issue_plane<R>(a, sm + (int)((zi + 2 * C::NS) % C::NS) * C::PLANE, zi, y0, x0);
      else cp_async_commit();
    }
    // this thread's outputs: rows y0 + 4 warp + j (j < 4), cols x0 + 2 lane + e
    const int ry = 4 * warp, cx = 2 * lane;
    const int64_t gy0 = a.gorg[1] + y0 + ry, gx0 = a.gorg[2] + x0 + cx;
    for (int64_t zo = z0; zo < z1; ++zo) {
      // planes up to zo+R have landed (this thread's copies), then everyone's (barrier); the
      // barrier also retires iteration zo-1, the last reader of plane zo-R-1, whose slot now
      // receives plane zo+R+1 while output plane zo is computed
      cp_async_wait_n<C::PF - 1>();
      __syncthreads();
      {
        const int64_t zn = zo + R + C::PF;  // its slot held plane zo-R-1, read last iteration
        if (zn < z1 + R) d3_issue_plane<R>(a, sm + (int)((zn + 2 * C::NS) % C::NS) * C::PLANE, zn, y0, x0);
        else cp_async_commit();
      }
      double acc[4][2];
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[j][0] = acc[j][1] = 0.0;
#pragma unroll
      for (int dz = 0; dz < N; ++dz) {
        if (!W.plane_nz[dz]) continue;
        const double* pl = sm + (int)((zo - R + dz + 2 * C::NS) % C::NS) * C::PLANE;
        // staged (row, col) of input (y0 + ry + ri - R, x0 + cx + c - LP)
        const double* rowp = pl + ry * C::PW + cx;
        if (W.plane_ctr[dz]) {  // one tap column: the lane's own pair of each needed row
#pragma unroll
          for (int ri = 0; ri < 4 + 2 * R; ++ri) {
            bool need = false;
#pragma unroll
            for (int j = 0; j < 4; ++j)
              if (ri - j >= 0 && ri - j <= 2 * R) need |= W.row_nz[dz][ri - j] != 0;
            if (!need) continue;
            const double2 v = *reinterpret_cast<const double2*>(rowp + ri * C::PW + C::LP);
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const int dy = ri - j;
              if (dy < 0 || dy > 2 * R) continue;
              const double wv = W.w[(dz * N + dy) * N + R];
              acc[j][0] = fma(wv, v.x, acc[j][0]);
              acc[j][1] = fma(wv, v.y, acc[j][1]);
            }
          }
        } else {
#pragma unroll
          for (int ri = 0; ri < 4 + 2 * R; ++ri) {
            bool need = false;
#pragma unroll
            for (int j = 0; j < 4; ++j)
              if (ri - j >= 0 && ri - j <= 2 * R) need |= W.row_nz[dz][ri - j] != 0;
            if (!need) continue;
            double v[2 + 2 * C::LP];
#pragma unroll
            for (int q = 0; q < 1 + C::LP; ++q) {
              const double2 t = *reinterpret_cast<const double2*>(rowp + ri * C::PW + 2 * q);
              v[2 * q] = t.x;
              v[2 * q + 1] = t.y;
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const int dy = ri - j;
              if (dy < 0 || dy > 2 * R) continue;
#pragma unroll
              for (int dx = 0; dx < N; ++dx) {
                if (STAR && dy != R && dx != R) continue;
                const double wv = W.w[(dz * N + dy) * N + dx];
                acc[j][0] = fma(wv, v[C::LP - R + dx], acc[j][0]);
                acc[j][1] = fma(wv, v[C::LP - R + dx + 1], acc[j][1]);
              }
            }
          }
        }
      }
      // FIXED: held frame values from the centre plane
      const double* ctr = sm + (int)((zo + 2 * C::NS) % C::NS) * C::PLANE + (ry + R) * C::PW + cx + C::LP;
      const int64_t gz = a.gorg[0] + zo;
      const bool zf = a.fixed_bc && (gz < R || gz >= a.GE[0] - R);
      double* out = a.dst.p + zo * a.dst.s0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int64_t y = y0 + ry + j, x = x0 + cx;
        if (y >= a.E[1] || x >= a.E[2]) continue;
        const int64_t gy = gy0 + j;
        const bool yf = zf || (a.fixed_bc && (gy < R || gy >= a.GE[1] - R));
        double v0 = acc[j][0], v1 = acc[j][1];
        if (yf || (a.fixed_bc && (gx0 < R || gx0 >= a.GE[2] - R))) v0 = ctr[j * C::PW];
        if (yf || (a.fixed_bc && (gx0 + 1 < R || gx0 + 1 >= a.GE[2] - R))) v1 = ctr[j * C::PW + 1];
        double* p = out + y * a.dst.s1 + x;
        if (x + 1 < a.E[2] && ((reinterpret_cast<uintptr_t>(p) & 15) == 0)) {
          *reinterpret_cast<double2*>(p) = make_double2(v0, v1);
        } else {
          p[0] = v0;
          if (x + 1 < a.E[2]) p[1] = v1;
        }
      }
    }
    __syncthreads();  // the ring is reused by the next item
  }
}

bool direct3d_exists(int r, int tf) { return tf == 1 && r >= 1 && r <= 3; }

template <int R>
static cudaError_t launch_d3(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  using C = D3Cfg<R>;
  constexpr int N = 2 * R + 1;
  static Direct3DW W;  // host staging (kernel parameters are copied at launch)
  for (int i = 0; i < 343; ++i) W.w[i] = i < N * N * N ? w_host[i] : 0.0;
  for (int dz = 0; dz < 7; ++dz) {
    W.plane_nz[dz] = 0;
    W.plane_ctr[dz] = 1;
    for (int dy = 0; dy < 7; ++dy) {
      W.row_nz[dz][dy] = 0;
      if (dz >= N || dy >= N) continue;
      for (int dx = 0; dx < N; ++dx)
        if (w_host[(dz * N + dy) * N + dx] != 0.0) {
          W.row_nz[dz][dy] = 1;
          W.plane_nz[dz] = 1;
          if (dx != R) W.plane_ctr[dz] = 0;
        }
    }
  }
  bool star = true;  // every non-zero on an axis through the centre
  for (int dz = 0; dz < N; ++dz)
    for (int dy = 0; dy < N; ++dy)
      for (int dx = 0; dx < N; ++dx)
        if (w_host[(dz * N + dy) * N + dx] != 0.0 && (dz != R) + (dy != R) + (dx != R) > 1) star = false;
  {
    const char* e = getenv("CSX_DIRECT3D_STAR");  // 0: the generic rows (A/B)
    if (e && e[0] == '0') star = false;
  }
  auto kern = star ? k_direct3d<R, true> : k_direct3d<R, false>;
  cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM);
  if (e != cudaSuccess) return e;
  int occ = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, C::NT, C::SMEM);
  if (e != cudaSuccess) return e;
  const int64_t nitems = ((a.E[2] + C::BX - 1) / C::BX) * ((a.E[1] + C::BY - 1) / C::BY) *
                         ((a.E[0] + C::ZC - 1) / C::ZC);
  const int64_t grid = persistent_grid(occ, a.max_ctas, nitems);
  if (grid < 1) return cudaSuccess;
  kern<<<(unsigned)grid, C::NT, C::SMEM, st>>>(a, W);
  return cudaGetLastError();
}

cudaError_t launch_direct3d(const DirectArgs& a, const double* w_host, cudaStream_t st) {
  if (a.tf != 1) return cudaErrorNotSupported;
  switch (a.r) {
    case 1: return launch_d3<1>(a, w_host, st);
    case 2: return launch_d3<2>(a, w_host, st);
    case 3: return launch_d3<3>(a, w_host, st);
  }
  return cudaErrorNotSupported;
}

}  // namespace csx
