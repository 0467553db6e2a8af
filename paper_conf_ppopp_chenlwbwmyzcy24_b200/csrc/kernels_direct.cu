// kernels_direct.cu — CUDA-core kernels of the csx hot path (product code):
//   * k_direct   : direct weighted sum with temporal blocking in shared memory (SURVEY §8(a)
//                  a10, N2).  Engine DIRECT runs it on every tile; for FIXED boundaries it is
//                  also the band fix-up after a fused TC pass (a7, reading A1): it recomputes
//                  the points within r*Tf of a face by Tf plain steps, holding the frame.
//   * k_pack     : user grid -> padded ping-pong grid interior.
//   * k_ghost_*  : PERIODIC ghost zones (depth r*Tf) refreshed from the wrapped interior.
#include <cuda_runtime.h>

#include "kernels.cuh"

namespace csx {

constexpr int kMaxTaps = 343;  // (2*3+1)^3

template <int NDIM>
__global__ void __launch_bounds__(256) k_direct(DirectArgs a) {
  extern __shared__ __align__(16) double sm[];
  const int h = a.r * a.tf;
  const int RB0 = a.B[0] + (a.real[0] ? 2 * h : 0);
  const int RB1 = a.B[1] + (a.real[1] ? 2 * h : 0);
  const int RB2 = a.B[2] + 2 * h;
  const int vol = RB0 * RB1 * RB2;
  double* tw = sm;
  int* toff = reinterpret_cast<int*>(sm + kMaxTaps);
  double* buf0 = sm + kMaxTaps + (kMaxTaps + 1) / 2 + 1;
  double* buf1 = buf0 + vol;
  __shared__ int ntaps;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nw = blockDim.x >> 5;
  if (tid == 0) {
    const int n = 2 * a.r + 1;
    int cnt = 0, dense = 1;
    for (int d = 0; d < NDIM; ++d) dense *= n;
    for (int i = 0; i < dense; ++i) {
      const double wv = a.w[i];
      if (wv == 0.0) continue;
      int rem = i, off[3] = {0, 0, 0};
      for (int d = NDIM - 1; d >= 0; --d) { off[d] = rem % n - a.r; rem /= n; }
      int d0 = 0, d1 = 0, d2 = off[NDIM - 1];
      if (NDIM >= 2) d1 = off[NDIM - 2];
      if (NDIM == 3) d0 = off[0];
      tw[cnt] = wv;
      toff[cnt] = (d0 * RB1 + d1) * RB2 + d2;
      ++cnt;
    }
    ntaps = cnt;
  }
  __syncthreads();
  const int nt = ntaps;
  for (int64_t it = blockIdx.x; it < a.ntiles; it += gridDim.x) {
    int64_t b0, b1, b2;  // tile origin (local coordinates of its first output)
    if (a.tile_org) {
      b0 = a.tile_org[3 * it];
      b1 = a.tile_org[3 * it + 1];
      b2 = a.tile_org[3 * it + 2];
    } else {
      const int64_t tid_lin = a.tile_list ? (int64_t)a.tile_list[it] : it;
      b2 = (tid_lin % a.tiles[2]) * a.B[2];
      b1 = ((tid_lin / a.tiles[2]) % a.tiles[1]) * a.B[1];
      b0 = (tid_lin / ((int64_t)a.tiles[2] * a.tiles[1])) * a.B[0];
    }
    const int64_t o0 = b0 - (a.real[0] ? h : 0);
    const int64_t o1 = b1 - (a.real[1] ? h : 0);
    const int64_t o2 = b2 - h;
    // load the region (halo h on real axes) from the padded source
    for (int row = warp; row < RB0 * RB1; row += nw) {
      const int z = row / RB1, y = row - z * RB1;
      const double* s = a.src.p + (o0 + z) * a.src.s0 + (o1 + y) * a.src.s1 + o2;
      double* d = buf0 + row * RB2;
      for (int x = lane; x < RB2; x += 32) d[x] = s[x];
    }
    __syncthreads();
    double* in = buf0;
    double* out = buf1;
    for (int s = 1; s <= a.tf; ++s) {
      const int sh = a.r * s;
      const int lo0 = a.real[0] ? sh : 0, hi0 = RB0 - lo0;
      const int lo1 = a.real[1] ? sh : 0, hi1 = RB1 - lo1;
      const int lo2 = sh, hi2 = RB2 - sh;
      const int ny = hi1 - lo1;
      const int cnt = (hi0 - lo0) * ny;
      for (int q = warp; q < cnt; q += nw) {
        const int z = lo0 + q / ny, y = lo1 + q % ny;
        const int64_t gz = a.gorg[0] + o0 + z, gy = a.gorg[1] + o1 + y;  // global coordinates
        const bool rowhold = a.fixed_bc && ((a.real[0] && (gz < a.r || gz >= a.GE[0] - a.r)) ||
                                            (a.real[1] && (gy < a.r || gy >= a.GE[1] - a.r)));
        const int rbase = (z * RB1 + y) * RB2;
        for (int x = lo2 + lane; x < hi2; x += 32) {
          const int64_t gx = a.gorg[2] + o2 + x;
          const bool hold = rowhold || (a.fixed_bc && (gx < a.r || gx >= a.GE[2] - a.r));
          const int idx = rbase + x;
          double v;
          if (hold) {
            v = in[idx];
          } else {
            v = 0.0;
            for (int k = 0; k < nt; ++k) v = fma(tw[k], in[idx + toff[k]], v);
          }
          out[idx] = v;
        }
      }
      __syncthreads();
      double* tmp = in; in = out; out = tmp;
    }
    // write the tile's outputs (band mode: only points within `band` of a face)
    const int h0 = a.real[0] ? h : 0, h1 = a.real[1] ? h : 0;
    for (int row = warp; row < a.B[0] * a.B[1]; row += nw) {
      const int z = row / a.B[1], y = row - z * a.B[1];
      const int64_t lz = b0 + z, ly = b1 + y;  // local coordinates
      if (lz >= a.E[0] || ly >= a.E[1]) continue;
      const int64_t gz = a.gorg[0] + lz, gy = a.gorg[1] + ly;
      const bool rowband = (a.real[0] && (gz < a.band || gz >= a.GE[0] - a.band)) ||
                           (a.real[1] && (gy < a.band || gy >= a.GE[1] - a.band));
      const double* src = in + ((z + h0) * RB1 + (y + h1)) * RB2 + h;
      double* dst = a.dst.p + lz * a.dst.s0 + ly * a.dst.s1;
      for (int x = lane; x < a.B[2]; x += 32) {
        const int64_t lx = b2 + x;
        if (lx >= a.E[2]) continue;
        const int64_t gx = a.gorg[2] + lx;
        if (a.band > 0 && !(rowband || gx < a.band || gx >= a.GE[2] - a.band)) continue;
        dst[lx] = src[x];
      }
    }
    __syncthreads();
  }
}

static int direct_smem(const DirectArgs& a) {
  const int h = a.r * a.tf;
  const int RB0 = a.B[0] + (a.real[0] ? 2 * h : 0);
  const int RB1 = a.B[1] + (a.real[1] ? 2 * h : 0);
  const int RB2 = a.B[2] + 2 * h;
  return (kMaxTaps + (kMaxTaps + 1) / 2 + 1 + 2 * RB0 * RB1 * RB2) * 8;
}

cudaError_t launch_direct(const DirectArgs& a, cudaStream_t st) {
  const int smem = direct_smem(a);
  if (a.ntiles <= 0) return cudaSuccess;
  cudaError_t e = cudaSuccess;
  int occ = 0;
  switch (a.ndim) {
    case 1:
      e = cudaFuncSetAttribute(k_direct<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct<1>, 256, smem);
      break;
    case 2:
      e = cudaFuncSetAttribute(k_direct<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct<2>, 256, smem);
      break;
    default:
      e = cudaFuncSetAttribute(k_direct<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
      if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_direct<3>, 256, smem);
  }
  if (e != cudaSuccess) return e;
  const int64_t grid = persistent_grid(occ, a.max_ctas, a.ntiles);
  switch (a.ndim) {
    case 1: k_direct<1><<<(unsigned)grid, 256, smem, st>>>(a); break;
    case 2: k_direct<2><<<(unsigned)grid, 256, smem, st>>>(a); break;
    default: k_direct<3><<<(unsigned)grid, 256, smem, st>>>(a); break;
  }
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------
// FIXED frame copy, one thread per frame element.  Local rows (z, y) are either entirely in
// the global frame (a frame plane or frame row: all E2 columns copied) or contribute only their
// 2r frame columns.  Work = O(frame size), not O(grid).
__global__ void k_frame_copy(CView src, View dst, int64_t E0, int64_t E1, int64_t E2, int64_t g0,
                             int64_t g1, int64_t g2, int64_t G0, int64_t G1, int64_t G2, int real0,
                             int real1, int r) {
  // local index ranges of the frame rows / planes
  const int64_t nrows = E0 * E1;
  const int64_t total = nrows * 2 * r;  // column part for every row (frame rows re-copy: harmless)
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t row = i / (2 * r);
    const int k = (int)(i - row * 2 * r);
    const int64_t z = row / E1, y = row - z * E1;
    const int64_t gx = k < r ? k : G2 - 2 * r + k;
    const int64_t x = gx - g2;
    if (x >= 0 && x < E2) dst.p[z * dst.s0 + y * dst.s1 + x] = src.p[z * src.s0 + y * src.s1 + x];
  }
  // full frame rows: rows whose plane or row index is in the global frame
  const int64_t nfr_y = real1 ? 2 * r : 0;           // frame rows per plane
  const int64_t nfr_z = real0 ? 2 * r : 0;           // frame planes
  const int64_t rows_a = nfr_z * E1;                 // rows of the frame planes
  const int64_t rows_b = (real1 ? E0 : 0) * nfr_y;   // frame rows of every plane
  const int64_t total2 = (rows_a + rows_b) * E2;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total2;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t rr = i / E2, x = i - rr * E2;
    int64_t z, y;
    if (rr < rows_a) {
      const int64_t kz = rr / E1;
      y = rr - kz * E1;
      const int64_t gz = kz < r ? kz : G0 - 2 * r + kz;
      z = gz - g0;
      if (z < 0 || z >= E0) continue;
    } else {
      const int64_t q = rr - rows_a;
      z = q / nfr_y;
      const int64_t ky = q - z * nfr_y;
      const int64_t gy = ky < r ? ky : G1 - 2 * r + ky;
      y = gy - g1;
      if (y < 0 || y >= E1) continue;
    }
    dst.p[z * dst.s0 + y * dst.s1 + x] = src.p[z * src.s0 + y * src.s1 + x];
  }
}

cudaError_t launch_frame_copy(CView src, View dst, const int64_t* E, const int64_t* gorg,
                              const int64_t* GE, const int* real, int r, cudaStream_t st) {
  k_frame_copy<<<4 * num_sms(), 256, 0, st>>>(src, dst, E[0], E[1], E[2], gorg[0], gorg[1], gorg[2],
                                             GE[0], GE[1], GE[2], real[0], real[1], r);
  return cudaGetLastError();
}

__global__ void k_pack(const double* __restrict__ in, View dst, int64_t E1, int64_t E2,
                       int64_t nrows) {
  for (int64_t row = blockIdx.x; row < nrows; row += gridDim.x) {
    const int64_t z = row / E1, y = row - z * E1;
    const double* s = in + row * E2;
    double* d = dst.p + z * dst.s0 + y * dst.s1;
    for (int64_t x = threadIdx.x; x < E2; x += blockDim.x) d[x] = s[x];
  }
}

// few long rows (1D): one thread per element
__global__ void k_pack_flat(const double* __restrict__ in, View dst, int64_t E1, int64_t E2,
                            int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t row = i / E2, x = i - row * E2;
    const int64_t z = row / E1, y = row - z * E1;
    dst.p[z * dst.s0 + y * dst.s1 + x] = in[i];
  }
}

cudaError_t launch_pack(const double* in, View dst, const int64_t* E, cudaStream_t st) {
  const int64_t nrows = E[0] * E[1];
  if (nrows < 4 * num_sms()) {
    k_pack_flat<<<8 * num_sms(), 256, 0, st>>>(in, dst, E[1], E[2], nrows * E[2]);
  } else {
    const int64_t grid = nrows < 65535 ? nrows : 65535;
    k_pack<<<(unsigned)grid, 256, 0, st>>>(in, dst, E[1], E[2], nrows);
  }
  return cudaGetLastError();
}

// axis 2 ghosts of interior rows
__global__ void k_ghost2(View b, int64_t E0, int64_t E1, int64_t E2, int H) {
  const int64_t n = E0 * E1 * 2 * H;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = i % (2 * H), row = i / (2 * H);
    const int64_t z = row / E1, y = row - z * E1;
    double* r = b.p + z * b.s0 + y * b.s1;
    if (k < H) r[-H + k] = r[E2 - H + k];
    else r[E2 + (k - H)] = r[k - H];
  }
}

// axis 1 ghost rows (full padded width) of interior planes
__global__ void k_ghost1(View b, int64_t E0, int64_t E1, int64_t E2, int H, int H2) {
  const int64_t W = E2 + 2 * H2;
  const int64_t n = E0 * 2 * H * W;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = i % W - H2;
    const int64_t k = (i / W) % (2 * H), z = i / (W * 2 * H);
    const int64_t y = k < H ? -H + k : E1 + (k - H);
    const int64_t ys = k < H ? E1 - H + k : k - H;
    b.p[z * b.s0 + y * b.s1 + x] = b.p[z * b.s0 + ys * b.s1 + x];
  }
}

// axis 0 ghost planes (full padded rows and width)
__global__ void k_ghost0(View b, int64_t E0, int64_t E1, int64_t E2, int H, int H1, int H2) {
  const int64_t W = E2 + 2 * H2, Hn = E1 + 2 * H1;
  const int64_t n = (int64_t)2 * H * Hn * W;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = i % W - H2;
    const int64_t y = (i / W) % Hn - H1;
    const int64_t k = i / (W * Hn);
    const int64_t z = k < H ? -H + k : E0 + (k - H);
    const int64_t zs = k < H ? E0 - H + k : k - H;
    b.p[z * b.s0 + y * b.s1 + x] = b.p[zs * b.s0 + y * b.s1 + x];
  }
}

// Refresh the ghosts of the axes with fill[a] != 0, fastest axis first so that corners are
// carried along (a slab-sharded run leaves its slab axis to the halo exchange).
cudaError_t launch_ghost_fill(View buf, const int64_t* E, const int* real, const int* fill, int H,
                              cudaStream_t st) {
  if (H <= 0) return cudaSuccess;
  const int grid = 4 * num_sms();
  const int H1 = real[1] ? H : 0;
  if (fill[2]) k_ghost2<<<grid, 256, 0, st>>>(buf, E[0], E[1], E[2], H);
  if (real[1] && fill[1]) k_ghost1<<<grid, 256, 0, st>>>(buf, E[0], E[1], E[2], H, H);
  if (real[0] && fill[0]) k_ghost0<<<grid, 256, 0, st>>>(buf, E[0], E[1], E[2], H, H1, H);
  return cudaGetLastError();
}

}  // namespace csx
