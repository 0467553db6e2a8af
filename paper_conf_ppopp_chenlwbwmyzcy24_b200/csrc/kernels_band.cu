// kernels_band.cu — FIXED-boundary band fix-up after a fused pass (DESIGN.md
// reading A1).  A pass with the composed window W^(Tf) is exact only at points >= r*Tf from a
// FIXED face (the composition runs through held frame points); the band b = r*Tf next to every
// GLOBAL face is recomputed here by Tf plain steps of the base stencil, holding the frame.
//
// One CTA per band segment: 128 columns of the top / bottom band or 128 rows of the left /
// right band (2D), or one end of the line (1D).  Level 0 is read from the pass's padded source;
// level s (s = 1..Tf) lives in shared memory on the segment dilated by r*(Tf-s).  The TC
// kernels skip (TC_TILE) or are overwritten at (TC_S2R) these points.
#include <cuda_runtime.h>

#include <cstdint>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

constexpr int kSeg = 128;

struct BandArgs {
  CView src;
  View dst;
  int64_t E1, E2;   // local extents (1D: E1 = 1)
  int64_t g1, g2;   // local origin in global coordinates
  int64_t G1, G2;   // global extents
  int tf, band, ndim;
  int nh, nv;       // segments per horizontal band (2D) and per vertical band
  double w[49];
};

template <int R, int NDIM>
__global__ void __launch_bounds__(256) k_band(BandArgs a) {
  extern __shared__ __align__(16) double sc[];
  constexpr int N = 2 * R + 1;
  const int b = a.band;
  int64_t qy0 = 0, qy1 = 1, qx0, qx1;
  int blk = blockIdx.x;
  if (NDIM == 1) {
    if (blk == 0) { qx0 = -a.g2; qx1 = b - a.g2; }
    else { qx0 = a.G2 - b - a.g2; qx1 = a.G2 - a.g2; }
  } else if (blk < 2 * a.nh) {
    const int seg = blk % a.nh;
    if (blk < a.nh) { qy0 = -a.g1; qy1 = b - a.g1; }
    else { qy0 = a.G1 - b - a.g1; qy1 = a.G1 - a.g1; }
    qx0 = (int64_t)seg * kSeg;
    qx1 = qx0 + kSeg;
  } else {
    blk -= 2 * a.nh;
    const int seg = blk % a.nv;
    qy0 = (int64_t)seg * kSeg;
    qy1 = qy0 + kSeg;
    if (blk < a.nv) { qx0 = -a.g2; qx1 = b - a.g2; }
    else { qx0 = a.G2 - b - a.g2; qx1 = a.G2 - a.g2; }
  }
  qy0 = max(qy0, (int64_t)0); qy1 = min(qy1, a.E1);
  qx0 = max(qx0, (int64_t)0); qx1 = min(qx1, a.E2);
  if (qy0 >= qy1 || qx0 >= qx1) return;
  const int r = R;
  const int tf = a.tf;
  const int mxW = (int)(qx1 - qx0) + 2 * r * (tf - 1);
  const int mxH = NDIM == 2 ? (int)(qy1 - qy0) + 2 * r * (tf - 1) : 1;
  double* lv[2] = {sc, sc + mxW * mxH};
  // previous level accessor: global level 0 or the smem level
  const double* pp = nullptr;
  int64_t py0 = 0, px0 = 0;
  int pW = 0;
  for (int s = 1; s <= tf; ++s) {
    const int d = r * (tf - s);
    const int64_t y0 = NDIM == 2 ? qy0 - d : 0, x0 = qx0 - d;
    const int W = (int)(qx1 - qx0) + 2 * d;
    const int H = NDIM == 2 ? (int)(qy1 - qy0) + 2 * d : 1;
    double* out = lv[s & 1];
    for (int i = threadIdx.x; i < H * W; i += blockDim.x) {
      const int iy = i / W, ix = i - iy * W;
      const int64_t y = y0 + iy, x = x0 + ix;
      const int64_t gy = y + a.g1, gx = x + a.g2;
      const bool hold = gx < R || gx >= a.G2 - R || (NDIM == 2 && (gy < R || gy >= a.G1 - R));
      double v;
      if (s == 1) {
        const double* c = a.src.p + (NDIM == 2 ? y * a.src.s1 : 0) + x;
        if (hold) {
          // a held point outside the GLOBAL grid feeds only held points: its value is never used,
          // and a dense source (first pass reading the user's grid) has no ghost cell there
          const bool out = gx < 0 || gx >= a.G2 || (NDIM == 2 && (gy < 0 || gy >= a.G1));
          v = out ? 0.0 : *c;
        } else {
          v = 0.0;
#pragma unroll
          for (int ii = 0; ii < (NDIM == 2 ? N : 1); ++ii)
#pragma unroll
            for (int jj = 0; jj < N; ++jj)
              v = fma(a.w[ii * N + jj], c[(NDIM == 2 ? (ii - R) * a.src.s1 : 0) + (jj - R)], v);
        }
      } else {
        const double* c = pp + (y - py0) * pW + (x - px0);
        if (hold) {
          v = *c;
        } else {
          v = 0.0;
#pragma unroll
          for (int ii = 0; ii < (NDIM == 2 ? N : 1); ++ii)
#pragma unroll
            for (int jj = 0; jj < N; ++jj)
              v = fma(a.w[ii * N + jj], c[(NDIM == 2 ? (ii - R) * pW : 0) + (jj - R)], v);
        }
      }
      out[i] = v;
    }
    __syncthreads();
    pp = out;
    py0 = y0;
    px0 = x0;
    pW = W;
  }
  const int W = (int)(qx1 - qx0);
  for (int i = threadIdx.x; i < (int)(qy1 - qy0) * W; i += blockDim.x) {
    const int iy = i / W, ix = i - iy * W;
    const int64_t y = qy0 + iy, x = qx0 + ix;
    a.dst.p[(NDIM == 2 ? y * a.dst.s1 : 0) + x] = pp[(y - py0) * pW + (x - px0)];
  }
}

template <int R, int NDIM>
static cudaError_t launch_band_rn(const BandArgs& a, int nblk, int smem, cudaStream_t st) {
  cudaError_t e = cudaFuncSetAttribute(k_band<R, NDIM>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  k_band<R, NDIM><<<nblk, 256, smem, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_band(int ndim, int r, int tf, CView src, View dst, const int64_t* E,
                        const int64_t* gorg, const int64_t* GE, const double* w_host,
                        cudaStream_t st, int* launched) {
  *launched = 0;
  if (ndim != 1 && ndim != 2) return cudaErrorNotSupported;
  BandArgs a;
  a.src = src;
  a.dst = dst;
  a.E1 = ndim == 2 ? E[1] : 1;
  a.E2 = E[2];
  a.g1 = gorg[1];
  a.g2 = gorg[2];
  a.G1 = ndim == 2 ? GE[1] : 1;
  a.G2 = GE[2];
  a.tf = tf;
  a.band = r * tf;
  a.ndim = ndim;
  const int n = 2 * r + 1;
  for (int i = 0; i < 49; ++i) a.w[i] = i < (ndim == 2 ? n * n : n) ? w_host[i] : 0.0;
  a.nh = (int)((a.E2 + kSeg - 1) / kSeg);
  a.nv = (int)((a.E1 + kSeg - 1) / kSeg);
  int nblk = ndim == 1 ? 2 : 2 * a.nh + 2 * a.nv;
  // two level buffers; the largest dilated segment is (band + 2d) x (128 + 2d), d = r (Tf-1)
  const int d = r * (tf - 1);
  const int bytes = 2 * (ndim == 2 ? (a.band + 2 * d) * (kSeg + 2 * d) : (a.band + 2 * d)) * 8;
  cudaError_t e = cudaErrorNotSupported;
  if (ndim == 1) {
    if (r == 1) e = launch_band_rn<1, 1>(a, nblk, bytes, st);
    else if (r == 2) e = launch_band_rn<2, 1>(a, nblk, bytes, st);
    else if (r == 3) e = launch_band_rn<3, 1>(a, nblk, bytes, st);
  } else {
    if (r == 1) e = launch_band_rn<1, 2>(a, nblk, bytes, st);
    else if (r == 2) e = launch_band_rn<2, 2>(a, nblk, bytes, st);
    else if (r == 3) e = launch_band_rn<3, 2>(a, nblk, bytes, st);
  }
  if (e == cudaSuccess) *launched = 1;
  return e;
}

}  // namespace csx
