// kernels_s2r_explicit.cu — breakdown variant I of the paper's Fig 6 (P.1865-1893, text
// P.1919-1926): EXPLICIT stencil2row.  The whole grid is first transformed into the
// stencil2row matrices A and B in global memory (HBM), with the div/mod address arithmetic of
// Eq 5 / Eq 6 (P.731-785) computed per element, and the dual tessellation (P.900-975) then runs
// on CUDA cores reading A and B back from HBM.  It exists to measure what the implicit,
// shared-memory stencil2row (variant II+) saves; it is not a production engine.
//
// Coordinates: the stencil2row input is the source grid shifted by the window radius,
// X'[x][y] = src[x - R][y - R] for x in [0, E1 + 2R), y in [0, nstrips*(nk+1) + nk), so that the
// window of output (i, j) starts at X'[i][j] (the paper's centre store, P.1326-1331).
//   Eq 5:  A[y / (nk+1)][nk*x + y mod (nk+1)]            for y mod (nk+1) != nk
//   Eq 6:  B[(y-nk) / (nk+1)][nk*x + (y-nk) mod (nk+1)]   for y >= nk, (y-nk) mod (nk+1) != nk
// Strip k (row k of A and B) yields outputs (i, k(nk+1) + c), c in [0, nk]:
//   out = sum_{q < nk^2} A[k][nk*i + q] W_A[q][c] + B[k][nk*i + q] W_B[q][c]
// with W_A[nk*a + b][c] = w[a][b - c] (b >= c), W_B[nk*a + b][c] = w[a][b + nk - c] (b < c)
// (P.961-975, Fig 3).
#include <cuda_runtime.h>

#include "kernels.cuh"

namespace csx {

__global__ void k_s2r_explicit_transform(CView src, double* A, double* B, int nk, int64_t rows,
                                         int64_t cols, int64_t ld, int64_t nstrips) {
  const int R = (nk - 1) / 2;
  const int64_t n = rows * cols;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t x = e / cols, y = e - x * cols;  // explicit div / mod (Eq 5/6 addressing)
    const double v = src.p[(x - R) * src.s1 + (y - R)];
    const int64_t ka = y / (nk + 1), ma = y % (nk + 1);
    if (ma != nk && ka < nstrips) A[ka * ld + nk * x + ma] = v;  // the last nk cols are B-only
    if (y >= nk) {
      const int64_t kb = (y - nk) / (nk + 1), mb = (y - nk) % (nk + 1);
      if (mb != nk) B[kb * ld + nk * x + mb] = v;
    }
  }
}

// one thread per output (i, k, c); c fastest so a warp stores contiguous output columns
__global__ void k_s2r_explicit_fma(const double* __restrict__ A, const double* __restrict__ B,
                                   const double* __restrict__ wc, View dst, int nk, int64_t E1,
                                   int64_t E2, int64_t nstrips, int64_t ld) {
  extern __shared__ double sw[];  // W_A then W_B, (nk*nk) x (nk+1) each
  const int K = nk * nk, N = nk + 1;
  for (int q = threadIdx.x; q < K * N; q += blockDim.x) {
    const int r = q / N, c = q - r * N, ai = r / nk, b = r - ai * nk;
    sw[q] = b >= c ? wc[ai * nk + (b - c)] : 0.0;
    sw[K * N + q] = b < c ? wc[ai * nk + (b + nk - c)] : 0.0;
  }
  __syncthreads();
  const int64_t per_row = nstrips * N;
  const int64_t n = E1 * per_row;
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = e / per_row, kc = e - i * per_row;
    const int64_t k = kc / N;
    const int c = (int)(kc - k * N);
    const int64_t col = k * N + c;
    if (col >= E2) continue;
    const double* a = A + k * ld + nk * i;
    const double* b = B + k * ld + nk * i;
    double acc = 0.0;
    for (int q = 0; q < K; ++q) acc = fma(a[q], sw[q * N + c], fma(b[q], sw[K * N + q * N + c], acc));
    dst.p[i * dst.s1 + col] = acc;
  }
}

int64_t s2r_explicit_elems(int nk, int64_t E1, int64_t E2) {
  const int R = (nk - 1) / 2;
  const int64_t nstrips = (E2 + nk) / (nk + 1);  // strips covering output columns [0, E2)
  return 2 * nstrips * (int64_t)nk * (E1 + 2 * R);
}

cudaError_t launch_s2r_explicit(int nk, CView src, View dst, const int64_t* E, const double* wc,
                                double* scratch, cudaStream_t st) {
  const int R = (nk - 1) / 2;
  const int64_t E1 = E[1], E2 = E[2];
  const int64_t nstrips = (E2 + nk) / (nk + 1);
  const int64_t rows = E1 + 2 * R;
  const int64_t ld = (int64_t)nk * rows;
  double* A = scratch;
  double* B = scratch + nstrips * ld;
  const int64_t cols = nstrips * (nk + 1) + nk;
  const int nsm = num_sms();
  k_s2r_explicit_transform<<<nsm * 8, 256, 0, st>>>(src, A, B, nk, rows, cols, ld, nstrips);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  const int smem = 2 * nk * nk * (nk + 1) * (int)sizeof(double);
  k_s2r_explicit_fma<<<nsm * 8, 256, smem, st>>>(A, B, wc, dst, nk, E1, E2, nstrips, ld);
  return cudaGetLastError();
}

}  // namespace csx
