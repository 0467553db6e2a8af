// 3D halo-reuse microbenchmark (debug harness): each CTA streams the z planes of one 64 x 64
// tile (+1 halo cell each side) of a 512^3 grid in the padded layout of the csx plans, with plain
// coalesced loads; items ordered like k_tile3d (tile fastest, 32-plane z chunks).  Reports the
// DRAM bytes per pass relative to the 1 GB interior.
#include <cstdio>
#include <cstdlib>
__global__ void k_halo(const double* __restrict__ g, int64_t s1, int64_t s0, int zch, int bx, int by,
                       double* sink, double* out, int wmode) {
  const int E = 512;
  const int tx_n = E / bx, ty_n = E / by, ncol = tx_n * ty_n;
  const int nitems = ncol * (E / zch);
  double acc = 0.0;
  for (int item = blockIdx.x; item < nitems; item += gridDim.x) {
    const int zc = item / ncol, t = item % ncol, ty = t / tx_n, tx = t % tx_n;
    for (int z = zc * zch - 1; z < zc * zch + zch + 1; ++z) {
      const double* pl = g + (int64_t)(z + 1) * s0 + (int64_t)(ty * by) * s1 + tx * bx + 16 - 2;
      const int w = bx + 4, h = by + 2;
      for (int i = threadIdx.x; i < w * h; i += blockDim.x) {
        const int r = i / w, c = i % w;
        acc += __ldcg(pl + (int64_t)r * s1 + c);
      }
      if (wmode && z >= zc * zch && z < zc * zch + zch) {  // write the tile's output plane
        double* po = out + (int64_t)(z + 1) * s0 + (int64_t)(ty * by + 1) * s1 + tx * bx + 16;
        for (int i = threadIdx.x; i < bx * by; i += blockDim.x) {
          double* q = po + (int64_t)(i / bx) * s1 + (i % bx);
          if (wmode == 1) *q = acc;
          else __stcs(q, acc);
        }
      }
      __syncthreads();
    }
  }
  if (acc == 1.2345) sink[0] = acc;
}
int main(int argc, char** argv) {
  const int zch = argc > 1 ? atoi(argv[1]) : 32;
  const int bx = argc > 2 ? atoi(argv[2]) : 64;
  const int by = argc > 3 ? atoi(argv[3]) : 64;
  const int wmode = argc > 4 ? atoi(argv[4]) : 0;
  const int64_t s1 = 736, rows = 644, s0 = s1 * rows, planes = 530;
  double *g, *sink, *out;
  cudaMalloc(&g, (size_t)s0 * planes * 8); cudaMalloc(&sink, 8); cudaMalloc(&out, (size_t)s0 * planes * 8);
  cudaMemset(g, 0, (size_t)s0 * planes * 8);
  k_halo<<<148, 512>>>(g, s1, s0, zch, bx, by, sink, out, wmode);
  cudaDeviceSynchronize();
  printf("zch %d tile %dx%d wmode %d: %s\n", zch, by, bx, wmode, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
