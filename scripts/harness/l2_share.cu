// L2 sharing microbenchmark (debug harness, not part of libcsx): does a line fetched by one SM
// serve a read of the same line by an SM on the other die?  Mode 0: every CTA reads the same
// 16 MB buffer (ideal DRAM traffic 16 MB).  Mode 1: CTA b reads chunk b and chunk b+1 of a
// 148 x 1 MB buffer, at the same time as CTA b+1 reads chunks b+1, b+2 (halo-like sharing between
// consecutive blockIdx).  Mode 2: as 1 but CTA pairs (b, b^1) share (both read chunk b>>1).
#include <cstdio>
#include <cstdlib>
__global__ void k_read(const double* __restrict__ p, size_t n_per, int mode, double* sink) {
  double acc = 0.0;
  const int b = blockIdx.x;
  for (int rep = 0; rep < 2; ++rep) {
    const double* base;
    if (mode == 0) base = p;
    else if (mode == 1) base = p + (size_t)(b + rep) * n_per;
    else base = p + (size_t)(b >> 1) * n_per;
    for (size_t i = threadIdx.x; i < n_per; i += blockDim.x) acc += __ldcg(base + i);
    if (mode == 0) break;
  }
  if (acc == 12345.678) sink[0] = acc;
}
int main(int argc, char** argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  const size_t n_per = (1 << 20) / 8;  // 1 MB
  size_t total = mode == 0 ? 16 * n_per : 150 * n_per;
  size_t nread = mode == 0 ? 16 * n_per : n_per;
  double *p, *sink;
  cudaMalloc(&p, total * 8); cudaMalloc(&sink, 8);
  cudaMemset(p, 0, total * 8);
  k_read<<<148, 1024>>>(p, nread, mode, sink);
  cudaDeviceSynchronize();
  printf("mode %d done: %s\n", mode, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
