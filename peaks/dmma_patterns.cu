// dmma_patterns.cu — how close to the DMMA.8x8x4 peak can an operand pattern like the TC_TILE
// kernel's get?  (1) constant operands (the peak test), (2) A/B from register arrays varying per
// DMMA, chains interleaved, (3) same with each accumulator chain issued back-to-back
// (serialised), (4) A fragments loaded from shared memory as in k_tile2d.  Prints JSON.
#include <cuda_runtime.h>

#include <cstdio>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s\n", cudaGetErrorString(e_)); return 1; } } while (0)

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

template <int MODE>
__global__ void k(double* out, int iters) {
  __shared__ double sm[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = 1.0 + i * 1e-9;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  double a[20], b[20];
#pragma unroll
  for (int i = 0; i < 20; ++i) { a[i] = 1.0 + (lane + i) * 1e-9; b[i] = 1.0 - (lane + i) * 1e-9; }
  double acc[8][2];
#pragma unroll
  for (int j = 0; j < 8; ++j) acc[j][0] = acc[j][1] = 0.0;
  const double* base = sm + (threadIdx.x >> 5) * 64 + (lane >> 2) * 2 + (lane & 3);
  for (int it = 0; it < iters; ++it) {
    if (MODE == 0) {
#pragma unroll
      for (int s = 0; s < 20; ++s)
#pragma unroll
        for (int j = 0; j < 8; ++j) dmma(acc[j][0], acc[j][1], a[0], b[0]);
    } else if (MODE == 1) {
#pragma unroll
      for (int s = 0; s < 20; ++s)
#pragma unroll
        for (int j = 0; j < 8; ++j) dmma(acc[j][0], acc[j][1], a[(s + j) % 20], b[s]);
    } else if (MODE == 2) {
#pragma unroll
      for (int j = 0; j < 8; ++j)
#pragma unroll
        for (int s = 0; s < 20; ++s) dmma(acc[j][0], acc[j][1], a[(s + j) % 20], b[s]);
    } else {
#pragma unroll
      for (int ra = 0; ra < 38; ++ra) {
        const double f0 = base[ra * 72], f1 = base[ra * 72 + 4];
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int rho = ra - 4 * j;
          if (rho >= 0 && rho < 10) {
            dmma(acc[j][0], acc[j][1], f0, b[2 * rho % 20]);
            dmma(acc[j][0], acc[j][1], f1, b[(2 * rho + 1) % 20]);
          }
        }
      }
    }
  }
  double s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += acc[j][0] + acc[j][1];
  if (s == 1234.5) out[threadIdx.x] = s;
}

template <int MODE>
static double run(int warps_per_cta, int ctas_per_sm, int sms, double* out) {
  const int iters = 200;
  dim3 grid(sms * ctas_per_sm), block(32 * warps_per_cta);
  k<MODE><<<grid, block>>>(out, 2);
  cudaDeviceSynchronize();
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<MODE><<<grid, block>>>(out, iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  const double per_warp = 160.0 * iters;  // 20 x 8 DMMA (mode 3: 160 too)
  return (double)grid.x * warps_per_cta * per_warp * 512.0 / (ms * 1e-3) / 1e12;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  double* out;
  CK(cudaMalloc(&out, 1 << 20));
  printf("{\n");
  const int cfg[][2] = {{8, 1}, {12, 1}, {16, 1}, {8, 2}};
  for (int c = 0; c < 4; ++c) {
    const int w = cfg[c][0], n = cfg[c][1];
    printf("  \"warps%d_ctas%d\": {\"const\": %.2f, \"var_interleaved\": %.2f, \"var_serial\": %.2f, \"smem_tile\": %.2f}%s\n",
           w, n, run<0>(w, n, sms, out), run<1>(w, n, sms, out), run<2>(w, n, sms, out),
           run<3>(w, n, sms, out), c < 3 ? "," : "");
  }
  printf("}\n");
  return 0;
}
