// fp64_peaks.cu — on-box FP64 roofline denominators for the csx hot path.
//
// MEASURED_PEAKS.json (driver-written) has no FP64 entries, so this program measures, on the
// B200 it runs on:
//   * DMMA.8x8x4 throughput (mma.sync.m8n8k4.f64; the only FP64 tensor instruction sm_100a has),
//     burst (~50 ms) and sustained (~3 s), and the single-chain DMMA latency;
//   * DFMA throughput (CUDA-core FP64), burst and sustained;
//   * DMMA and DFMA issued concurrently by different warps of the same CTA (are the pipes shared?);
//   * FP64 HBM copy bandwidth (read + write bytes);
//   * shared-memory LDS.64 bandwidth.
// Prints one JSON object on stdout.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <algorithm>

#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); exit(1); } } while (0)

__device__ __forceinline__ void dmma(double& d0, double& d1, double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
               : "+d"(d0), "+d"(d1) : "d"(a), "d"(b));
}

template <int NACC>
__global__ void k_dmma(double* out, long iters, double seed) {
  double a = seed + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
  double acc[NACC][2];
#pragma unroll
  for (int i = 0; i < NACC; ++i) { acc[i][0] = 0.0; acc[i][1] = 0.0; }
  for (long it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NACC; ++i) dmma(acc[i][0], acc[i][1], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < NACC; ++i) s += acc[i][0] + acc[i][1];
  if (s == 12345.678) out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

template <int NCH>
__global__ void k_dfma(double* out, long iters, double seed) {
  double x[NCH];
  const double a = 0.999999 + threadIdx.x * 1e-12, b = seed * 1e-7;
#pragma unroll
  for (int i = 0; i < NCH; ++i) x[i] = seed + i;
  for (long it = 0; it < iters; ++it) {
#pragma unroll
    for (int i = 0; i < NCH; ++i) x[i] = fma(x[i], a, b);
  }
  double s = 0;
#pragma unroll
  for (int i = 0; i < NCH; ++i) s += x[i];
  if (s == 12345.678) out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// Even warps DMMA, odd warps DFMA: if the two pipes are independent the mixed run takes
// max(T_dmma, T_dfma), if they share one FP64 datapath it takes the sum.
__global__ void k_mixed(double* out, long it_mma, long it_fma, double seed) {
  const int warp = threadIdx.x >> 5;
  double s = 0;
  if ((warp & 1) == 0) {
    double a = seed + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
    double acc[8][2];
#pragma unroll
    for (int i = 0; i < 8; ++i) { acc[i][0] = 0.0; acc[i][1] = 0.0; }
    for (long it = 0; it < it_mma; ++it) {
#pragma unroll
      for (int i = 0; i < 8; ++i) dmma(acc[i][0], acc[i][1], a, b);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) s += acc[i][0] + acc[i][1];
  } else {
    double x[8];
    const double a = 0.999999 + threadIdx.x * 1e-12, b = seed * 1e-7;
#pragma unroll
    for (int i = 0; i < 8; ++i) x[i] = seed + i;
    for (long it = 0; it < it_fma; ++it) {
#pragma unroll
      for (int i = 0; i < 8; ++i) x[i] = fma(x[i], a, b);
    }
#pragma unroll
    for (int i = 0; i < 8; ++i) s += x[i];
  }
  if (s == 12345.678) out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_copy(const double2* __restrict__ in, double2* __restrict__ out, size_t n) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  for (; i < n; i += stride) out[i] = in[i];
}

__global__ void k_lds(double* out, long iters) {
  __shared__ double buf[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) buf[i] = i;
  __syncthreads();
  double s0 = 0, s1 = 0, s2 = 0, s3 = 0;
  int idx = threadIdx.x & 1023;
  for (long it = 0; it < iters; ++it) {
    s0 += buf[idx];
    s1 += buf[(idx + 32) & 4095];
    s2 += buf[(idx + 64) & 4095];
    s3 += buf[(idx + 96) & 4095];
    idx = (idx + 128) & 4095;
  }
  double s = s0 + s1 + s2 + s3;
  if (s == 12345.678) out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void k_dmma_lat(double* out, long iters) {
  double a = 1.0, b = 1.0, d0 = 0, d1 = 0;
  for (long it = 0; it < iters; ++it) dmma(d0, d1, a, b);
  if (d0 + d1 == 12345.678) out[threadIdx.x] = d0;
}

template <class F>
static float time_ms(F launch, int reps = 1) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  launch();  // warm
  CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(a));
  for (int r = 0; r < reps; ++r) launch();
  CK(cudaEventRecord(b));
  CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  CK(cudaGetLastError());
  return ms / reps;
}

int main() {
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  int sms = p.multiProcessorCount;
  double* out; CK(cudaMalloc(&out, 1 << 24));
  printf("{\n  \"gpu\": \"%s\", \"sms\": %d,\n", p.name, sms);

  // DMMA throughput: grid = 4*sms CTAs x 256 threads (8 warps/CTA -> 32 warps/SM), 8 accumulators per warp.
  const int thr = 256, cta = 4 * sms;
  long it_burst = 4000;
  float ms = time_ms([&] { k_dmma<8><<<cta, thr>>>(out, it_burst, 1.0); }, 3);
  double n_mma = (double)cta * (thr / 32) * it_burst * 8;
  double dmma_tf = n_mma * 512.0 / (ms * 1e-3) / 1e12;
  // sustained: ~3 s
  long it_sus = (long)(it_burst * 3000.0 / ms);
  float ms_s = time_ms([&] { k_dmma<8><<<cta, thr>>>(out, it_sus, 1.0); }, 1);
  double dmma_tf_s = (double)cta * (thr / 32) * it_sus * 8 * 512.0 / (ms_s * 1e-3) / 1e12;
  // occupancy sweep (warps per SM) for DMMA
  printf("  \"dmma_tflops\": %.3f, \"dmma_tflops_sustained\": %.3f,\n", dmma_tf, dmma_tf_s);
  printf("  \"dmma_sweep\": [");
  const int wl[] = {4, 8, 16, 32, 48};
  for (int wi = 0; wi < 5; ++wi) {
    int w = wl[wi];
    int t = std::min(w, 32) * 32; int c = sms * std::max(1, w / 32) * (w > 32 ? 1 : 1);
    if (w == 48) { t = 384; c = 2 * sms; }
    float m = time_ms([&] { k_dmma<8><<<c, t>>>(out, it_burst, 1.0); }, 2);
    double tf = (double)c * (t / 32) * it_burst * 8 * 512.0 / (m * 1e-3) / 1e12;
    printf("%s{\"warps_per_sm\": %d, \"tflops\": %.3f}", wi ? ", " : "", (c / sms) * (t / 32), tf);
  }
  printf("],\n");
  // accumulator-count sweep at 32 warps/SM
  {
    float m1 = time_ms([&] { k_dmma<1><<<cta, thr>>>(out, it_burst * 8, 1.0); }, 2);
    float m2 = time_ms([&] { k_dmma<2><<<cta, thr>>>(out, it_burst * 4, 1.0); }, 2);
    float m4 = time_ms([&] { k_dmma<4><<<cta, thr>>>(out, it_burst * 2, 1.0); }, 2);
    double base = (double)cta * (thr / 32) * it_burst * 8 * 512.0 / 1e12;
    printf("  \"dmma_acc_sweep_tflops\": {\"1\": %.3f, \"2\": %.3f, \"4\": %.3f, \"8\": %.3f},\n",
           base / (m1 * 1e-3), base / (m2 * 1e-3), base / (m4 * 1e-3), dmma_tf);
  }
  // DMMA latency (one warp, one chain)
  {
    long li = 100000;
    float m = time_ms([&] { k_dmma_lat<<<1, 32>>>(out, li); }, 1);
    printf("  \"dmma_latency_ns\": %.3f,\n", m * 1e6 / li);
  }
  // DFMA
  long itf = 4000;
  float msf = time_ms([&] { k_dfma<8><<<cta, thr>>>(out, itf, 1.0); }, 3);
  double n_fma = (double)cta * thr * itf * 8;
  double dfma_tf = n_fma * 2 / (msf * 1e-3) / 1e12;
  long itf_s = (long)(itf * 3000.0 / msf);
  float msf_s = time_ms([&] { k_dfma<8><<<cta, thr>>>(out, itf_s, 1.0); }, 1);
  double dfma_tf_s = (double)cta * thr * itf_s * 8 * 2 / (msf_s * 1e-3) / 1e12;
  printf("  \"dfma_tflops\": %.3f, \"dfma_tflops_sustained\": %.3f,\n", dfma_tf, dfma_tf_s);
  // Mixed: 16 warps/CTA, 2 CTAs/SM; even warps DMMA, odd DFMA.  Pick iteration counts so that
  // each half alone would take about the same time.
  {
    const int t = 512, c = 2 * sms;
    long im = 2000;
    // half the warps doing DMMA: per-warp flops per it = 8*512; DFMA warp: 32*8*2 = 512/it
    long ifm = (long)(im * 8.0 * 512.0 / 512.0 * (dfma_tf / dmma_tf));
    float m_mma = time_ms([&] { k_mixed<<<c, t>>>(out, im, 0, 1.0); }, 2);
    float m_fma = time_ms([&] { k_mixed<<<c, t>>>(out, 0, ifm, 1.0); }, 2);
    float m_both = time_ms([&] { k_mixed<<<c, t>>>(out, im, ifm, 1.0); }, 2);
    double fl_mma = (double)c * 8 * im * 8 * 512.0, fl_fma = (double)c * 8 * 32 * ifm * 8 * 2.0;
    printf("  \"mixed\": {\"ms_dmma_only\": %.3f, \"ms_dfma_only\": %.3f, \"ms_both\": %.3f, "
           "\"combined_tflops\": %.3f, \"verdict\": \"%s\"},\n",
           m_mma, m_fma, m_both, (fl_mma + fl_fma) / (m_both * 1e-3) / 1e12,
           m_both < 0.75 * (m_mma + m_fma) ? "pipes overlap" : "pipes shared");
  }
  // HBM copy
  {
    size_t bytes = (size_t)2 << 30;  // 2 GiB each way
    size_t n = bytes / sizeof(double2);
    double2 *a, *b;
    CK(cudaMalloc(&a, bytes)); CK(cudaMalloc(&b, bytes));
    CK(cudaMemset(a, 0, bytes)); CK(cudaMemset(b, 0, bytes));
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      float m = time_ms([&] { k_copy<<<sms * 8, 512>>>(a, b, n); }, 1);
      best = std::min(best, m);
    }
    printf("  \"hbm_copy_gbs\": %.1f,\n", 2.0 * bytes / (best * 1e-3) / 1e9);
    CK(cudaFree(a)); CK(cudaFree(b));
  }
  // LDS.64
  {
    long il = 20000;
    float m = time_ms([&] { k_lds<<<sms * 4, 256>>>(out, il); }, 2);
    double bytes = (double)sms * 4 * 256 * il * 4 * 8;
    double clk_ghz = p.clockRate * 1e-6;
    printf("  \"lds64_tbs\": %.2f, \"lds64_bytes_per_clk_per_sm_at_max_clock\": %.1f,\n",
           bytes / (m * 1e-3) / 1e12, bytes / (m * 1e-3) / (sms * clk_ghz * 1e9));
  }
  printf("  \"clock_rate_mhz_attr\": %.0f\n}\n", p.clockRate * 1e-3);
  return 0;
}
