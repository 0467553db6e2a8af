// Standalone check of k_direct2d_wf (debug harness, not part of libcsx): R=1, TF=1, one strip.
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cmath>
#include "../../paper_conf_ppopp_chenlwbwmyzcy24_b200/csrc/kernels_direct2d_wf.cu"
namespace csx {
int num_sms() { return 148; }
int64_t persistent_grid(int occ, int max_ctas, int64_t items) { return items < 1 ? 1 : (items > 148 ? 148 : items); }
}
using namespace csx;
int main() {
  const int E1 = 20, E2 = 40, G = 16;
  const int A1 = E1 + 2 * G + 200, A2 = 128 + E2 + 256;
  std::vector<double> h((size_t)A1 * A2, 0.0), out((size_t)E1 * E2, -7.0);
  for (int y = 0; y < E1; ++y) for (int x = 0; x < E2; ++x) h[(size_t)(y + G) * A2 + x + 128] = 1000.0 * y + x;
  double *d, *o;
  cudaMalloc(&d, h.size() * 8); cudaMalloc(&o, out.size() * 8);
  cudaMemcpy(d, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(o, out.data(), out.size() * 8, cudaMemcpyHostToDevice);
  DirectArgs a{};
  a.src = CView{d + (size_t)G * A2 + 128, (int64_t)A1 * A2, A2};
  a.dst = View{o, (int64_t)E1 * E2, E2};
  a.E[0] = 1; a.E[1] = E1; a.E[2] = E2;
  a.GE[0] = 1; a.GE[1] = E1; a.GE[2] = E2;
  a.r = 1; a.tf = 1; a.fixed_bc = 0; a.ndim = 2;
  double w[9] = {0, 0, 0, 0, 0, 0, 0, 1, 0};  // pure shift: out[y][x] = in[y+1][x]
  const char* ws = getenv("W");
  if (ws && ws[0] == 'c') { for (int i = 0; i < 9; ++i) w[i] = 0; w[4] = 1; }
  if (ws && ws[0] == 'l') { for (int i = 0; i < 9; ++i) w[i] = 0; w[3] = 1; }
  if (ws && ws[0] == 'u') { for (int i = 0; i < 9; ++i) w[i] = 0; w[1] = 1; }
  cudaError_t e = launch_direct2d_wf(a, w, 0);
  printf("launch %s\n", cudaGetErrorString(e));
  e = cudaDeviceSynchronize();
  printf("sync %s\n", cudaGetErrorString(e));
  cudaMemcpy(out.data(), o, out.size() * 8, cudaMemcpyDeviceToHost);
  for (int y = 0; y < 6; ++y) {
    for (int x = 0; x < 8; ++x) printf("%8.0f ", out[(size_t)y * E2 + x]);
    printf("\n");
  }
  return 0;
}
