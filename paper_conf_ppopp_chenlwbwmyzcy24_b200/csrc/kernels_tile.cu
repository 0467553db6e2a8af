// kernels_tile.cu — engine TC_TILE (B200 variant of the stencil-as-GEMM).  Not built yet.
#include <cuda_runtime.h>

#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

bool tile_kernel_exists(int ndim, int nk) {
  (void)ndim;
  (void)nk;
  return false;
}

cudaError_t launch_tile(int ndim, int nk, const S2RArgs& a, cudaStream_t st) {
  (void)ndim; (void)nk; (void)a; (void)st;
  return cudaErrorNotSupported;
}

}  // namespace csx
