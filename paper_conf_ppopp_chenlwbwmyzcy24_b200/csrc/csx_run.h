// csx_run.h — pass-loop plumbing shared by api.cpp (single GPU) and comm.cpp (sharded).
#pragma once
#include <cuda_runtime.h>

#include <vector>

#include "csx_internal.h"
#include "kernels.cuh"

namespace csx {

// Everything one fused pass needs to know about the grid it runs on.
struct PassCtx {
  CView src;                      // padded source at its interior origin
  View dst;                       // destination at its interior origin
  int64_t E[3];                   // local interior extents (normalised)
  int64_t gorg[3];                // local origin in global coordinates (slab offset)
  int part = 0;                   // TC_TILE slab-tile subset: 0 all, 1 interior, 2 edge (+ fix-ups)
  int max_ctas = 0;               // persistent-grid cap (leaves SMs to NCCL while overlapping)
};

csx_status cuda_fail(cudaError_t e, const char* where);
csx_status ensure_device(csx_plan_s* p);
csx_status ensure_grid(csx_plan_s* p, Padded* pd, double** bufs, const int64_t* E);
csx_status run_pass(csx_plan_s* p, Pass& ps, const PassCtx& c, cudaStream_t st);
csx_status run_local(csx_plan_s* p, const double* d_in, double* d_out, int64_t T, cudaStream_t st);
void direct_tile(int ndim, int* B);
bool tile_kernel_exists(int ndim, int radius, int tf);
bool tile_reads_dense(const double* p, const int64_t* E);

}  // namespace csx
