// kernels_peer.cu — the slab halo exchange over NVLink peer memory, without NCCL on the data
// path (the paper is single-GPU, P.2757-2758).
//
// Every rank maps its neighbours' slab ping-pong buffers and flag blocks (CUDA IPC over
// NVLink / NVSwitch; a self-neighbour on a 1-rank ring uses its own pointers).  After a pass,
// k_peer_push copies this rank's first / last r*Tf slab rows of the new grid straight into the
// up / down neighbour's ghost rows of the SAME buffer (the neighbour's next-pass source), with
// peer stores issued by the SMs; the last CTA to finish publishes the epoch in the neighbours'
// READY flags (fence + st.release.sys, the classic last-block pattern).  Before writing, the
// push waits until the neighbour has finished reading those ghost rows in its previous pass
// (FREED flags).  k_peer_wait blocks the compute stream until this rank's own ghosts are READY.
// Flags are monotonically increasing 64-bit epochs (no reset between runs).
#include <cuda_runtime.h>

#include <cstdint>

#include "kernels.cuh"

namespace csx {

__device__ __forceinline__ unsigned long long ld_acquire_sys(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];\n" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_sys(unsigned long long* p, unsigned long long v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;\n" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ unsigned long long global_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Spin on a peer-written epoch.  A neighbour that never arrives (a rank died or called with a
// different T) must not hang the GPU: after 60 s the kernel traps, so the run fails with a CUDA
// error at the caller's next synchronisation instead of spinning forever.
__device__ __forceinline__ void spin_until(const unsigned long long* p, unsigned long long v) {
  if (!p) return;
  const unsigned long long t0 = global_ns();
  while (ld_acquire_sys(p) < v) {
    __nanosleep(256);
    if (global_ns() - t0 > 60ull * 1000000000ull) __trap();
  }
}

__global__ void k_peer_push(PeerPushArgs a) {
  if (threadIdx.x == 0) {  // the neighbour no longer reads the ghost rows we overwrite
    if (a.dst_up) spin_until(a.freed_up, a.wait_v);
    if (a.dst_down) spin_until(a.freed_down, a.wait_v);
  }
  __syncthreads();
  const int64_t tid = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.x;
  const bool vec = a.vec2 != 0;
  for (int side = 0; side < 2; ++side) {
    double* dst = side == 0 ? a.dst_up : a.dst_down;
    const double* src = side == 0 ? a.src_first : a.src_last;
    if (!dst) continue;
    if (vec) {
      const int64_t n2 = a.n / 2;
      const double2* s2 = reinterpret_cast<const double2*>(src);
      double2* d2 = reinterpret_cast<double2*>(dst);
      for (int64_t i = tid; i < n2; i += nth) d2[i] = s2[i];
      if ((a.n & 1) && tid == 0) dst[a.n - 1] = src[a.n - 1];
    } else {
      for (int64_t i = tid; i < a.n; i += nth) dst[i] = src[i];
    }
  }
  __threadfence_system();  // this CTA's peer stores are visible system-wide before it counts
  __syncthreads();
  if (threadIdx.x == 0) {
    const unsigned int done = atomicAdd(a.counter, 1u);
    if (done == gridDim.x - 1) {  // last CTA: every copy is performed -> publish the epochs
      *a.counter = 0u;
      __threadfence_system();
      if (a.ready_v) {
        if (a.ready_up_remote) st_release_sys(a.ready_up_remote, a.ready_v);
        if (a.ready_down_remote) st_release_sys(a.ready_down_remote, a.ready_v);
      }
      if (a.freed_v) {
        if (a.freed_up_remote) st_release_sys(a.freed_up_remote, a.freed_v);
        if (a.freed_down_remote) st_release_sys(a.freed_down_remote, a.freed_v);
      }
    }
  }
}

__global__ void k_peer_wait(const unsigned long long* ready_top, const unsigned long long* ready_bottom,
                            unsigned long long v) {
  if (threadIdx.x == 0) {
    spin_until(ready_top, v);
    spin_until(ready_bottom, v);
  }
}

cudaError_t launch_peer_push(const PeerPushArgs& a, cudaStream_t st) {
  int grid = 1;
  if (a.n > 0) {
    const int64_t per = 256LL * 8;  // doubles per CTA per sweep (double2 x 256 threads x 4)
    grid = (int)((a.n + per - 1) / per);
    if (grid > 16) grid = 16;
    if (grid < 1) grid = 1;
  }
  k_peer_push<<<grid, 256, 0, st>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_peer_wait(const unsigned long long* ready_top, const unsigned long long* ready_bottom,
                             unsigned long long v, cudaStream_t st) {
  k_peer_wait<<<1, 32, 0, st>>>(ready_top, ready_bottom, v);
  return cudaGetLastError();
}

}  // namespace csx
