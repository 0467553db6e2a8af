// comm.cpp — slab-sharded runs over NCCL (not in the paper, which is
// single-GPU, P.2757-2758).
//
// The grid is cut into slabs along the slowest axis (extents[0]); rank i owns rows
// [floor(i N0 / p), floor((i+1) N0 / p)).  Every fused pass of Tf steps needs a halo of r*Tf rows
// from each neighbour: before the pass, the ghost rows of the padded slab grid are filled by
// ncclSend/ncclRecv in one group (a ring for PERIODIC; the end ranks of a FIXED grid have no
// outer neighbour and keep zero ghosts, which only feed the held frame).  Then the local slab runs
// the same TC pass kernel as the single-GPU path, with the FIXED band fix-up told where the global
// faces are.
#include <cuda_runtime.h>
#include <nccl.h>

#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "csx_internal.h"
#include "csx_run.h"
#include "kernels.cuh"

struct csx_comm_s {
  ncclComm_t comm = nullptr;
  int rank = 0, nranks = 1;
  cudaStream_t cs = nullptr;       // halo-exchange stream (overlaps the interior kernels)
  cudaEvent_t ev_edge = nullptr;   // compute -> comm: this pass's edge tiles are written
  cudaEvent_t ev_x = nullptr;      // comm -> compute: the next pass's ghosts have arrived
};

namespace csx {

static csx_status nccl_fail(ncclResult_t r, const char* where) {
  return fail(CSX_ERR_NCCL, std::string(where) + ": " + ncclGetErrorString(r));
}

// Pointer to the first element of slab "row" k along the slab axis a0 in a padded grid (row
// = plane for 3D, grid row for 2D, cell for 1D), including the ghost columns of that row, and
// the element count of `h` consecutive such rows.
static void slab_rows(const Padded& pd, double* base, int a0, int64_t k, int h, double** ptr,
                      size_t* count) {
  if (a0 == 0) {
    *ptr = base + (pd.O[0] + k) * pd.s0;
    *count = (size_t)h * pd.s0;
  } else if (a0 == 1) {
    *ptr = base + (pd.O[1] + k) * pd.s1;
    *count = (size_t)h * pd.s1;
  } else {
    *ptr = base + pd.O[2] + k;
    *count = (size_t)h;
  }
}

// Halo-exchange schedule (csx_halo_schedule).  Every rank posts, in this order: send its last
// h rows down, receive its top ghost from up, send its first h rows up, receive its bottom ghost
// from down.  With that fixed order the k-th message between any pair is matched correctly even
// when up == down (two ranks, or one rank talking to itself on a PERIODIC ring).
static int halo_schedule(const csx_plan_s* p, int rank, int nranks, int64_t El, int64_t* ops) {
  const int h = p->halo;
  const bool periodic = p->bc == CSX_BC_PERIODIC;
  int up = rank - 1, down = rank + 1;
  if (periodic) {
    up = (up + nranks) % nranks;
    down = down % nranks;
  } else {
    if (up < 0) up = -1;
    if (down >= nranks) down = -1;
  }
  int n = 0;
  auto op = [&](int kind, int peer, int64_t row) {
    ops[4 * n] = kind; ops[4 * n + 1] = peer; ops[4 * n + 2] = row; ops[4 * n + 3] = h;
    ++n;
  };
  if (down >= 0) op(0, down, El - h);
  if (up >= 0) { op(1, up, -h); op(0, up, 0); }
  if (down >= 0) op(1, down, El);
  return n;
}

static csx_status exchange(csx_plan_s* p, csx_comm_s* c, double* base, int a0, int64_t El,
                           cudaStream_t st) {
  int64_t ops[16];
  const int nops = halo_schedule(p, c->rank, c->nranks, El, ops);
  ncclResult_t r = ncclGroupStart();
  if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
  for (int k = 0; k < nops; ++k) {
    double* ptr;
    size_t n;
    slab_rows(p->spad, base, a0, ops[4 * k + 2], (int)ops[4 * k + 3], &ptr, &n);
    if (ops[4 * k] == 0) r = ncclSend(ptr, n, ncclDouble, (int)ops[4 * k + 1], c->comm, st);
    else r = ncclRecv(ptr, n, ncclDouble, (int)ops[4 * k + 1], c->comm, st);
    if (r != ncclSuccess) return nccl_fail(r, ops[4 * k] == 0 ? "ncclSend" : "ncclRecv");
  }
  r = ncclGroupEnd();
  if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd");
  return CSX_OK;
}

}  // namespace csx

using namespace csx;

extern "C" {

csx_status csx_comm_create(const void* nccl_unique_id, int rank, int nranks, csx_comm_t* out) {
  if (!nccl_unique_id || !out || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad communicator arguments");
  *out = nullptr;
  csx_comm_s* c = new (std::nothrow) csx_comm_s();
  if (!c) return fail(CSX_ERR_OUT_OF_MEMORY, "comm allocation");
  ncclUniqueId id;
  std::memcpy(&id, nccl_unique_id, sizeof(id));
  ncclResult_t r = ncclCommInitRank(&c->comm, nranks, id, rank);
  if (r != ncclSuccess) {
    delete c;
    return nccl_fail(r, "ncclCommInitRank");
  }
  c->rank = rank;
  c->nranks = nranks;
  if (cudaStreamCreateWithFlags(&c->cs, cudaStreamNonBlocking) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_edge, cudaEventDisableTiming) != cudaSuccess ||
      cudaEventCreateWithFlags(&c->ev_x, cudaEventDisableTiming) != cudaSuccess) {
    ncclCommDestroy(c->comm);
    delete c;
    return fail(CSX_ERR_CUDA, "comm stream / event creation failed");
  }
  *out = c;
  return CSX_OK;
}

csx_status csx_comm_destroy(csx_comm_t c) {
  if (!c) return CSX_OK;
  if (c->comm) ncclCommDestroy(c->comm);
  if (c->ev_edge) cudaEventDestroy(c->ev_edge);
  if (c->ev_x) cudaEventDestroy(c->ev_x);
  if (c->cs) cudaStreamDestroy(c->cs);
  delete c;
  return CSX_OK;
}

csx_status csx_nccl_unique_id(void* out128) {
  if (!out128) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL");
  ncclUniqueId id;
  ncclResult_t r = ncclGetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  std::memcpy(out128, &id, sizeof(id));
  return CSX_OK;
}

csx_status csx_shard_rows(const csx_plan_t p, int rank, int nranks, int64_t* lo, int64_t* hi) {
  if (!p || !lo || !hi || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad shard arguments");
  const int64_t N0 = p->ext[0];
  *lo = (int64_t)rank * N0 / nranks;
  *hi = (int64_t)(rank + 1) * N0 / nranks;
  return CSX_OK;
}

csx_status csx_halo_schedule(const csx_plan_t p, int rank, int nranks, int64_t* ops, int* nops) {
  if (!p || !ops || !nops || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad arguments");
  int64_t lo, hi;
  csx_status s = csx_shard_rows(p, rank, nranks, &lo, &hi);
  if (s != CSX_OK) return s;
  *nops = halo_schedule(p, rank, nranks, hi - lo, ops);
  return CSX_OK;
}

csx_status csx_run_sharded(csx_plan_t p, csx_comm_t c, const double* d_in, double* d_out,
                           int64_t T, void* stream) {
  if (!p || !c || !d_in || !d_out) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  if (T < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "timesteps < 0");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int64_t lo, hi;
  csx_status s = csx_shard_rows(p, c->rank, c->nranks, &lo, &hi);
  if (s != CSX_OK) return s;
  const int a0 = 3 - p->ndim;  // normalised slab axis
  int64_t El[3] = {p->E[0], p->E[1], p->E[2]};
  El[a0] = hi - lo;
  if (El[a0] < p->halo || El[a0] < 1)
    return fail(CSX_ERR_UNSUPPORTED, "a rank owns fewer rows than the halo depth r*Tf");
  const int64_t n = El[0] * El[1] * El[2];
  s = ensure_device(p);
  if (s != CSX_OK) return s;
  if (T == 0) {
    if (d_in != d_out) {
      cudaError_t e = cudaMemcpyAsync(d_out, d_in, n * sizeof(double), cudaMemcpyDeviceToDevice, st);
      if (e != cudaSuccess) return cuda_fail(e, "copy");
    }
    return CSX_OK;
  }
  if (p->s_rank != c->rank || p->s_nranks != c->nranks) {
    cudaFree(p->d_sbuf[0]);
    cudaFree(p->d_sbuf[1]);
    p->d_sbuf[0] = p->d_sbuf[1] = nullptr;
    s = ensure_grid(p, &p->spad, p->d_sbuf, El);
    if (s != CSX_OK) return s;
    p->s_rank = c->rank;
    p->s_nranks = c->nranks;
    p->s_lo = lo;
    p->s_hi = hi;
  }
  const Padded& pd = p->spad;
  const int real[3] = {p->ndim == 3, p->ndim >= 2, 1};
  int fill[3] = {real[0], real[1], real[2]};
  fill[a0] = 0;  // the slab axis is filled by the exchange
  View b[2];
  for (int i = 0; i < 2; ++i) b[i] = View{p->d_sbuf[i] + pd.origin(), pd.s0, pd.s1};
  cudaError_t e = launch_pack(d_in, b[0], El, st);
  if (e != cudaSuccess) return cuda_fail(e, "pack");
  p->n_launches += 1;
  auto refresh = [&](int i) -> csx_status {
    if (p->bc == CSX_BC_PERIODIC) {
      cudaError_t e2 = launch_ghost_fill(b[i], El, real, fill, p->halo, st);
      if (e2 != cudaSuccess) return cuda_fail(e2, "ghost fill");
      p->n_launches += (real[0] && fill[0]) + (real[1] && fill[1]) + fill[2];
    }
    return exchange(p, c, p->d_sbuf[i], a0, El[a0], st);
  };
  s = refresh(0);
  if (s != CSX_OK) return s;
  const int64_t nmain = T / p->tf;
  const int rem = (int)(T % p->tf);
  const int64_t npass = nmain + (rem ? 1 : 0);
  const View out{d_out, El[1] * El[2], El[2]};
  // TC_TILE overlaps the halo exchange of pass i+1 with the interior tiles of pass i+1:
  //   compute: interior(i) -> [wait ghosts(i)] -> edge(i) + fix-ups -> ghost fill -> ev_edge
  //   comm:    [wait ev_edge] -> exchange into dst(i) -> ev_x
  // interior tiles never read ghost rows; edge tiles are the first / last slab tiles.
  // (CSX_FORCE_OVERLAP=1 exercises the overlapped schedule on a single rank, for tests)
  const char* fo = getenv("CSX_FORCE_OVERLAP");
  const bool overlap = p->engine == CSX_ENGINE_TC_TILE && (c->nranks > 1 || (fo && fo[0] == '1'));
  const int max_ctas = overlap ? num_sms() - 2 : 0;  // leave SMs for the NCCL kernels
  int cur = 0;
  for (int64_t i = 0; i < npass; ++i) {
    const int tfp = i < nmain ? p->tf : rem;
    const bool last = i == npass - 1;
    PassCtx pc;
    pc.src = CView{b[cur].p, b[cur].s0, b[cur].s1, pd.O[0], pd.O[1], pd.O[2], pd.A[0]};
    pc.dst = last ? out : b[cur ^ 1];
    for (int a = 0; a < 3; ++a) { pc.E[a] = El[a]; pc.gorg[a] = 0; }
    pc.gorg[a0] = lo;
    if (!overlap) {
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (!last) {
        s = refresh(cur ^ 1);
        if (s != CSX_OK) return s;
      }
    } else {
      pc.max_ctas = max_ctas;
      pc.part = 1;
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (i > 0) {
        cudaError_t e2 = cudaStreamWaitEvent(st, c->ev_x, 0);
        if (e2 != cudaSuccess) return cuda_fail(e2, "wait halo");
      }
      pc.part = 2;
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (!last) {
        if (p->bc == CSX_BC_PERIODIC) {
          cudaError_t e2 = launch_ghost_fill(b[cur ^ 1], El, real, fill, p->halo, st);
          if (e2 != cudaSuccess) return cuda_fail(e2, "ghost fill");
          p->n_launches += (real[0] && fill[0]) + (real[1] && fill[1]) + fill[2];
        }
        cudaError_t e2 = cudaEventRecord(c->ev_edge, st);
        if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(c->cs, c->ev_edge, 0);
        if (e2 != cudaSuccess) return cuda_fail(e2, "edge event");
        s = exchange(p, c, p->d_sbuf[cur ^ 1], a0, El[a0], c->cs);
        if (s != CSX_OK) return s;
        e2 = cudaEventRecord(c->ev_x, c->cs);
        if (e2 != cudaSuccess) return cuda_fail(e2, "halo event");
      }
    }
    cur ^= 1;
  }
  return CSX_OK;
}

}  // extern "C"
