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
#include <cuda.h>
#include <cudaTypedefs.h>
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
    if (r != ncclSuccess) {  // close the group before reporting, so later NCCL calls fail cleanly
      ncclGroupEnd();
      return nccl_fail(r, ops[4 * k] == 0 ? "ncclSend" : "ncclRecv");
    }
  }
  r = ncclGroupEnd();
  if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd");
  return CSX_OK;
}


// ---- NVLink peer-memory exchange (csx_run_sharded_peer) -----------------------------------

// Push this rank's first / last h slab rows of buffer `buf` into the neighbours' ghost rows of
// the same buffer, after they have finished reading them (FREED >= wait_v); publish READY /
// FREED epochs (0 = none).  n == 0 pushes only the flags.
static csx_status peer_push(csx_plan_s* p, csx_peer_s* q, int buf, bool copy, unsigned long long wait_v,
                            unsigned long long ready_v, unsigned long long freed_v, cudaStream_t st) {
  const int a0 = 3 - p->ndim;
  const int h = p->halo;
  const Padded& pd = p->spad;
  PeerPushArgs a;
  double* mine = p->d_sbuf[buf];
  size_t n = 0;
  double* ptr = nullptr;
  if (copy) {
    slab_rows(pd, mine, a0, 0, h, &ptr, &n);
    a.src_first = ptr;
    slab_rows(pd, mine, a0, q->El - h, h, &ptr, &n);
    a.src_last = ptr;
    if (q->up >= 0) {  // up's bottom ghost rows El_up .. El_up + h - 1 (same layout but El)
      slab_rows(pd, q->up_buf[buf], a0, q->El_up, h, &ptr, &n);
      a.dst_up = ptr;
    }
    if (q->down >= 0) {  // down's top ghost rows -h .. -1
      slab_rows(pd, q->down_buf[buf], a0, -h, h, &ptr, &n);
      a.dst_down = ptr;
    }
    a.n = (int64_t)n;
    auto al = [](const void* x) { return (reinterpret_cast<uintptr_t>(x) & 15) == 0; };
    a.vec2 = al(a.src_first) && al(a.src_last) && (!a.dst_up || al(a.dst_up)) &&
             (!a.dst_down || al(a.dst_down));
  }
  a.freed_up = q->flags + 2;
  a.freed_down = q->flags + 3;
  a.wait_v = wait_v;
  if (q->up >= 0) {
    a.ready_up_remote = q->up_flags + 1;  // my first rows are up's bottom ghosts
    a.freed_up_remote = q->up_flags + 3;  // I am up's down neighbour
  }
  if (q->down >= 0) {
    a.ready_down_remote = q->down_flags + 0;
    a.freed_down_remote = q->down_flags + 2;
  }
  a.ready_v = ready_v;
  a.freed_v = freed_v;
  a.counter = reinterpret_cast<unsigned int*>(q->flags + 4);
  cudaError_t e = launch_peer_push(a, st);
  if (e != cudaSuccess) return cuda_fail(e, "peer push");
  p->n_launches += 1;
  return CSX_OK;
}

static csx_status peer_wait(csx_plan_s* p, csx_peer_s* q, unsigned long long v, cudaStream_t st) {
  if (q->up < 0 && q->down < 0) return CSX_OK;
  cudaError_t e = launch_peer_wait(q->up >= 0 ? q->flags + 0 : nullptr,
                                   q->down >= 0 ? q->flags + 1 : nullptr, v, st);
  if (e != cudaSuccess) return cuda_fail(e, "peer wait");
  p->n_launches += 1;
  return CSX_OK;
}

// The sharded pass loop, shared by the NCCL (c != null) and the peer-memory (q != null)
// exchanges.  Epochs of the peer exchange for a run with base E and P passes:
//   initial push  : wait FREED >= E, write ghosts of buffer 0, READY = E + 1
//   pass i        : edge tiles wait READY >= E + i + 1
//   push after i  : wait FREED >= E + i, write ghosts of dst(i), READY = E + i + 2, FREED = E + i + 1
//   end of run    : FREED = E + P (every ghost read of this run is done); next base E + P
static csx_status run_sharded_impl(csx_plan_s* p, csx_comm_s* c, csx_peer_s* q, const double* d_in,
                                   double* d_out, int64_t T, cudaStream_t st) {
  if (T < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "timesteps < 0");
  const int rank = c ? c->rank : q->rank, nranks = c ? c->nranks : q->nranks;
  int64_t lo, hi;
  csx_status s = csx_shard_rows(p, rank, nranks, &lo, &hi);
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
  if (q) {
    if (p->s_rank != rank || p->s_nranks != nranks || !p->d_sbuf[0])
      return fail(CSX_ERR_INTERNAL, "peer slab buffers changed after export");
  } else if (p->s_rank != rank || p->s_nranks != nranks || p->s_p1 != 0) {
    cudaFree(p->d_sbuf[0]);
    cudaFree(p->d_sbuf[1]);
    p->d_sbuf[0] = p->d_sbuf[1] = nullptr;
    s = ensure_grid(p, &p->spad, p->d_sbuf, El);
    if (s != CSX_OK) return s;
    p->s_rank = rank;
    p->s_nranks = nranks;
    p->s_p0 = p->s_p1 = 0;
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
  auto fill_other_axes = [&](int i) -> csx_status {
    if (p->bc == CSX_BC_PERIODIC) {
      cudaError_t e2 = launch_ghost_fill(b[i], El, real, fill, p->halo, st);
      if (e2 != cudaSuccess) return cuda_fail(e2, "ghost fill");
      p->n_launches += (real[0] && fill[0]) + (real[1] && fill[1]) + fill[2];
    }
    return CSX_OK;
  };
  const int64_t nmain = T / p->tf;
  const int rem = (int)(T % p->tf);
  const int64_t npass = nmain + (rem ? 1 : 0);
  const unsigned long long E0 = q ? q->epoch : 0;
  // initial ghosts of buffer 0
  s = fill_other_axes(0);
  if (s != CSX_OK) return s;
  if (q) {
    s = peer_push(p, q, 0, true, E0, E0 + 1, 0, st);
    if (s == CSX_OK) s = peer_wait(p, q, E0 + 1, st);
  } else {
    s = exchange(p, c, p->d_sbuf[0], a0, El[a0], st);
  }
  if (s != CSX_OK) return s;
  const View out{d_out, El[1] * El[2], El[2]};
  // TC_TILE overlaps the halo exchange of pass i+1 with the interior tiles of pass i+1:
  //   compute: interior(i) -> [wait ghosts(i)] -> edge(i) + fix-ups -> ghost fill -> ev_edge
  //   comm:    [wait ev_edge] -> exchange / peer push into dst(i) -> ev_x
  // interior tiles never read ghost rows; edge tiles are the first / last slab tiles.
  // (CSX_FORCE_OVERLAP=1 exercises the overlapped schedule on a single rank, for tests)
  const char* fo = getenv("CSX_FORCE_OVERLAP");
  const bool overlap = p->engine == CSX_ENGINE_TC_TILE && (nranks > 1 || (fo && fo[0] == '1'));
  int max_ctas = overlap ? num_sms() - 2 : 0;  // leave SMs for the exchange kernels
  if (p->max_ctas > 0 && (max_ctas == 0 || p->max_ctas < max_ctas)) max_ctas = p->max_ctas;
  cudaStream_t cs = c ? c->cs : (cudaStream_t)q->cs;
  cudaEvent_t ev_edge = c ? c->ev_edge : (cudaEvent_t)q->ev_edge;
  cudaEvent_t ev_x = c ? c->ev_x : (cudaEvent_t)q->ev_x;
  int cur = 0;
  for (int64_t i = 0; i < npass; ++i) {
    const int tfp = i < nmain ? p->tf : rem;
    const bool last = i == npass - 1;
    PassCtx pc;
    pc.src = CView{b[cur].p, b[cur].s0, b[cur].s1, pd.O[0], pd.O[1], pd.O[2], pd.A[0]};
    pc.dst = last ? out : b[cur ^ 1];
    for (int a = 0; a < 3; ++a) { pc.E[a] = El[a]; pc.gorg[a] = 0; }
    pc.gorg[a0] = lo;
    pc.max_ctas = p->max_ctas;
    if (!overlap) {
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (!last) {
        s = fill_other_axes(cur ^ 1);
        if (s != CSX_OK) return s;
        if (q) {
          s = peer_push(p, q, cur ^ 1, true, E0 + i, E0 + i + 2, E0 + i + 1, st);
          if (s == CSX_OK) s = peer_wait(p, q, E0 + i + 2, st);
        } else {
          s = exchange(p, c, p->d_sbuf[cur ^ 1], a0, El[a0], st);
        }
        if (s != CSX_OK) return s;
      }
    } else {
      pc.max_ctas = max_ctas;
      pc.part = 1;
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (i > 0) {
        cudaError_t e2 = cudaStreamWaitEvent(st, ev_x, 0);
        if (e2 != cudaSuccess) return cuda_fail(e2, "wait halo");
        if (q) {
          s = peer_wait(p, q, E0 + i + 1, st);
          if (s != CSX_OK) return s;
        }
      }
      pc.part = 2;
      s = run_pass(p, p->passes[tfp - 1], pc, st);
      if (s != CSX_OK) return s;
      if (!last) {
        s = fill_other_axes(cur ^ 1);
        if (s != CSX_OK) return s;
        cudaError_t e2 = cudaEventRecord(ev_edge, st);
        if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(cs, ev_edge, 0);
        if (e2 != cudaSuccess) return cuda_fail(e2, "edge event");
        if (q) s = peer_push(p, q, cur ^ 1, true, E0 + i, E0 + i + 2, E0 + i + 1, cs);
        else s = exchange(p, c, p->d_sbuf[cur ^ 1], a0, El[a0], cs);
        if (s != CSX_OK) return s;
        e2 = cudaEventRecord(ev_x, cs);
        if (e2 != cudaSuccess) return cuda_fail(e2, "halo event");
      }
    }
    cur ^= 1;
  }
  if (q) {  // every ghost read of this run is done: release the neighbours' next writes
    s = peer_push(p, q, 0, false, 0, 0, E0 + (unsigned long long)npass, st);
    if (s != CSX_OK) return s;
    q->epoch = E0 + (unsigned long long)npass;
  }
  return CSX_OK;
}


// ---- Pencil (block) decomposition over a p0 x p1 process grid ----------
//
// The two slowest stencil axes are split: 3D (z, y) — every rank owns a pencil running the full
// x extent; 2D (rows, cols) — blocks.  Rank = i0 * p1 + i1 owns [lo, hi) along axis a (index
// i0 of p0) and axis b (i1 of p1), floor partitions as for slabs.  Ghosts (depth r*Tf) are
// exchanged in two phases per pass, so that corners (edges in 3D) travel through the face
// neighbours: phase 0 along axis b for the owned range of axis a (strided faces, packed into a
// contiguous staging buffer by cudaMemcpy2DAsync around the NCCL group); phase 1 along axis a
// with full padded rows of axis b — which now include the axis-b ghosts just received.

#define COMM_CUDA(call, where)                  \
  do {                                          \
    cudaError_t e_ = (call);                    \
    if (e_ != cudaSuccess) return cuda_fail(e_, where); \
  } while (0)

static void pencil_axes(const csx_plan_s* p, int* aa, int* ab) {
  *aa = p->ndim == 3 ? 0 : 1;
  *ab = *aa + 1;
}

static void pencil_box(const csx_plan_s* p, int rank, int p0, int p1, int64_t* lo, int64_t* hi) {
  int aa, ab;
  pencil_axes(p, &aa, &ab);
  for (int a = 0; a < 3; ++a) { lo[a] = 0; hi[a] = p->E[a]; }
  const int i0 = rank / p1, i1 = rank - (rank / p1) * p1;
  lo[aa] = (int64_t)i0 * p->E[aa] / p0;
  hi[aa] = (int64_t)(i0 + 1) * p->E[aa] / p0;
  lo[ab] = (int64_t)i1 * p->E[ab] / p1;
  hi[ab] = (int64_t)(i1 + 1) * p->E[ab] / p1;
}

// ops of 5 int64: {phase (0 axis b, 1 axis a), kind (0 send, 1 recv), peer, first row along the
// phase's axis (local interior index; negative = low ghosts, >= local extent = high ghosts), rows}.
// Per phase the slab order: send high rows to the high neighbour, recv low ghosts from the low
// one, send low rows to the low neighbour, recv high ghosts from the high one.
static int pencil_schedule(const csx_plan_s* p, int rank, int p0, int p1, const int64_t* El, int64_t* ops) {
  int aa, ab;
  pencil_axes(p, &aa, &ab);
  const int h = p->halo;
  const bool periodic = p->bc == CSX_BC_PERIODIC;
  const int i0 = rank / p1, i1 = rank - (rank / p1) * p1;
  int n = 0;
  for (int phase = 0; phase < 2; ++phase) {
    const int np = phase == 0 ? p1 : p0, me = phase == 0 ? i1 : i0;
    const int64_t Ex = El[phase == 0 ? ab : aa];
    auto peer_of = [&](int idx) { return phase == 0 ? i0 * p1 + idx : idx * p1 + i1; };
    int lo_n = me - 1, hi_n = me + 1;
    if (periodic) {
      lo_n = (lo_n + np) % np;
      hi_n = hi_n % np;
    } else {
      if (lo_n < 0) lo_n = -1;
      if (hi_n >= np) hi_n = -1;
    }
    auto op = [&](int kind, int peer, int64_t row) {
      int64_t* o = ops + 5 * n++;
      o[0] = phase; o[1] = kind; o[2] = peer; o[3] = row; o[4] = h;
    };
    if (hi_n >= 0) op(0, peer_of(hi_n), Ex - h);
    if (lo_n >= 0) { op(1, peer_of(lo_n), -h); op(0, peer_of(lo_n), 0); }
    if (hi_n >= 0) op(1, peer_of(hi_n), Ex);
  }
  return n;
}

// A face of h rows along axis b (phase 0) as a 2D copy: `height` runs of `width` contiguous
// doubles, `pitch` apart.  3D (b = y): one run per z plane of the owned range, h padded rows
// each; 2D (b = cols): one run per owned row, h cells each.
static void face_b(const csx_plan_s* p, const Padded& pd, double* base, int64_t row, int h,
                   const int64_t* El, double** ptr, size_t* width, size_t* height, size_t* pitch) {
  if (p->ndim == 3) {
    *ptr = base + pd.O[0] * pd.s0 + (pd.O[1] + row) * pd.s1;
    *width = (size_t)h * pd.s1;
    *height = (size_t)El[0];
    *pitch = (size_t)pd.s0;
  } else {
    *ptr = base + pd.O[1] * pd.s1 + pd.O[2] + row;
    *width = (size_t)h;
    *height = (size_t)El[1];
    *pitch = (size_t)pd.s1;
  }
}

static csx_status exchange_pencil(csx_plan_s* p, csx_comm_s* c, double* base, int p0, int p1,
                                  const int64_t* El, cudaStream_t st) {
  int64_t ops[40];
  const int nops = pencil_schedule(p, c->rank, p0, p1, El, ops);
  int aa, ab;
  pencil_axes(p, &aa, &ab);
  const Padded& pd = p->spad;
  for (int phase = 0; phase < 2; ++phase) {
    size_t stage_off = 0;
    // phase 0: pack the strided send faces
    if (phase == 0)
      for (int k = 0; k < nops; ++k) {
        const int64_t* o = ops + 5 * k;
        if (o[0] != 0) continue;
        double* ptr;
        size_t w, hgt, pitch;
        face_b(p, pd, base, o[3], (int)o[4], El, &ptr, &w, &hgt, &pitch);
        if (o[1] == 0)
          COMM_CUDA(cudaMemcpy2DAsync(p->d_pstage + stage_off, w * 8, ptr, pitch * 8, w * 8, hgt,
                                     cudaMemcpyDeviceToDevice, st), "pack face");
        stage_off += w * hgt;
      }
    ncclResult_t r = ncclGroupStart();
    if (r != ncclSuccess) return nccl_fail(r, "ncclGroupStart");
    stage_off = 0;
    for (int k = 0; k < nops; ++k) {
      const int64_t* o = ops + 5 * k;
      if (o[0] != phase) continue;
      double* ptr;
      size_t n;
      if (phase == 0) {
        size_t w, hgt, pitch;
        face_b(p, pd, base, o[3], (int)o[4], El, &ptr, &w, &hgt, &pitch);
        ptr = p->d_pstage + stage_off;
        n = w * hgt;
        stage_off += n;
      } else {
        slab_rows(pd, base, aa, o[3], (int)o[4], &ptr, &n);
      }
      if (o[1] == 0) r = ncclSend(ptr, n, ncclDouble, (int)o[2], c->comm, st);
      else r = ncclRecv(ptr, n, ncclDouble, (int)o[2], c->comm, st);
      if (r != ncclSuccess) {
        ncclGroupEnd();
        return nccl_fail(r, o[1] == 0 ? "ncclSend" : "ncclRecv");
      }
    }
    r = ncclGroupEnd();
    if (r != ncclSuccess) return nccl_fail(r, "ncclGroupEnd");
    // phase 0: unpack the received faces into the axis-b ghosts
    if (phase == 0) {
      stage_off = 0;
      for (int k = 0; k < nops; ++k) {
        const int64_t* o = ops + 5 * k;
        if (o[0] != 0) continue;
        double* ptr;
        size_t w, hgt, pitch;
        face_b(p, pd, base, o[3], (int)o[4], El, &ptr, &w, &hgt, &pitch);
        if (o[1] == 1)
          COMM_CUDA(cudaMemcpy2DAsync(ptr, pitch * 8, p->d_pstage + stage_off, w * 8, w * 8, hgt,
                                     cudaMemcpyDeviceToDevice, st), "unpack face");
        stage_off += w * hgt;
      }
    }
  }
  return CSX_OK;
}

static csx_status run_sharded_pencil_impl(csx_plan_s* p, csx_comm_s* c, int p0, int p1,
                                          const double* d_in, double* d_out, int64_t T,
                                          cudaStream_t st) {
  if (T < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "timesteps < 0");
  if (p->ndim < 2) return fail(CSX_ERR_UNSUPPORTED, "pencil decomposition needs ndim >= 2");
  if (p0 < 1 || p1 < 1 || p0 * p1 != c->nranks)
    return fail(CSX_ERR_INVALID_ARGUMENT, "process grid p0 x p1 must equal the communicator size");
  const int rank = c->rank, nranks = c->nranks;
  int aa, ab;
  pencil_axes(p, &aa, &ab);
  int64_t lo[3], hi[3], El[3];
  pencil_box(p, rank, p0, p1, lo, hi);
  for (int a = 0; a < 3; ++a) El[a] = hi[a] - lo[a];
  if (El[aa] < p->halo || El[ab] < p->halo || El[aa] < 1 || El[ab] < 1)
    return fail(CSX_ERR_UNSUPPORTED, "a rank owns fewer rows than the halo depth r*Tf along a split axis");
  const int64_t n = El[0] * El[1] * El[2];
  csx_status s = ensure_device(p);
  if (s != CSX_OK) return s;
  if (T == 0) {
    if (d_in != d_out) {
      cudaError_t e = cudaMemcpyAsync(d_out, d_in, n * sizeof(double), cudaMemcpyDeviceToDevice, st);
      if (e != cudaSuccess) return cuda_fail(e, "copy");
    }
    return CSX_OK;
  }
  if (p->peer) return fail(CSX_ERR_INVALID_ARGUMENT, "plan is bound to a peer slab exchange");
  if (p->s_rank != rank || p->s_nranks != nranks || p->s_p0 != p0 || p->s_p1 != p1) {
    cudaFree(p->d_sbuf[0]);
    cudaFree(p->d_sbuf[1]);
    p->d_sbuf[0] = p->d_sbuf[1] = nullptr;
    s = ensure_grid(p, &p->spad, p->d_sbuf, El);
    if (s != CSX_OK) return s;
    p->s_rank = rank;
    p->s_nranks = nranks;
    p->s_p0 = p0;
    p->s_p1 = p1;
    p->s_lo = lo[aa];
    p->s_hi = hi[aa];
  }
  const Padded& pd = p->spad;
  // staging: the 4 phase-0 faces (2 send, 2 recv) of h rows each
  {
    double* ptr;
    size_t w, hgt, pitch;
    face_b(p, pd, p->d_sbuf[0], 0, p->halo, El, &ptr, &w, &hgt, &pitch);
    const size_t need = 4 * w * hgt;
    if (need > p->pstage_elems) {
      cudaFree(p->d_pstage);
      p->d_pstage = nullptr;
      p->pstage_elems = 0;
      COMM_CUDA(cudaMalloc(&p->d_pstage, need * sizeof(double)), "cudaMalloc(pencil staging)");
      p->pstage_elems = need;
    }
  }
  const int real[3] = {p->ndim == 3, p->ndim >= 2, 1};
  int fill[3] = {real[0], real[1], real[2]};
  fill[aa] = fill[ab] = 0;  // the split axes are filled by the exchange
  View b[2];
  for (int i = 0; i < 2; ++i) b[i] = View{p->d_sbuf[i] + pd.origin(), pd.s0, pd.s1};
  cudaError_t e = launch_pack(d_in, b[0], El, st);
  if (e != cudaSuccess) return cuda_fail(e, "pack");
  p->n_launches += 1;
  auto ghosts = [&](int i) -> csx_status {
    if (p->bc == CSX_BC_PERIODIC && (fill[0] || fill[1] || fill[2])) {
      cudaError_t e2 = launch_ghost_fill(b[i], El, real, fill, p->halo, st);
      if (e2 != cudaSuccess) return cuda_fail(e2, "ghost fill");
      p->n_launches += fill[0] + fill[1] + fill[2];
    }
    return exchange_pencil(p, c, p->d_sbuf[i], p0, p1, El, st);
  };
  const int64_t nmain = T / p->tf;
  const int rem = (int)(T % p->tf);
  const int64_t npass = nmain + (rem ? 1 : 0);
  s = ghosts(0);
  if (s != CSX_OK) return s;
  const View out{d_out, El[1] * El[2], El[2]};
  int cur = 0;
  for (int64_t i = 0; i < npass; ++i) {
    const int tfp = i < nmain ? p->tf : rem;
    const bool last = i == npass - 1;
    PassCtx pc;
    pc.src = CView{b[cur].p, b[cur].s0, b[cur].s1, pd.O[0], pd.O[1], pd.O[2], pd.A[0]};
    pc.dst = last ? out : b[cur ^ 1];
    for (int a = 0; a < 3; ++a) { pc.E[a] = El[a]; pc.gorg[a] = lo[a]; }
    pc.max_ctas = p->max_ctas;
    s = run_pass(p, p->passes[tfp - 1], pc, st);
    if (s != CSX_OK) return s;
    if (!last) {
      s = ghosts(cur ^ 1);
      if (s != CSX_OK) return s;
    }
    cur ^= 1;
  }
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
  return run_sharded_impl(p, c, nullptr, d_in, d_out, T, reinterpret_cast<cudaStream_t>(stream));
}

csx_status csx_shard_box(const csx_plan_t p, int rank, int p0, int p1, int64_t* lo, int64_t* hi) {
  if (!p || !lo || !hi || p0 < 1 || p1 < 1 || rank < 0 || rank >= p0 * p1)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad shard arguments");
  if (p->ndim < 2) return fail(CSX_ERR_UNSUPPORTED, "pencil decomposition needs ndim >= 2");
  int64_t l3[3], h3[3];
  pencil_box(p, rank, p0, p1, l3, h3);
  for (int a = 0; a < p->ndim; ++a) {  // user axis order: axis a of ndim = normalised 3 - ndim + a
    lo[a] = l3[3 - p->ndim + a];
    hi[a] = h3[3 - p->ndim + a];
  }
  return CSX_OK;
}

csx_status csx_pencil_schedule(const csx_plan_t p, int rank, int p0, int p1, int64_t* ops, int* nops) {
  if (!p || !ops || !nops || p0 < 1 || p1 < 1 || rank < 0 || rank >= p0 * p1)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad arguments");
  if (p->ndim < 2) return fail(CSX_ERR_UNSUPPORTED, "pencil decomposition needs ndim >= 2");
  int64_t lo[3], hi[3], El[3];
  pencil_box(p, rank, p0, p1, lo, hi);
  for (int a = 0; a < 3; ++a) El[a] = hi[a] - lo[a];
  *nops = pencil_schedule(p, rank, p0, p1, El, ops);
  return CSX_OK;
}

csx_status csx_run_sharded_pencil(csx_plan_t p, csx_comm_t c, int p0, int p1, const double* d_in,
                                  double* d_out, int64_t T, void* stream) {
  if (!p || !c || !d_in || !d_out) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  return run_sharded_pencil_impl(p, c, p0, p1, d_in, d_out, T, reinterpret_cast<cudaStream_t>(stream));
}

csx_status csx_run_sharded_peer(csx_plan_t p, const double* d_in, double* d_out, int64_t T,
                                void* stream) {
  if (!p || !d_in || !d_out) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  if (!p->peer || !p->peer->connected)
    return fail(CSX_ERR_INVALID_ARGUMENT, "csx_peer_export / csx_peer_connect not done for this plan");
  return run_sharded_impl(p, nullptr, p->peer, d_in, d_out, T, reinterpret_cast<cudaStream_t>(stream));
}

namespace {
struct PeerDesc {  // one rank's exported description (CSX_PEER_DESC_BYTES, POD)
  uint32_t magic, version;
  int32_t rank, nranks;
  int64_t El, elems;
  int64_t E[3];
  int32_t halo, ndim;
  int64_t offset;          // bytes from the IPC allocation base to the peer block
  int64_t stride;          // doubles from slab buffer 0 to slab buffer 1 (and 1 to the flags)
  cudaIpcMemHandle_t mem;  // the allocation holding slab buffers 0, 1 and the flag block
};
static_assert(sizeof(PeerDesc) <= CSX_PEER_DESC_BYTES, "descriptor size");
constexpr uint32_t kPeerMagic = 0x43535850u;  // "CSXP"
}  // namespace

csx_status csx_peer_export(csx_plan_t p, int rank, int nranks, void* desc) {
  if (!p || !desc || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad peer export arguments");
  int64_t lo, hi;
  csx_status s = csx_shard_rows(p, rank, nranks, &lo, &hi);
  if (s != CSX_OK) return s;
  const int a0 = 3 - p->ndim;
  int64_t El[3] = {p->E[0], p->E[1], p->E[2]};
  El[a0] = hi - lo;
  if (El[a0] < p->halo || El[a0] < 1)
    return fail(CSX_ERR_UNSUPPORTED, "a rank owns fewer rows than the halo depth r*Tf");
  s = ensure_device(p);
  if (s != CSX_OK) return s;
  if (p->peer) return fail(CSX_ERR_INVALID_ARGUMENT, "peer exchange already exported for this plan");
  // the slab buffers are fixed from here on (neighbours map them): ONE allocation holds slab
  // buffers 0 and 1 and the flag block, so a single IPC handle covers all three (small
  // cudaMallocs may share an allocation, and a second mapping of it would fail)
  cudaFree(p->d_sbuf[0]);
  cudaFree(p->d_sbuf[1]);
  p->d_sbuf[0] = p->d_sbuf[1] = nullptr;
  layout_padded(p, El, &p->spad);
  const int64_t stride = (p->spad.elems() + 31) / 32 * 32;
  const size_t bytes = (size_t)(2 * stride) * sizeof(double) + 256;
  csx_peer_s* q = new (std::nothrow) csx_peer_s();
  if (!q) return fail(CSX_ERR_OUT_OF_MEMORY, "peer state");
  p->peer = q;  // owned by the plan from here on (freed by csx_plan_destroy)
  q->rank = rank;
  q->nranks = nranks;
  q->El = El[a0];
  cudaError_t e = cudaMalloc(&q->block, bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(CSX_ERR_OUT_OF_MEMORY, "cudaMalloc of the peer slab block failed");
  }
  e = cudaMemset(q->block, 0, bytes);
  double* blk = static_cast<double*>(q->block);
  p->d_sbuf[0] = blk;
  p->d_sbuf[1] = blk + stride;
  q->flags = reinterpret_cast<unsigned long long*>(blk + 2 * stride);
  p->s_rank = rank;
  p->s_nranks = nranks;
  p->s_lo = lo;
  p->s_hi = hi;
  cudaStream_t cs = nullptr;
  cudaEvent_t e1 = nullptr, e2 = nullptr;
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&e1, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&e2, cudaEventDisableTiming);
  q->cs = cs;
  q->ev_edge = e1;
  q->ev_x = e2;
  if (e != cudaSuccess) return cuda_fail(e, "peer block / stream");
  // the IPC handle names the whole allocation containing the block: export its base + offset
  static PFN_cuMemGetAddressRange_v3020 range = [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult qr;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &qr) != cudaSuccess ||
        qr != cudaDriverEntryPointSuccess) {
      cudaGetLastError();
      return (PFN_cuMemGetAddressRange_v3020) nullptr;
    }
    return reinterpret_cast<PFN_cuMemGetAddressRange_v3020>(fn);
  }();
  CUdeviceptr base = reinterpret_cast<CUdeviceptr>(q->block);
  size_t rsize = 0;
  if (!range || range(&base, &rsize, reinterpret_cast<CUdeviceptr>(q->block)) != CUDA_SUCCESS)
    return fail(CSX_ERR_CUDA, "cuMemGetAddressRange failed");
  PeerDesc d;
  std::memset(&d, 0, sizeof(d));
  d.magic = kPeerMagic;
  d.version = 2;
  d.rank = rank;
  d.nranks = nranks;
  d.El = El[a0];
  d.elems = p->spad.elems();
  for (int k = 0; k < 3; ++k) d.E[k] = p->E[k];
  d.halo = p->halo;
  d.ndim = p->ndim;
  d.offset = (int64_t)(reinterpret_cast<CUdeviceptr>(q->block) - base);
  d.stride = stride;
  e = cudaIpcGetMemHandle(&d.mem, reinterpret_cast<void*>(base));
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
  std::memset(desc, 0, CSX_PEER_DESC_BYTES);
  std::memcpy(desc, &d, sizeof(d));
  return CSX_OK;
}

csx_status csx_peer_connect(csx_plan_t p, const void* descs) {
  if (!p || !descs) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  csx_peer_s* q = p->peer;
  if (!q) return fail(CSX_ERR_INVALID_ARGUMENT, "csx_peer_export first");
  if (q->connected) return CSX_OK;
  const unsigned char* all = static_cast<const unsigned char*>(descs);
  auto desc_of = [&](int r, PeerDesc* d) -> csx_status {
    std::memcpy(d, all + (size_t)r * CSX_PEER_DESC_BYTES, sizeof(*d));
    if (d->magic != kPeerMagic || d->version != 2 || d->rank != r || d->nranks != q->nranks ||
        d->halo != p->halo || d->ndim != p->ndim)
      return fail(CSX_ERR_INVALID_ARGUMENT, "peer descriptor mismatch (rank order / plan parameters)");
    for (int k = 0; k < 3; ++k)
      if (d->E[k] != p->E[k]) return fail(CSX_ERR_INVALID_ARGUMENT, "peer descriptor: plans differ");
    return CSX_OK;
  };
  for (int r = 0; r < q->nranks; ++r) {  // every descriptor must belong to this collective
    PeerDesc d;
    csx_status s0 = desc_of(r, &d);
    if (s0 != CSX_OK) return s0;
  }
  const bool periodic = p->bc == CSX_BC_PERIODIC;
  q->up = q->rank - 1;
  q->down = q->rank + 1;
  if (periodic) {
    q->up = (q->up + q->nranks) % q->nranks;
    q->down %= q->nranks;
  } else {
    if (q->up < 0) q->up = -1;
    if (q->down >= q->nranks) q->down = -1;
  }
  // map one neighbour (own pointers for a self-neighbour; one mapping if up == down)
  auto map = [&](int r, double** buf, unsigned long long** flags, int64_t* El) -> csx_status {
    if (r < 0) return CSX_OK;
    PeerDesc d;
    csx_status s2 = desc_of(r, &d);
    if (s2 != CSX_OK) return s2;
    *El = d.El;
    if (r == q->rank) {
      buf[0] = p->d_sbuf[0];
      buf[1] = p->d_sbuf[1];
      *flags = q->flags;
      return CSX_OK;
    }
    if (r == q->up && q->up_flags && r == q->down) {  // already mapped as up
      buf[0] = q->up_buf[0];
      buf[1] = q->up_buf[1];
      *flags = q->up_flags;
      return CSX_OK;
    }
    void* ptr = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&ptr, d.mem, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) return cuda_fail(e, "cudaIpcOpenMemHandle");
    q->opened.push_back(ptr);
    double* blk = reinterpret_cast<double*>(static_cast<char*>(ptr) + d.offset);
    buf[0] = blk;
    buf[1] = blk + d.stride;
    *flags = reinterpret_cast<unsigned long long*>(blk + 2 * d.stride);
    return CSX_OK;
  };
  csx_status s = map(q->up, q->up_buf, &q->up_flags, &q->El_up);
  if (s == CSX_OK) s = map(q->down, q->down_buf, &q->down_flags, &q->El_down);
  if (s != CSX_OK) return s;
  q->connected = true;
  return CSX_OK;
}

}  // extern "C"
