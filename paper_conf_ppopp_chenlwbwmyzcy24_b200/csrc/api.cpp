// api.cpp — the C-ABI of libcsx.so (include/csx.h): argument validation, device state, and
// the pass loop of csx_run.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include "csx_internal.h"
#include "csx_run.h"
#include "kernels.cuh"

namespace csx {

static thread_local std::string g_err;

void set_error(const std::string& msg) { g_err = msg; }

csx_status fail(csx_status s, const std::string& msg) {
  g_err = msg;
  return s;
}

csx_status cuda_fail(cudaError_t e, const char* where) {
  g_err = std::string(where) + ": " + cudaGetErrorString(e);
  return CSX_ERR_CUDA;
}

#define CSX_CUDA(call, where)                   \
  do {                                          \
    cudaError_t e_ = (call);                    \
    if (e_ != cudaSuccess) return cuda_fail(e_, where); \
  } while (0)

// drop a captured csx_run graph (engine / variant changes make it stale)
static void graph_reset(csx_plan_s* p) {
  if (p->g_exec) {
    cudaGraphExecDestroy((cudaGraphExec_t)p->g_exec);
    p->g_exec = nullptr;
  }
  p->g_T = -1;
}

// Tile shape of the direct kernel (engine DIRECT and the FIXED band fix-up).
void direct_tile(int ndim, int* B) {
  if (ndim == 1) { B[0] = 1; B[1] = 1; B[2] = 1024; }
  else if (ndim == 2) { B[0] = 1; B[1] = 32; B[2] = 64; }
  else { B[0] = 8; B[1] = 8; B[2] = 32; }
}

static csx_status upload_pass(Pass& ps) {
  if (ps.uploaded) return CSX_OK;
  if (ps.s2r_ok) {
    CSX_CUDA(cudaMalloc(&ps.d_frags, ps.frags.size() * sizeof(double)), "cudaMalloc(frags)");
    CSX_CUDA(cudaMemcpy(ps.d_frags, ps.frags.data(), ps.frags.size() * sizeof(double),
                        cudaMemcpyHostToDevice), "upload frags");
    const size_t ne = ps.lut_g.size();
    std::vector<int32_t> il(2 * ne);
    for (size_t e = 0; e < ne; ++e) {
      il[2 * e] = ps.lut_g[e];
      il[2 * e + 1] = (int32_t)((uint32_t)ps.lut_a[e] | ((uint32_t)ps.lut_b[e] << 16));
    }
    CSX_CUDA(cudaMalloc(&ps.d_lut, il.size() * sizeof(int32_t)), "cudaMalloc(lut)");
    CSX_CUDA(cudaMemcpy(ps.d_lut, il.data(), il.size() * sizeof(int32_t), cudaMemcpyHostToDevice),
             "upload lut");
  }
  if (ps.tile_ok) {
    CSX_CUDA(cudaMalloc(&ps.d_tile_frags, ps.tile_frags.size() * sizeof(double)), "cudaMalloc");
    CSX_CUDA(cudaMemcpy(ps.d_tile_frags, ps.tile_frags.data(),
                        ps.tile_frags.size() * sizeof(double), cudaMemcpyHostToDevice), "upload");
  }
  CSX_CUDA(cudaMalloc(&ps.d_wc, ps.wc.size() * sizeof(double)), "cudaMalloc(wc)");
  CSX_CUDA(cudaMemcpy(ps.d_wc, ps.wc.data(), ps.wc.size() * sizeof(double), cudaMemcpyHostToDevice),
           "upload wc");
  ps.uploaded = true;
  return CSX_OK;
}

csx_status ensure_device(csx_plan_s* p) {
  int dev = 0;
  CSX_CUDA(cudaGetDevice(&dev), "cudaGetDevice");
  if (p->device >= 0) {
    if (dev != p->device) return fail(CSX_ERR_INVALID_ARGUMENT, "plan used on another device");
    for (auto& ps : p->passes) {
      csx_status s = upload_pass(ps);
      if (s != CSX_OK) return s;
    }
    return CSX_OK;
  }
  for (auto& ps : p->passes) {
    csx_status s = upload_pass(ps);
    if (s != CSX_OK) return s;
  }
  {
    cudaStream_t side;
    cudaEvent_t a, b;
    CSX_CUDA(cudaStreamCreateWithFlags(&side, cudaStreamNonBlocking), "side stream");
    CSX_CUDA(cudaEventCreateWithFlags(&a, cudaEventDisableTiming), "event");
    CSX_CUDA(cudaEventCreateWithFlags(&b, cudaEventDisableTiming), "event");
    p->side = side;
    p->ev_fork = a;
    p->ev_join = b;
  }
  CSX_CUDA(cudaMalloc(&p->d_wbase, p->w.size() * sizeof(double)), "cudaMalloc(w)");
  CSX_CUDA(cudaMemcpy(p->d_wbase, p->w.data(), p->w.size() * sizeof(double),
                      cudaMemcpyHostToDevice), "upload w");
  p->device = dev;
  return CSX_OK;
}

csx_status ensure_grid(csx_plan_s* p, Padded* pd, double** bufs, const int64_t* E) {
  if (bufs[0]) return CSX_OK;
  layout_padded(p, E, pd);
  const size_t bytes = (size_t)pd->elems() * sizeof(double);
  for (int i = 0; i < 2; ++i) {
    cudaError_t e = cudaMalloc(&bufs[i], bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(CSX_ERR_OUT_OF_MEMORY, "cudaMalloc of a padded grid failed");
    }
    CSX_CUDA(cudaMemset(bufs[i], 0, bytes), "cudaMemset");
  }
  return CSX_OK;
}

// One fused pass of Tf' steps from the padded source to dst (padded scratch or user output).
// ctx describes the local grid and its place in the global grid (sharded runs).
csx_status run_pass(csx_plan_s* p, Pass& ps, const PassCtx& c, cudaStream_t st) {
  csx_engine eng = p->engine;
  cudaError_t e = cudaSuccess;
  // TC_TILE 2D, FIXED, Tf > 1: the edge CTAs skip the band, so k_band (which writes only band
  // points) runs on the side stream concurrently with the TC kernel; the caller's stream waits
  // for it after the TC launch.
  const bool band_side = eng == CSX_ENGINE_TC_TILE && p->bc == CSX_BC_FIXED && p->ndim == 2 &&
                         ps.tf > 1 && c.part != 1;
  if (band_side) {
    cudaStream_t side = (cudaStream_t)p->side;
    CSX_CUDA(cudaEventRecord((cudaEvent_t)p->ev_fork, st), "fork");
    CSX_CUDA(cudaStreamWaitEvent(side, (cudaEvent_t)p->ev_fork, 0), "fork wait");
    int launched = 0;
    e = launch_band(p->ndim, p->radius, ps.tf, c.src, c.dst, c.E, c.gorg, p->E, p->w.data(), side,
                    &launched);
    if (e != cudaSuccess) return cuda_fail(e, "band fix-up launch");
    p->n_launches += launched;
    CSX_CUDA(cudaEventRecord((cudaEvent_t)p->ev_join, side), "join");
  }
  if (eng == CSX_ENGINE_TC_S2R || eng == CSX_ENGINE_TC_TILE) {
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    // time the main-pass (dominant) kernel only, every prof-th launch (events between kernels
    // break programmatic dependent launch, so bench.py samples rather than brackets them all)
    const bool prof = p->prof > 0 && ps.tf == p->tf && (p->n_tc_launches % p->prof) == 0;
    if (prof) {
      if (p->prof_used + 2 > p->prof_events.size()) {
        for (int k = 0; k < 64; ++k) {
          cudaEvent_t ev;
          CSX_CUDA(cudaEventCreate(&ev), "cudaEventCreate");
          p->prof_events.push_back(ev);
        }
      }
      ev0 = (cudaEvent_t)p->prof_events[p->prof_used++];
      ev1 = (cudaEvent_t)p->prof_events[p->prof_used++];
      CSX_CUDA(cudaEventRecord(ev0, st), "cudaEventRecord");
    }
    S2RArgs a;
    a.part = eng == CSX_ENGINE_TC_TILE ? c.part : 0;
    a.max_ctas = c.max_ctas;
    a.src = c.src;
    a.dst = c.dst;
    a.E0 = c.E[0]; a.E1 = c.E[1]; a.E2 = c.E[2];
    a.lut = reinterpret_cast<const int2*>(ps.d_lut);
    a.wc = ps.d_wc;
    if (eng == CSX_ENGINE_TC_TILE) {
      // 3D Tf = 2 runs the BASE stencil twice in shared memory (k_tile3d_tb): base fragments,
      // base weights and the base plane split
      const Pass& pw = (p->ndim == 3 && ps.tf == 2) ? p->passes[0] : ps;
      a.frags = pw.d_tile_frags;
      a.wc = pw.d_wc;
      a.pdl = !band_side && c.part == 0;  // no PDL across the band join / halo-exchange waits
      if (p->ndim == 3)
        for (int dz = 0; dz < pw.nk; ++dz) a.tc_mask |= pw.plane_is_tc[dz] << dz;
      if (p->bc == CSX_BC_FIXED && p->ndim == 1) {  // 1D band recomputed in-kernel
        a.fix_band = p->radius * ps.tf;
        a.r = p->radius;
        a.wbase = p->d_wbase;
        a.gorg2 = c.gorg[2];
        a.GE2 = p->E[2];
      }
      if (p->bc == CSX_BC_FIXED && p->ndim >= 2) {
        // 2D: the edge CTAs leave the band to k_band (Tf > 1) or write the held frame (Tf = 1);
        // 3D (Tf = 1): the frame is written from the staged plane
        a.fix_band = p->radius * ps.tf;
        a.hold_frame = ps.tf == 1 || p->ndim == 3;  // 3D Tf = 2 holds the frame at both levels
        a.r = p->radius;
        a.wbase = p->d_wbase;
        a.gorg0 = c.gorg[0];
        a.gorg1 = c.gorg[1];
        a.gorg2 = c.gorg[2];
        a.GE0 = p->E[0];
        a.GE1 = p->E[1];
        a.GE2 = p->E[2];
      }
      e = launch_tile(p->ndim, p->radius, ps.tf, a, st);
    } else {
      a.frags = ps.d_frags;
      a.s2r_variant = (p->s2r_pad ? 1 : 0) | (p->s2r_dirty ? 2 : 0) | (p->s2r_fma ? 4 : 0);
      int tc_mask = 0;
      if (p->ndim == 1) {
        a.tiles_x = (int)((c.E[2] + ps.bn - 1) / ps.bn);
        a.tiles_y = 1;
        a.ntiles = a.tiles_x;
      } else {
        a.tiles_x = (int)((c.E[2] + ps.bn - 1) / ps.bn);
        a.tiles_y = (int)((c.E[1] + ps.bm - 1) / ps.bm);
        a.ntiles = (int64_t)a.tiles_x * a.tiles_y;
        if (p->ndim == 3) {
          const int64_t zchunk = 64;
          a.ntiles *= (c.E[0] + zchunk - 1) / zchunk;
          for (int dz = 0; dz < ps.nk; ++dz) tc_mask |= ps.plane_is_tc[dz] << dz;
        }
      }
      if (p->s2r_explicit && p->ndim == 2) {
        const int64_t need = s2r_explicit_elems(ps.nk, c.E[1], c.E[2]);
        if (need > p->s2r_elems) {
          cudaFree(p->d_s2r);
          p->d_s2r = nullptr;
          p->s2r_elems = 0;
          CSX_CUDA(cudaMalloc(&p->d_s2r, (size_t)need * sizeof(double)), "cudaMalloc(stencil2row)");
          p->s2r_elems = need;
        }
        e = launch_s2r_explicit(ps.nk, c.src, c.dst, c.E, ps.d_wc, p->d_s2r, st);
        p->n_launches += 1;  // two kernels: transform + tessellation
      } else {
        e = launch_s2r(p->ndim, ps.nk, ps.nf, a, tc_mask, st);
      }
    }
    if (e != cudaSuccess) return cuda_fail(e, "TC pass launch");
    if (prof) CSX_CUDA(cudaEventRecord(ev1, st), "cudaEventRecord");
    if (ps.tf == p->tf) p->n_tc_launches += 1;
    p->n_launches += 1;
  }
  if (band_side) CSX_CUDA(cudaStreamWaitEvent(st, (cudaEvent_t)p->ev_join, 0), "join wait");
  const bool direct_all = eng == CSX_ENGINE_DIRECT;
  const int real[3] = {p->ndim == 3, p->ndim >= 2, 1};
  if (eng == CSX_ENGINE_TC_TILE && c.part == 1) return CSX_OK;  // fix-ups run with the edge part
  if (direct_all) {
    DirectArgs d;
    d.src = c.src;
    d.dst = c.dst;
    for (int a2 = 0; a2 < 3; ++a2) {
      d.E[a2] = c.E[a2];
      d.real[a2] = real[a2];
      d.gorg[a2] = c.gorg[a2];
      d.GE[a2] = p->E[a2];
    }
    d.r = p->radius;
    d.tf = ps.tf;
    d.fixed_bc = p->bc == CSX_BC_FIXED;
    d.w = p->d_wbase;
    d.ndim = p->ndim;
    d.tile_list = nullptr;
    d.tile_org = nullptr;
    d.band = 0;
    d.max_ctas = c.max_ctas;
    direct_tile(p->ndim, d.B);
    for (int a2 = 0; a2 < 3; ++a2) d.tiles[a2] = (int)((c.E[a2] + d.B[a2] - 1) / d.B[a2]);
    d.ntiles = (int64_t)d.tiles[0] * d.tiles[1] * d.tiles[2];
    if (p->ndim == 2 && direct2d_exists(p->radius, ps.tf))
      e = launch_direct2d(d, p->w.data(), st);
    else if (p->ndim == 1 && direct1d_exists(p->radius, ps.tf) && !getenv("CSX_DIRECT_GENERIC"))
      e = launch_direct1d(d, p->w.data(), st);
    else if (p->ndim == 3 && direct3d_exists(p->radius, ps.tf) && !getenv("CSX_DIRECT_GENERIC"))
      e = launch_direct3d(d, p->w.data(), st);
    else
      e = launch_direct(d, st);
    if (e != cudaSuccess) return cuda_fail(e, "direct launch");
    p->n_launches += 1;
  } else if (p->bc == CSX_BC_FIXED && !(eng == CSX_ENGINE_TC_TILE && p->ndim == 1) &&
             !(eng == CSX_ENGINE_TC_TILE && p->ndim >= 2 && ps.tf == 1) &&
             !(eng == CSX_ENGINE_TC_TILE && p->ndim == 3)) {  // else done in-kernel
    if (ps.tf == 1 || p->ndim == 3) {
      // the composed window is the plain stencil: only the held frame needs restoring
      e = launch_frame_copy(c.src, c.dst, c.E, c.gorg, p->E, real, p->radius, st);
      if (e != cudaSuccess) return cuda_fail(e, "frame copy launch");
      p->n_launches += 1;
    } else if (!band_side) {
      int launched = 0;
      e = launch_band(p->ndim, p->radius, ps.tf, c.src, c.dst, c.E, c.gorg, p->E, p->w.data(), st,
                      &launched);
      if (e != cudaSuccess) return cuda_fail(e, "band fix-up launch");
      p->n_launches += launched;
    }
  }
  return CSX_OK;
}

}  // namespace csx

using namespace csx;

extern "C" {

const char* csx_status_string(csx_status s) {
  switch (s) {
    case CSX_OK: return "CSX_OK";
    case CSX_ERR_INVALID_ARGUMENT: return "CSX_ERR_INVALID_ARGUMENT";
    case CSX_ERR_UNSUPPORTED: return "CSX_ERR_UNSUPPORTED";
    case CSX_ERR_OUT_OF_MEMORY: return "CSX_ERR_OUT_OF_MEMORY";
    case CSX_ERR_CUDA: return "CSX_ERR_CUDA";
    case CSX_ERR_NCCL: return "CSX_ERR_NCCL";
    case CSX_ERR_INTERNAL: return "CSX_ERR_INTERNAL";
  }
  return "CSX_ERR_UNKNOWN";
}

const char* csx_last_error(void) { return g_err.c_str(); }

static bool engine_ok(const csx_plan_s* p, csx_engine e) {
  for (const auto& ps : p->passes) {
    if (e == CSX_ENGINE_TC_S2R && !ps.s2r_ok) return false;
    if (e == CSX_ENGINE_TC_TILE && !(ps.tile_ok && tile_kernel_exists(p->ndim, p->radius, ps.tf))) return false;
  }
  return true;
}

csx_status csx_plan(int ndim, const int64_t* extents, csx_shape shape, int radius,
                    const double* weights, csx_boundary bc, int fuse_steps, csx_plan_t* out) {
  if (!out) return fail(CSX_ERR_INVALID_ARGUMENT, "out is NULL");
  *out = nullptr;
  if (!extents || !weights) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL extents or weights");
  if (ndim < 1 || ndim > 3) return fail(CSX_ERR_INVALID_ARGUMENT, "ndim must be 1, 2 or 3");
  if (radius < 1 || radius > 3) return fail(CSX_ERR_INVALID_ARGUMENT, "radius must be 1..3");
  if (shape != CSX_SHAPE_STAR && shape != CSX_SHAPE_BOX)
    return fail(CSX_ERR_INVALID_ARGUMENT, "unknown shape");
  if (bc != CSX_BC_FIXED && bc != CSX_BC_PERIODIC)
    return fail(CSX_ERR_INVALID_ARGUMENT, "unknown boundary");
  if (fuse_steps < 0 || fuse_steps > 16) return fail(CSX_ERR_INVALID_ARGUMENT, "fuse_steps out of range");
  csx_plan_s* p = new (std::nothrow) csx_plan_s();
  if (!p) return fail(CSX_ERR_OUT_OF_MEMORY, "plan allocation");
  p->ndim = ndim;
  p->radius = radius;
  p->shape = shape;
  p->bc = bc;
  for (int a = 0; a < ndim; ++a) {
    if (extents[a] < 1) { delete p; return fail(CSX_ERR_INVALID_ARGUMENT, "extent < 1"); }
    p->ext[a] = extents[a];
    p->E[3 - ndim + a] = extents[a];
  }
  const int n = 2 * radius + 1;
  int64_t dense = 1;
  for (int a = 0; a < ndim; ++a) dense *= n;
  p->w.assign(weights, weights + dense);
  for (int64_t i = 0; i < dense; ++i) {
    if (!std::isfinite(p->w[i])) { delete p; return fail(CSX_ERR_INVALID_ARGUMENT, "non-finite weight"); }
    if (p->w[i] != 0.0) ++p->nnz;
    if (shape == CSX_SHAPE_STAR && p->w[i] != 0.0) {
      int64_t rem = i;
      int offaxis = 0;
      for (int a = 0; a < ndim; ++a) { offaxis += (rem % n) != radius; rem /= n; }
      if (offaxis > 1) { delete p; return fail(CSX_ERR_INVALID_ARGUMENT, "STAR weight off the axes"); }
    }
  }
  p->tf = fuse_steps;
  csx_status s = build_plan(p);
  if (s != CSX_OK) { delete p; return s; }
  p->engine_req = CSX_ENGINE_AUTO;
  if (engine_ok(p, CSX_ENGINE_TC_TILE)) p->engine = CSX_ENGINE_TC_TILE;
  else if (engine_ok(p, CSX_ENGINE_TC_S2R)) p->engine = CSX_ENGINE_TC_S2R;
  else p->engine = CSX_ENGINE_DIRECT;
  *out = p;
  return CSX_OK;
}

int csx_auto_fuse_steps(int ndim, int radius, csx_engine engine) {
  if (ndim < 1 || ndim > 3 || radius < 1 || radius > 3) return 0;
  if (engine < CSX_ENGINE_AUTO || engine > CSX_ENGINE_DIRECT) return 0;
  return csx::auto_tf(ndim, radius, engine);
}

csx_status csx_plan_set_s2r_variant(csx_plan_t p, int padding, int dirty_bits) {
  if (p) graph_reset(p);
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  // padding = 2: breakdown variant II (padding + dirty bits, tessellation on CUDA cores);
  // padding = 3: breakdown variant I (explicit stencil2row in HBM, CUDA-core tessellation)
  if (padding < 0 || padding > 3) return fail(CSX_ERR_INVALID_ARGUMENT, "padding must be 0..3");
  if (padding == 3 && p->ndim != 2) return fail(CSX_ERR_UNSUPPORTED, "breakdown variants are 2D only");
  p->s2r_fma = padding == 2;
  p->s2r_explicit = padding == 3;
  if (p->s2r_fma || p->s2r_explicit) { padding = 1; dirty_bits = 1; }
  if (p->ndim != 2 && !(padding && dirty_bits))
    return fail(CSX_ERR_UNSUPPORTED, "breakdown variants are 2D only");
  p->s2r_pad = padding != 0;
  p->s2r_dirty = dirty_bits != 0;
  // rebuild the tables of every pass; device copies are re-uploaded at the next run
  std::vector<Pass> fresh(p->passes.size());
  for (size_t i = 0; i < p->passes.size(); ++i) {
    csx_status s = build_pass(p, (int)i + 1, &fresh[i]);
    if (s != CSX_OK) return s;
  }
  if (p->device >= 0) {
    for (auto& ps : p->passes) {
      cudaFree(ps.d_frags);
      cudaFree(ps.d_lut);
      cudaFree(ps.d_tile_frags);
      cudaFree(ps.d_wc);
    }
  }
  p->passes.swap(fresh);
  return CSX_OK;
}

csx_status csx_plan_set_engine(csx_plan_t p, csx_engine e) {
  if (p) graph_reset(p);
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  if (e == CSX_ENGINE_AUTO) {
    p->engine_req = e;
    if (engine_ok(p, CSX_ENGINE_TC_TILE)) p->engine = CSX_ENGINE_TC_TILE;
    else if (engine_ok(p, CSX_ENGINE_TC_S2R)) p->engine = CSX_ENGINE_TC_S2R;
    else p->engine = CSX_ENGINE_DIRECT;
    return CSX_OK;
  }
  if (e != CSX_ENGINE_TC_S2R && e != CSX_ENGINE_TC_TILE && e != CSX_ENGINE_DIRECT)
    return fail(CSX_ERR_INVALID_ARGUMENT, "unknown engine");
  if (!engine_ok(p, e)) return fail(CSX_ERR_UNSUPPORTED, "engine cannot run this plan");
  p->engine_req = e;
  p->engine = e;
  return CSX_OK;
}

csx_status csx_run(csx_plan_t p, const double* d_in, double* d_out, int64_t T, void* stream) {
  if (!p || !d_in || !d_out) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  if (T < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "timesteps < 0");
  if ((reinterpret_cast<uintptr_t>(d_in) | reinterpret_cast<uintptr_t>(d_out)) & 7)
    return fail(CSX_ERR_INVALID_ARGUMENT, "grids must be 8-byte aligned");
  const int64_t n = p->E[0] * p->E[1] * p->E[2];
  if (d_in != d_out && d_in < d_out + n && d_out < d_in + n)
    return fail(CSX_ERR_INVALID_ARGUMENT, "d_in and d_out overlap");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  csx_status s = ensure_device(p);
  if (s != CSX_OK) return s;
  if (T == 0) {
    if (d_in != d_out)
      CSX_CUDA(cudaMemcpyAsync(d_out, d_in, n * sizeof(double), cudaMemcpyDeviceToDevice, st), "copy");
    return CSX_OK;
  }
  s = ensure_grid(p, &p->pad, p->d_buf, p->E);
  if (s != CSX_OK) return s;
  if (!p->graph_on || p->prof > 0) return run_local(p, d_in, d_out, T, st);
  // Graph mode: replay the captured pass sequence if (d_in, d_out, T) match; otherwise run
  // eagerly (first use: lazy allocations, tensor maps) and capture the same sequence on the
  // plan's non-blocking stream for the next call.  The replay is one cudaGraphLaunch on the
  // caller's stream (the legacy default stream included); PDL edges are kept in the graph.
  if (p->g_exec && p->g_in == d_in && p->g_out == d_out && p->g_T == T) {
    CSX_CUDA(cudaGraphLaunch((cudaGraphExec_t)p->g_exec, st), "cudaGraphLaunch");
    p->n_launches += p->g_launches;
    p->n_tc_launches += p->g_tc_launches;
    return CSX_OK;
  }
  s = run_local(p, d_in, d_out, T, st);
  if (s != CSX_OK) return s;
  if (p->g_exec) {
    cudaGraphExecDestroy((cudaGraphExec_t)p->g_exec);
    p->g_exec = nullptr;
  }
  if (!p->g_stream) {
    cudaStream_t cs;
    CSX_CUDA(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking), "capture stream");
    p->g_stream = cs;
  }
  cudaStream_t cs = (cudaStream_t)p->g_stream;
  const int64_t l0 = p->n_launches, t0 = p->n_tc_launches;
  CSX_CUDA(cudaStreamBeginCapture(cs, cudaStreamCaptureModeRelaxed), "begin capture");
  s = run_local(p, d_in, d_out, T, cs);
  cudaGraph_t g = nullptr;
  const cudaError_t ec = cudaStreamEndCapture(cs, &g);
  if (s != CSX_OK) {
    if (g) cudaGraphDestroy(g);
    return s;
  }
  if (ec != cudaSuccess) return cuda_fail(ec, "end capture");
  cudaGraphExec_t ge = nullptr;
  const cudaError_t ei = cudaGraphInstantiate(&ge, g, 0);
  cudaGraphDestroy(g);
  if (ei != cudaSuccess) return cuda_fail(ei, "cudaGraphInstantiate");
  p->g_exec = ge;
  p->g_in = d_in;
  p->g_out = d_out;
  p->g_T = T;
  p->g_launches = p->n_launches - l0;  // capture counted the launches without running them
  p->g_tc_launches = p->n_tc_launches - t0;
  p->n_launches = l0;
  p->n_tc_launches = t0;
  return CSX_OK;
}

csx_status csx_plan_set_max_ctas(csx_plan_t p, int max_ctas) {
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  if (max_ctas < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "max_ctas must be >= 0");
  p->max_ctas = max_ctas;
  graph_reset(p);
  return CSX_OK;
}

csx_status csx_plan_set_graph(csx_plan_t p, int on) {
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  p->graph_on = on != 0;
  graph_reset(p);
  return CSX_OK;
}

// csx_run_host, pipelined: the grid is cut along its slowest axis into K chunks; chunk k's
// input is its rows plus a ghost zone of H = (T + 1) r rows on each side (wrapped for PERIODIC,
// clipped at the global faces for FIXED), advanced T steps by a sub-plan of the same stencil,
// boundary and fusion depth, and only its own rows are copied back.  Information travels r rows
// per base step, and the sub-plan's artificial faces (held or wrapped) disturb at most the
// T r + r rows next to them, so the kept rows equal the whole-grid run up to rounding order.  The
// H2D copy of chunk k + 1, the run of chunk k and the D2H copy of chunk k - 1 overlap on three
// streams (PCIe is full duplex), which hides most of the two copies behind the compute: 1 + 2H/C
// of the work for two copies that took ~2/3 of the serial call.  Used when the host buffers are
// pinned and do not overlap, and K >= 2 chunks of >= 4H rows and >= 8M points exist (K <= 4;
// CSX_HOST_CHUNKS: 0 off, n forces n).
static int host_chunks(const csx_plan_s* p, const double* h_in, double* h_out, int64_t T) {
  const char* e = getenv("CSX_HOST_CHUNKS");
  const int forced = e ? atoi(e) : -1;
  if (forced == 0 || T <= 0) return 0;
  {  // overlapping host buffers (in place or not): the serial path reads all input first
    const int64_t n = p->E[0] * p->E[1] * p->E[2];
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(h_in), a1 = a0 + (uintptr_t)n * sizeof(double);
    const uintptr_t b0 = reinterpret_cast<uintptr_t>(h_out), b1 = b0 + (uintptr_t)n * sizeof(double);
    if (a0 < b1 && b0 < a1) return 0;
  }
  cudaPointerAttributes ai, ao;
  if (cudaPointerGetAttributes(&ai, h_in) != cudaSuccess || cudaPointerGetAttributes(&ao, h_out) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  if (ai.type != cudaMemoryTypeHost || ao.type != cudaMemoryTypeHost) return 0;  // pageable: serial
  const int64_t N = p->ext[0];
  const int64_t H = (T + 1) * p->radius;
  if (forced > 0) return (int)std::min<int64_t>(forced, std::max<int64_t>(1, N / (H + 1)));
  // up to 4 chunks of >= 4H rows (ghost rows <= 50 % of a chunk) and >= 8M points each (so each
  // chunk's passes stay long kernels, not launch-bound): measured on C2, 4 chunks 367 GSt/s,
  // 8: 332, 12: 310, 16: 285 (serial 220); 8 chunks of the 10.24M-point 1D grid ran slower
  // than the serial call (their 77 passes of 1.3M points each are launch-bound)
  // Where the ghost rows are cheap (<= 10 % of the grid over all chunks) up to 8 chunks: the
  // 102.4M-point 1D grid ran 3597 GSt/s with 8 chunks, 3236 with 4.
  const int64_t plane = p->E[0] * p->E[1] * p->E[2] / N;
  int64_t k = std::min<int64_t>(8, (N / 10) / (2 * H));
  if (k < 2) k = std::min<int64_t>(4, N / (4 * H));
  while (k >= 2 && (N / k) * plane < (int64_t(8) << 20)) --k;
  return k >= 2 ? (int)k : 0;
}

static csx_status host_subplan(csx_plan_s* p, int64_t rows, csx_plan_s** out) {
  for (auto& q : p->hsub)
    if (q.first == rows) { *out = q.second; return CSX_OK; }
  int64_t ext[3] = {p->ext[0], p->ext[1], p->ext[2]};
  ext[0] = rows;
  csx_plan_s* q = nullptr;
  csx_status s = csx_plan(p->ndim, ext, p->shape, p->radius, p->w.data(), p->bc, p->tf, &q);
  if (s != CSX_OK) return s;
  s = csx_plan_set_engine(q, p->engine);
  if (s == CSX_OK) s = csx_plan_set_max_ctas(q, p->max_ctas);
  if (s != CSX_OK) { csx_plan_destroy(q); return s; }
  p->hsub.emplace_back(rows, q);
  *out = q;
  return CSX_OK;
}

static csx_status run_host_chunked(csx_plan_s* p, const double* h_in, double* h_out, int64_t T,
                                   cudaStream_t st, int K) {
  const int64_t N = p->ext[0];
  const int64_t plane = p->E[0] * p->E[1] * p->E[2] / N;  // doubles per slowest-axis row
  const int64_t H = (T + 1) * p->radius;
  const int64_t C = (N + K - 1) / K;
  const bool per = p->bc == CSX_BC_PERIODIC;
  const int64_t slot_rows = std::min<int64_t>(C + 2 * H, per ? C + 2 * H : N);
  if (slot_rows * plane > p->h_slot_elems) {
    for (auto& b : p->h_slot) { cudaFree(b); b = nullptr; }
    p->h_slot_elems = 0;
    for (auto& b : p->h_slot) {
      cudaError_t e = cudaMalloc(&b, (size_t)(slot_rows * plane) * sizeof(double));
      if (e != cudaSuccess) { cudaGetLastError(); return fail(CSX_ERR_OUT_OF_MEMORY, "cudaMalloc(host pipeline slot)"); }
    }
    p->h_slot_elems = slot_rows * plane;
  }
  if (!p->h_s_in) {
    cudaStream_t a = nullptr, b = nullptr;
    CSX_CUDA(cudaStreamCreateWithFlags(&a, cudaStreamNonBlocking), "stream");
    p->h_s_in = a;
    CSX_CUDA(cudaStreamCreateWithFlags(&b, cudaStreamNonBlocking), "stream");
    p->h_s_out = b;
    for (auto& ev : p->h_ev) {
      cudaEvent_t x = nullptr;
      CSX_CUDA(cudaEventCreateWithFlags(&x, cudaEventDisableTiming), "event");
      ev = x;
    }
  }
  cudaStream_t sin = (cudaStream_t)p->h_s_in, sout = (cudaStream_t)p->h_s_out;
  cudaEvent_t* ev = reinterpret_cast<cudaEvent_t*>(p->h_ev);
  // the caller's prior work on st (e.g. writes to h_in by an earlier D2H) precedes our copies
  CSX_CUDA(cudaEventRecord(ev[2], st), "event");
  CSX_CUDA(cudaStreamWaitEvent(sin, ev[2], 0), "wait");
  const size_t rowb = (size_t)plane * sizeof(double);
  // every chunk's sub-plan first: a chunk shorter than its composed window (tiny grids, few
  // steps, deep fusion) is refused by csx_plan, and then the whole call takes the serial path
  for (int k = 0; k < K; ++k) {
    const int64_t lo = k * C, hi = std::min(N, lo + C);
    if (lo >= hi) break;
    const int64_t r0 = per ? lo - H : std::max<int64_t>(0, lo - H);
    const int64_t r1 = per ? hi + H : std::min(N, hi + H);
    csx_plan_s* q = nullptr;
    if (host_subplan(p, r1 - r0, &q) != CSX_OK) return CSX_ERR_UNSUPPORTED;
  }
  p->h_last_chunks = 0;
  p->h_last_h2d = p->h_last_d2h = 0;
  for (int k = 0; k < K; ++k) {
    const int64_t lo = k * C, hi = std::min(N, lo + C);
    if (lo >= hi) break;
    const int s = k & 1;
    const int64_t r0 = per ? lo - H : std::max<int64_t>(0, lo - H);
    const int64_t r1 = per ? hi + H : std::min(N, hi + H);
    const int64_t rows = r1 - r0;
    csx_plan_s* q = nullptr;
    csx_status cs = host_subplan(p, rows, &q);
    if (cs != CSX_OK) return cs;
    double* din = p->h_slot[s];
    double* dout = p->h_slot[2 + s];
    // H2D of rows [r0, r1) (wrapped into [0, N) for PERIODIC: at most three runs)
    if (k >= 2) CSX_CUDA(cudaStreamWaitEvent(sin, ev[2 + s], 0), "wait");  // chunk k-2's run done
    for (int64_t r = r0; r < r1;) {
      const int64_t g = ((r % N) + N) % N;
      const int64_t len = std::min(r1 - r, N - g);
      CSX_CUDA(cudaMemcpyAsync(din + (r - r0) * plane, h_in + g * plane, (size_t)len * rowb,
                               cudaMemcpyHostToDevice, sin), "H2D");
      r += len;
    }
    CSX_CUDA(cudaEventRecord(ev[s], sin), "event");
    CSX_CUDA(cudaStreamWaitEvent(st, ev[s], 0), "wait");
    if (k >= 2) CSX_CUDA(cudaStreamWaitEvent(st, ev[4 + s], 0), "wait");  // chunk k-2's D2H done
    cs = csx_run(q, din, dout, T, st);
    if (cs != CSX_OK) return cs;
    CSX_CUDA(cudaEventRecord(ev[2 + s], st), "event");
    CSX_CUDA(cudaStreamWaitEvent(sout, ev[2 + s], 0), "wait");
    CSX_CUDA(cudaMemcpyAsync(h_out + lo * plane, dout + (lo - r0) * plane, (size_t)(hi - lo) * rowb,
                             cudaMemcpyDeviceToHost, sout), "D2H");
    CSX_CUDA(cudaEventRecord(ev[4 + s], sout), "event");
    p->h_last_chunks += 1;
    p->h_last_h2d += rows * (int64_t)rowb;
    p->h_last_d2h += (hi - lo) * (int64_t)rowb;
  }
  CSX_CUDA(cudaStreamSynchronize(sout), "sync");
  CSX_CUDA(cudaStreamSynchronize(st), "sync");
  return CSX_OK;
}

csx_status csx_run_host(csx_plan_t p, const double* h_in, double* h_out, int64_t T, void* stream) {
  if (!p || !h_in || !h_out) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  if (T < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "timesteps < 0");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int64_t n = p->E[0] * p->E[1] * p->E[2];
  csx_status s = ensure_device(p);
  if (s != CSX_OK) return s;
  const int K = host_chunks(p, h_in, h_out, T);
  if (K >= 2) {
    s = run_host_chunked(p, h_in, h_out, T, st, K);
    if (s != CSX_ERR_UNSUPPORTED) return s;
    set_error("");  // a chunk too short for its sub-plan: serial path below
  }
  p->h_last_chunks = 1;
  p->h_last_h2d = p->h_last_d2h = n * (int64_t)sizeof(double);
  if (!p->d_dense) {
    cudaError_t e = cudaMalloc(&p->d_dense, n * sizeof(double));
    if (e != cudaSuccess) { cudaGetLastError(); return fail(CSX_ERR_OUT_OF_MEMORY, "cudaMalloc(dense)"); }
  }
  CSX_CUDA(cudaMemcpyAsync(p->d_dense, h_in, n * sizeof(double), cudaMemcpyHostToDevice, st), "H2D");
  s = csx_run(p, p->d_dense, p->d_dense, T, stream);
  if (s != CSX_OK) return s;
  CSX_CUDA(cudaMemcpyAsync(h_out, p->d_dense, n * sizeof(double), cudaMemcpyDeviceToHost, st), "D2H");
  CSX_CUDA(cudaStreamSynchronize(st), "sync");
  return CSX_OK;
}

csx_status csx_host_last(const csx_plan_t p, int* chunks, int64_t* h2d_bytes, int64_t* d2h_bytes) {
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  if (chunks) *chunks = p->h_last_chunks;
  if (h2d_bytes) *h2d_bytes = p->h_last_h2d;
  if (d2h_bytes) *d2h_bytes = p->h_last_d2h;
  return CSX_OK;
}

csx_status csx_profile_enable(csx_plan_t p, int enable) {
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  if (enable < 0) return fail(CSX_ERR_INVALID_ARGUMENT, "profile period must be >= 0");
  p->prof = enable;
  return CSX_OK;
}

csx_status csx_profile_read(csx_plan_t p, double* tc_ms, int64_t* tc_launches, int64_t* total,
                            int reset) {
  if (!p) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL plan");
  double ms = 0.0;
  int64_t timed = 0;
  for (size_t i = 0; i + 1 < p->prof_used; i += 2, ++timed) {
    cudaEvent_t a = (cudaEvent_t)p->prof_events[i], b = (cudaEvent_t)p->prof_events[i + 1];
    CSX_CUDA(cudaEventSynchronize(b), "cudaEventSynchronize");
    float f = 0.f;
    CSX_CUDA(cudaEventElapsedTime(&f, a, b), "cudaEventElapsedTime");
    ms += f;
  }
  // sampled launches: scale the mean timed duration to every main-pass launch
  if (tc_ms) *tc_ms = timed > 0 ? ms / (double)timed * (double)p->n_tc_launches : 0.0;
  if (tc_launches) *tc_launches = p->n_tc_launches;
  if (total) *total = p->n_launches;
  if (reset) {
    p->prof_used = 0;
    p->n_tc_launches = 0;
    p->n_launches = 0;
  }
  return CSX_OK;
}

csx_status csx_plan_destroy(csx_plan_t p) {
  if (!p) return CSX_OK;
  for (auto& q : p->hsub) csx_plan_destroy(q.second);  // csx_run_host chunk sub-plans
  p->hsub.clear();
  for (void* ev : p->prof_events) cudaEventDestroy((cudaEvent_t)ev);
  if (p->side) cudaStreamDestroy((cudaStream_t)p->side);
  if (p->ev_fork) cudaEventDestroy((cudaEvent_t)p->ev_fork);
  if (p->ev_join) cudaEventDestroy((cudaEvent_t)p->ev_join);
  if (p->device >= 0) {
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(p->device);
    for (auto& ps : p->passes) {
      cudaFree(ps.d_frags);
      cudaFree(ps.d_lut);
      cudaFree(ps.d_tile_frags);
      cudaFree(ps.d_wc);
    }
    cudaFree(p->d_buf[0]);
    cudaFree(p->d_buf[1]);
    cudaFree(p->d_wbase);
    cudaFree(p->d_dense);
    for (auto& b : p->h_slot) cudaFree(b);
    if (p->h_s_in) cudaStreamDestroy((cudaStream_t)p->h_s_in);
    if (p->h_s_out) cudaStreamDestroy((cudaStream_t)p->h_s_out);
    for (void* e : p->h_ev)
      if (e) cudaEventDestroy((cudaEvent_t)e);
    if (!p->peer) {  // (peer plans keep their slab buffers inside the peer block)
      cudaFree(p->d_sbuf[0]);
      cudaFree(p->d_sbuf[1]);
    }
    cudaFree(p->d_s2r);
    cudaFree(p->d_pstage);
    cudaFree(p->d_halo);
    p->d_s2r = nullptr;
    p->d_pstage = nullptr;
    p->d_halo = nullptr;
    if (p->g_exec) cudaGraphExecDestroy((cudaGraphExec_t)p->g_exec);
    if (p->g_stream) cudaStreamDestroy((cudaStream_t)p->g_stream);
    p->g_exec = nullptr;
    p->g_stream = nullptr;
    // NVLink peer exchange (comm.cpp): the block holds both slab buffers and the flag words a
    // neighbour's last k_peer_push writes into, so the caller must have synchronised every rank
    // (e.g. a barrier after the last csx_run_sharded_peer) before destroying a peer plan.
    if (p->peer) {
      csx_peer_s* q = p->peer;
      if (q->cs) cudaStreamSynchronize((cudaStream_t)q->cs);
      for (void* ptr : q->opened) cudaIpcCloseMemHandle(ptr);
      cudaFree(q->block);
      if (q->cs) cudaStreamDestroy((cudaStream_t)q->cs);
      if (q->ev_edge) cudaEventDestroy((cudaEvent_t)q->ev_edge);
      if (q->ev_x) cudaEventDestroy((cudaEvent_t)q->ev_x);
      delete q;
      p->peer = nullptr;
      p->d_sbuf[0] = p->d_sbuf[1] = nullptr;
    }
    cudaSetDevice(cur);
  }
  delete p;
  return CSX_OK;
}

csx_status csx_plan_info(const csx_plan_t p, csx_plan_info_t* info) {
  if (!p || !info) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  const Pass& ps = p->passes[p->tf - 1];
  std::memset(info, 0, sizeof(*info));
  info->ndim = p->ndim;
  info->radius = p->radius;
  info->fuse_steps = p->tf;
  info->nk = ps.nk;
  info->engine = p->engine;
  info->tile_m = ps.bm;
  info->tile_n = ps.bn;
  info->s2r_pitch = ps.pitch;
  info->mma_per_pass = p->engine == CSX_ENGINE_TC_TILE ? ps.tile_mma_per_pass
                       : p->engine == CSX_ENGINE_TC_S2R ? ps.mma_per_pass : 0;
  const double pts = (double)(p->E[0] * p->E[1] * p->E[2]);
  info->tc_flops_per_point_step = 512.0 * (double)info->mma_per_pass / (pts * ps.tf);
  info->useful_flops_per_point_step = 2.0 * p->nnz;
  return CSX_OK;
}

csx_status csx_compose_weights(int ndim, int radius, const double* w, int tf, double* out) {
  if (!w || !out || ndim < 1 || ndim > 3 || radius < 1 || radius > 7 || tf < 1 || tf > 16)
    return fail(CSX_ERR_INVALID_ARGUMENT, "bad argument");
  int64_t dense = 1;
  for (int a = 0; a < ndim; ++a) dense *= 2 * radius + 1;
  std::vector<double> base(w, w + dense);
  std::vector<double> c = compose(ndim, radius, base, tf);
  std::memcpy(out, c.data(), c.size() * sizeof(double));
  return CSX_OK;
}

csx_status csx_weight_matrices(int nk, int ndim1, const double* w, double* wa, double* wb) {
  if (!w || !wa || !wb || nk < 1 || nk > 31) return fail(CSX_ERR_INVALID_ARGUMENT, "bad argument");
  weight_matrices(nk, ndim1, w, wa, wb);
  return CSX_OK;
}

int csx_stencil2row_index(int nk, int which, int64_t x, int64_t y, int64_t* row, int64_t* col) {
  if (!row || !col || nk < 1 || x < 0 || y < 0) return 0;
  return s2r_index(nk, which, x, y, row, col) ? 1 : 0;
}

int csx_fragment_bank_conflicts(int pitch, int col) { return fragment_conflicts(pitch, col); }

csx_status csx_plan_lut(const csx_plan_t p, int32_t* lut_a, int32_t* lut_b, int64_t* count,
                        int* region_rows, int* region_cols) {
  if (!p || !count) return fail(CSX_ERR_INVALID_ARGUMENT, "NULL argument");
  const Pass& ps = p->passes[p->tf - 1];
  if (!ps.s2r_ok) return fail(CSX_ERR_UNSUPPORTED, "plan has no stencil2row LUT");
  *count = (int64_t)ps.lut_a.size();
  if (region_rows) *region_rows = ps.rr;
  if (region_cols) *region_cols = ps.rc;
  if (lut_a) std::memcpy(lut_a, ps.lut_a.data(), ps.lut_a.size() * sizeof(int32_t));
  if (lut_b) std::memcpy(lut_b, ps.lut_b.data(), ps.lut_b.size() * sizeof(int32_t));
  return CSX_OK;
}

}  // extern "C"

namespace csx {

// The pass loop: pack d_in into the padded grid, then floor(T/Tf) fused
// passes plus one remainder pass of T mod Tf steps, ping-ponging between the two padded
// grids; the last pass writes straight into d_out.  PERIODIC ghosts are refreshed after every
// pass; FIXED bands are recomputed by the fix-up inside run_pass.
csx_status run_local(csx_plan_s* p, const double* d_in, double* d_out, int64_t T, cudaStream_t st) {
  const Padded& pd = p->pad;
  const int real[3] = {p->ndim == 3, p->ndim >= 2, 1};
  View b[2];
  for (int i = 0; i < 2; ++i) b[i] = View{p->d_buf[i] + pd.origin(), pd.s0, pd.s1};
  const int64_t nmain = T / p->tf;
  const int rem = (int)(T % p->tf);
  const int64_t npass = nmain + (rem ? 1 : 0);
  // Pass depths (reading A8): nmain passes of Tf then the remainder.  A remainder of 1 after at
  // least one full pass of Tf >= 3 is folded with the last full pass into two passes of
  // ceil/floor((Tf+1)/2) — same pass count, and on the DMMA-bound 2D path two nk = 5 passes cost
  // less than nk = 7 + nk = 3 (12 + 12 vs 20 + 6 DMMAs per 64 outputs, the nk = 3 pass being
  // HBM-bound at its full sweep).  Kept when CSX_FOLD_REMAINDER=0.
  const char* fr = getenv("CSX_FOLD_REMAINDER");
  const bool fold = rem == 1 && nmain >= 1 && p->tf >= 3 && p->ndim >= 2 && !(fr && fr[0] == '0');
  auto depth = [&](int64_t i) -> int {
    if (fold && i >= nmain - 1) return i == nmain - 1 ? (p->tf + 2) / 2 : (p->tf + 1) / 2;
    return i < nmain ? p->tf : rem;
  };
  // FIXED TC_TILE 2D / 3D: the first pass stages its tiles straight from the user's dense d_in
  // through a TMA tensor map (out-of-grid halo boxes zero-filled; only held frame points and
  // the k_band-recomputed band see them), so no pack into the padded layout.  Not in place for a
  // single pass (its tiles would read halos other tiles already overwrote).
  const bool dense_src = p->engine == CSX_ENGINE_TC_TILE && p->ndim >= 2 && p->bc == CSX_BC_FIXED &&
                         (d_in != d_out || npass > 1) && tile_reads_dense(d_in, p->E);
  cudaError_t e = cudaSuccess;
  if (!dense_src) {
    e = launch_pack(d_in, b[0], p->E, st);
    if (e != cudaSuccess) return cuda_fail(e, "pack");
    p->n_launches += 1;
  }
  const int nghost = real[0] + real[1] + real[2];
  if (p->bc == CSX_BC_PERIODIC) {
    e = launch_ghost_fill(b[0], p->E, real, real, p->halo, st);
    if (e != cudaSuccess) return cuda_fail(e, "ghost fill");
    p->n_launches += nghost;
  }
  const View out{d_out, p->E[1] * p->E[2], p->E[2]};
  int cur = 0;
  for (int64_t i = 0; i < npass; ++i) {
    const int tfp = depth(i);
    const bool last = i == npass - 1;
    PassCtx c;
    c.src = CView{b[cur].p, b[cur].s0, b[cur].s1, pd.O[0], pd.O[1], pd.O[2], pd.A[0]};
    if (i == 0 && dense_src) c.src = CView{d_in, p->E[1] * p->E[2], p->E[2], 0, 0, 0, p->E[0]};
    c.dst = last ? out : b[cur ^ 1];
    for (int a = 0; a < 3; ++a) { c.E[a] = p->E[a]; c.gorg[a] = 0; }
    c.max_ctas = p->max_ctas;
    csx_status s = run_pass(p, p->passes[tfp - 1], c, st);
    if (s != CSX_OK) return s;
    if (!last && p->bc == CSX_BC_PERIODIC) {
      e = launch_ghost_fill(b[cur ^ 1], p->E, real, real, p->halo, st);
      if (e != cudaSuccess) return cuda_fail(e, "ghost fill");
      p->n_launches += nghost;
    }
    cur ^= 1;
  }
  return CSX_OK;
}

}  // namespace csx
