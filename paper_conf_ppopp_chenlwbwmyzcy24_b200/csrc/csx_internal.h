// csx_internal.h — plan representation shared by the host planner (planner.cpp), the C-ABI
// (api.cpp) and the kernel launchers (*.cu).  Product code only; nothing here is shared with
// oracle/.
#pragma once
#include <cstdint>
#include <string>
#include <utility>
#include <vector>

#include "../../include/csx.h"

namespace csx {

constexpr int kMaxNK = 15;          // largest composed window edge any engine accepts
constexpr int kWarp = 32;

// Set the thread-local error detail returned by csx_last_error().
void set_error(const std::string& msg);
csx_status fail(csx_status s, const std::string& msg);

// ---- host planning (planner.cpp) -------------------------------------------------------

// W^(Tf): Tf-fold discrete convolution of the offset-indexed (2r+1)^d array (P.1466-1482).
std::vector<double> compose(int ndim, int radius, const std::vector<double>& w, int tf);

// Paper weight matrices (P.961-975): (nk*nk) x (nk+1) row-major (2D) or nk x (nk+1) (1D).
void weight_matrices(int nk, int ndim1, const double* w, double* wa, double* wb);

// Eq 5 / Eq 6 mapping.  Returns true if (x, y) lands in matrix `which` (0 = A, 1 = B).
bool s2r_index(int nk, int which, int64_t x, int64_t y, int64_t* row, int64_t* col);

// Max 8-byte words per 4-byte bank over the two 4x4 requests of one m8n8k4 A fragment
// read from a stencil2row tile with pitch `pitch` (doubles), fragment column `col`.
int fragment_conflicts(int pitch, int col);

// Smallest pitch >= min_pitch that is conflict-free for every fragment column (Fig 5).
int choose_pitch(int min_pitch);

// One fused-pass configuration (a "sub-plan"): Tf' steps, composed window nk = 2 r Tf' + 1.
struct Pass {
  int tf = 0;
  int nk = 0;
  std::vector<double> wc;          // composed weights, nk^ndim
  // --- TC_S2R geometry (2D: nk x nk window; 1D: nk; 3D: per-plane 2D windows) ---
  int sw = 0;                      // strip width nk + 1 (outputs per strip)
  int ks = 0;                      // k-slices per weight matrix (ceil(K/4))
  int nf = 0;                      // N fragments ceil((nk+1)/8)
  int bm = 0, bn = 0;              // CTA output tile (rows, cols)
  int rr = 0, rc = 0;              // CTA input region rows, cols
  int pitch = 0;                   // stencil2row smem pitch (doubles)
  int planes = 1;                  // 3D: number of z offsets (nk); 1D/2D: 1
  int tc_planes = 1;               // 3D: planes computed on tensor cores
  std::vector<int> plane_is_tc;    // 3D: per z offset, 1 = TC, 0 = CUDA-core single tap
  std::vector<double> frags;       // per-lane DMMA B fragments [plane][A|B][nf][ks][32]
  std::vector<int32_t> lut_g;      // per region element: offset in the padded source grid
  std::vector<int32_t> lut_a;      // per region element: smem offset in stencil2row A
  std::vector<int32_t> lut_b;      // per region element: smem offset in stencil2row B
  int64_t mma_per_pass = 0;        // DMMA instructions per pass over the whole grid
  // --- TC_TILE geometry ---
  int tile_ok = 0;
  bool s2r_ok = false;              // a TC_S2R kernel exists for (ndim, nk)
  std::vector<double> tile_frags;  // [plane][slice][32] fragments for the 4x2-block GEMM
  int tile_ks = 0;                 // k-slices per output block (K / 4)
  int tile_a = 0, tile_b = 0;      // output block a rows x b cols (a * b = 8 = DMMA N)
  int tile_kc = 0;                 // padded region row length of one block (multiple of 4)
  int64_t tile_mma_per_pass = 0;
  // device copies (owned)
  double* d_frags = nullptr;
  int32_t* d_lut = nullptr;        // interleaved {g, a | b << 16} pairs
  double* d_tile_frags = nullptr;
  double* d_wc = nullptr;          // composed weights on the device (direct / 3D CUDA-core taps)
  bool uploaded = false;
};

// A padded ping-pong grid: 3 normalised axes (missing leading axes have extent 1).
struct Padded {
  int64_t E[3] = {1, 1, 1};        // interior extents
  int64_t O[3] = {0, 0, 0};        // interior origin inside the allocation
  int64_t A[3] = {1, 1, 1};        // allocated extents (A[2] is the row pitch)
  int64_t s0 = 0, s1 = 0;          // strides of axes 0 and 1 (axis 2 stride is 1)
  int64_t elems() const { return A[0] * A[1] * A[2]; }
  int64_t origin() const { return O[0] * s0 + O[1] * s1 + O[2]; }
};

// DMMAs per output point, pass and TC plane of the 3D Tf = 2 kernel that runs (kernels_tile.cu)
double tile3d_tb_mma_per_point();

}  // namespace csx

// NVLink peer-memory halo exchange state of a sharded plan (comm.cpp, kernels_peer.cu).
struct csx_peer_s {
  int rank = 0, nranks = 1, up = -1, down = -1;  // neighbours along the slab axis (-1 none)
  int64_t El = 0, El_up = 0, El_down = 0;         // slab rows owned by this rank / neighbours
  double* up_buf[2] = {nullptr, nullptr};         // neighbour slab buffers (allocation bases)
  double* down_buf[2] = {nullptr, nullptr};
  // local flag block: [0] READY_TOP (written by up), [1] READY_BOTTOM (by down),
  // [2] FREED_BY_UP (by up), [3] FREED_BY_DOWN (by down), [4] last-CTA counter
  unsigned long long* flags = nullptr;
  void* block = nullptr;                          // one allocation: slab buffers 0, 1 + flags
  unsigned long long* up_flags = nullptr;         // the neighbours' flag blocks (peer memory)
  unsigned long long* down_flags = nullptr;
  std::vector<void*> opened;                      // IPC mappings to close
  unsigned long long epoch = 0;                   // epoch base of the next run
  void* cs = nullptr;                             // cudaStream_t: push stream
  void* ev_edge = nullptr;                        // cudaEvent_t
  void* ev_x = nullptr;
  bool connected = false;
};

struct csx_plan_s {
  int ndim = 0;
  int64_t ext[3] = {1, 1, 1};      // user extents (ext[0] slowest), ndim of them valid
  int64_t E[3] = {1, 1, 1};        // normalised to 3 axes
  int radius = 0;
  csx_shape shape = CSX_SHAPE_BOX;
  csx_boundary bc = CSX_BC_FIXED;
  std::vector<double> w;           // base weights (2r+1)^ndim
  int nnz = 0;
  int tf = 1;                      // main fusion depth
  int halo = 0;                    // r * tf
  csx_engine engine_req = CSX_ENGINE_AUTO;
  bool s2r_pad = true;             // TC_S2R 2D: conflict-free pitch (Fig 5)
  bool s2r_dirty = true;           // TC_S2R 2D: dirty-bits padding instead of branches
  bool s2r_fma = false;            // TC_S2R 2D: breakdown II, tessellation on CUDA cores
  bool s2r_explicit = false;       // TC_S2R 2D: breakdown I, explicit stencil2row in HBM
  double* d_s2r = nullptr;         // breakdown I: global stencil2row A|B scratch
  int64_t s2r_elems = 0;
  csx_engine engine = CSX_ENGINE_TC_S2R;
  std::vector<csx::Pass> passes;   // index tf' - 1, for tf' = 1..tf
  // device state (allocated at the first run)
  int device = -1;
  csx::Padded pad;
  double* d_buf[2] = {nullptr, nullptr};
  double* d_wbase = nullptr;       // base weights (direct engine, fix-up)
  // sharded state
  csx::Padded spad;                // per-rank slab grid
  double* d_sbuf[2] = {nullptr, nullptr};
  double* d_halo = nullptr;        // 4 halo staging slabs (send lo/hi, recv lo/hi)
  int64_t s_lo = -1, s_hi = -1;
  int s_rank = -1, s_nranks = 0;
  int s_p0 = 0, s_p1 = 0;          // pencil process grid of the sharded buffers (0: slabs)
  double* d_pstage = nullptr;      // pencil halo staging (4 strided faces packed contiguously)
  size_t pstage_elems = 0;
  double* d_dense = nullptr;       // csx_run_host staging grid
  // csx_run_host chunked pipeline (ghost-zone chunks along the slowest axis): sub-plans by
  // chunk extent, two device slots (input / output), copy streams and per-slot events
  std::vector<std::pair<int64_t, csx_plan_s*>> hsub;
  double* h_slot[4] = {nullptr, nullptr, nullptr, nullptr};  // in0, in1, out0, out1
  int64_t h_slot_elems = 0;
  void* h_s_in = nullptr;          // cudaStream_t (H2D)
  void* h_s_out = nullptr;         // cudaStream_t (D2H)
  void* h_ev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};  // h2d[2], comp[2], d2h[2]
  int h_last_chunks = 0;           // what the last csx_run_host did (csx_host_last)
  int64_t h_last_h2d = 0, h_last_d2h = 0;
  csx_peer_s* peer = nullptr;      // NVLink peer halo exchange (csx_peer_export / _connect)
  // side stream: the FIXED band fix-up of a TC_TILE 2D pass runs concurrently with the pass
  void* side = nullptr;            // cudaStream_t
  void* ev_fork = nullptr;         // cudaEvent_t
  void* ev_join = nullptr;
  // CUDA graph replay of csx_run (csx_plan_set_graph): the pass sequence of one
  // (d_in, d_out, T) captured once and replayed with one cudaGraphLaunch
  int graph_on = 0;
  int max_ctas = 0;                // persistent-grid cap of every launch (csx_plan_set_max_ctas)
  void* g_exec = nullptr;          // cudaGraphExec_t
  void* g_stream = nullptr;        // non-blocking capture stream
  const double* g_in = nullptr;
  double* g_out = nullptr;
  int64_t g_T = -1, g_launches = 0, g_tc_launches = 0;
  // measurement hooks
  int prof = 0;  // 0 off, n: time every n-th main-pass TC launch
  std::vector<void*> prof_events;  // cudaEvent_t pairs around TC launches
  size_t prof_used = 0;
  int64_t n_tc_launches = 0, n_launches = 0;
};

namespace csx {
// planner.cpp
csx_status build_plan(csx_plan_s* p);
int auto_tf(int ndim, int radius, int engine);  // automatic fusion depth (reading A4)
csx_status build_pass(const csx_plan_s* p, int tf, Pass* out);
void layout_padded(const csx_plan_s* p, const int64_t* E, Padded* pd);
}  // namespace csx
