// planner.cpp — host-side planning for the csx hot path.
//
//  a1  fusion depth + weight composition  (PAPER.md P.1466-1482, Fig 4)
//  a2  weight matrices W_A / W_B -> per-lane DMMA B fragments  (P.961-975, P.1304-1325, Fig 3)
//  a3  lookup table + dirty-bits padding   (P.1711-1721, P.1759-1773, Fig 5)
//      with the conflict-free stencil2row pitch (P.1722-1757)
//
// Everything here runs once per plan on the host; the kernels only read the tables.
#include <algorithm>
#include <cmath>
#include <cstring>

#include "csx_internal.h"
#include "s2r_geom.h"

namespace csx {

std::vector<double> compose(int ndim, int radius, const std::vector<double>& w, int tf) {
  // Tf-fold discrete convolution of the offset-indexed arrays: applying a correlation with w
  // Tf times equals one correlation with W^(Tf) = w * w * ... * w (on a torus).
  std::vector<double> cur = w;
  int cr = radius;  // radius of cur
  const int n = 2 * radius + 1;
  for (int step = 1; step < tf; ++step) {
    const int nr = cr + radius, nn = 2 * nr + 1, cn = 2 * cr + 1;
    std::vector<double> nxt((size_t)std::pow(nn, ndim), 0.0);
    const int64_t csz = (int64_t)std::pow(cn, ndim), wsz = (int64_t)std::pow(n, ndim);
    for (int64_t a = 0; a < csz; ++a) {
      if (cur[a] == 0.0) continue;
      int ca[3] = {0, 0, 0};
      int64_t t = a;
      for (int d = ndim - 1; d >= 0; --d) { ca[d] = (int)(t % cn) - cr; t /= cn; }
      for (int64_t b = 0; b < wsz; ++b) {
        if (w[b] == 0.0) continue;
        int wb[3] = {0, 0, 0};
        int64_t u = b;
        for (int d = ndim - 1; d >= 0; --d) { wb[d] = (int)(u % n) - radius; u /= n; }
        int64_t idx = 0;
        for (int d = 0; d < ndim; ++d) idx = idx * nn + (ca[d] + wb[d] + nr);
        nxt[idx] += cur[a] * w[b];
      }
    }
    cur.swap(nxt);
    cr = nr;
  }
  return cur;
}

void weight_matrices(int nk, int ndim1, const double* w, double* wa, double* wb) {
  // P.961-975 / Fig 3:  W_A[nk*i + j][c] = w[i][j - c]        (j >= c; lower triangles)
  //                     W_B[nk*i + j][c] = w[i][j + nk - c]   (j <  c; upper triangles)
  // c in [0, nk]; W_A's last column and W_B's first column are zero.
  const int rows_w = ndim1 ? 1 : nk;
  const int cols = nk + 1;
  for (int i = 0; i < rows_w; ++i)
    for (int j = 0; j < nk; ++j)
      for (int c = 0; c < cols; ++c) {
        const int k = nk * i + j;
        wa[k * cols + c] = (j >= c) ? w[i * nk + (j - c)] : 0.0;
        wb[k * cols + c] = (j < c) ? w[i * nk + (j + nk - c)] : 0.0;
      }
}

bool s2r_index(int nk, int which, int64_t x, int64_t y, int64_t* row, int64_t* col) {
  // Eq 5 (A): (x, y) -> [floor(y/(nk+1))][nk*x + y mod (nk+1)]   where (y+1) mod (nk+1) != 0
  // Eq 6 (B): (x, y) -> [floor((y-nk)/(nk+1))][nk*x + (y-nk) mod (nk+1)]
  //           where (y-nk+1) mod (nk+1) != 0 and y >= nk   (reading A6 of the garbled P.785)
  const int64_t s = nk + 1;
  int64_t yy = y;
  if (which == 1) {
    yy = y - nk;
    if (yy < 0) return false;
  }
  if ((yy + 1) % s == 0) return false;
  *row = yy / s;
  *col = (int64_t)nk * x + yy % s;
  return true;
}

int fragment_conflicts(int pitch, int col) {
  // P.1736-1757: a warp's 8x4 FP64 fragment is two requests of 16 lanes (rows 0-3, rows 4-7),
  // each a 4x4 block; 32 banks of 4 bytes, one double = 2 banks.  Conflict degree = the max
  // number of distinct 8-byte words that map to one bank within a request.
  int worst = 1;
  for (int half = 0; half < 2; ++half) {
    int count[32] = {0};
    for (int g = 4 * half; g < 4 * half + 4; ++g)
      for (int t = 0; t < 4; ++t) {
        const int64_t word = (int64_t)g * pitch + col + t;  // double index
        const int bank = (int)((word * 2) % 32);
        count[bank] += 1;  // the word also occupies bank+1; symmetric, count one
      }
    for (int b = 0; b < 32; ++b) worst = std::max(worst, count[b]);
  }
  return worst;
}

int choose_pitch(int min_pitch) {
  for (int p = min_pitch;; ++p) {
    bool ok = true;
    for (int c = 0; c < 16 && ok; ++c) ok = fragment_conflicts(p, c) == 1;
    if (ok) return p;
  }
}

// ----------------------------------------------------------------------------------------
// Padded ping-pong grid layout: interior at O, halo of depth >= r*Tf on every real axis,
// the fastest axis aligned so that interior rows start on a 128-byte boundary.
void layout_padded(const csx_plan_s* p, const int64_t* E, Padded* pd) {
  const int H = p->halo;
  const int real0 = p->ndim == 3, real1 = p->ndim >= 2;
  // slack beyond the interior for CTA tiles that overhang the last row / column (every
  // kernel's tile is <= 128 rows and <= 128 + 32 columns including its halo)
  for (int a = 0; a < 3; ++a) pd->E[a] = E[a];
  pd->O[0] = real0 ? H : 0;
  pd->O[1] = real1 ? H : 0;
  pd->O[2] = 16 * ((H + 15) / 16);  // >= H, interior rows 128-byte aligned
  if (pd->O[2] < 16) pd->O[2] = 16;
  pd->A[0] = real0 ? (E[0] + 2 * H + 16) : 1;  // direct-kernel z tiles (8) overhang the last plane
  pd->A[1] = real1 ? (pd->O[1] + E[1] + 128 + H + 2) : 1;
  const int64_t need2 = pd->O[2] + E[2] + 160 + H + 32;
  pd->A[2] = 32 * ((need2 + (p->ndim == 1 ? 2048 : 0) + 31) / 32);  // 1D tiles overhang more
  pd->s1 = pd->A[2];
  pd->s0 = pd->A[1] * pd->A[2];
}

template <class G>
static void fill_geom(Pass* P, int bm, int rr) {
  P->ks = G::KS;
  P->bm = bm;
  P->bn = G::BN;
  P->rr = rr;
  P->rc = G::RC;
  P->pitch = G::PITCH;
}

// TC_S2R kernels exist for 1D nk in {3..15}, 2D nk in {3,5,7}, 3D nk = 3.
static bool s2r_geometry(int ndim, int nk, Pass* P) {
  if (ndim == 1) {
    switch (nk) {
      case 3: fill_geom<S2R1D<3>>(P, 1, 1); return true;
      case 5: fill_geom<S2R1D<5>>(P, 1, 1); return true;
      case 7: fill_geom<S2R1D<7>>(P, 1, 1); return true;
      case 9: fill_geom<S2R1D<9>>(P, 1, 1); return true;
      case 11: fill_geom<S2R1D<11>>(P, 1, 1); return true;
      case 13: fill_geom<S2R1D<13>>(P, 1, 1); return true;
      case 15: fill_geom<S2R1D<15>>(P, 1, 1); return true;
    }
    return false;
  }
  if (ndim == 2) {
    switch (nk) {
      case 3: fill_geom<S2R2D<3>>(P, S2R2D<3>::BM, S2R2D<3>::RR); return true;
      case 5: fill_geom<S2R2D<5>>(P, S2R2D<5>::BM, S2R2D<5>::RR); return true;
      case 7: fill_geom<S2R2D<7>>(P, S2R2D<7>::BM, S2R2D<7>::RR); return true;
    }
    return false;
  }
  if (nk == 3) {
    fill_geom<S2R3D<3>>(P, S2R3D<3>::BM, S2R3D<3>::RR);
    return true;
  }
  return false;
}

csx_status build_pass(const csx_plan_s* p, int tf, Pass* out) {
  Pass P;
  P.tf = tf;
  P.nk = 2 * p->radius * tf + 1;
  P.wc = compose(p->ndim, p->radius, p->w, tf);
  const int nk = P.nk;
  P.sw = nk + 1;
  P.nf = (P.sw + 7) / 8;
  const int ndim = p->ndim;
  // Plane structure (3D, §4.2 P.1788-1800): z offset dz carries the 2D window W[dz].  A plane
  // with a single tap (the +-z arms of star shapes) goes to CUDA cores (reading A9).
  if (ndim == 3) {
    P.planes = nk;
    P.plane_is_tc.assign(nk, 1);
    P.tc_planes = 0;
    for (int dz = 0; dz < nk; ++dz) {
      int taps = 0;
      for (int i = 0; i < nk * nk; ++i) taps += P.wc[(size_t)dz * nk * nk + i] != 0.0;
      P.plane_is_tc[dz] = taps > 1;
      P.tc_planes += P.plane_is_tc[dz];
    }
  }
  // ---------------- TC_S2R geometry (s2r_geom.h) ----------------
  const int nplanes = ndim == 3 ? nk : 1;
  P.s2r_ok = s2r_geometry(ndim, nk, &P);
  if (P.s2r_ok) {
  const int strips = P.bn / P.sw;  // stencil2row rows covered by one CTA tile
  // the kernels' constexpr pitch must be the conflict-free pitch of the bank model
  if (P.pitch != choose_pitch(ndim == 1 ? 4 * P.ks : nk * P.rr))
    return fail(CSX_ERR_INTERNAL, "stencil2row pitch disagrees with the bank-conflict model");
  // Breakdown variants (Fig 6, P.1865-1950), 2D only: without padding the pitch is the bare
  // nk*rr (266 for the 32x64 tile: 2-way conflicts, Fig 5); without dirty bits the elements
  // that belong to neither matrix get a sentinel and the copy loop branches on it.
  const bool pad = ndim != 2 || p->s2r_pad;
  const bool dirty_bits = ndim != 2 || p->s2r_dirty;
  if (!pad) P.pitch = nk * P.rr;
  // LUT: every input-region element -> (global offset, smem offset in A, in B).  Elements
  // that belong to neither matrix are routed to the dirty row (row index `strips`), so the
  // copy loop has no branches (P.1759-1773).
  const int64_t ne = (int64_t)P.rr * P.rc;
  P.lut_g.resize(ne);
  P.lut_a.resize(ne);
  P.lut_b.resize(ne);
  int64_t sp[3];
  {
    int64_t E[3] = {p->E[0], p->E[1], p->E[2]};
    Padded tmp;
    layout_padded(p, E, &tmp);
    sp[1] = tmp.s1;
  }
  const int dirty_base = strips * P.pitch;
  for (int x = 0; x < P.rr; ++x)
    for (int y = 0; y < P.rc; ++y) {
      const int64_t e = (int64_t)x * P.rc + y;
      P.lut_g[e] = (int32_t)(ndim == 1 ? y : x * sp[1] + y);
      int64_t row, col;
      const int dirty = dirty_bits ? dirty_base + (int)(e % P.pitch) : 0xffff;
      // Eq 5 on tile-local coordinates: for 1D the "row" of the input is x = 0 and the
      // stencil2row row length is nk (P.1779-1786).
      if (s2r_index(nk, 0, ndim == 1 ? 0 : x, y, &row, &col) && row < strips)
        P.lut_a[e] = (int32_t)(row * P.pitch + col);
      else
        P.lut_a[e] = dirty;
      if (s2r_index(nk, 1, ndim == 1 ? 0 : x, y, &row, &col) && row < strips)
        P.lut_b[e] = (int32_t)(row * P.pitch + col);
      else
        P.lut_b[e] = dirty;
    }
  // Per-lane DMMA B fragments: slice s, lane l holds W[4s + l%4][8f + l/4]  (m8n8k4 .col B).
  // 2D layout per plane: [A|B][nf][ks][32].
  const int K = ndim == 1 ? nk : nk * nk;
  const int cols = nk + 1;
  std::vector<double> wa((size_t)K * cols), wb((size_t)K * cols);
  P.frags.assign((size_t)nplanes * 2 * P.nf * P.ks * 32, 0.0);
  for (int pl = 0; pl < nplanes; ++pl) {
    const double* w2 = P.wc.data() + (size_t)pl * (ndim == 3 ? nk * nk : 0);
    weight_matrices(nk, ndim == 1, w2, wa.data(), wb.data());
    for (int m = 0; m < 2; ++m)
      for (int f = 0; f < P.nf; ++f)
        for (int s = 0; s < P.ks; ++s)
          for (int l = 0; l < 32; ++l) {
            const int k = 4 * s + (l % 4), c = 8 * f + l / 4;
            double v = 0.0;
            if (k < K && c < cols) v = (m == 0 ? wa : wb)[(size_t)k * cols + c];
            P.frags[((((size_t)pl * 2 + m) * P.nf + f) * P.ks + s) * 32 + l] = v;
          }
  }
  }  // s2r_ok
  // Eq 13, generalised by reading A7 (N fragments) and 3D planes: DMMAs per pass over the
  // whole grid = (points / (8 (nk+1))) * 2 ceil(K/4) * nf * tc_planes.
  const int64_t pts = p->E[0] * p->E[1] * p->E[2];
  const int tcp = ndim == 3 ? P.tc_planes : 1;
  P.mma_per_pass = (int64_t)((double)pts / (8.0 * P.sw) * 2 * P.ks * P.nf * tcp + 0.5);
  // ---------------- TC_TILE geometry (2D nk <= 13, 3D planes nk <= 7) ----------------
  // The same GEMM with the 8 N columns of a DMMA holding an a x b block of outputs (a*b = 8)
  // instead of 1 x (nk+1): K = the (a+nk-1) x (b+nk-1) input region of the block, each region
  // row padded to kc (a multiple of 4) so that every k-slice is 4 consecutive cells of one
  // input row.  Block shape per nk minimises K: nk=3 -> 4x2 (K=24), nk=5 -> 2x4 (K=48),
  // nk=7 -> 4x2 (K=80) versus the paper's 2*ceil(nk^2/4)*4 = 24 / 56 / 104; fused windows
  // past one N fragment of the paper's layout (reading A7): nk=9 -> 2x4 (K=120), nk=11 -> 4x2
  // (K=168), nk=13 -> 2x4 (K=224) versus 2*ceil(nk^2/4)*4*nf = 168 / 248 / 344.
  if (ndim == 1) {
    // 1D TC_TILE: the 8 N columns are 8 consecutive outputs, so the weight operand is the banded
    // Toeplitz matrix W[k][n] = w[k - n] (0 <= k - n < nk), K = nk + 7 rounded up to 4.
    P.tile_ok = 1;
    P.tile_a = 1;
    P.tile_b = 8;
    P.tile_ks = (nk + 7 + 3) / 4;
    P.tile_kc = 4 * P.tile_ks;
    P.tile_frags.assign((size_t)P.tile_ks * 32, 0.0);
    for (int s = 0; s < P.tile_ks; ++s)
      for (int l = 0; l < 32; ++l) {
        const int k = 4 * s + (l % 4), n = l / 4, j = k - n;
        P.tile_frags[(size_t)s * 32 + l] = (j >= 0 && j < nk) ? P.wc[j] : 0.0;
      }
    P.tile_mma_per_pass = (int64_t)((double)pts / 64.0 * P.tile_ks + 0.5);
  }
  if ((ndim == 2 && nk <= 13) || (ndim == 3 && nk <= 7)) {
    // block shape: the one of 4x2 / 2x4 with the smaller K = (a+nk-1) * kc
    auto kdim = [nk](int a_, int b_) { return (a_ + nk - 1) * 4 * ((b_ + nk - 1 + 3) / 4); };
    int a = 4, b = 2;
    if (kdim(2, 4) < kdim(4, 2)) { a = 2; b = 4; }
    const int krows = a + nk - 1;
    const int kc = 4 * ((b + nk - 1 + 3) / 4);
    P.tile_ok = 1;
    P.tile_a = a;
    P.tile_b = b;
    P.tile_kc = kc;
    P.tile_ks = krows * kc / 4;
    P.tile_frags.assign((size_t)nplanes * P.tile_ks * 32, 0.0);
    for (int pl = 0; pl < nplanes; ++pl) {
      const double* w2 = P.wc.data() + (size_t)pl * (ndim == 3 ? nk * nk : 0);
      for (int s = 0; s < P.tile_ks; ++s)
        for (int l = 0; l < 32; ++l) {
          const int k = 4 * s + (l % 4), n = l / 4;  // n = output (alpha, beta) of the block
          const int rho = k / kc, kap = k % kc;
          const int alpha = n / b, beta = n % b;
          const int i = rho - alpha, j = kap - beta;
          double v = 0.0;
          if (i >= 0 && i < nk && j >= 0 && j < nk) v = w2[i * nk + j];
          P.tile_frags[((size_t)pl * P.tile_ks + s) * 32 + l] = v;
        }
    }
    P.tile_mma_per_pass = (int64_t)((double)pts / 64.0 * P.tile_ks * tcp + 0.5);
  }
  if (ndim == 3 && tf == 2 && p->radius == 1) {
    // 3D Tf = 2 runs the BASE stencil twice by temporal blocking (k_tile3d_tb2), not the composed
    // window: per 32 x 64 output tile and plane, level 1 computes 45 DMMA tiles (4 x 16) on the
    // grown 36 x 80 tile for 34 of every 32 planes (the z-chunk's two extra step-1 planes) and
    // level 2 32 tiles, 6 DMMAs (K = 24) per tile and TC plane of the base window (k_tile3d_tb3:
    // 39 level-1 tiles; tile3d_tb_mma_per_point follows the geometry the launch will pick).
    int base_tc = 0;
    for (int dz = 0; dz < 3; ++dz) {
      int taps = 0;
      for (int i = 0; i < 9; ++i) taps += p->w[(size_t)dz * 9 + i] != 0.0;
      base_tc += taps > 1;
    }
    P.tile_mma_per_pass = (int64_t)((double)pts * tile3d_tb_mma_per_point() * base_tc + 0.5);
  }
  *out = std::move(P);
  return CSX_OK;
}

int auto_tf(int ndim, int radius, int engine) {
  // DESIGN.md "Fusion depth" (reading A4): 2D r=1 -> 2 (TC_TILE on B200; TC_S2R keeps the
  // paper's Box-2D9P choice of 3, P.1478-1480); r >= 2 in 2D and all 3D -> 1 (one N fragment, lowest DMMA count per
  // point-step on B200).  1D is HBM-bound, so deeper fusion pays until the DMMA work of the
  // Toeplitz blocks (K = nk + 7) meets the HBM time: TC_TILE takes nk ~ 27..29 (r=1 -> 13,
  // r=2 -> 7, r=3 -> 3; round-2 sweep on Heat-1D / 1D5P, 10.24M and 102.4M points: Tf 9 / 11 /
  // 13 / 15 = 2845 / 3136 / 3263 / 3166 and 3060 / 3509 / 3877 / 4152 GSt/s; 1D5P Tf 4..7 best
  // at 7); TC_S2R's paper layout keeps nk + 1 <= 16 (two N fragments): r=1 -> 7, r=2 -> 3,
  // r=3 -> 2.
  if (ndim == 1) {
    if (engine == CSX_ENGINE_TC_S2R) return radius == 1 ? 7 : (radius == 2 ? 3 : 2);
    return radius == 1 ? 13 : (radius == 2 ? 7 : 3);
  }
  // the CUDA-core comparator's own best depth: 2D r = 1 -> 4 (register wavefront, Box-2D9P
  // 10240^2: Tf 1/2/3/4 = 310 / 640 / 681 / 766 GSt/s), r >= 2 -> 1
  if (ndim == 2 && engine == CSX_ENGINE_DIRECT) return radius == 1 ? 4 : 1;
  // 2D r = 1: the paper fuses 3 steps (Box-2D9P, P.1478-1480) and so does its layout here
  // (TC_S2R: 26 DMMAs per 64 outputs at nk = 7 vs 14 per 48 at nk = 5).  TC_TILE on B200 runs 2:
  // nk = 5 executes 48 tensor flops per point-step against nk = 7's 53.3 and moves 8 B instead
  // of 5.3, which the 6.5 TB/s HBM still covers — Box-2D9P / Heat-2D 10240^2, T = 100: 640 /
  // 640 GSt/s at Tf = 2 against 618 / 618 at Tf = 3 and 510 at Tf = 4 (profiles/r02/ab/)
  if (ndim == 2 && engine == CSX_ENGINE_TC_S2R) return radius == 1 ? 3 : 1;
  if (ndim == 2) return radius == 1 ? 2 : 1;
  return 1;
}

csx_status build_plan(csx_plan_s* p) {
  if (p->tf <= 0) {
    p->tf = auto_tf(p->ndim, p->radius, CSX_ENGINE_AUTO);
    // 3D r = 1 stars (single-tap z arms: one TC plane): two steps per pass by temporal blocking
    // (k_tile3d_tb2, Heat-3D 313 vs 293 GSt/s at Tf = 1); boxes keep Tf = 1 (150 vs 196)
    if (p->ndim == 3 && p->radius == 1) {
      bool star = true;
      for (int dz = 0; dz < 3; dz += 2) {
        int taps = 0;
        for (int i = 0; i < 9; ++i) taps += p->w[(size_t)dz * 9 + i] != 0.0;
        star = star && taps <= 1;
      }
      if (star) p->tf = 2;
    }
  }
  const int nk = 2 * p->radius * p->tf + 1;
  // 1D: TC_S2R (the paper's layout, nf <= 2 N fragments) takes nk <= 15, TC_TILE (Toeplitz
  // blocks) nk <= 31 — the FIXED band code's 32-lane cone needs 2 r (Tf-1) <= 31.
  if (p->ndim == 1 && nk > 31)
    return fail(CSX_ERR_UNSUPPORTED, "1D: composed window 2*r*Tf+1 must be <= 31");
  // 2D: TC_S2R (the paper's layout, one N fragment) takes nk <= 7; TC_TILE and DIRECT nk <= 13
  // (C3's "multi-step fused" r = 3, Tf = 2 is nk = 13).
  if (p->ndim == 2 && nk > 13)
    return fail(CSX_ERR_UNSUPPORTED, "2D: composed window 2*r*Tf+1 must be <= 13");
  if (p->ndim == 3 && p->tf > 2)
    return fail(CSX_ERR_UNSUPPORTED, "3D: Tf <= 2 (reading A4)");
  if (p->ndim == 3 && p->tf == 2 && p->radius != 1)
    return fail(CSX_ERR_UNSUPPORTED, "3D: Tf = 2 (temporal blocking) needs radius 1");
  for (int a = 0; a < 3; ++a)
    if ((a >= 3 - p->ndim) && p->E[a] < nk)
      return fail(CSX_ERR_INVALID_ARGUMENT, "extent smaller than the composed window 2*r*Tf+1");
  p->halo = p->radius * p->tf;
  p->passes.clear();
  p->passes.resize(p->tf);
  for (int t = 1; t <= p->tf; ++t) {
    csx_status s = build_pass(p, t, &p->passes[t - 1]);
    if (s != CSX_OK) return s;
  }
  return CSX_OK;
}

}  // namespace csx
