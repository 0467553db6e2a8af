/* oracle.c — CPU ORACLE for the csx hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this.  It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ppopp_chenlwbwmyzcy24_b200/csrc); neither includes nor links the other.
 *
 * What it computes — the plain definition the method reaches (up to FP reassociation):
 *   PAPER.md P.146-149 (§1) and P.277-287 (§2.1): "The value of one point at time t is a
 *   weighted sum of itself and neighboring points at the previous time t-1"; star / box
 *   shapes of radius r.  Orientation (correlation): w[i][j] multiplies X[x+i][y+j] with the
 *   result at the window centre (Fig 3, P.966-970, P.1326-1330; readings A2/A3).
 *
 *   u_{t+1}[p] = sum_{o in {-r..r}^d, w[o] != 0} w[o] * u_t[p + o]
 *   FIXED    : points within r of any face keep u_t[p]          (reading A1)
 *   PERIODIC : p + o is taken modulo the extents                 (reading A1)
 *
 * Plain C, double, built with -O2 -ffp-contract=off (no FMA contraction), fixed summation
 * order (row-major over offsets), ping-pong arrays, no blocking, no fusion, no intrinsics.
 * "#pragma omp parallel for" over the flattened point index is deterministic because each
 * output is computed independently.
 *
 * Pins (tests/test_oracle.py, -m "not gpu"): dense-matrix brute force, scipy.ndimage
 * correlate (wrap), constant-field invariant, closed-form Fourier decay (Heat-1D/2D/3D),
 * pure-shift stencils (np.roll), and window-sampling vs full runs.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#ifdef _OPENMP
#include <omp.h>
#endif

enum { ORACLE_BC_FIXED = 0, ORACLE_BC_PERIODIC = 1 };

/* A window of the global grid, normalised to 3 axes (missing leading axes have extent 1 and
 * radius 0).  Axis a covers global coordinates lo[a] .. lo[a]+len[a]-1 (mod E[a] when
 * PERIODIC).  full[a] != 0 means the window is the whole axis. */
typedef struct {
  int64_t E[3], lo[3], len[3];
  int full[3];
  int rad[3];
} window_t;

/* One base time step on a window (PAPER.md P.146-149).  A window point is held (copied
 * through) if it is in the FIXED frame of the global grid, or if one of its neighbours
 * would fall outside the window (an artificial window edge; only used when sampling, see
 * oracle_sample — those points are wrong but never reach the sampled centre). */
static void step_window(const window_t* W, const double* w, int bc, const double* in,
                        double* out) {
  const int64_t L0 = W->len[0], L1 = W->len[1], L2 = W->len[2];
  const int r0 = W->rad[0], r1 = W->rad[1], r2 = W->rad[2];
  const int n1 = 2 * r1 + 1, n2 = 2 * r2 + 1;
  const int64_t total = L0 * L1 * L2;
#pragma omp parallel for schedule(static)
  for (int64_t p = 0; p < total; ++p) {
    const int64_t i0 = p / (L1 * L2), i1 = (p / L2) % L1, i2 = p % L2;
    const int64_t ii[3] = {i0, i1, i2};
    int hold = 0;
    for (int a = 0; a < 3; ++a) {
      const int r = W->rad[a];
      if (r == 0) continue;
      if (bc == ORACLE_BC_FIXED) {
        const int64_t g = W->lo[a] + ii[a];
        if (g < r || g >= W->E[a] - r) hold = 1;  /* FIXED frame of the global grid */
        if (ii[a] < r || ii[a] >= W->len[a] - r) hold = 1;  /* window edge (or frame) */
      } else if (!W->full[a]) {
        if (ii[a] < r || ii[a] >= W->len[a] - r) hold = 1;  /* artificial window edge */
      }
    }
    if (hold) {
      out[p] = in[p];
      continue;
    }
    double s = 0.0;
    for (int a = -r0; a <= r0; ++a) {
      int64_t j0 = i0 + a;
      if (j0 < 0) j0 += L0; else if (j0 >= L0) j0 -= L0;   /* only reachable on a full periodic axis */
      for (int b = -r1; b <= r1; ++b) {
        int64_t j1 = i1 + b;
        if (j1 < 0) j1 += L1; else if (j1 >= L1) j1 -= L1;
        for (int c = -r2; c <= r2; ++c) {
          const double wt = w[((a + r0) * n1 + (b + r1)) * n2 + (c + r2)];
          if (wt == 0.0) continue;
          int64_t j2 = i2 + c;
          if (j2 < 0) j2 += L2; else if (j2 >= L2) j2 -= L2;
          s += wt * in[(j0 * L1 + j1) * L2 + j2];
        }
      }
    }
    out[p] = s;
  }
}

static int normalise(int ndim, const int64_t* extents, int radius, window_t* W) {
  if (ndim < 1 || ndim > 3 || radius < 0) return -1;
  for (int a = 0; a < 3; ++a) {
    const int k = a - (3 - ndim);
    W->E[a] = k >= 0 ? extents[k] : 1;
    if (W->E[a] < 1) return -1;
    W->rad[a] = k >= 0 ? radius : 0;
    W->lo[a] = 0;
    W->len[a] = W->E[a];
    W->full[a] = 1;
    if (k >= 0 && W->E[a] < 2 * radius + 1) return -1;
  }
  return 0;
}

static double now_s(void) {
  struct timespec ts;
  clock_gettime(CLOCK_MONOTONIC, &ts);
  return ts.tv_sec + 1e-9 * ts.tv_nsec;
}

/* Run T base steps on the whole grid.  extents[0] is the slowest axis (C order).  weights is
 * the dense (2r+1)^ndim array, row-major over offsets -r..r.  u0 and out are grids of
 * prod(extents) doubles (may alias).  nthreads <= 0 keeps the OpenMP default.  If seconds
 * is non-NULL it receives the CLOCK_MONOTONIC time of the T-step loop alone.
 * Returns 0, or -1 on invalid arguments, -2 on allocation failure. */
int oracle_run(int ndim, const int64_t* extents, int radius, const double* weights, int bc,
               const double* u0, double* out, int64_t T, int nthreads, double* seconds) {
  window_t W;
  if (normalise(ndim, extents, radius, &W) != 0 || T < 0) return -1;
  if (bc != ORACLE_BC_FIXED && bc != ORACLE_BC_PERIODIC) return -1;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  const int64_t n = W.E[0] * W.E[1] * W.E[2];
  double* a = (double*)malloc(n * sizeof(double));
  double* b = (double*)malloc(n * sizeof(double));
  if (!a || !b) { free(a); free(b); return -2; }
  memcpy(a, u0, n * sizeof(double));
  const double t0 = now_s();
  for (int64_t t = 0; t < T; ++t) {
    step_window(&W, weights, bc, a, b);
    double* tmp = a; a = b; b = tmp;
  }
  const double t1 = now_s();
  if (seconds) *seconds = t1 - t0;
  memcpy(out, a, n * sizeof(double));
  free(a);
  free(b);
  return 0;
}

/* u_T at npts sampled points, each computed on its own dependence cone: the window of
 * half-width r*T around the point (clipped at FIXED faces, wrapped for PERIODIC, or the
 * whole axis when the cone covers it).  Errors from the window's artificial edges advance r
 * points per step, so after T steps the centre is exact.  pts is npts x ndim global
 * coordinates (extents[0] slowest).  Returns 0 or a negative error. */
int oracle_sample(int ndim, const int64_t* extents, int radius, const double* weights, int bc,
                  const double* u0, int64_t T, int64_t npts, const int64_t* pts, double* vals,
                  int nthreads) {
  window_t G;
  if (normalise(ndim, extents, radius, &G) != 0 || T < 0) return -1;
#ifdef _OPENMP
  if (nthreads > 0) omp_set_num_threads(nthreads);
#else
  (void)nthreads;
#endif
  const int64_t R = (int64_t)radius * T;
  for (int64_t k = 0; k < npts; ++k) {
    window_t W = G;
    int64_t c[3];
    for (int a = 0; a < 3; ++a) {
      const int q = a - (3 - ndim);
      c[a] = q >= 0 ? pts[k * ndim + q] : 0;
      if (c[a] < 0 || c[a] >= G.E[a]) return -1;
      if (G.rad[a] == 0 || 2 * R + 1 >= G.E[a]) {
        W.lo[a] = 0; W.len[a] = G.E[a]; W.full[a] = 1;
      } else if (bc == ORACLE_BC_FIXED) {
        const int64_t lo = c[a] - R < 0 ? 0 : c[a] - R;
        const int64_t hi = c[a] + R >= G.E[a] ? G.E[a] - 1 : c[a] + R;
        W.lo[a] = lo; W.len[a] = hi - lo + 1; W.full[a] = (lo == 0 && hi == G.E[a] - 1);
      } else {
        W.lo[a] = c[a] - R; W.len[a] = 2 * R + 1; W.full[a] = 0;
      }
    }
    const int64_t n = W.len[0] * W.len[1] * W.len[2];
    double* a = (double*)malloc(n * sizeof(double));
    double* b = (double*)malloc(n * sizeof(double));
    if (!a || !b) { free(a); free(b); return -2; }
    /* gather the window from the global grid */
    for (int64_t i0 = 0; i0 < W.len[0]; ++i0)
      for (int64_t i1 = 0; i1 < W.len[1]; ++i1)
        for (int64_t i2 = 0; i2 < W.len[2]; ++i2) {
          int64_t g0 = W.lo[0] + i0, g1 = W.lo[1] + i1, g2 = W.lo[2] + i2;
          g0 = ((g0 % G.E[0]) + G.E[0]) % G.E[0];
          g1 = ((g1 % G.E[1]) + G.E[1]) % G.E[1];
          g2 = ((g2 % G.E[2]) + G.E[2]) % G.E[2];
          a[(i0 * W.len[1] + i1) * W.len[2] + i2] = u0[(g0 * G.E[1] + g1) * G.E[2] + g2];
        }
    for (int64_t t = 0; t < T; ++t) {
      step_window(&W, weights, bc, a, b);
      double* tmp = a; a = b; b = tmp;
    }
    const int64_t l0 = c[0] - W.lo[0], l1 = c[1] - W.lo[1], l2 = c[2] - W.lo[2];
    vals[k] = a[(l0 * W.len[1] + l1) * W.len[2] + l2];
    free(a);
    free(b);
  }
  return 0;
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}
