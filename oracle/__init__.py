"""CPU oracle for the csx hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` and
``--impl reference`` legs) may import this package.  It shares no code with the CUDA path
(``paper_conf_ppopp_chenlwbwmyzcy24_b200``) and never imports it.

* ``run``       — T plain base steps of the direct weighted sum (oracle.c, PAPER.md P.146-149,
                  P.277-287), FIXED or PERIODIC boundary (reading A1).
* ``sample``    — u_T at chosen points, each from its own dependence cone (oracle.c).
* ``brute``     — an independent formulation: the step as a dense matrix, applied T times
                  (numpy; tiny grids only).  Used to pin ``run``.

Pinned in tests/test_oracle.py; no function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import time

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")

FIXED, PERIODIC = 0, 1
_BC = {"fixed": FIXED, "periodic": PERIODIC, FIXED: FIXED, PERIODIC: PERIODIC}


def build(force: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (plain C, -O2 -ffp-contract=off, OpenMP)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fopenmp", "-fPIC", "-shared",
                               "-std=c99", "-D_POSIX_C_SOURCE=199309L", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


_lib = None


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i64p = ctypes.POINTER(ctypes.c_int64)
        dp = ctypes.POINTER(ctypes.c_double)
        lib.oracle_run.argtypes = [ctypes.c_int, i64p, ctypes.c_int, dp, ctypes.c_int, dp, dp,
                                   ctypes.c_int64, ctypes.c_int, dp]
        lib.oracle_run.restype = ctypes.c_int
        lib.oracle_sample.argtypes = [ctypes.c_int, i64p, ctypes.c_int, dp, ctypes.c_int, dp,
                                      ctypes.c_int64, ctypes.c_int64, i64p, dp, ctypes.c_int]
        lib.oracle_sample.restype = ctypes.c_int
        lib.oracle_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _i64p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def _radius_of(weights: np.ndarray) -> int:
    n = weights.shape[0]
    if n % 2 != 1 or any(s != n for s in weights.shape):
        raise ValueError("weights must be (2r+1)^ndim")
    return (n - 1) // 2


def max_threads() -> int:
    return _load().oracle_max_threads()


def run(u0: np.ndarray, weights: np.ndarray, bc, T: int, nthreads: int = 0,
        return_seconds: bool = False):
    """u_T after T base steps (float64, same shape as u0)."""
    lib = _load()
    u0 = np.ascontiguousarray(u0, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float64)
    if w.ndim != u0.ndim:
        raise ValueError("weights and grid dimensionality differ")
    ext = np.array(u0.shape, dtype=np.int64)
    out = np.empty_like(u0)
    secs = ctypes.c_double(0.0)
    rc = lib.oracle_run(u0.ndim, _i64p(ext), _radius_of(w), _dp(w), _BC[bc], _dp(u0), _dp(out),
                        int(T), int(nthreads), ctypes.byref(secs))
    if rc != 0:
        raise ValueError(f"oracle_run failed ({rc})")
    return (out, secs.value) if return_seconds else out


def sample(u0: np.ndarray, weights: np.ndarray, bc, T: int, points, nthreads: int = 0):
    """u_T at each of ``points`` (k x ndim global coordinates), via its dependence cone."""
    lib = _load()
    u0 = np.ascontiguousarray(u0, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float64)
    pts = np.ascontiguousarray(np.asarray(points, dtype=np.int64).reshape(-1, u0.ndim))
    ext = np.array(u0.shape, dtype=np.int64)
    vals = np.empty(pts.shape[0], dtype=np.float64)
    rc = lib.oracle_sample(u0.ndim, _i64p(ext), _radius_of(w), _dp(w), _BC[bc], _dp(u0), int(T),
                           pts.shape[0], _i64p(pts), _dp(vals), int(nthreads))
    if rc != 0:
        raise ValueError(f"oracle_sample failed ({rc})")
    return vals


def brute_matrix(shape, weights: np.ndarray, bc) -> np.ndarray:
    """The one-step operator as a dense matrix M (u_{t+1} = M @ u_t), built entry by entry:
    M[p, q] += w[o] for q = p + o (wrapped for PERIODIC); identity rows for FIXED-frame
    points (P.146-149; reading A1).  Tiny grids only."""
    shape = tuple(int(s) for s in shape)
    r = _radius_of(weights)
    n = int(np.prod(shape))
    M = np.zeros((n, n))
    offsets = list(np.ndindex(*weights.shape))
    for p in np.ndindex(*shape):
        ip = np.ravel_multi_index(p, shape)
        if _BC[bc] == FIXED and any(c < r or c >= s - r for c, s in zip(p, shape)):
            M[ip, ip] = 1.0
            continue
        for o in offsets:
            wt = weights[o]
            if wt == 0.0:
                continue
            q = tuple((c + oi - r) % s for c, oi, s in zip(p, o, shape))
            M[ip, np.ravel_multi_index(q, shape)] += wt
    return M


def brute(u0: np.ndarray, weights: np.ndarray, bc, T: int) -> np.ndarray:
    """u_T = M^T u_0 by repeated dense mat-vec."""
    M = brute_matrix(u0.shape, weights, bc)
    v = u0.reshape(-1).astype(np.float64)
    for _ in range(T):
        v = M @ v
    return v.reshape(u0.shape)


def timed_run(u0, weights, bc, T, nthreads=0):
    """(u_T, seconds of the T-step loop measured inside oracle.c, wall seconds)."""
    t0 = time.perf_counter()
    out, secs = run(u0, weights, bc, T, nthreads=nthreads, return_seconds=True)
    return out, secs, time.perf_counter() - t0
