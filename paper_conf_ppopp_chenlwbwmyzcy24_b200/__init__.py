"""Thin Python binding of libcsx.so — the B200-native ConvStencil hot path (include/csx.h).

Argument marshalling only: every step of the stencil sweep runs in the CUDA kernels of
``csrc/``.  Device grids are passed as torch CUDA float64 tensors (``data_ptr()``) and streams
as ``torch.cuda.Stream``; PyTorch is plumbing (memory, streams, process groups).  There is no
CPU fallback: if ``libcsx.so`` is missing, importing this package raises.

Function names mirror the C-ABI: ``csx_plan``, ``csx_run``, ``csx_run_host``,
``csx_run_sharded``, ``csx_comm_create`` ... ; ``Plan`` is a small owner object around them.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libcsx.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python -m paper_conf_ppopp_chenlwbwmyzcy24_b200.build` "
        "(there is no CPU fallback)")

_lib = ctypes.CDLL(LIB_PATH)

# ---- enums (csx.h) ---------------------------------------------------------------------
CSX_OK, CSX_ERR_INVALID_ARGUMENT, CSX_ERR_UNSUPPORTED, CSX_ERR_OUT_OF_MEMORY, CSX_ERR_CUDA, \
    CSX_ERR_NCCL, CSX_ERR_INTERNAL = range(7)
CSX_SHAPE_STAR, CSX_SHAPE_BOX = 0, 1
CSX_BC_FIXED, CSX_BC_PERIODIC = 0, 1
CSX_ENGINE_AUTO, CSX_ENGINE_TC_S2R, CSX_ENGINE_TC_TILE, CSX_ENGINE_DIRECT = 0, 1, 2, 3
ENGINES = {"auto": 0, "tc_s2r": 1, "tc_tile": 2, "direct": 3}
ENGINE_NAMES = {v: k for k, v in ENGINES.items()}

_i64p = ctypes.POINTER(ctypes.c_int64)
_dp = ctypes.POINTER(ctypes.c_double)
_i32p = ctypes.POINTER(ctypes.c_int32)
_vp = ctypes.c_void_p


class csx_plan_info_t(ctypes.Structure):
    _fields_ = [("ndim", ctypes.c_int), ("radius", ctypes.c_int), ("fuse_steps", ctypes.c_int),
                ("nk", ctypes.c_int), ("remainder_steps", ctypes.c_int), ("engine", ctypes.c_int),
                ("tile_m", ctypes.c_int), ("tile_n", ctypes.c_int), ("s2r_pitch", ctypes.c_int),
                ("mma_per_pass", ctypes.c_int64), ("tc_flops_per_point_step", ctypes.c_double),
                ("useful_flops_per_point_step", ctypes.c_double)]


def _sig(name, res, args):
    f = getattr(_lib, name)
    f.restype = res
    f.argtypes = args
    return f


_sig("csx_plan", ctypes.c_int, [ctypes.c_int, _i64p, ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int,
                                ctypes.c_int, ctypes.POINTER(_vp)])
_sig("csx_plan_set_engine", ctypes.c_int, [_vp, ctypes.c_int])
_sig("csx_auto_fuse_steps", ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int])
_sig("csx_plan_set_s2r_variant", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int])
_sig("csx_run", ctypes.c_int, [_vp, _vp, _vp, ctypes.c_int64, _vp])
_sig("csx_run_host", ctypes.c_int, [_vp, _dp, _dp, ctypes.c_int64, _vp])
_sig("csx_comm_create", ctypes.c_int, [ctypes.c_char_p, ctypes.c_int, ctypes.c_int, ctypes.POINTER(_vp)])
_sig("csx_comm_destroy", ctypes.c_int, [_vp])
_sig("csx_nccl_unique_id", ctypes.c_int, [ctypes.c_char_p])
_sig("csx_shard_rows", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int, _i64p, _i64p])
_sig("csx_run_sharded", ctypes.c_int, [_vp, _vp, _vp, _vp, ctypes.c_int64, _vp])
_sig("csx_peer_export", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int, ctypes.c_char_p])
_sig("csx_peer_connect", ctypes.c_int, [_vp, ctypes.c_char_p])
_sig("csx_run_sharded_peer", ctypes.c_int, [_vp, _vp, _vp, ctypes.c_int64, _vp])
_sig("csx_plan_destroy", ctypes.c_int, [_vp])
_sig("csx_status_string", ctypes.c_char_p, [ctypes.c_int])
_sig("csx_last_error", ctypes.c_char_p, [])
_sig("csx_plan_info", ctypes.c_int, [_vp, ctypes.POINTER(csx_plan_info_t)])
_sig("csx_compose_weights", ctypes.c_int, [ctypes.c_int, ctypes.c_int, _dp, ctypes.c_int, _dp])
_sig("csx_weight_matrices", ctypes.c_int, [ctypes.c_int, ctypes.c_int, _dp, _dp, _dp])
_sig("csx_stencil2row_index", ctypes.c_int, [ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                             ctypes.c_int64, _i64p, _i64p])
_sig("csx_fragment_bank_conflicts", ctypes.c_int, [ctypes.c_int, ctypes.c_int])
_sig("csx_plan_lut", ctypes.c_int, [_vp, _i32p, _i32p, _i64p, ctypes.POINTER(ctypes.c_int),
                                    ctypes.POINTER(ctypes.c_int)])

_sig("csx_profile_enable", ctypes.c_int, [_vp, ctypes.c_int])
_sig("csx_profile_read", ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_double), _i64p, _i64p, ctypes.c_int])
_sig("csx_host_last", ctypes.c_int, [_vp, ctypes.POINTER(ctypes.c_int), _i64p, _i64p])

_sig("csx_halo_schedule", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int, _i64p, ctypes.POINTER(ctypes.c_int)])
_sig("csx_plan_set_graph", ctypes.c_int, [_vp, ctypes.c_int])
_sig("csx_plan_set_max_ctas", ctypes.c_int, [_vp, ctypes.c_int])
_sig("csx_shard_box", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, _i64p, _i64p])
_sig("csx_pencil_schedule", ctypes.c_int, [_vp, ctypes.c_int, ctypes.c_int, ctypes.c_int, _i64p,
                                           ctypes.POINTER(ctypes.c_int)])
_sig("csx_run_sharded_pencil", ctypes.c_int, [_vp, _vp, ctypes.c_int, ctypes.c_int, _vp, _vp,
                                              ctypes.c_int64, _vp])

EXPORTED = ["csx_host_last", "csx_plan_set_graph", "csx_plan_set_max_ctas", "csx_shard_box", "csx_pencil_schedule", "csx_run_sharded_pencil", "csx_peer_export", "csx_peer_connect", "csx_run_sharded_peer", "csx_auto_fuse_steps", "csx_plan_set_s2r_variant", "csx_halo_schedule", "csx_profile_enable", "csx_profile_read", "csx_plan", "csx_plan_set_engine", "csx_run", "csx_run_host", "csx_comm_create",
            "csx_comm_destroy", "csx_nccl_unique_id", "csx_shard_rows", "csx_run_sharded",
            "csx_plan_destroy", "csx_status_string", "csx_last_error", "csx_plan_info",
            "csx_compose_weights", "csx_weight_matrices", "csx_stencil2row_index",
            "csx_fragment_bank_conflicts", "csx_plan_lut"]


class CsxError(RuntimeError):
    def __init__(self, status: int, where: str):
        self.status = status
        msg = _lib.csx_status_string(status).decode()
        detail = _lib.csx_last_error().decode()
        super().__init__(f"{where}: {msg}: {detail}")


def _check(status: int, where: str):
    if status != CSX_OK:
        raise CsxError(status, where)


def _dptr(a: np.ndarray):
    return a.ctypes.data_as(_dp)


def _stream_handle(stream):
    if stream is None:
        import torch
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(int(getattr(stream, "cuda_stream", stream)))


def _device_ptr(t, n: int, name: str):
    import torch
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{name} must be a torch.Tensor")
    if t.device.type != "cuda" or t.dtype != torch.float64 or not t.is_contiguous():
        raise ValueError(f"{name} must be a contiguous float64 CUDA tensor")
    if t.numel() != n:
        raise ValueError(f"{name} has {t.numel()} elements, expected {n}")
    return ctypes.c_void_p(t.data_ptr())


# ---- C-ABI mirrors ----------------------------------------------------------------------
def csx_plan(ndim: int, extents, shape: int, radius: int, weights, bc: int, fuse_steps: int = 0):
    ext = np.ascontiguousarray(extents, dtype=np.int64)
    w = np.ascontiguousarray(weights, dtype=np.float64).reshape(-1)
    h = _vp()
    _check(_lib.csx_plan(int(ndim), ext.ctypes.data_as(_i64p), int(shape), int(radius), _dptr(w),
                         int(bc), int(fuse_steps), ctypes.byref(h)), "csx_plan")
    return h


def csx_plan_set_engine(plan, engine: int):
    _check(_lib.csx_plan_set_engine(plan, int(engine)), "csx_plan_set_engine")


def csx_plan_set_s2r_variant(plan, padding=True, dirty_bits: bool = True):
    """padding: True/False, 2 for breakdown variant II (CUDA-core tessellation) or 3 for
    variant I (explicit stencil2row in global memory)."""
    pad = padding if (padding in (2, 3) and not isinstance(padding, bool)) else int(bool(padding))
    _check(_lib.csx_plan_set_s2r_variant(plan, pad, int(bool(dirty_bits))), "csx_plan_set_s2r_variant")


def csx_run(plan, d_in, d_out, timesteps: int, n: int, stream=None):
    _check(_lib.csx_run(plan, _device_ptr(d_in, n, "d_in"), _device_ptr(d_out, n, "d_out"),
                        int(timesteps), _stream_handle(stream)), "csx_run")


def csx_run_host(plan, h_in: np.ndarray, h_out: np.ndarray, timesteps: int, stream=None):
    if h_in.dtype != np.float64 or h_out.dtype != np.float64:
        raise ValueError("host grids must be float64")
    if not (h_in.flags.c_contiguous and h_out.flags.c_contiguous):
        raise ValueError("host grids must be C-contiguous")
    _check(_lib.csx_run_host(plan, _dptr(h_in), _dptr(h_out), int(timesteps), _stream_handle(stream)),
           "csx_run_host")


def csx_plan_destroy(plan):
    _check(_lib.csx_plan_destroy(plan), "csx_plan_destroy")


def csx_plan_info(plan) -> dict:
    info = csx_plan_info_t()
    _check(_lib.csx_plan_info(plan, ctypes.byref(info)), "csx_plan_info")
    d = {k: getattr(info, k) for k, _ in info._fields_}
    d["engine_name"] = ENGINE_NAMES.get(d["engine"], "?")
    return d


def csx_compose_weights(weights: np.ndarray, fuse_steps: int) -> np.ndarray:
    w = np.ascontiguousarray(weights, dtype=np.float64)
    ndim = w.ndim
    r = (w.shape[0] - 1) // 2
    n = 2 * r * fuse_steps + 1
    out = np.empty((n,) * ndim)
    _check(_lib.csx_compose_weights(ndim, r, _dptr(w), int(fuse_steps), _dptr(out)),
           "csx_compose_weights")
    return out


def csx_weight_matrices(w: np.ndarray):
    w = np.ascontiguousarray(w, dtype=np.float64)
    nk = w.shape[0]
    k = nk * nk if w.ndim == 2 else nk
    wa = np.empty((k, nk + 1))
    wb = np.empty((k, nk + 1))
    _check(_lib.csx_weight_matrices(nk, int(w.ndim == 1), _dptr(w), _dptr(wa), _dptr(wb)),
           "csx_weight_matrices")
    return wa, wb


def csx_stencil2row_index(nk: int, which: int, x: int, y: int):
    r = ctypes.c_int64()
    c = ctypes.c_int64()
    ok = _lib.csx_stencil2row_index(nk, which, x, y, ctypes.byref(r), ctypes.byref(c))
    return (r.value, c.value) if ok else None


def csx_fragment_bank_conflicts(pitch: int, col: int) -> int:
    return _lib.csx_fragment_bank_conflicts(int(pitch), int(col))


def csx_plan_lut(plan):
    n = ctypes.c_int64()
    rr = ctypes.c_int()
    rc = ctypes.c_int()
    _check(_lib.csx_plan_lut(plan, None, None, ctypes.byref(n), ctypes.byref(rr), ctypes.byref(rc)),
           "csx_plan_lut")
    a = np.empty(n.value, dtype=np.int32)
    b = np.empty(n.value, dtype=np.int32)
    _check(_lib.csx_plan_lut(plan, a.ctypes.data_as(_i32p), b.ctypes.data_as(_i32p), ctypes.byref(n),
                             None, None), "csx_plan_lut")
    return a.reshape(rr.value, rc.value), b.reshape(rr.value, rc.value)


def csx_profile_enable(plan, enable=True):
    """enable: False/0 off, True/1 time every main-pass TC launch, n > 1 every n-th."""
    _check(_lib.csx_profile_enable(plan, int(enable)), "csx_profile_enable")


def csx_profile_read(plan, reset: bool = True):
    """(summed TC kernel ms, TC launches, all kernel launches) since the last reset."""
    ms = ctypes.c_double()
    tc = ctypes.c_int64()
    tot = ctypes.c_int64()
    _check(_lib.csx_profile_read(plan, ctypes.byref(ms), ctypes.byref(tc), ctypes.byref(tot),
                                 int(bool(reset))), "csx_profile_read")
    return ms.value, tc.value, tot.value


def csx_host_last(plan):
    """(chunks, H2D bytes, D2H bytes) of the last csx_run_host on `plan`."""
    k = ctypes.c_int()
    hi = ctypes.c_int64()
    ho = ctypes.c_int64()
    _check(_lib.csx_host_last(plan, ctypes.byref(k), ctypes.byref(hi), ctypes.byref(ho)), "csx_host_last")
    return k.value, hi.value, ho.value


def csx_nccl_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(_lib.csx_nccl_unique_id(buf), "csx_nccl_unique_id")
    return buf.raw


def csx_comm_create(unique_id: bytes, rank: int, nranks: int):
    h = _vp()
    _check(_lib.csx_comm_create(unique_id, int(rank), int(nranks), ctypes.byref(h)), "csx_comm_create")
    return h


def csx_comm_destroy(comm):
    _check(_lib.csx_comm_destroy(comm), "csx_comm_destroy")


def csx_shard_rows(plan, rank: int, nranks: int):
    lo = ctypes.c_int64()
    hi = ctypes.c_int64()
    _check(_lib.csx_shard_rows(plan, rank, nranks, ctypes.byref(lo), ctypes.byref(hi)), "csx_shard_rows")
    return lo.value, hi.value


def csx_halo_schedule(plan, rank: int, nranks: int):
    """[(kind 'send'|'recv', peer, first_row, nrows), ...] in posting order."""
    ops = np.zeros(16, dtype=np.int64)
    n = ctypes.c_int()
    _check(_lib.csx_halo_schedule(plan, rank, nranks, ops.ctypes.data_as(_i64p), ctypes.byref(n)),
           "csx_halo_schedule")
    return [("send" if ops[4 * k] == 0 else "recv", int(ops[4 * k + 1]), int(ops[4 * k + 2]),
             int(ops[4 * k + 3])) for k in range(n.value)]


def csx_run_sharded(plan, comm, d_in, d_out, timesteps: int, n_local: int, stream=None):
    _check(_lib.csx_run_sharded(plan, comm, _device_ptr(d_in, n_local, "d_in"),
                                _device_ptr(d_out, n_local, "d_out"), int(timesteps),
                                _stream_handle(stream)), "csx_run_sharded")


def csx_shard_box(plan, rank: int, p0: int, p1: int):
    """([lo per axis], [hi per axis]) of rank's block on the p0 x p1 process grid."""
    lo = np.zeros(3, dtype=np.int64)
    hi = np.zeros(3, dtype=np.int64)
    _check(_lib.csx_shard_box(plan, rank, p0, p1, lo.ctypes.data_as(_i64p), hi.ctypes.data_as(_i64p)),
           "csx_shard_box")
    nd = int(csx_plan_info(plan)["ndim"])
    return [int(v) for v in lo[:nd]], [int(v) for v in hi[:nd]]


def csx_pencil_schedule(plan, rank: int, p0: int, p1: int):
    """[(phase 0 (second split axis) | 1 (first split axis), 'send'|'recv', peer, first_row,
    nrows), ...] in posting order."""
    ops = np.zeros(40, dtype=np.int64)
    n = ctypes.c_int()
    _check(_lib.csx_pencil_schedule(plan, rank, p0, p1, ops.ctypes.data_as(_i64p), ctypes.byref(n)),
           "csx_pencil_schedule")
    return [(int(ops[5 * k]), "send" if ops[5 * k + 1] == 0 else "recv", int(ops[5 * k + 2]),
             int(ops[5 * k + 3]), int(ops[5 * k + 4])) for k in range(n.value)]


def csx_run_sharded_pencil(plan, comm, p0: int, p1: int, d_in, d_out, timesteps: int, n_local: int,
                           stream=None):
    _check(_lib.csx_run_sharded_pencil(plan, comm, int(p0), int(p1), _device_ptr(d_in, n_local, "d_in"),
                                       _device_ptr(d_out, n_local, "d_out"), int(timesteps),
                                       _stream_handle(stream)), "csx_run_sharded_pencil")


CSX_PEER_DESC_BYTES = 512


def csx_peer_export(plan, rank: int, nranks: int) -> bytes:
    buf = ctypes.create_string_buffer(CSX_PEER_DESC_BYTES)
    _check(_lib.csx_peer_export(plan, int(rank), int(nranks), buf), "csx_peer_export")
    return buf.raw


def csx_peer_connect(plan, descs):
    blob = b"".join(descs)
    if any(len(d) != CSX_PEER_DESC_BYTES for d in descs):
        raise ValueError("peer descriptors must be CSX_PEER_DESC_BYTES each")
    _check(_lib.csx_peer_connect(plan, blob), "csx_peer_connect")


def csx_run_sharded_peer(plan, d_in, d_out, timesteps: int, n_local: int, stream=None):
    _check(_lib.csx_run_sharded_peer(plan, _device_ptr(d_in, n_local, "d_in"),
                                     _device_ptr(d_out, n_local, "d_out"), int(timesteps),
                                     _stream_handle(stream)), "csx_run_sharded_peer")


# ---- owner object ------------------------------------------------------------------------
class Plan:
    """Owns a csx plan.  ``weights`` is the dense (2r+1)^ndim array (correlation orientation)."""

    def __init__(self, extents, weights, shape: str = "box", bc: str = "periodic",
                 fuse_steps: int = 0, engine: str = "auto"):
        w = np.asarray(weights, dtype=np.float64)
        self.extents = tuple(int(e) for e in extents)
        self.ndim = len(self.extents)
        if w.ndim != self.ndim:
            raise ValueError("weights must have one axis per grid axis")
        self.radius = (w.shape[0] - 1) // 2
        self.n = int(np.prod(self.extents))
        if fuse_steps == 0 and engine in ("tc_s2r", "direct"):
            # the automatic depth for the requested engine (TC_S2R 1D keeps nk + 1 <= 16)
            fuse_steps = int(_lib.csx_auto_fuse_steps(self.ndim, self.radius, ENGINES[engine]))
        self._h = csx_plan(self.ndim, self.extents, CSX_SHAPE_BOX if shape == "box" else CSX_SHAPE_STAR,
                           self.radius, w, CSX_BC_FIXED if bc == "fixed" else CSX_BC_PERIODIC,
                           fuse_steps)
        if engine != "auto":
            csx_plan_set_engine(self._h, ENGINES[engine])

    @property
    def handle(self):
        return self._h

    def set_s2r_variant(self, padding=True, dirty_bits: bool = True):
        csx_plan_set_s2r_variant(self._h, padding, dirty_bits)

    def set_engine(self, engine: str):
        csx_plan_set_engine(self._h, ENGINES[engine])

    def info(self) -> dict:
        return csx_plan_info(self._h)

    def run(self, d_in, d_out, timesteps: int, stream=None):
        csx_run(self._h, d_in, d_out, timesteps, self.n, stream)

    def run_host(self, h_in: np.ndarray, timesteps: int, h_out: np.ndarray | None = None, stream=None):
        h_in = np.ascontiguousarray(h_in, dtype=np.float64)
        if h_out is None:
            h_out = np.empty_like(h_in)
        csx_run_host(self._h, h_in, h_out, timesteps, stream)
        return h_out

    def host_last(self):
        """(chunks, H2D bytes, D2H bytes) of the last run_host."""
        return csx_host_last(self._h)

    def shard_rows(self, rank: int, nranks: int):
        return csx_shard_rows(self._h, rank, nranks)

    def run_sharded(self, comm, d_in, d_out, timesteps: int, n_local: int, stream=None):
        csx_run_sharded(self._h, comm, d_in, d_out, timesteps, n_local, stream)

    def peer_setup(self, rank: int, nranks: int, all_gather=None):
        """Bootstrap the NVLink peer-memory halo exchange: export this rank's descriptor,
        all-gather them (default: torch.distributed.all_gather_object on the default group)
        and connect to the neighbours."""
        desc = csx_peer_export(self._h, rank, nranks)
        if nranks == 1:
            descs = [desc]
        elif all_gather is not None:
            descs = all_gather(desc)
        else:
            import torch.distributed as dist
            descs = [None] * nranks
            dist.all_gather_object(descs, desc)
        csx_peer_connect(self._h, descs)

    def run_sharded_peer(self, d_in, d_out, timesteps: int, n_local: int, stream=None):
        csx_run_sharded_peer(self._h, d_in, d_out, timesteps, n_local, stream)

    def halo_schedule(self, rank: int, nranks: int):
        return csx_halo_schedule(self._h, rank, nranks)

    def set_graph(self, on: bool = True):
        """CUDA-graph replay of run() for repeated (d_in, d_out, T) (csx_plan_set_graph)."""
        _check(_lib.csx_plan_set_graph(self._h, int(bool(on))), "csx_plan_set_graph")

    def set_max_ctas(self, max_ctas: int):
        """Cap every persistent grid the plan launches (0 = occupancy x SMs;
        csx_plan_set_max_ctas).  Results do not depend on it."""
        _check(_lib.csx_plan_set_max_ctas(self._h, int(max_ctas)), "csx_plan_set_max_ctas")

    def shard_box(self, rank: int, p0: int, p1: int):
        return csx_shard_box(self._h, rank, p0, p1)

    def pencil_schedule(self, rank: int, p0: int, p1: int):
        return csx_pencil_schedule(self._h, rank, p0, p1)

    def run_sharded_pencil(self, comm, p0: int, p1: int, d_in, d_out, timesteps: int, n_local: int,
                           stream=None):
        csx_run_sharded_pencil(self._h, comm, p0, p1, d_in, d_out, timesteps, n_local, stream)

    def lut(self):
        return csx_plan_lut(self._h)

    def close(self):
        if self._h:
            csx_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
