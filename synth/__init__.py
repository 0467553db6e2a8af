"""Seeded synthetic inputs shared by the oracle tests, the CUDA parity tests and bench.py.

This module holds NONE of the method's arithmetic: it only draws numbers and names the
stencil shapes of the paper's benchmark table (Table 4, P.1841-1859; Table 3
P.888-898 for Star-2D9P / Box-2D25P).  Both sides of every parity check (``oracle/`` and
the CUDA path in ``paper_conf_ppopp_chenlwbwmyzcy24_b200``) receive the arrays built here;
neither side imports the other.

Input recipe: u0[i] = (splitmix64(seed XOR i) >> 11) * 2**-53 in [0, 1),
i = row-major flat index into the GLOBAL grid, seed = 20240302.  Weights come in two
families: the dyadic "physical" set (exact in binary, sums to 1) and seeded random
asymmetric positive weights normalised to sum 1 (asymmetric so a flipped kernel cannot
pass, reading A3).
"""
from __future__ import annotations

from dataclasses import dataclass
from math import comb

import numpy as np

SEED = 20240302

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64(x: np.ndarray) -> np.ndarray:
    """Vigna's splitmix64 finaliser applied to each uint64 of ``x`` (wrapping arithmetic)."""
    with np.errstate(over="ignore"):
        z = (x.astype(np.uint64) + _GOLDEN) & _M64
        z = ((z ^ (z >> np.uint64(30))) * _C1) & _M64
        z = ((z ^ (z >> np.uint64(27))) * _C2) & _M64
        return z ^ (z >> np.uint64(31))


def uniform01(seed: int, start: int, count: int) -> np.ndarray:
    """float64 values (splitmix64(seed ^ i) >> 11) * 2^-53 for i in [start, start+count)."""
    out = np.empty(count, dtype=np.float64)
    chunk = 1 << 24
    s = np.uint64(seed)
    for lo in range(0, count, chunk):
        n = min(chunk, count - lo)
        idx = np.arange(start + lo, start + lo + n, dtype=np.uint64)
        out[lo:lo + n] = (splitmix64(idx ^ s) >> np.uint64(11)).astype(np.float64) * (2.0 ** -53)
    return out


def grid(extents, seed: int = SEED, rows: tuple[int, int] | None = None) -> np.ndarray:
    """The seeded initial grid u0 (C order, extents[0] slowest).

    ``rows=(lo, hi)`` returns only the slab of slowest-axis rows [lo, hi) of the same global
    grid (what one rank of a slab-sharded run owns), with identical values.
    """
    extents = tuple(int(e) for e in extents)
    inner = int(np.prod(extents[1:], dtype=np.int64)) if len(extents) > 1 else 1
    lo, hi = (0, extents[0]) if rows is None else rows
    vals = uniform01(seed, lo * inner, (hi - lo) * inner)
    return vals.reshape((hi - lo,) + extents[1:])


def grid_window(extents, lo, hi, seed: int = SEED) -> np.ndarray:
    """The box [lo, hi) (one bound per axis, clipped to the grid by the caller) of the same
    global grid as ``grid(extents)``, without building the whole grid."""
    extents = tuple(int(e) for e in extents)
    lo = tuple(int(v) for v in lo)
    hi = tuple(int(v) for v in hi)
    shape = tuple(h - l for l, h in zip(lo, hi))
    out = np.empty(shape, dtype=np.float64)
    strides = [int(np.prod(extents[a + 1:], dtype=np.int64)) for a in range(len(extents))]
    for idx in np.ndindex(*shape[:-1]):
        base = sum((lo[a] + idx[a]) * strides[a] for a in range(len(idx)))
        out[idx] = uniform01(seed, base + lo[-1], shape[-1])
    return out


def grid_torch(extents, device, seed: int = SEED, chunk: int = 1 << 26):
    """``grid(extents)`` generated on a torch device (same values, bit for bit): for grids too
    large to build on the host (the maximum-size parity test).  int64 arithmetic wraps like the
    uint64 reference; right shifts are made logical with a mask."""
    import torch
    extents = tuple(int(e) for e in extents)
    n = int(np.prod(extents, dtype=np.int64))
    s64 = lambda v: v - (1 << 64) if v >= 1 << 63 else v  # noqa: E731
    g, c1, c2 = s64(0x9E3779B97F4A7C15), s64(0xBF58476D1CE4E5B9), s64(0x94D049BB133111EB)
    shr = lambda z, k: (z >> k) & ((1 << (64 - k)) - 1)  # noqa: E731
    out = torch.empty(n, dtype=torch.float64, device=device)
    for lo in range(0, n, chunk):
        m = min(chunk, n - lo)
        z = torch.arange(lo, lo + m, dtype=torch.int64, device=device) ^ seed
        z = z + g
        z = (z ^ shr(z, 30)) * c1
        z = (z ^ shr(z, 27)) * c2
        z = z ^ shr(z, 31)
        out[lo:lo + m] = shr(z, 11).to(torch.float64) * (2.0 ** -53)
    return out.view(extents)


@dataclass(frozen=True)
class Shape:
    """One benchmark stencil: name, dimension, radius, star/box footprint."""
    name: str
    ndim: int
    radius: int
    kind: str  # "star" | "box"
    shape_id: int

    @property
    def points(self) -> int:
        return int(self.footprint().sum())

    def footprint(self) -> np.ndarray:
        """Boolean (2r+1)^d mask of taps the shape may use (star = axial only, P.278-283)."""
        n = 2 * self.radius + 1
        if self.kind == "box" or self.ndim == 1:
            return np.ones((n,) * self.ndim, dtype=bool)
        m = np.zeros((n,) * self.ndim, dtype=bool)
        c = self.radius
        for ax in range(self.ndim):
            idx = [c] * self.ndim
            for k in range(n):
                idx[ax] = k
                m[tuple(idx)] = True
        return m


# Table 4 (P.1848-1859) plus the two extra Table 3 shapes (P.888-898).
SHAPES = {
    s.name: s
    for s in [
        Shape("heat1d", 1, 1, "star", 1),
        Shape("1d5p", 1, 2, "star", 2),
        Shape("heat2d", 2, 1, "star", 3),
        Shape("box2d9p", 2, 1, "box", 4),
        Shape("star2d13p", 2, 3, "star", 5),
        Shape("box2d49p", 2, 3, "box", 6),
        Shape("heat3d", 3, 1, "star", 7),
        Shape("box3d27p", 3, 1, "box", 8),
        Shape("star2d9p", 2, 2, "star", 9),
        Shape("box2d25p", 2, 2, "box", 10),
        # general radius in 3D (r <= 3 in every dimension; the paper's 3D
        # method is a sum of per-plane 2D ConvStencils for any plane window, P.1788-1800)
        Shape("star3d13p", 3, 2, "star", 11),
        Shape("box3d125p", 3, 2, "box", 12),
        Shape("star3d19p", 3, 3, "star", 13),
        Shape("box3d343p", 3, 3, "box", 14),
    ]
}


def _binomial(n: int) -> np.ndarray:
    return np.array([comb(n, k) for k in range(n + 1)], dtype=np.float64)


def physical_weights(name: str) -> np.ndarray:
    """Dyadic weights summing exactly to 1 (SURVEY.md §8(d) "Weights", family 1)."""
    s = SHAPES[name]
    n = 2 * s.radius + 1
    c = s.radius
    if s.kind == "box" or s.ndim == 1:
        b = _binomial(n - 1)
        w = b
        for _ in range(s.ndim - 1):
            w = np.multiply.outer(w, b)
        return w / w.sum()
    w = np.zeros((n,) * s.ndim)
    if name == "heat2d":
        centre, arms = 0.5, [0.125]
    elif name == "star2d13p":
        centre, arms = 0.5, [1 / 16, 1 / 32, 1 / 32]
    elif name == "star2d9p":
        centre, arms = 0.5, [1 / 16, 1 / 16]
    elif name == "heat3d":
        centre, arms = 0.625, [0.0625]
    elif name == "star3d13p":
        centre, arms = 0.25, [1 / 16, 1 / 16]
    elif name == "star3d19p":
        centre, arms = 0.25, [1 / 16, 1 / 32, 1 / 32]
    else:
        raise KeyError(name)
    w[(c,) * s.ndim] = centre
    for ax in range(s.ndim):
        for d, a in enumerate(arms, start=1):
            for sgn in (-1, 1):
                idx = [c] * s.ndim
                idx[ax] = c + sgn * d
                w[tuple(idx)] = a
    assert abs(w.sum() - 1.0) == 0.0
    return w


def random_weights(name: str, seed: int = SEED) -> np.ndarray:
    """Seeded asymmetric positive weights on the shape's footprint, normalised to sum 1."""
    s = SHAPES[name]
    fp = s.footprint()
    vals = uniform01(seed + s.shape_id * 1000003, 0, fp.size).reshape(fp.shape)
    w = np.where(fp, 0.05 + vals, 0.0)
    return w / w.sum()


def random_signed_weights(ndim: int, radius: int, seed: int = SEED, box: bool = True) -> np.ndarray:
    """Seeded weights of mixed sign (not normalised) for general-r parity cases."""
    n = 2 * radius + 1
    vals = uniform01(seed + 7919 * (ndim * 10 + radius), 0, n ** ndim).reshape((n,) * ndim)
    w = (vals - 0.5) / (0.5 * n ** ndim)
    if not box:
        w = np.where(Shape("x", ndim, radius, "star", 0).footprint(), w, 0.0)
    return w
