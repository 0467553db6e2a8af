"""Pins for the CPU oracle (oracle/), checked against things other than itself.

Each pin is chosen so that a plausible mistake in oracle.c (a dropped tap, a flipped offset
= convolution instead of correlation, a transposed axis, a wrong wrap, a wrong FIXED frame)
fails at least one of them:

* dense-matrix brute force (oracle.brute — an independent formulation)  [P.146-149]
* scipy.ndimage.correlate(mode="wrap") — a library routine that IS one periodic step
* pure-shift stencils -> np.roll (exact, catches orientation/axis errors; reading A3)
* constant field invariant for weights summing to 1 (bit-exact with dyadic data)
* closed-form Fourier-mode decay for Heat-1D/2D/3D and centro-symmetric boxes
* linear data is a fixed point of FIXED-boundary heat (discrete Laplacian of a line = 0)
* oracle.sample (dependence cone) equals the full run bit for bit
"""
import numpy as np
import pytest
import scipy.ndimage as ndi

import oracle
import synth

RNG = np.random.default_rng(12345)


def rel_err(a, b):
    return float(np.max(np.abs(a - b)) / max(np.max(np.abs(b)), 1e-300))


CASES = [
    ((41,), 1), ((41,), 2), ((41,), 3),
    ((11, 13), 1), ((11, 13), 2), ((9, 10), 3),
    ((7, 8, 9), 1), ((6, 5, 7), 2),
]


@pytest.mark.parametrize("shape,r", CASES)
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("box", [True, False])
def test_brute_force(shape, r, bc, box):
    """oracle.run == dense-matrix power on tiny grids, asymmetric signed weights."""
    if min(shape) < 2 * r + 1:
        pytest.skip("grid smaller than the window")
    w = synth.random_signed_weights(len(shape), r, seed=77 + r, box=box)
    u0 = synth.grid(shape, seed=99)
    T = 5
    got = oracle.run(u0, w, bc, T)
    ref = oracle.brute(u0, w, bc, T)
    assert rel_err(got, ref) <= 1e-14


@pytest.mark.parametrize("name", list(synth.SHAPES))
def test_scipy_correlate_periodic(name):
    """One PERIODIC step is scipy.ndimage.correlate(mode='wrap'); T steps likewise."""
    s = synth.SHAPES[name]
    shape = {1: (97,), 2: (23, 31), 3: (11, 12, 13)}[s.ndim]
    w = synth.random_weights(name)
    u0 = synth.grid(shape)
    ref = u0.copy()
    for _ in range(4):
        ref = ndi.correlate(ref, w, mode="wrap")
    got = oracle.run(u0, w, "periodic", 4)
    assert rel_err(got, ref) <= 1e-14


@pytest.mark.parametrize("name", list(synth.SHAPES))
def test_scipy_correlate_fixed(name):
    """FIXED: interior = correlate, frame of width r restored to the previous values."""
    s = synth.SHAPES[name]
    r = s.radius
    shape = {1: (97,), 2: (23, 31), 3: (11, 12, 13)}[s.ndim]
    w = synth.random_weights(name)
    u0 = synth.grid(shape)
    ref = u0.copy()
    inner = tuple(slice(r, n - r) for n in shape)
    for _ in range(3):
        nxt = ref.copy()
        nxt[inner] = ndi.correlate(ref, w, mode="wrap")[inner]
        ref = nxt
    got = oracle.run(u0, w, "fixed", 3)
    assert rel_err(got, ref) <= 1e-14


@pytest.mark.parametrize("ndim", [1, 2, 3])
def test_pure_shift_is_roll(ndim):
    """w = unit tap at offset o: u_T[p] = u0[p + T*o] exactly (correlation orientation)."""
    r = 2
    shape = {1: (53,), 2: (17, 19), 3: (9, 10, 11)}[ndim]
    u0 = synth.grid(shape, seed=5)
    for trial in range(6):
        o = tuple(int(v) for v in RNG.integers(-r, r + 1, size=ndim))
        w = np.zeros((2 * r + 1,) * ndim)
        w[tuple(x + r for x in o)] = 1.0
        T = 3
        got = oracle.run(u0, w, "periodic", T)
        ref = np.roll(u0, shift=tuple(-T * x for x in o), axis=tuple(range(ndim)))
        assert np.array_equal(got, ref), (o,)


@pytest.mark.parametrize("name", list(synth.SHAPES))
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_constant_field(name, bc):
    """Weights summing to 1 keep a constant field constant; bit-exact for dyadic data."""
    s = synth.SHAPES[name]
    shape = {1: (64,), 2: (20, 24), 3: (10, 11, 12)}[s.ndim]
    c = 0.375
    u0 = np.full(shape, c)
    got = oracle.run(u0, synth.physical_weights(name), bc, 7)
    assert np.all(got == c)


def _heat_lambda(alpha, ks, ns):
    return 1.0 - 4.0 * alpha * sum(np.sin(np.pi * k / n) ** 2 for k, n in zip(ks, ns))


@pytest.mark.parametrize("name,alpha", [("heat1d", 0.25), ("heat2d", 0.125), ("heat3d", 0.0625)])
def test_fourier_decay_heat(name, alpha):
    """Heat on a torus: u0 = cos(2 pi k.p/N) decays as lambda^T, lambda = 1 - 4a sum sin^2(pi k/N)."""
    s = synth.SHAPES[name]
    shape = {1: (64,), 2: (32, 40), 3: (16, 12, 20)}[s.ndim]
    ks = {1: (3,), 2: (2, 5), 3: (1, 2, 3)}[s.ndim]
    grids = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    phase = sum(2 * np.pi * k * g / n for k, g, n in zip(ks, grids, shape))
    u0 = np.cos(phase)
    T = 40
    got = oracle.run(u0, synth.physical_weights(name), "periodic", T)
    ref = _heat_lambda(alpha, ks, shape) ** T * u0
    assert np.max(np.abs(got - ref)) <= 1e-14


@pytest.mark.parametrize("name", ["box2d9p", "box2d49p", "box3d27p", "1d5p", "star2d13p", "box3d125p",
                                  "star3d19p"])
def test_fourier_decay_symbol(name):
    """Centro-symmetric w: lambda(k) = sum_o w_o cos(2 pi k.o/N) (the stencil's symbol)."""
    s = synth.SHAPES[name]
    w = synth.physical_weights(name)
    r = s.radius
    shape = {1: (60,), 2: (28, 36), 3: (14, 16, 18)}[s.ndim]
    ks = {1: (4,), 2: (3, 2), 3: (1, 3, 2)}[s.ndim]
    lam = 0.0
    for o in np.ndindex(*w.shape):
        lam += w[o] * np.cos(sum(2 * np.pi * k * (oi - r) / n for k, oi, n in zip(ks, o, shape)))
    grids = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
    u0 = np.cos(sum(2 * np.pi * k * g / n for k, g, n in zip(ks, grids, shape)))
    T = 25
    got = oracle.run(u0, w, "periodic", T)
    assert np.max(np.abs(got - lam ** T * u0)) <= 1e-14


def test_fixed_linear_fixed_point():
    """FIXED heat keeps linear data exactly (dyadic slope/intercept): a closed-form steady state."""
    for name, shape in [("heat1d", (64,)), ("heat2d", (24, 32)), ("heat3d", (10, 12, 14))]:
        grids = np.meshgrid(*[np.arange(n) for n in shape], indexing="ij")
        u0 = 0.5 + sum((d + 1) * 2.0 ** -8 * g for d, g in enumerate(grids))
        got = oracle.run(u0, synth.physical_weights(name), "fixed", 30)
        assert np.array_equal(got, u0)


def test_fixed_frame_held():
    """FIXED: the frame of width r never changes, whatever the weights."""
    w = synth.random_weights("box2d49p")
    u0 = synth.grid((20, 22), seed=3)
    got = oracle.run(u0, w, "fixed", 6)
    r = 3
    frame = np.ones_like(u0, dtype=bool)
    frame[r:-r, r:-r] = False
    assert np.array_equal(got[frame], u0[frame])
    assert not np.array_equal(got[~frame], u0[~frame])


def test_T0_identity():
    u0 = synth.grid((13, 17))
    assert np.array_equal(oracle.run(u0, synth.physical_weights("box2d9p"), "fixed", 0), u0)


@pytest.mark.parametrize("ndim,shape,r,T", [
    (1, (200,), 2, 9), (2, (40, 50), 1, 7), (2, (40, 50), 3, 4), (3, (18, 19, 20), 1, 4),
    (2, (12, 13), 1, 20),  # cone covers the whole grid
])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_sample_matches_run(ndim, shape, r, T, bc):
    """oracle.sample (window = dependence cone) == oracle.run at the same points, bit for bit."""
    w = synth.random_signed_weights(ndim, r, seed=11)
    u0 = synth.grid(shape, seed=21)
    full = oracle.run(u0, w, bc, T)
    pts = [tuple(int(RNG.integers(0, n)) for n in shape) for _ in range(12)]
    pts += [tuple(0 for _ in shape), tuple(n - 1 for n in shape), tuple(r for _ in shape)]
    vals = oracle.sample(u0, w, bc, T, pts)
    ref = np.array([full[p] for p in pts])
    assert np.array_equal(vals, ref)


def test_threads_deterministic():
    u0 = synth.grid((64, 70))
    w = synth.random_weights("box2d49p")
    a = oracle.run(u0, w, "periodic", 5, nthreads=1)
    b = oracle.run(u0, w, "periodic", 5, nthreads=4)
    assert np.array_equal(a, b)


def test_invalid_arguments():
    with pytest.raises(ValueError):
        oracle.run(np.zeros((4, 4)), np.ones((7, 7)), "fixed", 1)  # grid smaller than window
