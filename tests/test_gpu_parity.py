"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle, element by element.

Tolerance (north_star): max |u_gpu - u_oracle| / max |u_oracle| <= 1e-12 after T steps.
DESIGN.md "Tolerance" derives why FP64 reassociation stays ~1e-15 here: weights are a convex
(or |w|-sum <= 1) combination, so each step adds at most ~nnz*eps relative error.

Sizes span several CTA tiles plus ragged tails; T spans several fused passes plus a remainder
pass (T mod Tf != 0).  Weights are seeded random ASYMMETRIC (a flipped kernel fails).
"""
import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

TOL = 1e-12


@pytest.fixture(scope="module")
def csx():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ppopp_chenlwbwmyzcy24_b200 as m
    return m


def rel(a, b):
    return float(np.max(np.abs(a - b)) / np.max(np.abs(b)))


def run_gpu(csx, u0, w, shape, bc, T, engine="auto", fuse_steps=0, inplace=False):
    p = csx.Plan(u0.shape, w, shape=shape, bc=bc, fuse_steps=fuse_steps, engine=engine)
    d_in = torch.from_numpy(u0).cuda()
    d_out = d_in if inplace else torch.empty_like(d_in)
    p.run(d_in, d_out, T)
    torch.cuda.synchronize()
    out = d_out.cpu().numpy()
    info = p.info()
    p.close()
    return out, info


SMALL = {1: (5003,), 2: (100, 150), 3: (21, 19, 70)}
TSTEPS = {1: 17, 2: 7, 3: 3}


@pytest.mark.parametrize("name", list(synth.SHAPES))
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("engine", ["tc_s2r", "tc_tile", "direct"])
def test_parity_small(csx, name, bc, engine):
    s = synth.SHAPES[name]
    ext = SMALL[s.ndim]
    u0 = synth.grid(ext, seed=1234 + s.shape_id)
    w = synth.random_weights(name)
    T = TSTEPS[s.ndim]
    try:
        got, info = run_gpu(csx, u0, w, s.kind, bc, T, engine=engine)
    except csx.CsxError as e:
        if e.status == csx.CSX_ERR_UNSUPPORTED and engine != "direct":
            pytest.skip(f"{engine} does not cover {name}")
        raise
    assert info["engine_name"] == engine
    ref = oracle.run(u0, w, bc, T)
    assert rel(got, ref) <= TOL, (name, bc, engine, info)


@pytest.mark.parametrize("tf", [1, 2, 3])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("engine", ["tc_s2r", "tc_tile"])
def test_parity_fusion_depths_2d(csx, tf, bc, engine):
    u0 = synth.grid((67, 130), seed=5)
    w = synth.random_weights("box2d9p")
    for T in (1, 2, 3, 4, 5, 10):
        got, info = run_gpu(csx, u0, w, "box", bc, T, engine=engine, fuse_steps=tf)
        assert info["fuse_steps"] == tf
        assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (tf, T)


@pytest.mark.parametrize("name,tf", [("box2d9p", 4), ("heat2d", 5), ("box2d9p", 6), ("box2d25p", 2),
                                     ("box2d25p", 3), ("star2d13p", 2), ("box2d49p", 2)])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("engine", ["tc_tile", "direct"])
def test_parity_deep_fusion_2d(csx, name, tf, bc, engine):
    """2D composed windows past the paper's one N fragment (nk = 9, 11, 13; C3's "multi-step
    fused" r = 3, Tf = 2): several CTA tiles + ragged tails, T with and without a remainder
    pass, the FIXED band of depth r*Tf recomputed by k_band."""
    s = synth.SHAPES[name]
    u0 = synth.grid((150, 203), seed=9)
    w = synth.random_weights(name)
    for T in (tf, 2 * tf + 1, 13):
        got, info = run_gpu(csx, u0, w, s.kind, bc, T, engine=engine, fuse_steps=tf)
        assert info["fuse_steps"] == tf and info["engine_name"] == engine
        assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (name, tf, T, bc, engine)


@pytest.mark.parametrize("tf", [1, 2, 3, 5, 7])
def test_parity_fusion_depths_1d(csx, tf):
    u0 = synth.grid((3000,), seed=6)
    w = synth.random_weights("heat1d")
    for bc in ("fixed", "periodic"):
        got, _ = run_gpu(csx, u0, w, "box", bc, 23, engine="tc_s2r", fuse_steps=tf)
        assert rel(got, oracle.run(u0, w, bc, 23)) <= TOL, (tf, bc)


@pytest.mark.parametrize("r,tf", [(1, 1), (1, 3), (1, 7), (1, 8), (1, 11), (1, 13), (1, 15), (2, 3), (2, 5),
                                  (2, 7), (3, 2), (3, 5)])
def test_parity_fusion_depths_1d_tile(csx, r, tf):
    """TC_TILE 1D (Toeplitz blocks, nk = 2 r Tf + 1 up to 31): 3 full tiles of 8 x 256 outputs
    plus a ragged tail; T = 2 Tf + 3 covers fused passes and a remainder pass."""
    u0 = synth.grid((3 * 2048 + 777,), seed=60 + r)
    w = {1: synth.random_weights("heat1d"), 2: synth.random_weights("1d5p")}.get(r)
    if w is None:
        w = synth.random_signed_weights(1, r, seed=61)
    T = 2 * tf + 3
    for bc in ("fixed", "periodic"):
        got, info = run_gpu(csx, u0, w, "box", bc, T, engine="tc_tile", fuse_steps=tf)
        assert info["nk"] == 2 * r * tf + 1
        assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (r, tf, bc)


def test_1d_deep_fusion_minimum_extent(csx):
    """Extent = nk exactly (every point is within the band of some face)."""
    w = synth.random_weights("heat1d")
    for tf in (8, 15):
        u0 = synth.grid((2 * tf + 1,), seed=62)
        for bc in ("fixed", "periodic"):
            got, _ = run_gpu(csx, u0, w, "box", bc, 2 * tf + 1, engine="tc_tile", fuse_steps=tf)
            assert rel(got, oracle.run(u0, w, bc, 2 * tf + 1)) <= TOL, (tf, bc)


def test_signed_weights_general_radius(csx):
    for ndim, r, ext in [(1, 3, (999,)), (2, 2, (70, 90)), (2, 3, (50, 77))]:
        w = synth.random_signed_weights(ndim, r, seed=9)
        u0 = synth.grid(ext, seed=10)
        for bc in ("fixed", "periodic"):
            for engine in ("tc_s2r", "auto"):
                got, _ = run_gpu(csx, u0, w, "box", bc, 4, engine=engine)
                assert rel(got, oracle.run(u0, w, bc, 4)) <= TOL, (ndim, r, bc, engine)


@pytest.mark.parametrize("name,ext", [("box2d9p", (130, 200)), ("box2d9p", (131, 201)),
                                      ("heat2d", (64, 66)), ("box2d49p", (90, 130)),
                                      ("heat3d", (40, 35, 70)), ("box3d27p", (33, 40, 66))])
def test_dense_source_first_pass(csx, monkeypatch, name, ext):
    """FIXED TC_TILE 2D/3D: the first pass stages tiles straight from the user's dense grid
    (TMA zero-fills the out-of-grid halo; no pack).  Bitwise equal to the packed path
    (CSX_DENSE_SRC=0), equal to the oracle, in place and out of place, T below / at / above Tf
    (odd row lengths fall back to the pack)."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=17)
    for T in (1, 3, 4, 7):
        for inplace in (False, True):
            got, info = run_gpu(csx, u0, w, s.kind, "fixed", T, inplace=inplace)
            assert info["engine_name"] == "tc_tile"
            monkeypatch.setenv("CSX_DENSE_SRC", "0")
            packed, _ = run_gpu(csx, u0, w, s.kind, "fixed", T, inplace=inplace)
            monkeypatch.delenv("CSX_DENSE_SRC")
            assert np.array_equal(got, packed), (name, ext, T, inplace)
            assert rel(got, oracle.run(u0, w, "fixed", T)) <= TOL, (name, ext, T, inplace)


def test_edge_cases(csx):
    w = synth.random_weights("box2d9p")
    u0 = synth.grid((40, 72), seed=3)
    # T = 0 copies
    got, _ = run_gpu(csx, u0, w, "box", "fixed", 0)
    assert np.array_equal(got, u0)
    # in place, T < Tf, T = Tf, remainder
    for T in (1, 2, 3, 4):
        got, _ = run_gpu(csx, u0, w, "box", "periodic", T, inplace=True)
        assert rel(got, oracle.run(u0, w, "periodic", T)) <= TOL
    # minimum extents: exactly the composed window (nk = 7)
    u1 = synth.grid((7, 7), seed=4)
    got, _ = run_gpu(csx, u1, w, "box", "periodic", 6, fuse_steps=3)
    assert rel(got, oracle.run(u1, w, "periodic", 6)) <= TOL
    # constant field stays exactly constant with dyadic weights (both BCs)
    c = np.full((64, 100), 0.375)
    for bc in ("fixed", "periodic"):
        got, _ = run_gpu(csx, c, synth.physical_weights("box2d9p"), "box", bc, 9)
        assert np.all(got == 0.375)


def test_run_host_e2e(csx):
    w = synth.random_weights("heat2d")
    u0 = synth.grid((90, 200), seed=12)
    p = csx.Plan(u0.shape, w, shape="star", bc="fixed")
    got = p.run_host(u0, 11)
    p.close()
    assert rel(got, oracle.run(u0, w, "fixed", 11)) <= TOL


def test_sharded_single_rank(csx):
    """csx_run_sharded through NCCL with one rank (the exchange talks to itself on the ring)."""
    for bc in ("fixed", "periodic"):
        w = synth.random_weights("box2d9p")
        u0 = synth.grid((96, 130), seed=13)
        p = csx.Plan(u0.shape, w, bc=bc)
        uid = csx.csx_nccl_unique_id()
        comm = csx.csx_comm_create(uid, 0, 1)
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run_sharded(comm, d_in, d_out, 10, u0.size)
        torch.cuda.synchronize()
        csx.csx_comm_destroy(comm)
        p.close()
        assert rel(d_out.cpu().numpy(), oracle.run(u0, w, bc, 10)) <= TOL, bc


def test_full_size_sampled_box2d9p(csx):
    """BASELINE config C2 (Box-2D9P, 10240^2, T=100) in bench.py's launch configuration:
    sampled outputs (incl. corners and the FIXED band) against the oracle's dependence cones."""
    ext, T = (10240, 10240), 100
    w = synth.random_weights("box2d9p")
    u0 = synth.grid(ext)
    got, info = run_gpu(csx, u0, w, "box", "fixed", T)
    assert info["engine_name"] == "tc_tile"  # bench.py's default engine for this config
    rng = np.random.default_rng(0)
    pts = [(int(rng.integers(0, ext[0])), int(rng.integers(0, ext[1]))) for _ in range(24)]
    pts += [(0, 0), (1, 1), (2, 5), (3, 3), (10239, 10239), (10237, 4000), (5000, 10238), (64, 63)]
    ref = oracle.sample(u0, w, "fixed", T, pts)
    vals = np.array([got[p] for p in pts])
    assert np.max(np.abs(vals - ref)) / np.max(np.abs(got)) <= TOL
    # a property that holds everywhere: convex weights keep values inside [min u0, max u0]
    assert got.min() >= u0.min() and got.max() <= u0.max()


@pytest.mark.parametrize("name,ext,T,tf", [("box2d49p", (10240, 10240), 100, 0),
                                           ("star2d13p", (10240, 10240), 100, 0),
                                           ("star2d13p", (10240, 10240), 100, 2),
                                           ("box2d49p", (10240, 10240), 100, 2),
                                           ("heat2d", (10240, 10240), 100, 0),
                                           ("box3d27p", (512, 512, 512), 50, 0),
                                           ("heat3d", (512, 512, 512), 50, 0),
                                           ("heat1d", (10240000,), 1000, 0),
                                           ("1d5p", (10240000,), 1000, 0)])
def test_full_size_sampled(csx, name, ext, T, tf):
    """Every BASELINE config at full size and full T in bench.py's launch configuration (auto
    engine; C3 also at its "multi-step fused" Tf = 2): sampled outputs, incl. corners and the
    FIXED frame / band, against the oracle's dependence cones."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext)
    got, info = run_gpu(csx, u0, w, s.kind, "fixed", T, fuse_steps=tf)
    rng = np.random.default_rng(1)
    pts = [tuple(int(rng.integers(0, e)) for e in ext) for _ in range(6)]
    band = s.radius * info["fuse_steps"]
    pts += [tuple(0 for _ in ext), tuple(e - 1 for e in ext), tuple(s.radius for _ in ext),
            tuple(band - 1 for _ in ext), tuple(e - band for e in ext)]
    ref = oracle.sample(u0, w, "fixed", T, pts)
    vals = np.array([got[p] for p in pts])
    assert np.max(np.abs(vals - ref)) / np.max(np.abs(got)) <= TOL, info


@pytest.mark.parametrize("name", ["heat3d", "box3d27p"])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_parity_3d_two_step_blocking(csx, name, bc):
    """3D Tf = 2 (k_tile3d_tb: the base stencil run twice per pass through a step-1 plane ring in
    shared memory): ragged tiles and z chunks, T even / odd (remainder pass of Tf = 1), thin grids,
    both boundaries, the dense first-pass source."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    for ext in ((40, 50, 70), (70, 37, 45), (9, 130, 66), (33, 5, 200)):
        u0 = synth.grid(ext, seed=81)
        for T in (2, 5, 8):
            got, info = run_gpu(csx, u0, w, s.kind, bc, T, engine="tc_tile", fuse_steps=2)
            assert info["fuse_steps"] == 2 and info["engine_name"] == "tc_tile"
            assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (name, ext, T, bc)
    # the overlapped sharded schedule (interior / edge z chunks, halo 2) on one rank
    import os
    os.environ["CSX_FORCE_OVERLAP"] = "1"
    try:
        u0 = synth.grid((100, 30, 40), seed=82)
        p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc, fuse_steps=2)
        comm = csx.csx_comm_create(csx.csx_nccl_unique_id(), 0, 1)
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run_sharded(comm, d_in, d_out, 5, u0.size)
        torch.cuda.synchronize()
        csx.csx_comm_destroy(comm)
        p.close()
        assert rel(d_out.cpu().numpy(), oracle.run(u0, w, bc, 5)) <= TOL, (name, bc, "sharded")
    finally:
        del os.environ["CSX_FORCE_OVERLAP"]


@pytest.mark.parametrize("variant", ["0", "1", "2", "3", "4", "5", "6", "7", "8", "9", "a", "b",
                                     "i", "j", "m", "n", "w", "x", "z", "u"])
def test_parity_3d_tile_variants(csx, monkeypatch, variant):
    """Every TC_TILE 3D CTA geometry / DMMA order (CSX_TILE3D_VARIANT), star and box, ragged
    (y, x) tiles and z chunks, both boundaries (i / j / m / n / w / x: box-only variants — the
    plane-interleaved order, two 8-warp CTAs per SM, 16-warp CTAs; z / u: 32 x 128 tiles of 16 /
    8 warps; stars take the default unless noted)."""
    monkeypatch.setenv("CSX_TILE3D_VARIANT", variant)
    for name, ext in (("heat3d", (70, 37, 45)), ("box3d27p", (9, 70, 150)), ("box3d27p", (37, 5, 9))):
        s = synth.SHAPES[name]
        u0 = synth.grid(ext, seed=33)
        w = synth.random_weights(name)
        for bc in ("fixed", "periodic"):
            got, info = run_gpu(csx, u0, w, s.kind, bc, 3, engine="tc_tile", fuse_steps=1)
            assert rel(got, oracle.run(u0, w, bc, 3)) <= TOL, (name, ext, bc, variant)


@pytest.mark.parametrize("name", ["heat3d", "box3d27p"])
@pytest.mark.parametrize("engine", ["tc_tile", "tc_s2r"])
def test_parity_3d_zchunks(csx, name, engine):
    """3D grids spanning several z chunks (ragged last chunk) and ragged (y, x) tiles."""
    s = synth.SHAPES[name]
    u0 = synth.grid((70, 37, 45), seed=31)
    w = synth.random_weights(name)
    for bc in ("fixed", "periodic"):
        got, info = run_gpu(csx, u0, w, s.kind, bc, 4, engine=engine, fuse_steps=1)
        assert info["engine_name"] == engine
        assert rel(got, oracle.run(u0, w, bc, 4)) <= TOL, (name, engine, bc)


def test_direct_comparator_2d_all_radii(csx):
    """The 2D CUDA-core comparator (k_direct2d_wf for r = 1 (Tf <= 4) and r = 2 (Tf = 1), the
    shared-memory kernels otherwise) for r = 1..3 and its temporal-blocking depths; the second
    grid spans several 256-row chunks and 56-64-column strips with ragged tails."""
    for ndim, r, tf in [(2, 1, 1), (2, 1, 2), (2, 1, 3), (2, 1, 4), (2, 2, 1), (2, 2, 2), (2, 3, 1),
                        (2, 3, 2)]:
        w = synth.random_signed_weights(ndim, r, seed=40 + r)
        for ext in ((131, 150), (601, 333)):
            u0 = synth.grid(ext, seed=41)
            for bc in ("fixed", "periodic"):
                got, info = run_gpu(csx, u0, w, "box", bc, 9, engine="direct", fuse_steps=tf)
                assert rel(got, oracle.run(u0, w, bc, 9)) <= TOL, (r, tf, bc, ext)


@pytest.mark.parametrize("generic", [False, True])
def test_direct_comparator_1d_3d(csx, monkeypatch, generic):
    """The 1D (register window + shuffles, Tf fused) and 3D (z-march, cp.async plane ring)
    comparator kernels, and the generic smem kernel they replace (CSX_DIRECT_GENERIC=1), for
    r = 1..3, several fusion depths, ragged extents, both boundaries, signed weights."""
    if generic:
        monkeypatch.setenv("CSX_DIRECT_GENERIC", "1")
    cases = [(1, 1, 1, (9001,), 13), (1, 1, 11, (20000,), 25), (1, 2, 5, (7777,), 12),
             (1, 3, 5, (4099,), 11), (1, 1, 15, (3000,), 33),
             (3, 1, 1, (37, 45, 70), 3), (3, 2, 1, (19, 33, 130), 2), (3, 3, 1, (16, 40, 66), 2)]
    for ndim, r, tf, ext, T in cases:
        w = synth.random_signed_weights(ndim, r, seed=60 + r)
        u0 = synth.grid(ext, seed=61)
        for bc in ("fixed", "periodic"):
            got, info = run_gpu(csx, u0, w, "box", bc, T, engine="direct", fuse_steps=tf)
            assert rel(got, oracle.run(u0, w, bc, T)) <= TOL, (ndim, r, tf, bc, generic)
    # star (Heat-3D) exercises the single-column planes
    w = synth.random_weights("heat3d")
    u0 = synth.grid((45, 70, 99), seed=62)
    for bc in ("fixed", "periodic"):
        got, _ = run_gpu(csx, u0, w, "star", bc, 4, engine="direct")
        assert rel(got, oracle.run(u0, w, bc, 4)) <= TOL, ("heat3d", bc, generic)


@pytest.mark.parametrize("pad,dirty", [(0, 0), (1, 0), (0, 1), (1, 1), (2, 1), (3, 1)])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_s2r_breakdown_variants(csx, pad, dirty, bc):
    """Fig 6 breakdown variants of TC_S2R (I explicit stencil2row, II CUDA-core tessellation, no
    padding / no dirty bits) compute the same result, over ragged extents and a remainder pass."""
    for name in ("box2d9p", "heat2d", "box2d49p", "box2d25p"):
        s = synth.SHAPES[name]
        w = synth.random_weights(name)
        u0 = synth.grid((99, 140), seed=51)
        p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc, engine="tc_s2r")
        p.set_s2r_variant(pad if pad in (2, 3) else bool(pad), bool(dirty))
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run(d_in, d_out, 7)
        torch.cuda.synchronize()
        p.close()
        assert rel(d_out.cpu().numpy(), oracle.run(u0, w, bc, 7)) <= TOL, (name, pad, dirty)


@pytest.mark.parametrize("name,ext,T", [("box2d9p", (400, 130), 10), ("heat1d", (30000,), 23),
                                        ("box3d27p", (100, 30, 40), 4), ("box2d49p", (300, 90), 3)])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_sharded_overlap_schedule(csx, monkeypatch, name, ext, T, bc):
    """The overlapped sharded schedule (interior tiles, then edge tiles after the halo event,
    exchange on its own stream) forced on one rank: same result as the oracle."""
    monkeypatch.setenv("CSX_FORCE_OVERLAP", "1")
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=14)
    p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc)
    assert p.info()["engine_name"] == "tc_tile"
    comm = csx.csx_comm_create(csx.csx_nccl_unique_id(), 0, 1)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    p.run_sharded(comm, d_in, d_out, T, u0.size)
    torch.cuda.synchronize()
    csx.csx_comm_destroy(comm)
    p.close()
    assert rel(d_out.cpu().numpy(), oracle.run(u0, w, bc, T)) <= TOL, (name, bc)


@pytest.mark.parametrize("name,ext,T", [("box2d9p", (200, 150), 7), ("heat3d", (40, 33, 50), 3),
                                        ("box3d27p", (21, 40, 35), 2), ("box2d49p", (90, 70), 3)])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_sharded_pencil_single_rank(csx, name, ext, T, bc):
    """csx_run_sharded_pencil on a 1 x 1 process grid: the two-phase face exchange runs through
    NCCL (PERIODIC: self send/recv of packed strided faces + full padded rows), then the same pass
    kernels; equal to the oracle."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=15)
    p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc)
    comm = csx.csx_comm_create(csx.csx_nccl_unique_id(), 0, 1)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    with pytest.raises(csx.CsxError):
        p.run_sharded_pencil(comm, 2, 1, d_in, d_out, T, u0.size)  # grid != communicator size
    p.run_sharded_pencil(comm, 1, 1, d_in, d_out, T, u0.size)
    torch.cuda.synchronize()
    got = d_out.cpu().numpy()
    p.run_sharded(comm, d_in, d_out, T, u0.size)  # back to slabs on the same plan
    torch.cuda.synchronize()
    got_slab = d_out.cpu().numpy()
    csx.csx_comm_destroy(comm)
    p.close()
    ref = oracle.run(u0, w, bc, T)
    assert rel(got, ref) <= TOL, (name, bc)
    assert rel(got_slab, ref) <= TOL, (name, bc)


@pytest.mark.parametrize("name,ext,T", [("box2d9p", (300, 260), 10), ("heat1d", (50000,), 40),
                                        ("box3d27p", (40, 50, 70), 3), ("heat1d", (1024,), 16)])
def test_graph_replay(csx, name, ext, T):
    """csx_plan_set_graph: the first call runs eagerly and captures, later calls with the same
    (d_in, d_out, T) replay the CUDA graph; a new triple re-captures.  Bitwise equal to eager
    runs and equal to the oracle (C1 = Heat-1D N=1024, T=16 is the last case)."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=71)
    ref = oracle.run(u0, w, "fixed", T)
    p = csx.Plan(u0.shape, w, shape=s.kind, bc="fixed")
    d_in = torch.from_numpy(u0).cuda()
    eager = torch.empty_like(d_in)
    p.run(d_in, eager, T)
    p.set_graph(True)
    outs = [torch.full_like(d_in, -1.0) for _ in range(2)]
    for k in range(3):                       # capture, replay, replay
        outs[0].fill_(-1.0)
        p.run(d_in, outs[0], T)
        torch.cuda.synchronize()
        assert torch.equal(outs[0], eager), k
    p.run(d_in, outs[1], T)                  # new output pointer -> re-capture
    torch.cuda.synchronize()
    assert torch.equal(outs[1], eager)       # the re-captured graph computes the same T steps
    p.run(d_in, outs[1], T - 1)              # new T -> re-capture
    torch.cuda.synchronize()
    p.set_graph(False)
    p.close()
    assert rel(outs[0].cpu().numpy(), ref) <= TOL
    assert rel(outs[1].cpu().numpy(), oracle.run(u0, w, "fixed", T - 1)) <= TOL


@pytest.mark.parametrize("name,ext,T", [("box2d9p", (50000, 50000), 4), ("heat3d", (1400, 1400, 1400), 3),
                                        ("box3d27p", (1360, 1400, 1410), 2), ("heat1d", (2900000000,), 23)])
def test_max_size_beyond_int32(csx, name, ext, T):
    """Maximum-size cases: 2.5-2.7e9-point grids (20-22 GB per buffer, flat indices past 2^31)
    generated on the device by the same seeded generator: 2D Box-2D9P (two folded passes of
    Tf = 2, dense first-pass source, k_band) and 3D Heat-3D / Box-3D27P (z-plane rings), FIXED.
    Sampled outputs (corners, faces, band, interior, indices beyond 2^31) against the oracle
    run on each point's dependence window (half-width T*r + 1, so the window's own held edge
    cannot reach the point)."""
    s = synth.SHAPES[name]
    r = s.radius
    free = torch.cuda.mem_get_info()[0]
    need = 5 * 8 * int(np.prod(ext, dtype=np.int64))
    if free < need:
        pytest.skip(f"needs ~{need >> 30} GB of free device memory, {free >> 30} GB free")
    w = synth.random_weights(name)
    d_in = synth.grid_torch(ext, "cuda")
    d_out = torch.empty_like(d_in)
    p = csx.Plan(ext, w, shape=s.kind, bc="fixed")
    p.run(d_in, d_out, T)
    torch.cuda.synchronize()
    rng = np.random.default_rng(5)
    nd = len(ext)
    pts = [tuple(0 for _ in ext), tuple(e - 1 for e in ext), tuple(1 for _ in ext),
           tuple(e - 2 for e in ext), tuple(e // 2 for e in ext),
           tuple([1] + [e // 3 for e in ext[1:]]), tuple([e - 2 for e in ext[:-1]] + [7]),
           tuple(int(e * 0.9) for e in ext)]
    pts += [tuple(int(rng.integers(0, e)) for e in ext) for _ in range(10)]
    h = T * r + 1
    for pt in pts:
        lo = tuple(max(0, c - h) for c in pt)
        hi = tuple(min(e, c + h + 1) for c, e in zip(pt, ext))
        u0w = synth.grid_window(ext, lo, hi)
        loc = tuple(c - l for c, l in zip(pt, lo))
        assert float(d_in[pt]) == u0w[loc]  # device generator == host generator
        ref = oracle.run(u0w, w, "fixed", T)[loc]
        got = float(d_out[pt])
        assert abs(got - ref) <= TOL, (name, pt, got, ref)  # values in [0, 1): max|u| ~ 1
    p.close()
    del d_in, d_out
    torch.cuda.empty_cache()


def test_graph_invalidated_by_engine_change(csx):
    """A captured graph must not outlive an engine switch: after set_engine the same
    (d_in, d_out, T) runs the new engine (bitwise equal to a fresh plan of that engine)."""
    w = synth.random_weights("box2d9p")
    u0 = synth.grid((200, 260), seed=91)
    d_in = torch.from_numpy(u0).cuda()
    out = torch.empty_like(d_in)
    p = csx.Plan(u0.shape, w, shape="box", bc="fixed")
    p.set_graph(True)
    for _ in range(2):
        p.run(d_in, out, 9)        # eager + capture, then replay (TC_TILE)
    p.set_engine("direct")
    p.run(d_in, out, 9)
    torch.cuda.synchronize()
    q = csx.Plan(u0.shape, w, shape="box", bc="fixed", engine="direct")
    ref = torch.empty_like(d_in)
    q.run(d_in, ref, 9)
    torch.cuda.synchronize()
    p.close()
    q.close()
    assert torch.equal(out, ref)
    assert rel(out.cpu().numpy(), oracle.run(u0, w, "fixed", 9)) <= TOL


_D1_VARIANT_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for r, tf, n, T in [(1, 1, 9001, 13), (1, 11, 20000, 25), (2, 5, 7777, 12), (3, 5, 4099, 11), (1, 15, 3000, 33)]:
    w = synth.random_signed_weights(1, r, seed=60 + r)
    u0 = synth.grid((n,), seed=61)
    for bc in ("fixed", "periodic"):
        p = csx.Plan(u0.shape, w, shape="box", bc=bc, fuse_steps=tf, engine="direct")
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run(d_in, d_out, T)
        torch.cuda.synchronize()
        ref = oracle.run(u0, w, bc, T)
        worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
        p.close()
print(worst)
"""


_D2_VARIANT_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for r, tf in [(1, 1), (1, 2), (1, 3), (1, 4), (2, 1), (2, 2), (3, 1)]:
    w = synth.random_signed_weights(2, r, seed=40 + r)
    u0 = synth.grid((601, 333), seed=41)
    for bc in ("fixed", "periodic"):
        p = csx.Plan(u0.shape, w, shape="box", bc=bc, fuse_steps=tf, engine="direct")
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run(d_in, d_out, 9)
        torch.cuda.synchronize()
        ref = oracle.run(u0, w, bc, 9)
        worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
        p.close()
print(worst)
"""


@pytest.mark.parametrize("env", [{"CSX_DIRECT2D": "smem"}, {"CSX_DIRECT2D": "smem", "CSX_DIRECT_WS": "0"},
                                 {"CSX_DIRECT2D_V": "4"}, {"CSX_DIRECT2D_UNR": "1"}])
def test_direct_comparator_2d_variants(env):
    """Every 2D comparator kernel variant (register wavefront V = 2 / 4, row loop unrolled by 2R+1 or
    not, the
    shared-memory kernels with and without warp specialisation; knobs read once per process,
    hence a subprocess each) matches the oracle."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", _D2_VARIANT_SCRIPT, root], env=dict(os.environ, **env),
                         cwd=root, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    assert float(out.stdout.strip().splitlines()[-1]) <= TOL, (env, out.stdout)


_S2R_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for name in ("box2d9p", "heat2d", "box2d25p", "box2d49p"):
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid((99, 140), seed=51)
    for bc in ("fixed", "periodic"):
        for pad, dirty in ((1, 1), (0, 0), (1, 0), (0, 1)):
            p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc, engine="tc_s2r")
            p.set_max_ctas(3)
            p.set_s2r_variant(bool(pad), bool(dirty))
            d_in = torch.from_numpy(u0).cuda()
            d_out = torch.empty_like(d_in)
            p.run(d_in, d_out, 7)
            torch.cuda.synchronize()
            ref = oracle.run(u0, w, bc, 7)
            worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
            p.close()
print(worst)
"""


@pytest.mark.parametrize("ws", ["0", "1"])
def test_s2r_2d_kernel_variants(ws):
    """The TC_S2R 2D kernels with the LUT scatter on dedicated warps (CSX_S2R_WS=1, default) and
    on the tessellation warps (0), every padding / dirty-bits variant, persistent grid capped at 3
    CTAs so that both A/B buffers and the raw ring wrap many times; read once per process."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", _S2R_SCRIPT, root], env=dict(os.environ, CSX_S2R_WS=ws),
                         cwd=root, capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    assert float(out.stdout.strip().splitlines()[-1]) <= TOL, (ws, out.stdout)


@pytest.mark.parametrize("v,pf", [(4, 0), (4, 1), (8, 1), (16, 0), (16, 1), (32, 0)])
def test_direct_comparator_1d_variants(v, pf):
    """Every k_direct1d variant (points per lane V x register prefetch, CSX_DIRECT1D_V /
    CSX_DIRECT1D_PF; read once per process, hence a subprocess each) matches the oracle; the
    default (V = 8, no prefetch) is covered by test_direct_comparator_1d_3d."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, CSX_DIRECT1D_V=str(v), CSX_DIRECT1D_PF=str(pf))
    out = subprocess.run([sys.executable, "-c", _D1_VARIANT_SCRIPT, root], env=env, cwd=root,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    assert float(out.stdout.strip().splitlines()[-1]) <= TOL, (v, pf, out.stdout)


_TILE2D_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for name, tf, T in (("box2d9p", 1, 3), ("box2d9p", 2, 5), ("box2d9p", 3, 7), ("box2d25p", 1, 3), ("heat2d", 2, 4)):
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid((301, 261), seed=71)
    for bc in ("fixed", "periodic"):
        p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc, fuse_steps=tf, engine="tc_tile")
        p.set_max_ctas(5)
        d_in = torch.from_numpy(u0).cuda()
        d_out = torch.empty_like(d_in)
        p.run(d_in, d_out, T)
        torch.cuda.synchronize()
        ref = oracle.run(u0, w, bc, T)
        worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
        p.close()
print(worst)
"""


@pytest.mark.parametrize("variant", ["0", "2", "3", "4", "5", "6", "7", "8"])
def test_tile2d_variants(variant):
    """Every 2D TC_TILE CTA geometry / DMMA order (CSX_TILE_VARIANT, read once per process: a
    subprocess each; variant 1 is the default the rest of the suite runs) for nk = 3, 5, 7,
    ragged tiles, both boundaries, persistent grid capped at 5 CTAs."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", _TILE2D_SCRIPT, root],
                         env=dict(os.environ, CSX_TILE_VARIANT=variant), cwd=root,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    assert float(out.stdout.strip().splitlines()[-1]) <= TOL, (variant, out.stdout)


_TILE1D_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import oracle, synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx
worst = 0.0
for name, tf, T in (("heat1d", 7, 15), ("heat1d", 11, 23), ("heat1d", 13, 27), ("1d5p", 5, 11), ("1d5p", 7, 15)):
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid((70001,), seed=73)
    for bc in ("fixed", "periodic"):
        for cap in (3, 0):
            p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc, fuse_steps=tf, engine="tc_tile")
            if cap:
                p.set_max_ctas(cap)
            d_in = torch.from_numpy(u0).cuda()
            d_out = torch.empty_like(d_in)
            p.run(d_in, d_out, T)
            torch.cuda.synchronize()
            ref = oracle.run(u0, w, bc, T)
            worst = max(worst, float(np.max(np.abs(d_out.cpu().numpy() - ref)) / np.max(np.abs(ref))))
            p.close()
print(worst)
"""


@pytest.mark.parametrize("variant", ["1", "2", "3", "4", "5", "6", "7", "8"])
def test_tile1d_variants(variant):
    """Every 1D TC_TILE tile / warp / ring geometry (CSX_TILE1D_VARIANT, read once per process: a
    subprocess each; the default — 8 DMMA warps for nk >= 21, variant 8's 4 warps below — runs in
    the rest of the suite) at nk = 15, 23, 27 (r = 1) and 21, 29 (r = 2), with a remainder pass,
    ragged tail, both boundaries, persistent grid capped at 3 CTAs and uncapped."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, "-c", _TILE1D_SCRIPT, root],
                         env=dict(os.environ, CSX_TILE1D_VARIANT=variant), cwd=root,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    assert float(out.stdout.strip().splitlines()[-1]) <= TOL, (variant, out.stdout)


@pytest.mark.parametrize("name, ext, T", [
    ("heat1d", (40001,), 23), ("1d5p", (30001,), 11), ("box2d9p", (301, 130), 7), ("heat2d", (257, 96), 10),
    ("box2d49p", (200, 70), 3), ("heat3d", (70, 33, 40), 5), ("box3d27p", (61, 20, 36), 3)])
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_run_host_chunked_pipeline(csx, monkeypatch, name, ext, T, bc):
    """csx_run_host with pinned host buffers runs ghost-zone chunks along the slowest axis on
    three streams (H2D of chunk k+1 / run of chunk k / D2H of chunk k-1): forced to 2, 3 and 5
    chunks (CSX_HOST_CHUNKS) — chunks whose ghost zones wrap (PERIODIC) or clip at the global
    faces (FIXED), a short last chunk — and compared element by element with the oracle; pageable
    buffers and CSX_HOST_CHUNKS = 0 take the serial path."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=77)
    ref = oracle.run(u0, w, bc, T)
    p = csx.Plan(u0.shape, w, shape=s.kind, bc=bc)
    h_in = torch.from_numpy(u0).pin_memory().numpy()
    for k in ("2", "3", "5", "0"):
        monkeypatch.setenv("CSX_HOST_CHUNKS", k)
        h_out = torch.empty(u0.shape, dtype=torch.float64).pin_memory().numpy()
        h_out[...] = np.nan
        p.run_host(h_in, T, h_out)
        assert rel(h_out, ref) <= TOL, (name, bc, k)
    monkeypatch.delenv("CSX_HOST_CHUNKS")
    got = p.run_host(u0.copy(), T)            # pageable: serial path
    assert rel(got, ref) <= TOL
    p.close()


def test_run_host_chunks_fall_back(csx, monkeypatch):
    """Forced chunks too short for the fused window (nk = 27 sub-plans on 12-row chunks) and
    overlapping host buffers take the serial path; results stay equal to the oracle."""
    w = synth.random_weights("heat1d")
    u0 = synth.grid((60,), seed=5)
    ref = oracle.run(u0, w, "fixed", 3)
    p = csx.Plan(u0.shape, w, shape="star", bc="fixed", fuse_steps=13)
    monkeypatch.setenv("CSX_HOST_CHUNKS", "5")      # 5 chunks of 12 + 2 x 4 ghost rows < 27
    h_in = torch.from_numpy(u0).pin_memory().numpy()
    h_out = torch.empty(u0.shape, dtype=torch.float64).pin_memory().numpy()
    p.run_host(h_in, 3, h_out)
    assert rel(h_out, ref) <= TOL
    assert p.host_last()[0] == 1
    p.close()
    w2 = synth.random_weights("box2d9p")
    u2 = synth.grid((300, 64), seed=6)
    ref2 = oracle.run(u2, w2, "periodic", 7)
    p2 = csx.Plan(u2.shape, w2, shape="box", bc="periodic")
    big = torch.from_numpy(np.concatenate([u2.ravel(), np.zeros(64)])).pin_memory().numpy()
    src = big[:u2.size].reshape(u2.shape)
    dst = big[64:64 + u2.size].reshape(u2.shape)       # overlaps src, shifted by one row
    monkeypatch.setenv("CSX_HOST_CHUNKS", "3")
    p2.run_host(src, 7, dst)
    assert p2.host_last()[0] == 1
    assert rel(dst, ref2) <= TOL
    p2.close()
