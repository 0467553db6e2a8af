"""GPU parity, round 2: general radius in 3D, persistent CTAs wrapping their rings, every
BASELINE config compared element by element at full size, and plan teardown.

Every comparison is against the CPU oracle (``oracle.run``) on the same seeded inputs, with the
north_star tolerance max|u_gpu - u_oracle| / max|u_oracle| <= 1e-12.
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


def run_gpu(csx, u0, w, shape, bc, T, engine="auto", fuse_steps=0, max_ctas=0, graph=False):
    p = csx.Plan(u0.shape, w, shape=shape, bc=bc, fuse_steps=fuse_steps, engine=engine)
    if max_ctas:
        p.set_max_ctas(max_ctas)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    if graph:
        p.set_graph(True)
        p.run(d_in, d_out, T)       # eager run + capture
        d_out.fill_(-1.0)
    p.run(d_in, d_out, T)           # (graph: replay)
    torch.cuda.synchronize()
    out = d_out.cpu().numpy()
    info = p.info()
    p.close()
    return out, info


# ---- 3D radius 2 and 3 (PAPER.md P.1788-1800: the 3D method is a sum of
# ---- per-plane 2D ConvStencils for any plane window) ----------------------------------------

R3D = ["star3d13p", "box3d125p", "star3d19p", "box3d343p"]


@pytest.mark.parametrize("name", R3D)
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
@pytest.mark.parametrize("engine", ["auto", "tc_tile", "tc_s2r", "direct"])
def test_parity_3d_general_radius(csx, name, bc, engine):
    """3D r = 2 / 3, star and box, on every engine: ragged (y, x) tiles, two z chunks, T = 3.
    TC_S2R has no 3D kernel past nk = 3 and must refuse (UNSUPPORTED) rather than run."""
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid((45, 37, 70), seed=201 + s.shape_id)
    if engine == "tc_s2r":
        with pytest.raises(csx.CsxError) as ei:
            run_gpu(csx, u0, w, s.kind, bc, 3, engine=engine)
        assert ei.value.status == csx.CSX_ERR_UNSUPPORTED
        return
    got, info = run_gpu(csx, u0, w, s.kind, bc, 3, engine=engine)
    assert info["engine_name"] == ("tc_tile" if engine == "auto" else engine)
    assert info["nk"] == 2 * s.radius + 1 and info["fuse_steps"] == 1
    assert rel(got, oracle.run(u0, w, bc, 3)) <= TOL, (name, bc, engine)


@pytest.mark.parametrize("r", [2, 3])
def test_parity_3d_general_radius_signed(csx, r):
    """Signed, non-normalised box weights at r = 2 / 3 (every plane on the tensor cores), thin and
    ragged grids, both boundaries; and fuse_steps = 2 at r >= 2 is refused (no 3D kernel)."""
    w = synth.random_signed_weights(3, r, seed=300 + r)
    for ext in ((2 * r + 1, 40, 66), (33, 2 * r + 1, 9), (70, 33, 130)):
        u0 = synth.grid(ext, seed=301)
        for bc in ("fixed", "periodic"):
            got, info = run_gpu(csx, u0, w, "box", bc, 2, engine="tc_tile")
            assert rel(got, oracle.run(u0, w, bc, 2)) <= TOL, (r, ext, bc)
    with pytest.raises(csx.CsxError):
        csx.Plan((40, 40, 40), w, shape="box", bc="fixed", fuse_steps=2)


# ---- persistent CTAs wrapping their smem rings many times (max_ctas cap) -------------------

CAP_CASES = [
    # (shape name, extents, T, engine, fuse_steps): one case per persistent kernel family
    ("box2d9p", (300, 260), 7, "tc_tile", 3),     # k_tile2d nk = 7 (+ folded remainder nk = 5)
    ("box2d9p", (300, 260), 5, "tc_tile", 1),     # k_tile2d nk = 3
    ("box2d9p", (300, 260), 5, "tc_tile", 2),     # k_tile2d nk = 5
    ("box2d9p", (300, 260), 9, "tc_tile", 4),     # k_tile2d nk = 9
    ("box2d25p", (300, 260), 5, "tc_tile", 2),    # k_tile2d nk = 9 (r = 2)
    ("heat2d", (300, 260), 10, "tc_tile", 5),     # k_tile2d nk = 11
    ("box2d49p", (300, 260), 4, "tc_tile", 2),    # k_tile2d nk = 13
    ("heat1d", (50000,), 23, "tc_tile", 11),      # k_tile1d nk = 23
    ("1d5p", (50000,), 11, "tc_tile", 5),         # k_tile1d nk = 21
    ("heat3d", (70, 37, 130), 3, "tc_tile", 1),   # k_tile3d nk = 3, star variant
    ("box3d27p", (70, 37, 130), 3, "tc_tile", 1),  # k_tile3d nk = 3, box variant
    ("box3d125p", (70, 37, 130), 2, "tc_tile", 1),  # k_tile3d nk = 5
    ("star3d19p", (70, 37, 130), 2, "tc_tile", 1),  # k_tile3d nk = 7 (star: 76-column pitch)
    ("star3d13p", (70, 37, 130), 2, "tc_tile", 1),  # k_tile3d nk = 5 (star: column-major blocks)
    ("heat3d", (70, 37, 130), 4, "tc_tile", 2),   # k_tile3d_tb
    ("box2d9p", (300, 260), 7, "tc_s2r", 3),      # k_s2r2d nk = 7
    ("box2d25p", (300, 260), 3, "tc_s2r", 1),     # k_s2r2d nk = 5
    ("heat1d", (50000,), 15, "tc_s2r", 7),        # k_s2r1d nk = 15
    ("box3d27p", (70, 37, 130), 3, "tc_s2r", 1),  # k_s2r3d
    ("box2d9p", (300, 260), 7, "direct", 3),      # k_direct2d_ws
    ("heat1d", (50000,), 23, "direct", 11),       # k_direct1d
    ("box3d27p", (70, 37, 130), 3, "direct", 1),  # k_direct3d
]


@pytest.mark.parametrize("case", CAP_CASES, ids=lambda c: f"{c[0]}-{c[3]}-tf{c[4]}")
@pytest.mark.parametrize("bc", ["fixed", "periodic"])
def test_persistent_ctas_wrap(csx, case, bc):
    """With the persistent grid capped at 1, 3 and 7 CTAs each CTA walks tens to hundreds of
    tiles / z items through its STAGES-deep ring (slot reuse, mbarrier phase flips, empty-slot
    waits, PDL across passes): fully compared with the oracle, and bitwise equal across caps."""
    name, ext, T, engine, tf = case
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext, seed=400 + s.shape_id)
    ref = oracle.run(u0, w, bc, T)
    outs = []
    for cap in (1, 3, 7, 0):
        got, info = run_gpu(csx, u0, w, s.kind, bc, T, engine=engine, fuse_steps=tf, max_ctas=cap)
        assert info["engine_name"] == engine and info["fuse_steps"] == tf
        assert rel(got, ref) <= TOL, (name, engine, tf, bc, cap)
        outs.append(got)
    for o in outs[1:]:
        assert np.array_equal(o, outs[0])


# ---- every BASELINE config, every element, full extents and full T --------------------------

FULL = [
    # (name, extents, T, fuse_steps list): BASELINE.json configs C1-C4 plus the north-star 1D list
    ("heat1d", (1024,), 16, [0]),                       # C1
    ("box2d9p", (10240, 10240), 100, [0, 3]),           # C2 (the headline; auto Tf = 2, and the paper's 3)
    ("star2d13p", (10240, 10240), 100, [0, 2]),         # C3, auto (Tf = 1) and "multi-step fused"
    ("box2d49p", (10240, 10240), 100, [0, 2]),          # C3
    ("heat3d", (512, 512, 512), 50, [0]),               # C4
    ("box3d27p", (512, 512, 512), 50, [0]),             # C4
    ("heat1d", (10240000,), 1000, [0]),                 # extra (north-star shape list)
    ("1d5p", (10240000,), 1000, [0]),
]


@pytest.mark.parametrize("case", FULL, ids=lambda c: f"{c[0]}-{'x'.join(map(str, c[1]))}")
def test_full_extent_parity(csx, case):
    """bench.py's launch configuration (auto engine, CUDA-graph replay) at the config's full
    extents and full T, FIXED, seeded asymmetric weights: EVERY output compared with the oracle
    run on the box's host cores (SURVEY §8(c) "Direct parity"; PAPER.md P.2829-2836)."""
    name, ext, T, tfs = case
    s = synth.SHAPES[name]
    w = synth.random_weights(name)
    u0 = synth.grid(ext)
    ref = oracle.run(u0, w, "fixed", T)
    for tf in tfs:
        got, info = run_gpu(csx, u0, w, s.kind, "fixed", T, fuse_steps=tf, graph=True)
        assert info["engine_name"] == "tc_tile"
        if tf:
            assert info["fuse_steps"] == tf
        err = rel(got, ref)
        assert err <= TOL, (name, ext, T, info["fuse_steps"], err)
        del got
    if name == "box2d9p":  # C2 also on the paper's layout (warp-specialised TC_S2R)
        got, info = run_gpu(csx, u0, w, s.kind, "fixed", T, engine="tc_s2r", graph=True)
        assert info["engine_name"] == "tc_s2r"
        assert rel(got, ref) <= TOL, (name, "tc_s2r")


# ---- teardown: plan destruction returns every byte ------------------------------------------

def _free_bytes():
    torch.cuda.synchronize()
    return torch.cuda.mem_get_info()[0]


def test_peer_plan_teardown_frees_memory(csx):
    """A single-rank NVLink-peer plan (ring onto itself) created, run and destroyed 20 times:
    device memory returns to its baseline (the peer block holds both padded slab grids)."""
    w = synth.random_weights("box2d9p")
    u0 = synth.grid((1024, 2048), seed=501)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    ref = oracle.run(u0, w, "periodic", 4)
    base = None
    for k in range(21):
        if k == 1:  # after one full cycle (lazily loaded modules, context resources)
            base = _free_bytes()
        p = csx.Plan(u0.shape, w, shape="box", bc="periodic")
        p.peer_setup(0, 1)
        p.run_sharded_peer(d_in, d_out, 4, u0.size)
        torch.cuda.synchronize()
        if k == 0:
            assert rel(d_out.cpu().numpy(), ref) <= TOL
        p.close()
    # one leaked peer block (two padded 1024 x 2048 slabs) is ~35 MB; 20 would be ~700 MB
    leak = base - _free_bytes()
    assert leak < (8 << 20), f"{leak >> 20} MB not returned after 20 peer plans"


def test_graph_plan_variant_switch_teardown(csx):
    """Graph mode, then breakdown variant I (explicit stencil2row scratch), run again, destroy:
    results stay right, nothing is double-freed, memory returns to baseline."""
    w = synth.random_weights("box2d9p")
    u0 = synth.grid((500, 700), seed=502)
    d_in = torch.from_numpy(u0).cuda()
    d_out = torch.empty_like(d_in)
    ref = oracle.run(u0, w, "fixed", 7)
    base = None
    for k in range(9):
        if k == 1:  # after one full cycle (lazily loaded modules, graph resources)
            base = _free_bytes()
        p = csx.Plan(u0.shape, w, shape="box", bc="fixed", engine="tc_s2r")
        p.set_graph(True)
        for _ in range(2):
            p.run(d_in, d_out, 7)
        torch.cuda.synchronize()
        assert rel(d_out.cpu().numpy(), ref) <= TOL
        p.set_s2r_variant(padding=3, dirty_bits=True)   # variant I: allocates the HBM scratch
        for _ in range(2):
            d_out.fill_(-1.0)
            p.run(d_in, d_out, 7)
        torch.cuda.synchronize()
        assert rel(d_out.cpu().numpy(), ref) <= TOL
        p.set_s2r_variant(padding=True, dirty_bits=True)
        p.run(d_in, d_out, 7)
        torch.cuda.synchronize()
        assert rel(d_out.cpu().numpy(), ref) <= TOL
        p.close()
    # 8 cycles: any leaked grid (>= 2.8 MB) or stencil2row scratch (~5 MB) adds up past 8 MB
    leak = base - _free_bytes()
    assert leak < (8 << 20), f"{leak >> 20} MB not returned"


@pytest.mark.parametrize("env", [{"CSX_TILE3D_KO": "0"}, {"CSX_TILE3D5_G8": "1"}, {"CSX_TILE3D5_G8": "0"},
                                 {"CSX_STAR_CF": "0"}, {"CSX_TILE3D_W16": "0"}, {"CSX_TILE3D_W16": "1"}])
def test_parity_3d_general_radius_variants(csx, monkeypatch, env):
    """The other 3D r = 2 / 3 tile configurations (row-outer DMMA order; 8 or 4 blocks per warp
    for both stars and boxes; the round-2 star layouts without the conflict-free DFMA planes;
    read at every launch): ragged tiles and z chunks, both boundaries."""
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    for name in R3D:
        s = synth.SHAPES[name]
        w = synth.random_weights(name)
        u0 = synth.grid((40, 70, 90), seed=601)
        for bc in ("fixed", "periodic"):
            got, _ = run_gpu(csx, u0, w, s.kind, bc, 2, engine="tc_tile", max_ctas=5)
            assert rel(got, oracle.run(u0, w, bc, 2)) <= TOL, (name, bc, env)


def test_randomized_plans_against_oracle(csx):
    """Seeded fuzzing over the plan space the C-ABI accepts: dimension, radius, star / box,
    signed weights, ragged extents (including extents equal to the composed window), boundary,
    fusion depth, engine, T with and without a remainder, persistent-grid caps, in place or not.
    Every run is compared element by element with the oracle; refusals must be UNSUPPORTED."""
    rng = np.random.default_rng(20241017)
    ran = 0
    for case in range(200):
        ndim = int(rng.integers(1, 4))
        r = int(rng.integers(1, 4))
        box = bool(rng.integers(0, 2)) or ndim == 1
        maxtf = {1: 15 // r, 2: 6 // r, 3: 2 if r == 1 else 1}[ndim]
        tf = int(rng.integers(1, max(1, maxtf) + 1))
        nk = 2 * r * tf + 1
        if ndim == 1:
            ext = (int(rng.integers(nk, 9000)),)
        elif ndim == 2:
            ext = tuple(int(rng.integers(nk, 300)) for _ in range(2))
        else:
            ext = tuple(int(rng.integers(nk, 60)) for _ in range(3))
        bc = ("fixed", "periodic")[int(rng.integers(0, 2))]
        engine = ("auto", "tc_tile", "tc_s2r", "direct")[int(rng.integers(0, 4))]
        T = int(rng.integers(1, 3 * tf + 2))
        cap = int((0, 0, 1, 3, 7)[int(rng.integers(0, 5))])
        w = synth.random_signed_weights(ndim, r, seed=1000 + case, box=box)
        u0 = synth.grid(ext, seed=2000 + case)
        try:
            p = csx.Plan(ext, w, shape="box" if box else "star", bc=bc, fuse_steps=tf, engine=engine)
        except csx.CsxError as e:
            assert e.status == csx.CSX_ERR_UNSUPPORTED, (case, ndim, r, tf, engine, str(e))
            continue
        if cap:
            p.set_max_ctas(cap)
        d_in = torch.from_numpy(u0).cuda()
        d_out = d_in if rng.integers(0, 4) == 0 else torch.empty_like(d_in)
        p.run(d_in, d_out, T)
        torch.cuda.synchronize()
        got = d_out.cpu().numpy()
        p.close()
        ref = oracle.run(u0, w, bc, T)
        assert rel(got, ref) <= TOL, (case, ndim, r, box, tf, ext, bc, engine, T, cap)
        ran += 1
    assert ran >= 120, ran


@pytest.mark.parametrize("geom", ["0", "1", "3", "4", "5", "6", "8", "a", "b", "c", "h", "t"])
def test_tb2_geometries(csx, monkeypatch, geom):
    """Every k_tile3d_tb2 / k_tile3d_tb3 geometry (CSX_TB_GEOM; a-c: tb3's strip tiles with three
    ring depths, t: the balanced-role tb2 32 x 64 tile):
    Heat-3D and Box-3D27P at Tf = 2, ragged tiles and z chunks, both boundaries, persistent grid
    capped at 3 CTAs and uncapped, element-wise against the oracle."""
    monkeypatch.setenv("CSX_TB_GEOM", geom)
    for name, ext in (("heat3d", (70, 61, 150)), ("box3d27p", (40, 57, 130)), ("heat3d", (9, 29, 65))):
        s = synth.SHAPES[name]
        w = synth.random_weights(name)
        u0 = synth.grid(ext, seed=5)
        for bc in ("fixed", "periodic"):
            ref = oracle.run(u0, w, bc, 5)
            for cap in (3, 0):
                got, info = run_gpu(csx, u0, w, s.kind, bc, 5, engine="tc_tile", fuse_steps=2, max_ctas=cap)
                assert info["fuse_steps"] == 2
                assert rel(got, ref) <= TOL, (geom, name, ext, bc, cap)


def test_heat3d_tf1_16_warps(csx, monkeypatch):
    """The 16-DMMA-warp Heat-3D Tf = 1 tile (CSX_TILE3D_W16 = 1, an A/B variant): ragged tiles,
    z chunks, both boundaries, capped and uncapped persistent grids."""
    monkeypatch.setenv("CSX_TILE3D_W16", "1")
    s = synth.SHAPES["heat3d"]
    w = synth.random_weights("heat3d")
    u0 = synth.grid((45, 70, 130), seed=11)
    for bc in ("fixed", "periodic"):
        ref = oracle.run(u0, w, bc, 3)
        for cap in (3, 0):
            got, _ = run_gpu(csx, u0, w, s.kind, bc, 3, engine="tc_tile", fuse_steps=1, max_ctas=cap)
            assert rel(got, ref) <= TOL, (bc, cap)
