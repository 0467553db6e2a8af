"""Host logic of libcsx.so (no GPU needed): the C-ABI loads and exports what include/csx.h
declares, and the planner reproduces the paper's worked examples.

Pins (each a value printed in the paper or a closed form, not a re-typed formula):
  Fig 2 stencil2row letters           tests/golden/fig2_stencil2row.txt   (Eq 5/6, P.731-785)
  Fig 3 weight matrices               tests/golden/fig3_weight_matrices.txt (P.961-975)
  Table 3 memory expansion factors    tests/golden/table3_memory.txt      (Eq 7-11, P.814-898)
  Fig 5 bank rule: pitch 266 conflicts, 268 does not                      (P.1736-1757)
  First tessellation = centres [3][3:66]                                   (P.1326-1330)
  Eq 13 DMMA count                                                         (P.1512-1524)
  Fig 4 fusion: 3 x (3x3) = 7x7, equal to 3 oracle steps on a torus         (P.1466-1482)
"""
import os
import re

import numpy as np
import pytest

import oracle
import synth
import paper_conf_ppopp_chenlwbwmyzcy24_b200 as csx

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def letters(n):
    return [chr(ord("A") + i) for i in range(n)]


def test_library_exports_every_declared_symbol():
    decl = open(os.path.join(ROOT, "include", "csx.h")).read()
    names = set(re.findall(r"\b(csx_[a-z0-9_]+)\s*\(", decl))
    assert len(names) >= 15
    for n in names:
        assert hasattr(csx._lib, n), n
    assert names == set(csx.EXPORTED)


def _s2r_matrices(nk, m, n):
    """Apply the library's Eq 5/6 mapping to a lettered m x n input."""
    A, B = {}, {}
    for x in range(m):
        for y in range(n):
            lab = letters(m)[x] + letters(n)[y]
            for which, M in ((0, A), (1, B)):
                rc = csx.csx_stencil2row_index(nk, which, x, y)
                if rc is not None:
                    M[rc] = lab
    def rows(M):
        out = {}
        for (r, c), lab in M.items():
            out.setdefault(r, {})[c] = lab
        return {r: [d[c] for c in sorted(d)] for r, d in out.items()}
    return rows(A), rows(B)


def test_fig2_stencil2row_letters():
    A, B = _s2r_matrices(7, 8, 22)
    gold = {}
    for line in open(os.path.join(GOLDEN, "fig2_stencil2row.txt")):
        if line.startswith("#") or not line.strip():
            continue
        k, v = line.split(":")
        gold[k.strip()] = v.split()
    assert A[0][:14] == gold["A0"]
    assert A[0][-14:] == gold["A0_tail_from_row_G"]
    assert A[1][:7] == gold["A1"]
    assert A[1][-14:] == gold["A1_tail_from_row_G"]
    assert B[0][:7] == gold["B0"]
    assert B[0][-14:] == gold["B0_tail_from_row_G"]
    assert B[1][:7] == gold["B1"]
    assert B[1][-14:] == gold["B1_tail_from_row_G"]
    # Eq 7 / Eq 8: m_s2r = n/(nk+1) rows, n_s2r = nk*m columns (here n = 22 -> 2 full rows + part)
    assert len(A[0]) == 7 * 8 and len(A[1]) == 7 * 8


def test_fig3_weight_matrices():
    a = np.arange(1, 50, dtype=np.float64).reshape(7, 7)  # a1..a49 row-major
    wa, wb = csx.csx_weight_matrices(a)
    assert wa.shape == (49, 8) and wb.shape == (49, 8)
    def sym(v):
        return "0" if v == 0 else f"a{int(v)}"
    for line in open(os.path.join(GOLDEN, "fig3_weight_matrices.txt")):
        if line.startswith("#") or not line.strip():
            continue
        head, vals = line.split(":")
        mat, row = head.split()
        row = int(row)
        vals = vals.split()
        if mat == "WA":
            assert [sym(v) for v in wa[row, :7]] == vals, row
            assert wa[row, 7] == 0.0
        else:
            assert [sym(v) for v in wb[row, 1:7]] == vals, row
            assert wb[row, 0] == 0.0
    # survey check: W_B row 0 = 0 a7 a6 a5 a4 a3 a2 a1, row 48 = 0 ... 0 a49
    assert [sym(v) for v in wb[0]] == ["0", "a7", "a6", "a5", "a4", "a3", "a2", "a1"]
    assert [sym(v) for v in wb[48]] == ["0"] * 7 + ["a49"]


@pytest.mark.parametrize("nk", [3, 5, 7])
def test_dual_tessellation_first_tile_centres(nk):
    """Tile_A . W_A + Tile_B . W_B (numpy GEMM on the library's matrices and Eq 5/6 mapping)
    equals the direct window sum at the centres; for nk = 7 these are [3][3:66] (P.1329-1330)."""
    r = (nk - 1) // 2
    m, n = nk + 2, 8 * (nk + 1) + nk
    X = synth.grid((m, n), seed=3)
    w = synth.uniform01(11, 0, nk * nk).reshape(nk, nk) - 0.5  # asymmetric
    wa, wb = csx.csx_weight_matrices(w)
    # build stencil2row A and B through the mapping
    rows = n // (nk + 1) + 1
    SA = np.zeros((rows, nk * m + 8))
    SB = np.zeros((rows, nk * m + 8))
    for x in range(m):
        for y in range(n):
            for which, S in ((0, SA), (1, SB)):
                rc = csx.csx_stencil2row_index(nk, which, x, y)
                if rc is not None:
                    S[rc] = X[x, y]
    # the first tessellation: tile rows 0..7, columns [0, nk^2) (Eq 12, i = 0)
    TA = SA[:8, :nk * nk]
    TB = SB[:8, :nk * nk]
    res = TA @ wa + TB @ wb          # 8 x (nk+1): strip g, output column c
    out = res.reshape(-1)             # 8 (nk+1) contiguous outputs
    ref = oracle.run(X, w, "periodic", 1)[r, r:r + 8 * (nk + 1)]
    assert np.max(np.abs(out - ref)) < 1e-14
    if nk == 7:
        assert (r, r, r + 8 * (nk + 1) - 1) == (3, 3, 66)


def test_table3_memory_factors():
    for line in open(os.path.join(GOLDEN, "table3_memory.txt")):
        if line.startswith("#") or not line.strip():
            continue
        name, nk, im2row, s2r, saving = line.split()
        nk, im2row, s2r, saving = int(nk), int(im2row), float(s2r), float(saving)
        n = 2000 * (nk + 1)
        cnt = 0
        for y in range(n):
            for which in (0, 1):
                cnt += csx.csx_stencil2row_index(nk, which, 0, y) is not None
        factor = cnt / n  # elements of A and B per input element (same for every row x)
        assert abs(factor - s2r) <= 0.0051 and abs(factor - 2 * nk / (nk + 1)) < 1e-3
        closed = 100.0 * (1 - (2 * nk / (nk + 1)) / im2row)
        assert abs(closed - saving) <= 0.011  # 81.48 vs printed 81.49 (reading A13)


def test_fig5_bank_rule():
    assert max(csx.csx_fragment_bank_conflicts(266, c) for c in range(16)) == 2
    assert max(csx.csx_fragment_bank_conflicts(268, c) for c in range(16)) == 1
    for p in range(200, 300):
        ok = max(csx.csx_fragment_bank_conflicts(p, c) for c in range(16)) == 1
        assert ok == (p % 16 in (4, 12))


def test_fusion_composition_equals_steps():
    w = synth.random_weights("box2d9p")
    wc = csx.csx_compose_weights(w, 3)
    assert wc.shape == (7, 7)
    assert abs(wc.sum() - 1.0) < 1e-15
    u0 = synth.grid((20, 24), seed=8)
    a = oracle.run(u0, wc, "periodic", 1)
    b = oracle.run(u0, w, "periodic", 3)
    assert np.max(np.abs(a - b)) < 1e-15
    # Fig 4: Box-2D9P composed twice more is a 7x7 (Box-2D49P-like) kernel with full support
    assert np.all(csx.csx_compose_weights(synth.physical_weights("box2d9p"), 3) > 0)


@pytest.mark.parametrize("name,ext", [("box2d9p", (320, 640)), ("box2d49p", (256, 512)),
                                      ("heat2d", (128, 96)), ("star2d13p", (64, 64))])
def test_eq13_mma_count(name, ext):
    s = synth.SHAPES[name]
    p = csx.Plan(ext, synth.physical_weights(name), shape=s.kind, engine="tc_s2r")
    info = p.info()
    nk = info["nk"]
    m, n = ext
    eq13 = 2 * m * n / (8 * (nk + 1)) * -(-nk * nk // 4)
    assert info["mma_per_pass"] == round(eq13)
    assert info["engine_name"] == "tc_s2r"
    p.close()


def test_plan_lut_structure():
    p = csx.Plan((320, 640), synth.physical_weights("box2d9p"), engine="tc_s2r")
    info = p.info()
    nk, pitch = info["nk"], info["s2r_pitch"]
    la, lb = p.lut()
    rr, rc = la.shape
    assert (rr, rc) == (32 + nk - 1, 8 * (nk + 1) + nk - 1) == (38, 70)  # Fig 5 tile
    assert pitch == 268                                                  # Fig 5: 266 -> 268
    dirty = 8 * pitch
    # every slot of the 8 stencil2row rows (first nk*rr columns) is written exactly once
    for L, off in ((la, 0), (lb, nk)):
        live = L[L < dirty]
        assert len(np.unique(live)) == len(live) == 8 * nk * rr
        assert np.all(L[L >= dirty] < 9 * pitch)
    p.close()


def test_plan_validation():
    w = synth.physical_weights("heat2d")
    with pytest.raises(csx.CsxError):
        csx.Plan((4, 4), w, shape="star", fuse_steps=3)  # grid smaller than the window
    bad = w.copy()
    bad[0, 0] = 0.1
    with pytest.raises(csx.CsxError):
        csx.Plan((64, 64), bad, shape="star")             # off-axis star weight
    with pytest.raises(csx.CsxError):
        csx.Plan((64, 64), np.full((3, 3), np.nan))
    p = csx.Plan((64, 64), w, shape="star")
    with pytest.raises(csx.CsxError):
        p.set_engine("tc_s2r") or csx.csx_plan_set_engine(p.handle, 99)
    p.close()


def test_1d_fusion_limits():
    """1D: TC_TILE (Toeplitz 8-output blocks, K = nk + 7 rounded up to 4) runs nk <= 31, the
    paper's stencil2row layout (TC_S2R, nf <= 2) nk <= 15; nk = 33 is refused."""
    w = synth.physical_weights("heat1d")
    p = csx.Plan((4096,), w, fuse_steps=15, engine="tc_tile")
    info = p.info()
    assert info["nk"] == 31
    assert info["mma_per_pass"] == 4096 // 64 * 10
    with pytest.raises(csx.CsxError):
        p.set_engine("tc_s2r")
    p.set_engine("auto")
    p.close()
    p = csx.Plan((4096,), w, fuse_steps=7, engine="tc_tile")
    assert p.info()["mma_per_pass"] == 4096 // 64 * 6      # nk = 15: K = 22 -> 24
    p.set_engine("tc_s2r")                                   # Eq 13: 2 ceil(15/4) nf=2 per 8x16
    assert p.info()["mma_per_pass"] == 4096 // (8 * 16) * 2 * 4 * 2
    p.close()
    with pytest.raises(csx.CsxError):
        csx.Plan((4096,), w, fuse_steps=16)


def test_2d_fusion_limits():
    """2D: TC_TILE runs composed windows up to nk = 13 (C3's "multi-step fused" r = 3, Tf = 2)
    with the block shape of smaller K: nk = 9 -> 2x4 (K = 120), 11 -> 4x2 (168), 13 -> 2x4
    (224); the paper's layout (TC_S2R, one N fragment) stops at nk = 7; nk = 15 is refused."""
    ext = (640, 512)
    pts = ext[0] * ext[1]
    for name, tf, nk, ks in (("box2d9p", 4, 9, 30), ("box2d9p", 5, 11, 42),
                             ("box2d49p", 2, 13, 56), ("star2d13p", 2, 13, 56), ("box2d25p", 3, 13, 56)):
        s = synth.SHAPES[name]
        p = csx.Plan(ext, synth.physical_weights(name), shape=s.kind, fuse_steps=tf)
        info = p.info()
        assert info["nk"] == nk and info["engine_name"] == "tc_tile", name
        assert info["mma_per_pass"] == pts // 64 * ks, name
        with pytest.raises(csx.CsxError):
            p.set_engine("tc_s2r")
        p.set_engine("direct")
        p.close()
    with pytest.raises(csx.CsxError):
        csx.Plan(ext, synth.physical_weights("box2d9p"), shape="box", fuse_steps=7)


def test_auto_fusion_depths():
    # (3D r = 1 stars run two steps per pass by temporal blocking; boxes and r >= 2 one)
    cases = {"heat1d": 13, "1d5p": 7, "heat2d": 2, "box2d9p": 2, "star2d13p": 1, "box2d49p": 1,
             "heat3d": 2, "box3d27p": 1, "star3d13p": 1, "box3d125p": 1}
    for name, tf in cases.items():
        s = synth.SHAPES[name]
        ext = {1: (4096,), 2: (128, 128), 3: (32, 32, 32)}[s.ndim]
        p = csx.Plan(ext, synth.physical_weights(name), shape=s.kind)
        assert p.info()["fuse_steps"] == tf, name
        p.close()
    # an explicit engine gets its own automatic depth: the paper's 1D layout keeps nk + 1 <= 16
    for name, tf in {"heat1d": 7, "1d5p": 3}.items():
        p = csx.Plan((4096,), synth.physical_weights(name), engine="tc_s2r")
        assert p.info()["fuse_steps"] == tf and p.info()["engine_name"] == "tc_s2r", name
        p.close()
    # 2D r = 1: TC_TILE fuses 2 steps on B200, the paper's layout (TC_S2R) keeps its 3
    p = csx.Plan((128, 128), synth.physical_weights("box2d9p"), engine="tc_s2r")
    assert p.info()["fuse_steps"] == 3 and p.info()["nk"] == 7
    p.close()
    assert csx._lib.csx_auto_fuse_steps(1, 3, csx.ENGINES["tc_tile"]) == 3
    # the CUDA-core comparator's own depth (2D r = 1: 4 steps)
    assert csx._lib.csx_auto_fuse_steps(2, 1, csx.ENGINES["direct"]) == 4
    p = csx.Plan((64, 64), synth.physical_weights("box2d9p"), engine="direct")
    assert p.info()["fuse_steps"] == 4
    p.close()
    assert csx._lib.csx_auto_fuse_steps(4, 1, 0) == 0


def test_shard_rows_partition():
    p = csx.Plan((1003, 64), synth.physical_weights("box2d9p"))
    for nr in (1, 2, 3, 8):
        spans = [p.shard_rows(i, nr) for i in range(nr)]
        assert spans[0][0] == 0 and spans[-1][1] == 1003
        assert all(a[1] == b[0] for a, b in zip(spans, spans[1:]))
        assert max(h - l for l, h in spans) - min(h - l for l, h in spans) <= 1
    p.close()


def test_s2r_variant_tables():
    """Breakdown variants: no padding -> pitch 266 (Fig 5); no dirty bits -> sentinel entries."""
    p = csx.Plan((320, 640), synth.physical_weights("box2d9p"), engine="tc_s2r")
    p.set_s2r_variant(padding=False, dirty_bits=False)
    assert p.info()["s2r_pitch"] == 266
    la, lb = p.lut()
    assert np.count_nonzero(la == 0xFFFF) > 0 and np.count_nonzero(lb == 0xFFFF) > 0
    live = la[la != 0xFFFF]
    assert len(np.unique(live)) == len(live) == 8 * 7 * 38
    p.set_s2r_variant(padding=True, dirty_bits=True)
    assert p.info()["s2r_pitch"] == 268
    p.set_s2r_variant(padding=3)  # breakdown I: explicit stencil2row (same LUT/pitch tables)
    assert p.info()["s2r_pitch"] == 268
    assert csx._lib.csx_plan_set_s2r_variant(p.handle, 4, 1) == csx.CSX_ERR_INVALID_ARGUMENT
    p.close()
    q = csx.Plan((4096,), synth.physical_weights("heat1d"), engine="tc_s2r")
    assert csx._lib.csx_plan_set_s2r_variant(q.handle, 3, 1) == csx.CSX_ERR_UNSUPPORTED
    q.close()


def test_run_argument_validation_without_gpu():
    """csx_run / csx_run_sharded reject bad pointers synchronously, before touching a device."""
    import ctypes
    p = csx.Plan((64, 64), synth.physical_weights("box2d9p"))
    lib, h = csx._lib, p.handle
    vp = ctypes.c_void_p
    n = 64 * 64
    assert lib.csx_run(h, None, vp(0x10000), 1, None) == csx.CSX_ERR_INVALID_ARGUMENT
    assert lib.csx_run(h, vp(0x10001), vp(0x90000), 1, None) == csx.CSX_ERR_INVALID_ARGUMENT  # misaligned
    assert lib.csx_run(h, vp(0x10000), vp(0x10000 + 8 * (n // 2)), 1, None) == csx.CSX_ERR_INVALID_ARGUMENT  # overlap
    assert "overlap" in csx._lib.csx_last_error().decode()
    assert lib.csx_run(h, vp(0x10000), vp(0x90000), -1, None) == csx.CSX_ERR_INVALID_ARGUMENT
    assert "timesteps" in csx._lib.csx_last_error().decode()
    assert lib.csx_run(None, vp(0x10000), vp(0x90000), 1, None) == csx.CSX_ERR_INVALID_ARGUMENT
    assert "NULL" in csx._lib.csx_last_error().decode()
    assert lib.csx_plan_set_max_ctas(h, -1) == csx.CSX_ERR_INVALID_ARGUMENT
    assert lib.csx_plan_set_max_ctas(h, 3) == csx.CSX_OK
    p.close()


def test_status_strings():
    for code in range(7):
        assert csx._lib.csx_status_string(code).decode().startswith("CSX_")


@pytest.mark.parametrize("geom, l1_tiles, rows, cols", [
    (None, 45, 32, 64), ("t", 45, 32, 64), ("1", 45, 32, 64), ("a", 39, 32, 64), ("c", 39, 32, 64),
    ("3", 40, 28, 64), ("0", 36, 32, 62), ("h", 25, 16, 64)])
def test_3d_two_step_mma_count(monkeypatch, geom, l1_tiles, rows, cols):
    """3D Tf = 2 (temporal blocking of the base r = 1 window): the planner's DMMA count per pass
    follows the geometry CSX_TB_GEOM selects — (level-1 DMMA tiles x 34/32 planes + level-2
    tiles) x 6 DMMAs per tile and TC plane, over the output tile's points: 1 TC plane for
    Heat-3D, 3 for Box-3D27P."""
    if geom is None:
        monkeypatch.delenv("CSX_TB_GEOM", raising=False)
    else:
        monkeypatch.setenv("CSX_TB_GEOM", geom)
    ext = (64, 96, 128)
    pts = ext[0] * ext[1] * ext[2]
    l2_tiles = rows // 4 * 4
    per_pt = (l1_tiles * 34 / 32 + l2_tiles) * 6 / (rows * cols)
    for name, ntc in (("heat3d", 1), ("box3d27p", 3)):
        s = synth.SHAPES[name]
        p = csx.Plan(ext, synth.physical_weights(name), shape=s.kind, fuse_steps=2)
        assert p.info()["mma_per_pass"] == int(pts * per_pt * ntc + 0.5), (geom, name)
        p.close()
