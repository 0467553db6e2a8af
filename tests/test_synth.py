"""The seeded input generator (synth/) — holds no method arithmetic, only draws numbers."""
import numpy as np

import synth


def test_splitmix64_known_value():
    # First output of Vigna's splitmix64 from state 0 (published test value).
    assert int(synth.splitmix64(np.array([0], dtype=np.uint64))[0]) == 0xE220A8397B1DCDAF


def test_grid_deterministic_and_slab_consistent():
    g = synth.grid((50, 30))
    assert np.array_equal(g, synth.grid((50, 30)))
    assert np.array_equal(g[17:31], synth.grid((50, 30), rows=(17, 31)))
    assert g.min() >= 0.0 and g.max() < 1.0


def test_weights_sum_and_footprint():
    for name, s in synth.SHAPES.items():
        w = synth.physical_weights(name)
        assert w.sum() == 1.0
        assert np.all(w[~s.footprint()] == 0)
        rw = synth.random_weights(name)
        assert abs(rw.sum() - 1.0) < 1e-15
        assert np.all(rw[~s.footprint()] == 0) and np.all(rw[s.footprint()] > 0)
        assert int(np.count_nonzero(w)) == s.points


def test_points_match_paper_names():
    # Table 4 (P.1848-1859): point counts are part of the shape names.
    pts = {n: s.points for n, s in synth.SHAPES.items()}
    assert pts == {"heat1d": 3, "1d5p": 5, "heat2d": 5, "box2d9p": 9, "star2d13p": 13,
                   "box2d49p": 49, "heat3d": 7, "box3d27p": 27, "star2d9p": 9, "box2d25p": 25,
                   "star3d13p": 13, "box3d125p": 125, "star3d19p": 19, "box3d343p": 343}


def test_grid_window_and_torch_generator_match_grid():
    """The windowed and the torch (device-side) generators reproduce grid() bit for bit."""
    import torch
    ext = (37, 41, 29)
    full = synth.grid(ext)
    w = synth.grid_window(ext, (3, 5, 7), (20, 41, 28))
    assert np.array_equal(w, full[3:20, 5:41, 7:28])
    t = synth.grid_torch(ext, "cpu", chunk=1000).numpy()
    assert np.array_equal(t, full)
    big = (3000, 70001)  # flat indices past 2^27, several chunks
    tb = synth.grid_torch(big, "cpu", chunk=1 << 24)
    assert np.array_equal(tb[2999, -50:].numpy(), synth.grid_window(big, (2999, 69951), (3000, 70001))[0])
