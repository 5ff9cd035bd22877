"""Input generator checks (shared input machinery; CPU only)."""
import numpy as np

import gen


def test_thresholds_match_graph500_probabilities():
    """Integer thresholds of gen.c encode A=.57 B=.19 C=.19 D=.05."""
    A, B, C, D = 0.57, 0.19, 0.19, 0.05
    T_ab, T_a, T_c = 3264175145, 3221225472, 3400182443
    assert abs((1 - T_ab / 2**32) - (C + D)) < 1e-9
    assert abs((1 - T_a / 2**32) - B / (A + B)) < 1e-9
    assert abs((1 - T_c / 2**32) - D / (C + D)) < 1e-9


def test_quadrant_frequencies():
    src, dst = gen.kronecker_edges(1, edgefactor=1 << 17, seed=3, scramble=False)
    q = np.bincount(src.astype(np.int64) * 2 + dst, minlength=4) / len(src)
    assert np.allclose(q, [0.57, 0.19, 0.19, 0.05], atol=0.005)


def test_scramble_is_bijection():
    for scale in (1, 2, 5, 10, 11):
        img = sorted(gen.scramble(x, scale, 17) for x in range(1 << scale))
        assert img == list(range(1 << scale))


def test_deterministic_and_thread_independent():
    a = gen.kronecker(12, 8, seed=9, nthreads=1)
    b = gen.kronecker(12, 8, seed=9, nthreads=7)
    assert (a.row == b.row).all() and (a.col == b.col).all() and (a.w == b.w).all()
    c = gen.kronecker(12, 8, seed=10)
    assert not (len(c.col) == len(a.col) and (c.col == a.col).all())


def test_csr_structure():
    g = gen.kronecker(12, 16, seed=1)
    assert g.row[0] == 0 and (np.diff(g.row) >= 0).all() and g.row[-1] == len(g.col)
    assert g.col.max() < g.V and g.w.min() >= 1 and g.w.max() <= 100
    u = np.repeat(np.arange(g.V), np.diff(g.row))
    assert (u != g.col).all()  # self-loops dropped
    fwd = np.sort(u.astype(np.int64) * g.V + g.col)
    rev = np.sort(g.col.astype(np.int64) * g.V + u)
    assert (fwd == rev).all()  # symmetric
    for v in range(0, g.V, 97):  # adjacency sorted by dst
        assert (np.diff(g.col[g.row[v]:g.row[v + 1]].astype(np.int64)) >= 0).all()


def test_f32_weights_range_and_exact():
    g = gen.kronecker(10, 8, seed=2, weights="f32")
    assert g.w.min() > 0 and g.w.max() <= 1
    scaled = g.w.astype(np.float64) * (1 << 24)
    assert (scaled == np.round(scaled)).all()


def test_grid_shape():
    g = gen.grid(50, 40, p=0.2, seed=2)
    assert g.V == 2000
    deg = np.diff(g.row)
    assert deg.max() <= 4 and deg.min() >= 1
    assert 2.2 < g.A / g.V < 2.6  # road_USA-like average degree
    u = np.repeat(np.arange(g.V), deg)
    d = np.abs(u - g.col.astype(np.int64))
    assert set(np.unique(d).tolist()) <= {1, 50}


def test_sources_have_degree():
    g = gen.kronecker(12, 16, seed=1)
    s = gen.sample_sources(g, 64, seed=7)
    assert len(s) == 64 and len(set(s.tolist())) == 64
    assert (np.diff(g.row)[s] > 0).all()
