"""Pins for the CPU oracle: values the paper prints, hand-worked examples,
closed forms, brute force and invariants -- never the oracle checked against
a retyped copy of itself. CPU only (no GPU marker)."""
import itertools
from collections import deque

import numpy as np
import pytest

import oracle

INF = oracle.INF_U32


def csr_from_arcs(V, arcs, wdtype=np.uint32):
    """Tiny CSR from directed arcs (u, v, w), arcs grouped by u in input order."""
    arcs = sorted(arcs, key=lambda a: a[0])  # stable: keeps input order per u
    row = np.zeros(V + 1, dtype=np.int64)
    for u, _, _ in arcs:
        row[u + 1] += 1
    row = np.cumsum(row).astype(np.int64)
    col = np.array([a[1] for a in arcs], dtype=np.uint32)
    w = np.array([a[2] for a in arcs], dtype=wdtype)
    return row, col, w


def undirected(edges):
    out = []
    for u, v, w in edges:
        out.append((u, v, w))
        out.append((v, u, w))
    return out


# ------------------------------------------------------------ Fig. 1 ----
def fig1_csr(golden):
    g = golden("fig1_csr.json")
    adj = g["adj_printed_rows_0_4"] + g["adj_rows_5_7_by_symmetry"]
    val = g["val_printed_rows_0_4"] + [g["w67"] if x == "w67" else x for x in g["val_rows_5_7_by_symmetry"]]
    return g, np.array(g["row"], np.int64), np.array(adj, np.uint32), np.array(val, np.uint32)


def test_fig1_csr_is_undirected(golden):
    """The printed rows 0-4 plus symmetry form a consistent undirected CSR."""
    g, row, col, w = fig1_csr(golden)
    arcs = {(u, int(col[e]), int(w[e])) for u in range(8) for e in range(row[u], row[u + 1])}
    assert len(arcs) == 26
    for u, v, ww in arcs:
        assert (v, u, ww) in arcs


def test_fig1_distances(golden):
    g, row, col, w = fig1_csr(golden)
    for fn in (oracle.dijkstra, oracle.bellman_ford):
        assert fn(row, col, w, 0).tolist() == g["dist_from_0"]


def test_fig1_light_heavy_of_vertex4(golden):
    """vertex 4's weights 1, 7, 1 are light, heavy, light at Delta=3."""
    g, row, col, w = fig1_csr(golden)
    ws = w[row[4]:row[5]]
    assert (ws < g["delta"]).tolist() == g["vertex4_light_mask"]


# ------------------------------------------------------------ Fig. 4 ----
def fig4_csr(golden, wdtype=np.uint32):
    g = golden("fig4_pro.json")
    arcs = sorted(undirected(g["edges"]), key=lambda a: (a[0], a[1]))
    return g, csr_from_arcs(g["V"], arcs, wdtype)


def test_fig4_degrees(golden):
    g, (row, col, w) = fig4_csr(golden)
    assert np.diff(row).tolist() == g["degrees"]


@pytest.mark.parametrize("wdtype", [np.uint32, np.float32])
def test_fig4_pro_exact(golden, wdtype):
    """Property-driven reordering reproduces every printed array of Fig. 4(c)."""
    g, (row, col, w) = fig4_csr(golden, wdtype)
    r = oracle.pro_reorder(row, col, w)
    assert r["new2old"].tolist() == g["new2old"]
    assert r["adj"].tolist() == g["adj"]
    assert r["val"].astype(np.int64).tolist() == g["val"]
    rl = oracle.pro_rowlist(r["row"], r["val"], g["delta"])
    assert rl.tolist() == g["rowlist"]
    assert rl[1::2][: g["V"]].tolist() == g["heavy_offsets"]
    assert (r["old2new"][r["new2old"]] == np.arange(g["V"])).all()


@pytest.mark.parametrize("delta", ["1", "2", "3", "5", "10"])
def test_fig4_heavy_offsets_other_delta(golden, delta):
    g, (row, col, w) = fig4_csr(golden)
    r = oracle.pro_reorder(row, col, w)
    assert oracle.pro_rowlist(r["row"], r["val"], float(delta)).tolist() == g["rowlist_by_delta"][delta]


def test_fig4_heavy_offsets_fractional_delta(golden):
    """u32 graphs round Delta up: light iff w < ceil(Delta) iff w < Delta."""
    g, (row, col, w) = fig4_csr(golden)
    r = oracle.pro_reorder(row, col, w)
    assert oracle.pro_rowlist(r["row"], r["val"], 2.5).tolist() == g["rowlist_by_delta"]["3"]


def test_fig4_all_pairs(golden):
    g, (row, col, w) = fig4_csr(golden)
    D = oracle.floyd_warshall(row, col, w)
    assert D.astype(np.int64).tolist() == g["dist"]
    for s in range(g["V"]):
        assert oracle.dijkstra(row, col, w, s).tolist() == g["dist"][s]
    # distances are invariant under the reordering (topology unchanged)
    r = oracle.pro_reorder(row, col, w)
    for s in range(g["V"]):
        dn = oracle.dijkstra(r["row"], r["adj"], r["val"], int(r["old2new"][s]))
        assert dn[r["old2new"]].tolist() == g["dist"][s]


def test_fig4_bucket_histogram(golden):
    """B_i = [i*Delta,(i+1)*Delta): from 0, d=[0,2,3,6,4], Delta=3 -> [2,2,1]."""
    g, (row, col, w) = fig4_csr(golden)
    d = oracle.dijkstra(row, col, w, 0)
    assert oracle.bucket_histogram(d, 3).tolist() == [2, 2, 1]


# ------------------------------------------------------------- f32 pin --
def test_f32_left_to_right_path(golden):
    g = golden("f32_path.json")
    w = np.array([np.float32(x) / np.float32(1 << 24) for x in g["u24_plus_1"]], dtype=np.float32)
    assert [hex(int(b)) for b in w.view(np.uint32)] == g["weight_bits"]
    edges = [(0, 1, w[0]), (1, 2, w[1]), (2, 3, w[2])]
    row, col, ww = csr_from_arcs(4, undirected(edges), np.float32)
    for fn in (oracle.dijkstra, oracle.bellman_ford):
        d = fn(row, col, ww, 0)
        assert [("0x%08x" % int(b)) for b in d.view(np.uint32)] == g["dist_bits"]
    assert "0x%08x" % int(d.view(np.uint32)[3]) != g["f64_once_rounded_d3_bits"]


def test_f32_bucket_index():
    """f32 bucket = (u32)(d * fl32(1/Delta)): 0.25 at Delta=0.1 -> 2.5 -> bucket 2."""
    d = np.array([0.0, 0.25, 0.0999, np.inf], dtype=np.float32)
    assert oracle.bucket_histogram(d, 0.1).tolist() == [2, 0, 1]


# -------------------------------------------------------- closed forms --
def test_unit_grid_is_manhattan():
    W, H = 7, 5
    edges = []
    for r in range(H):
        for c in range(W):
            if c + 1 < W:
                edges.append((r * W + c, r * W + c + 1, 1))
            if r + 1 < H:
                edges.append((r * W + c, (r + 1) * W + c, 1))
    row, col, w = csr_from_arcs(W * H, undirected(edges))
    s = 2 * W + 3
    d = oracle.dijkstra(row, col, w, s)
    exp = [abs(v // W - 2) + abs(v % W - 3) for v in range(W * H)]
    assert d.tolist() == exp


def test_path_prefix_sums():
    rng = np.random.default_rng(0)
    ws = rng.integers(1, 1000, size=50)
    row, col, w = csr_from_arcs(51, undirected([(i, i + 1, int(ws[i])) for i in range(50)]))
    assert oracle.dijkstra(row, col, w, 0).tolist() == [0] + np.cumsum(ws).tolist()
    d = oracle.dijkstra(row, col, w, 50)
    assert d.tolist() == (np.cumsum(ws[::-1])[::-1].tolist() + [0])


def test_star():
    ws = [5, 3, 9, 1, 7]
    row, col, w = csr_from_arcs(6, undirected([(0, i + 1, x) for i, x in enumerate(ws)]))
    assert oracle.dijkstra(row, col, w, 0).tolist() == [0] + ws
    assert oracle.dijkstra(row, col, w, 3).tolist() == [9, 14, 12, 0, 10, 16]


def test_unit_weights_equal_bfs_hops():
    import gen

    g = gen.kronecker(10, 8, seed=11)
    w1 = np.ones_like(g.w)
    src = int(gen.sample_sources(g, 1, seed=3)[0])
    hops = np.full(g.V, INF, dtype=np.int64)
    hops[src] = 0
    q = deque([src])
    while q:  # textbook BFS
        u = q.popleft()
        for e in range(g.row[u], g.row[u + 1]):
            v = int(g.col[e])
            if hops[v] == INF:
                hops[v] = hops[u] + 1
                q.append(v)
    assert (oracle.dijkstra(g.row, g.col, w1, src).astype(np.int64) == hops).all()


def test_unreachable_and_directed():
    row, col, w = csr_from_arcs(4, [(0, 1, 4), (2, 0, 1)])  # 2 -> 0 only; 3 isolated
    assert oracle.dijkstra(row, col, w, 0).tolist() == [0, 4, INF, INF]
    assert oracle.dijkstra(row, col, w, 2).tolist() == [1, 5, 0, INF]


def test_u32_overflow_detected():
    row, col, w = csr_from_arcs(3, [(0, 1, 0xFFFFFFF0), (1, 2, 0x20)])
    with pytest.raises(OverflowError):
        oracle.dijkstra(row, col, w, 0)


# ---------------------------------------------------------- brute force --
def random_tiny(rng, V, nE, wmax, f32=False):
    arcs = []
    for _ in range(nE):
        u, v = int(rng.integers(V)), int(rng.integers(V))  # self-loops, multi-edges allowed
        if f32:
            x = np.float32(int(rng.integers(0, 1 << 24)) + 1) / np.float32(1 << 24)
            if rng.random() < 0.1:
                x = np.float32(0.0)
            arcs.append((u, v, x))
        else:
            arcs.append((u, v, int(rng.integers(0, wmax + 1))))
        if rng.random() < 0.5:
            arcs.append((v, u, arcs[-1][2]))
    return csr_from_arcs(V, arcs, np.float32 if f32 else np.uint32)


def paths_min(row, col, w, s, f32):
    """Enumerate every simple path (DFS) and take the min left-to-right sum."""
    V = len(row) - 1
    best = [None] * V
    zero = np.float32(0) if f32 else 0

    def dfs(u, acc, seen):
        if best[u] is None or acc < best[u]:
            best[u] = acc
        for e in range(row[u], row[u + 1]):
            v = int(col[e])
            if v in seen:
                continue
            nacc = np.float32(acc + w[e]) if f32 else acc + int(w[e])
            dfs(v, nacc, seen | {v})

    dfs(s, zero, {s})
    if f32:
        return np.array([np.inf if b is None else b for b in best], dtype=np.float32)
    return np.array([INF if b is None else b for b in best], dtype=np.uint64)


def test_brute_force_u32():
    rng = np.random.default_rng(1)
    for trial in range(400):
        V = int(rng.integers(1, 8))
        row, col, w = random_tiny(rng, V, int(rng.integers(0, 14)), wmax=int(rng.choice([1, 3, 50])))
        D = oracle.floyd_warshall(row, col, w)
        for s in range(V):
            d = oracle.dijkstra(row, col, w, s)
            assert (d == oracle.bellman_ford(row, col, w, s)).all()
            exp = np.where(D[s] == np.iinfo(np.uint64).max, INF, D[s]).astype(np.uint64)
            assert (d.astype(np.uint64) == exp).all()
            assert (d.astype(np.uint64) == paths_min(row, col, w, s, False)).all()


def test_brute_force_f32():
    rng = np.random.default_rng(2)
    for trial in range(300):
        V = int(rng.integers(1, 8))
        row, col, w = random_tiny(rng, V, int(rng.integers(0, 14)), 0, f32=True)
        for s in range(V):
            d = oracle.dijkstra(row, col, w, s)
            assert (d.view(np.uint32) == oracle.bellman_ford(row, col, w, s).view(np.uint32)).all()
            assert (d.view(np.uint32) == paths_min(row, col, w, s, True).view(np.uint32)).all()


def test_dijkstra_vs_bellman_ford_medium():
    import gen

    for wt in ("u32", "f32"):
        g = gen.kronecker(11, 8, seed=5, weights=wt)
        for s in gen.sample_sources(g, 3, seed=9):
            a = oracle.dijkstra(g.row, g.col, g.w, int(s))
            b = oracle.bellman_ford(g.row, g.col, g.w, int(s))
            assert (a.view(np.uint32) == b.view(np.uint32)).all()


# ---------------------------------------------------------- certificate --
def test_certificate_accepts_and_rejects():
    import gen

    g = gen.kronecker(10, 8, seed=12)
    s = int(gen.sample_sources(g, 1, seed=1)[0])
    d = oracle.dijkstra(g.row, g.col, g.w, s)
    assert oracle.certificate(g.row, g.col, g.w, s, d) == -1
    reach = np.flatnonzero((d != INF) & (np.arange(g.V) != s))
    rng = np.random.default_rng(0)
    for v in rng.choice(reach, 20, replace=False):
        for delta in (-1, +1):
            bad = d.copy()
            bad[v] = np.uint32(int(bad[v]) + delta)
            assert oracle.certificate(g.row, g.col, g.w, s, bad) != -1
        bad = d.copy()
        bad[v] = INF
        assert oracle.certificate(g.row, g.col, g.w, s, bad) != -1
    bad = d.copy()
    bad[s] = 1
    assert oracle.certificate(g.row, g.col, g.w, s, bad) == g.V
    # an unreachable vertex given a finite value has no tight in-arc
    iso = np.flatnonzero(d == INF)
    if len(iso):
        bad = d.copy()
        bad[iso[0]] = 7
        assert oracle.certificate(g.row, g.col, g.w, s, bad) != -1


# ---------------------------------------------------------------- PRO ----
@pytest.mark.parametrize("wt", ["u32", "f32"])
def test_pro_invariants_random(wt):
    import gen

    g = gen.kronecker(9, 8, seed=21, weights=wt)
    r = oracle.pro_reorder(g.row, g.col, g.w)
    deg = np.diff(g.row)
    n2o = r["new2old"].astype(np.int64)
    nd = deg[n2o]
    assert (np.diff(nd) <= 0).all()  # descending degree
    ties = np.flatnonzero(np.diff(nd) == 0)
    assert (n2o[ties] < n2o[ties + 1]).all()  # ties by ascending original id
    assert (np.diff(r["row"]) == nd).all()
    # each segment sorted by (weight, new id) and a relabelled copy of the old one
    o2n = r["old2new"]
    for i in range(g.V):
        a, b = r["row"][i], r["row"][i + 1]
        seg = list(zip(r["val"][a:b].view(np.uint32).tolist(), r["adj"][a:b].tolist()))
        assert seg == sorted(seg)
        o = n2o[i]
        old = sorted(zip(g.w[g.row[o]:g.row[o + 1]].view(np.uint32).tolist(),
                         o2n[g.col[g.row[o]:g.row[o + 1]]].tolist()))
        assert seg == old


def test_pro_rowlist_heavy_is_lower_bound():
    import gen

    g = gen.kronecker(9, 8, seed=22)
    r = oracle.pro_reorder(g.row, g.col, g.w)
    for delta in (1, 7, 32, 100, 101, 1e9):
        rl = oracle.pro_rowlist(r["row"], r["val"], delta)
        for i in range(0, g.V, 7):
            a, b = r["row"][i], r["row"][i + 1]
            assert rl[2 * i] == a
            assert rl[2 * i + 1] == a + np.searchsorted(r["val"][a:b], np.ceil(delta), side="left")
