"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (default parameters, PRO on, the configs' Delta). Distances are compared
element by element with the oracle for sampled sources; further sources are
checked with the shortest-path certificate (a complete proof for integer
weights >= 1). PRO is checked against the oracle at C1 and by its
defining properties at C4."""
import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

INF = oracle.INF_U32


@pytest.fixture(scope="module")
def sssp():
    import torch

    assert torch.cuda.is_available()
    import paper_conf_icppw_zhangczsdhay23_b200 as m

    return m


_graphs = {}


def graph(name):
    if name not in _graphs:
        _graphs[name] = gen.make_config(name)
    return _graphs[name]


def check(got, exp, what):
    gb, eb = got.view(np.uint32), exp.view(np.uint32)
    bad = np.flatnonzero(gb != eb)
    assert len(bad) == 0, f"{what}: {len(bad)} mismatches, first {bad[:5].tolist()}"


@pytest.mark.parametrize("name,n_exact,n_cert", [("C1", 4, 8), ("C3", 1, 0), ("C2", 1, 1), ("C4", 1, 3)])
def test_config_parity(sssp, name, n_exact, n_cert):
    g = graph(name)
    delta = gen.CONFIGS[name]["delta"]
    srcs = gen.sample_sources(g, n_exact + n_cert, seed=7)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)  # as bench.py (symmetric generator graphs)
        for i, s in enumerate(srcs):
            got = G.sssp(int(s), delta).copy()
            st = G.stats()
            reach = int((got.view(np.uint32) != (0x7F800000 if g.wtype == "f32" else INF)).sum())
            assert st["reachable"] == reach
            if i < n_exact:
                check(got, oracle.dijkstra(g.row, g.col, g.w, int(s)), f"{name} src={s}")
            else:
                assert oracle.certificate(g.row, g.col, g.w, int(s), got) == -1, f"{name} certificate src={s}"
            if g.wtype == "u32":
                assert st["updates"] >= reach - 1


def test_c1_delta_sweep_and_reorder_off(sssp):
    g = graph("C1")
    s = int(gen.sample_sources(g, 1, seed=11)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        for d in (8, 16, 64):
            check(G.sssp(s, d), exp, f"C1 reorder off delta={d}")
        G.reorder()
        for d in (8, 16, 64):
            check(G.sssp(s, d), exp, f"C1 reorder on delta={d}")


def test_c1_pro_matches_oracle(sssp):
    g = graph("C1")
    ref = oracle.pro_reorder(g.row, g.col, g.w)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        ex = G.export_csr(32)
    assert np.array_equal(ex["new2old"], ref["new2old"])
    assert np.array_equal(ex["adj"], ref["adj"])
    assert np.array_equal(ex["val"], ref["val"])
    assert np.array_equal(ex["rowlist"], oracle.pro_rowlist(ref["row"], ref["val"], 32))


def test_c4_pro_properties(sssp):
    """PRO at scale 24: degree order, ties by id, segments sorted by (w, new dst),
    heavy offsets = first w >= Delta, multiset of arcs preserved (order-free sum of hashed triples)."""
    g = graph("C4")
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        ex = G.export_csr(32)
    n2o = ex["new2old"].astype(np.int64)
    deg = np.diff(g.row)
    assert np.array_equal(np.sort(n2o), np.arange(g.V))
    nd = deg[n2o]
    assert (np.diff(nd) <= 0).all()
    ties = np.flatnonzero(np.diff(nd) == 0)
    assert (n2o[ties] < n2o[ties + 1]).all()
    rl = ex["rowlist"]
    starts = rl[0:-1:2]
    assert np.array_equal(np.diff(np.append(starts, rl[-1])), nd)
    key = (ex["val"].astype(np.uint64) << np.uint64(32)) | ex["adj"].astype(np.uint64)
    inc = key[1:] >= key[:-1]
    boundary = np.zeros(len(key) - 1, dtype=bool)
    b = starts[1:] - 1
    boundary[b[(b >= 0) & (b < len(boundary))]] = True
    assert (inc | boundary).all()
    heavy = rl[1:-1:2]
    ends = np.append(starts[1:], rl[-1])
    assert ((heavy >= starts) & (heavy <= ends)).all()
    w = ex["val"]
    hv = heavy[heavy < ends]
    assert (w[hv] >= 32).all()
    hl = heavy[heavy > starts]
    assert (w[hl - 1] < 32).all()
    # the arc multiset is preserved: relabel back and compare order-free checksums
    o2n = np.empty(g.V, dtype=np.int64)
    o2n[n2o] = np.arange(g.V)
    src_old = np.repeat(np.arange(g.V, dtype=np.int64), deg)
    h_ref = np.uint64(0)
    h_new = np.uint64(0)
    mix = lambda a, b, c: ((a * np.uint64(0x9E3779B97F4A7C15)) ^ (b * np.uint64(0xC2B2AE3D27D4EB4F))
                           ^ (c * np.uint64(0x165667B19E3779F9)))
    with np.errstate(over="ignore"):
        h_ref = np.sum(mix(o2n[src_old].astype(np.uint64), o2n[g.col].astype(np.uint64),
                                          g.w.astype(np.uint64)), dtype=np.uint64)
        src_new = np.repeat(np.arange(g.V, dtype=np.int64), nd)
        h_new = np.sum(mix(src_new.astype(np.uint64), ex["adj"].astype(np.uint64),
                                          ex["val"].astype(np.uint64)), dtype=np.uint64)
    assert h_ref == h_new


@pytest.mark.parametrize("name,n_exact", [("C4", 1), ("C3", 1), ("C1", 4)])
def test_multi_source_full_size(sssp, name, n_exact):
    """sssp_run_multi at full size in the bench --multi launch configuration
    (one 32-source group, bench.MULTI_DELTA): rows bit-exact against the oracle
    for the first sources, the shortest-path certificate for the other rows of
    u32 configs, and every row equal to the single-source kernel's result for
    a sample of lanes (both paths must give the unique distances)."""
    import torch

    import bench

    g = graph(name)
    delta = bench.MULTI_DELTA[name]
    srcs = [int(s) for s in gen.sample_sources(g, 32, seed=7)]
    f32 = g.wtype == "f32"
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        out = torch.empty((32, g.V), dtype=torch.float32 if f32 else torch.int32, device="cuda")
        G.run_multi(srcs, delta, out)
        rows = out.cpu().numpy()
        for i in range(n_exact):
            check(rows[i], oracle.dijkstra(g.row, g.col, g.w, srcs[i]), f"{name} multi src={srcs[i]}")
        if not f32:
            for i in (5, 17, 31):
                assert oracle.certificate(g.row, g.col, g.w, srcs[i], rows[i]) == -1, f"{name} multi cert lane {i}"
        for i in (2, 9, 30):
            check(rows[i], G.sssp(srcs[i], gen.CONFIGS[name]["delta"]).copy(), f"{name} multi vs single lane {i}")


def test_c5_full_size_certificates(sssp):
    """C5 (Kronecker scale 26, 2.1 G arcs, int64 row offsets) in both bench launch
    configurations: one single-source run (config Delta) and one 32-source
    sssp_run_multi group (bench.MULTI_DELTA), each checked with the complete
    shortest-path certificate (u32 weights >= 1: d[s] = 0, every arc satisfied,
    every reachable vertex tight on some arc, unreachable = no finite neighbour)."""
    import torch

    import bench

    g = graph("C5")
    srcs = [int(s) for s in gen.sample_sources(g, 32, seed=7)]
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)  # as bench.py
        d = G.sssp(srcs[0], gen.CONFIGS["C5"]["delta"]).copy()
        assert oracle.certificate(g.row, g.col, g.w, srcs[0], d) == -1, "C5 single-source certificate"
        out = torch.empty((32, g.V), dtype=torch.int32, device="cuda")
        G.run_multi(srcs, bench.MULTI_DELTA["C5"], out)
        for i in (0, 13, 31):
            row = out[i].cpu().numpy().view(np.uint32)
            assert oracle.certificate(g.row, g.col, g.w, srcs[i], row) == -1, f"C5 multi certificate lane {i}"
        assert np.array_equal(out[0].cpu().numpy().view(np.uint32), d.view(np.uint32))
    _graphs.pop("C5", None)
