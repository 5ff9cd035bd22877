"""GPU parity: the CUDA path (through the C-ABI) vs the CPU oracle, element by
element, on seeded inputs. u32 distances must be bit-exact; f32 distances are
bit-exact too (the f32 result is the unique min over left-to-right binary32
path sums), which is stricter than north_star's 1e-6."""
import math

import numpy as np
import pytest

import gen
import oracle

pytestmark = pytest.mark.gpu

INF = oracle.INF_U32


@pytest.fixture(scope="module")
def sssp():
    import torch

    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import __graft_entry__

    __graft_entry__.build_cuda()
    import paper_conf_icppw_zhangczsdhay23_b200 as m

    return m


def bits(a):
    return np.ascontiguousarray(a).view(np.uint32)


def assert_same(got, exp, what=""):
    gb, eb = bits(got), bits(exp)
    if not np.array_equal(gb, eb):
        bad = np.flatnonzero(gb != eb)
        raise AssertionError(f"{what}: {len(bad)} mismatches; first {bad[:8].tolist()} "
                             f"got {gb[bad[:8]].tolist()} exp {eb[bad[:8]].tolist()}")


def csr_from_arcs(V, arcs, wdtype=np.uint32):
    arcs = sorted(arcs, key=lambda a: a[0])
    row = np.zeros(V + 1, dtype=np.int64)
    for u, _, _ in arcs:
        row[u + 1] += 1
    row = np.cumsum(row).astype(np.int64)
    col = np.array([a[1] for a in arcs], dtype=np.uint32)
    w = np.array([a[2] for a in arcs], dtype=wdtype)
    return row, col, w


# ------------------------------------------------------ paper examples ----
def test_fig4_pro_on_gpu(sssp, golden):
    g = golden("fig4_pro.json")
    arcs = []
    for u, v, w in g["edges"]:
        arcs += [(u, v, w), (v, u, w)]
    arcs.sort(key=lambda a: (a[0], a[1]))
    for wd in (np.uint32, np.float32):
        row, col, w = csr_from_arcs(g["V"], arcs, wd)
        with sssp.Graph(row, col, w) as G:
            G.reorder()
            ex = G.export_csr(g["delta"])
            assert ex["new2old"].tolist() == g["new2old"]
            assert ex["rowlist"].tolist() == g["rowlist"]
            assert ex["adj"].tolist() == g["adj"]
            assert ex["val"].astype(np.int64).tolist() == g["val"]
            for d, rl in g["rowlist_by_delta"].items():
                assert G.export_csr(float(d))["rowlist"].tolist() == rl
            for s in range(g["V"]):
                assert G.sssp(s, g["delta"]).astype(np.int64).tolist() == g["dist"][s]


def test_fig1_distances_on_gpu(sssp, golden):
    g = golden("fig1_csr.json")
    adj = g["adj_printed_rows_0_4"] + g["adj_rows_5_7_by_symmetry"]
    val = g["val_printed_rows_0_4"] + [g["w67"] if x == "w67" else x for x in g["val_rows_5_7_by_symmetry"]]
    row = np.array(g["row"], np.int64)
    col, w = np.array(adj, np.uint32), np.array(val, np.uint32)
    for reorder in (False, True):
        with sssp.Graph(row, col, w) as G:
            if reorder:
                G.reorder()
            assert G.sssp(0, g["delta"]).tolist() == g["dist_from_0"]


# ------------------------------------------------------------- random -----
CASES = [
    # scale, ef, weights, deltas
    (10, 16, "u32", (1, 7, 32, 1e9, float("inf"))),
    (13, 16, "u32", (16, 100)),
    (10, 16, "f32", (0.01, 0.1, 1.0, float("inf"))),
    (13, 8, "f32", (0.1,)),
]


@pytest.mark.parametrize("scale,ef,wt,deltas", CASES)
@pytest.mark.parametrize("flags", [3, 0, 1, 2])
def test_kronecker_parity(sssp, scale, ef, wt, deltas, flags):
    g = gen.kronecker(scale, ef, seed=100 + scale, weights=wt)
    srcs = gen.sample_sources(g, 3, seed=scale)
    exp = {int(s): oracle.dijkstra(g.row, g.col, g.w, int(s)) for s in srcs}
    with sssp.Graph(g.row, g.col, g.w) as G:
        if flags:
            G.reorder(flags)
        for d in deltas:
            for s in srcs:
                assert_same(G.sssp(int(s), d), exp[int(s)], f"s{scale} {wt} flags={flags} delta={d} src={s}")


def test_grid_many_buckets(sssp):
    g = gen.grid(300, 200, p=0.2, seed=5)
    s = int(gen.sample_sources(g, 1, seed=1)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    for reorder in (True, False):
        with sssp.Graph(g.row, g.col, g.w) as G:
            if reorder:
                G.reorder()
            G.set_param(sssp.SSSP_PARAM_BF_TAIL, 0)  # every bucket on its own
            for d in (50, 400, 1600):
                assert_same(G.sssp(s, d), exp, f"grid reorder={reorder} delta={d}")
                st = G.stats()
                assert st["buckets"] >= int(exp[exp != INF].max()) // max(d, 1) // 2


# ---------------------------------------------------------- edge cases ----
def test_single_vertex_and_no_arcs(sssp):
    with sssp.Graph(np.zeros(2, np.int64), np.zeros(0, np.uint32), np.zeros(0, np.uint32)) as G:
        assert G.sssp(0, 5).tolist() == [0]
    row = np.zeros(6, np.int64)
    with sssp.Graph(row, np.zeros(0, np.uint32), np.zeros(0, np.float32)) as G:
        G.reorder()
        d = G.sssp(3, 1.0)
        assert d[3] == 0 and np.isinf(np.delete(d, 3)).all()


def test_self_loops_multi_edges_zero_weights(sssp):
    rng = np.random.default_rng(7)
    for trial in range(20):
        V = int(rng.integers(2, 40))
        arcs = []
        for _ in range(int(rng.integers(0, 150))):
            u, v = int(rng.integers(V)), int(rng.integers(V))
            arcs.append((u, v, int(rng.integers(0, 5))))
        row, col, w = csr_from_arcs(V, arcs)
        s = int(rng.integers(V))
        exp = oracle.dijkstra(row, col, w, s)
        with sssp.Graph(row, col, w) as G:
            if trial % 2:
                G.reorder()
            for d in (1, 3, 1e9):
                assert_same(G.sssp(s, d), exp, f"trial {trial} delta {d}")


def test_hub_chunks(sssp):
    """A star with 20000 leaves plus a ring: light and heavy ranges > 4096 arcs."""
    n = 20000
    rng = np.random.default_rng(3)
    arcs = []
    for i in range(1, n + 1):
        w = int(rng.integers(1, 100))
        arcs += [(0, i, w), (i, 0, w)]
        j = i % n + 1
        arcs += [(i, j, 3), (j, i, 3)]
    row, col, w = csr_from_arcs(n + 1, arcs)
    for s in (0, 17):
        exp = oracle.dijkstra(row, col, w, s)
        with sssp.Graph(row, col, w) as G:
            G.reorder()
            G.set_param(sssp.SSSP_PARAM_P2_EDGE_BALANCED, -1)  # heavy hubs through the chunk list too
            for d in (10, 60):
                assert_same(G.sssp(s, d), exp, f"hub src={s} delta={d}")
                assert G.stats()["hub_chunks"] > 0


def test_forced_overflow_rescans(sssp):
    """Tiny queues and ring force the dropped-push -> rescan fall-back."""
    g = gen.kronecker(14, 16, seed=9)
    s = int(gen.sample_sources(g, 1, seed=2)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_SLOT_CAPACITY, 4096)
        assert_same(G.sssp(s, 64), exp, "slot capacity 4096")
        assert G.stats()["rescans"] > 0
        G.set_param(sssp.SSSP_PARAM_SLOT_CAPACITY, 0)
        G.set_param(sssp.SSSP_PARAM_RING_SLOTS, 4)
        assert_same(G.sssp(s, 4), exp, "ring 4, delta 4")
        assert G.stats()["rescans"] > 0


@pytest.mark.parametrize("param,value", [(1, 1), (3, 1), (3, 17)])
def test_launch_shapes(sssp, param, value):
    g = gen.kronecker(12, 16, seed=4)
    s = int(gen.sample_sources(g, 1, seed=5)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(param, value)
        assert_same(G.sssp(s, 32), exp, f"param {param}={value}")


def test_determinism_repeated(sssp):
    g = gen.kronecker(12, 16, seed=6)
    s = int(gen.sample_sources(g, 1, seed=5)[0])
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        first = G.sssp(s, 16).copy()
        for _ in range(50):
            assert_same(G.sssp(s, 16), first, "repeat")


# ---------------------------------------------------- PRO vs oracle -------
@pytest.mark.parametrize("wt", ["u32", "f32"])
def test_pro_matches_oracle(sssp, wt):
    g = gen.kronecker(12, 16, seed=31, weights=wt)
    ref = oracle.pro_reorder(g.row, g.col, g.w)
    delta = 32 if wt == "u32" else 0.25
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        ex = G.export_csr(delta)
    assert np.array_equal(ex["new2old"], ref["new2old"])
    assert np.array_equal(ex["adj"], ref["adj"])
    assert np.array_equal(bits(ex["val"]), bits(ref["val"]))
    assert np.array_equal(ex["rowlist"], oracle.pro_rowlist(ref["row"], ref["val"], delta))


# --------------------------------------------- edge-balanced phase 2 -----
@pytest.mark.parametrize("eb", [0, -1, 64])
@pytest.mark.parametrize("wt,deltas", [("u32", (1, 8, 32, 200)), ("f32", (0.01, 0.1, 0.5))])
@pytest.mark.parametrize("flags", [3, 0])
def test_p2_edge_balanced_parity(sssp, eb, wt, deltas, flags):
    """Phases 2&3 with equal heavy arcs per warp for every bucket
    (eb=0), never (-1), or buckets of >= 64 settled entries; with and without
    PRO (without: the whole adjacency with a per-arc heavy predicate)."""
    g = gen.kronecker(13, 16, seed=77, weights=wt)
    srcs = gen.sample_sources(g, 2, seed=13)
    with sssp.Graph(g.row, g.col, g.w) as G:
        if flags:
            G.reorder(flags)
        G.set_param(sssp.SSSP_PARAM_P2_EDGE_BALANCED, eb)
        for s in srcs:
            exp = oracle.dijkstra(g.row, g.col, g.w, int(s))
            for d in deltas:
                assert_same(G.sssp(int(s), d), exp, f"eb={eb} {wt} flags={flags} delta={d} src={s}")


def test_p2_edge_balanced_hubs_and_grid(sssp):
    """Hubs far above 4096 heavy arcs (one entry spread over many warps) and a
    grid with hundreds of small buckets, every bucket edge-balanced."""
    n = 30000
    rng = np.random.default_rng(5)
    arcs = []
    for i in range(1, n + 1):
        w = int(rng.integers(1, 100))
        arcs += [(0, i, w), (i, 0, w), (1, i, w + 1), (i, 1, w + 1)]
    row, col, w = csr_from_arcs(n + 1, arcs)
    exp = oracle.dijkstra(row, col, w, 5)
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_P2_EDGE_BALANCED, 0)
        for d in (2, 10, 50):
            assert_same(G.sssp(5, d), exp, f"hubs delta={d}")
    g = gen.grid(300, 200, p=0.2, seed=5)
    s = int(gen.sample_sources(g, 1, seed=1)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_P2_EDGE_BALANCED, 0)
        for d in (50, 400):
            assert_same(G.sssp(s, d), exp, f"grid eb delta={d}")


# ------------------------------------------------------------- stats ------
def test_stats_invariants(sssp):
    g = gen.kronecker(13, 16, seed=8)
    s = int(gen.sample_sources(g, 1, seed=1)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    reach = int((exp != INF).sum())
    ref = oracle.pro_reorder(g.row, g.col, g.w)
    rl = oracle.pro_rowlist(ref["row"], ref["val"], 32)
    heavy_deg = rl[2::2] - rl[1::2]  # end - heavy per new vertex
    reach_new = exp[ref["new2old"]] != INF
    for eb in (0, -1):  # edge-balanced phase 2 in every bucket / never
        with sssp.Graph(g.row, g.col, g.w) as G:
            G.reorder()
            G.set_param(sssp.SSSP_PARAM_P2_EDGE_BALANCED, eb)
            G.set_param(sssp.SSSP_PARAM_BF_TAIL, 0)  # per-bucket heavy relaxations to the end
            G.sssp(s, 32)
            st = G.stats()
        _check_stats(st, reach, heavy_deg, reach_new)


def _check_stats(st, reach, heavy_deg, reach_new):
    assert st["reachable"] == reach
    # valid updates = reachable - 1; every update is >= valid
    assert st["updates"] >= reach - 1
    # each reachable vertex's heavy arcs are relaxed exactly once (u32 weights)
    assert st["heavy_vertices"] == reach
    assert st["heavy_arcs"] == int(heavy_deg[reach_new].sum())
    assert st["vertices_settled"] >= reach


# ---------------------------------------------------------- ABI errors ----
def test_abi_errors_on_device(sssp):
    g = gen.kronecker(8, 8, seed=1)
    with sssp.Graph(g.row, g.col, g.w) as G:
        with pytest.raises(sssp.SSSPError) as e:
            G.distances()
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
        for bad in (0, -1, float("nan")):
            with pytest.raises(sssp.SSSPError) as e:
                G.run(0, bad)
            assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT
        for src in (-1, g.V):
            with pytest.raises(sssp.SSSPError):
                G.run(src, 4)
        G.run(int(gen.sample_sources(g, 1)[0]), 4)
        G.distances()
        G.reorder()
        G.reorder()  # idempotent
        with pytest.raises(sssp.SSSPError) as e:
            G.distances()  # reorder invalidates the result
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
    bad_col = g.col.copy()
    bad_col[5] = g.V
    with pytest.raises(sssp.SSSPError) as e:
        sssp.Graph(g.row, bad_col, g.w)
    assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT
    bad_row = g.row.copy()
    bad_row[3], bad_row[4] = bad_row[4], bad_row[3] - 1
    with pytest.raises(sssp.SSSPError):
        sssp.Graph(bad_row, g.col, g.w)
    for x in (-1.0, float("nan"), float("inf")):
        wf = g.w.astype(np.float32)
        wf[2] = x
        with pytest.raises(sssp.SSSPError):
            sssp.Graph(g.row, g.col, wf)


def test_u32_overflow_reported(sssp):
    row, col, w = csr_from_arcs(3, [(0, 1, 0xFFFFFFF0), (1, 2, 0x20)])
    with sssp.Graph(row, col, w) as G:
        G.run(0, 1e9)
        with pytest.raises(sssp.SSSPError) as e:
            G.distances()
        assert e.value.status == sssp.SSSP_ERR_OVERFLOW


def test_negative_zero_weight_canonicalised(sssp):
    row, col, w = csr_from_arcs(3, [(0, 1, np.float32(-0.0)), (1, 2, np.float32(0.5))], np.float32)
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        d = G.sssp(0, 0.25)
    assert bits(d).tolist() == bits(np.array([0, 0, 0.5], np.float32)).tolist()


# --------------------------------------------------- device memory path ---
def test_device_inputs_and_outputs(sssp):
    import torch

    g = gen.kronecker(11, 16, seed=12)
    s = int(gen.sample_sources(g, 1, seed=1)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    row = torch.from_numpy(g.row).cuda()
    col = torch.from_numpy(g.col.view(np.int32)).cuda()
    w = torch.from_numpy(g.w.view(np.int32)).cuda()
    stream = torch.cuda.Stream()
    with sssp.Graph(row, col, w, stream=stream) as G:
        G.reorder()
        out = torch.empty(g.V, dtype=torch.int32, device="cuda")
        G.run(s, 32)
        G.distances(out)
        torch.cuda.synchronize()
        assert_same(out.cpu().numpy().view(np.uint32), exp, "device out")
        # batch into a device matrix
        srcs = gen.sample_sources(g, 4, seed=9)
        mat = torch.empty((4, g.V), dtype=torch.int32, device="cuda")
        G.run_batch(srcs, 32, mat)
        torch.cuda.synchronize()
        for i, ss in enumerate(srcs):
            assert_same(mat[i].cpu().numpy().view(np.uint32), oracle.dijkstra(g.row, g.col, g.w, int(ss)), "batch")


# ------------------------------------------------------- ablation modes ---
@pytest.mark.parametrize("sync,adwl,flags", [(1, 0, 0), (0, 0, 0), (0, 0, 3), (0, 1, 0), (1, 1, 3)])
@pytest.mark.parametrize("wt", ["u32", "f32"])
def test_ablation_modes_parity(sssp, sync, adwl, flags, wt):
    """BL (sync, static), BASYN, +PRO, +ADWL: every ablation mode is exact."""
    g = gen.kronecker(12, 16, seed=77, weights=wt)
    srcs = gen.sample_sources(g, 2, seed=3)
    delta = 32 if wt == "u32" else 0.1
    with sssp.Graph(g.row, g.col, g.w) as G:
        if flags:
            G.reorder(flags)
        G.set_param(sssp.SSSP_PARAM_SYNC, sync)
        G.set_param(sssp.SSSP_PARAM_ADWL, adwl)
        for s in srcs:
            assert_same(G.sssp(int(s), delta), oracle.dijkstra(g.row, g.col, g.w, int(s)),
                        f"sync={sync} adwl={adwl} flags={flags} src={s}")
            st = G.stats()
            if sync:
                assert st["levels"] > 0
            if not adwl:
                assert st["hub_chunks"] == 0 and st["bin_warp"] == 0 and st["bin_cta"] == 0


# ------------------------------------------------ adaptive Delta (NEXT-1) --
@pytest.mark.parametrize("mode", [1, 2])
@pytest.mark.parametrize("wt,deltas", [("u32", (1, 3, 16, 64)), ("f32", (0.05, 0.1, 0.4))])
@pytest.mark.parametrize("flags", [3, 0])
def test_adaptive_delta_parity(sssp, mode, wt, deltas, flags):
    """Eq. (1)-(2) bucket widths leave the distances unchanged
    (Delta-stepping is exact for every Delta), with PRO (light
    levels from the heavy-offset table per level) and without (predicate)."""
    g = gen.kronecker(13, 16, seed=91, weights=wt)
    srcs = gen.sample_sources(g, 2, seed=17)
    with sssp.Graph(g.row, g.col, g.w) as G:
        if flags:
            G.reorder(flags)
        G.set_param(sssp.SSSP_PARAM_ADAPTIVE_DELTA, mode)
        for s in srcs:
            exp = oracle.dijkstra(g.row, g.col, g.w, int(s))
            for d in deltas:
                assert_same(G.sssp(int(s), d), exp, f"adaptive={mode} {wt} flags={flags} delta={d} src={s}")


def _adapt_records(tr):
    return [e for e in tr if e["which"] == 8]


def _closed_buckets(tr):
    """(first slot, end slot, kernel C) of every bucket the scheduler closed, in order: the
    closing entry names the bucket (closed_b), its end is the cur_end (pad) that the
    preceding entries recorded for it."""
    out, end = [], {}
    for e in tr:
        if e["closed_b"] != INF:
            out.append((e["closed_b"], end[e["closed_b"]], e["closed_c"]))
        if e["which"] != 8:
            end[e["cur"]] = e["pad"]
    return out


@pytest.mark.parametrize("mode,reading", [(1, "A"), (2, "B")])
def test_adaptive_delta_follows_eq1(sssp, mode, reading):
    """The widths the kernel used are the oracle's Eq. (1)-(2) applied to
    C_i = vertices whose final distance (oracle Dijkstra) lies in bucket i's
    recorded bounds -- checked equal to the kernel's own count -- and the
    kernel's T_i (phase-1 queue items: schedule-dependent)."""
    g = gen.grid(400, 300, p=0.2, seed=8)  # many buckets
    s = int(gen.sample_sources(g, 1, seed=3)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_ADAPTIVE_DELTA, mode)
        assert_same(G.sssp(s, 400), exp, "grid adaptive")
        tr = G.trace()
        recs = _adapt_records(tr)
        st = G.stats()
    assert len(recs) >= 20 and st["rescans"] == 0
    fine = 100  # Delta_0 = 400 = 4 ring slots of g = 100
    closed = _closed_buckets(tr)
    assert len(closed) == len(recs) + 1  # the last bucket closes without an Eq. (1) record
    C = []
    for i, (r, (b0, b1, kc)) in enumerate(zip(recs, closed)):
        oc = int(np.count_nonzero((exp != INF) & (exp >= b0 * fine) & (exp < b1 * fine)))
        assert r["cur"] == kc == oc, f"C_{i}: Eq. (1) record {r['cur']}, trace {kc}, oracle {oc} ([{b0},{b1}))"
        C.append(oc)
    T = [r["tail"] for r in recs]
    ref = oracle.adaptive_delta(C, T, 4.0, reading)  # Delta_0 = 400 = 4 ring slots of g = 100
    got = [float(np.array([r["far_min"]], dtype=np.uint32).view(np.float32)[0]) for r in recs]
    for i, (a, b) in enumerate(zip(got, ref[1:])):
        assert abs(a - b) <= 1e-4 * max(1.0, abs(b)), f"Delta_{i + 1}: kernel {a} oracle {b}"
        m = recs[i]["mode"]
        want = min(max(int(round(b)), 1), 16)
        assert m == want or abs(b - math.floor(b) - 0.5) < 1e-3, f"width {i + 1}: {m} vs {want}"
    assert len(set(r["mode"] for r in recs)) > 1, "Delta never changed"
    assert sum(c for _, _, c in closed) == int((exp != INF).sum())


@pytest.mark.parametrize("case", ["kron-pull", "kron-push", "grid", "kron-noreorder"])
def test_bucket_settled_counts_match_oracle(sssp, case):
    """SURVEY §8(c) scheduler stat (ii): for a fixed Delta and u32 weights, the
    vertices settled in bucket b (trace closed_c) equal #{v : floor(d(v)/Delta) = b}
    of the oracle's Dijkstra distances (oracle.bucket_histogram; bucket
    definition), bucket by bucket; every non-empty bucket is closed
    exactly once and the counts sum to the reachable vertices."""
    if case == "grid":
        g, deltas = gen.grid(300, 200, p=0.2, seed=5), (400, 1600, 50)
    else:
        g, deltas = gen.kronecker(13, 16, seed=31), (8, 16, 64)
    srcs = [int(x) for x in gen.sample_sources(g, 2, seed=4)]
    with sssp.Graph(g.row, g.col, g.w) as G:
        if case != "kron-noreorder":
            G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1 if case == "kron-pull" else 0)
        G.set_param(sssp.SSSP_PARAM_BF_TAIL, 0)  # every bucket closed on its own
        if case == "grid":  # with the local chase on (auto here) the counts are not kept
            G.sssp(srcs[0], 1600)
            assert all(e["closed_c"] == INF for e in G.trace() if e["closed_b"] != INF)
            G.set_param(sssp.SSSP_PARAM_LOCAL_CHASE, 0)
        for s in srcs:
            exp = oracle.dijkstra(g.row, g.col, g.w, s)
            for d in deltas:
                assert_same(G.sssp(s, d), exp, f"{case} delta={d}")
                closed = [(b, c) for b, _, c in _closed_buckets(G.trace())]
                hist = oracle.bucket_histogram(exp, d)
                got = {}
                for b, c in closed:
                    assert b not in got, f"bucket {b} closed twice"
                    got[b] = c
                for b, c in got.items():
                    want = int(hist[b]) if b < len(hist) else 0
                    assert c == want, f"{case} delta={d} src={s} bucket {b}: kernel {c} oracle {want}"
                nonempty = {b for b in range(len(hist)) if hist[b]}
                assert nonempty <= set(got), f"buckets never closed: {sorted(nonempty - set(got))[:5]}"
                assert sum(got.values()) == int((exp != INF).sum())


# --------------------------------------- batched multi-source (NEXT-4) ----
def _multi(sssp, G, srcs, delta, V, f32):
    import torch

    out = torch.empty((len(srcs), V), dtype=torch.float32 if f32 else torch.int32, device="cuda")
    G.run_multi(srcs, delta, out)
    return out.cpu().numpy().view(np.float32 if f32 else np.uint32)


@pytest.mark.parametrize("wt,deltas", [("u32", (1, 16, 64, float("inf"))), ("f32", (0.02, 0.1, float("inf")))])
@pytest.mark.parametrize("flags", [3, 0])
def test_multi_source_parity(sssp, wt, deltas, flags):
    """sssp_run_multi: 40 sources (a full 32-lane group + a partial one, with a
    repeated source) bit-exact against per-source Dijkstra."""
    g = gen.kronecker(12, 16, seed=55, weights=wt)
    srcs = [int(s) for s in gen.sample_sources(g, 39, seed=21)]
    srcs.append(srcs[3])
    exp = np.stack([oracle.dijkstra(g.row, g.col, g.w, s) for s in srcs])
    with sssp.Graph(g.row, g.col, g.w) as G:
        if flags:
            G.reorder(flags)
        for d in deltas:
            got = _multi(sssp, G, srcs, d, g.V, wt == "f32")
            for i in range(len(srcs)):
                assert_same(got[i], exp[i], f"multi {wt} flags={flags} delta={d} src#{i}={srcs[i]}")
            st = G.multi_stats()
            assert st["expansions"] > 0 and st["arcs"] > 0


def test_multi_source_grid_and_hubs(sssp):
    """Many buckets (grid), ring-horizon rescans (delta 1 with weights up to
    100), and adjacencies split into 256-arc items (two 30000-arc hubs)."""
    g = gen.grid(300, 200, p=0.2, seed=5)
    srcs = [int(s) for s in gen.sample_sources(g, 8, seed=4)]
    exp = np.stack([oracle.dijkstra(g.row, g.col, g.w, s) for s in srcs])
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        for d in (1, 400):
            got = _multi(sssp, G, srcs, d, g.V, False)
            for i in range(len(srcs)):
                assert_same(got[i], exp[i], f"grid multi delta={d} src={srcs[i]}")
        assert G.multi_stats()["buckets"] > 50
    n = 30000
    rng = np.random.default_rng(5)
    arcs = []
    for i in range(1, n + 1):
        w = int(rng.integers(1, 100))
        arcs += [(0, i, w), (i, 0, w), (1, i, w + 1), (i, 1, w + 1)]
    row, col, w = csr_from_arcs(n + 1, arcs)
    srcs = [0, 1, 5, 77, 29999]
    exp = np.stack([oracle.dijkstra(row, col, w, s) for s in srcs])
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        for d in (1, 10):
            got = _multi(sssp, G, srcs, d, n + 1, False)
            for i in range(len(srcs)):
                assert_same(got[i], exp[i], f"hub multi delta={d} src={srcs[i]}")
            assert G.multi_stats()["split_items"] > 0
            if d == 1:
                assert G.multi_stats()["rescans"] >= 0


def test_multi_source_abi_errors(sssp):
    import torch

    g = gen.kronecker(8, 8, seed=3)
    with sssp.Graph(g.row, g.col, g.w) as G:
        with pytest.raises(sssp.SSSPError) as e:
            G.multi_stats()
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
        out = torch.empty((4, g.V), dtype=torch.int32, device="cuda")
        for bad_src in ([-1], [g.V]):
            with pytest.raises(sssp.SSSPError) as e:
                G.run_multi(bad_src, 16, out)
            assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT
        for bad in (0, -1, float("nan")):
            with pytest.raises(sssp.SSSPError) as e:
                G.run_multi([0], bad, out)
            assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT
        with pytest.raises(sssp.SSSPError) as e:
            G.run_multi([0], 16, out, ld=g.V - 1)
        assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT
        G.run_multi([], 16, out)  # empty batch: no-op
        # the hub run of the lane alignment replaces the last single-source result
        G.sssp(0, 16)
        G.run_multi([1, 2], 16, out)
        with pytest.raises(sssp.SSSPError) as e:
            G.distances()
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
        # alignment off: same rows
        a = out[:2].cpu().numpy().copy()
        G.set_param(sssp.SSSP_PARAM_MULTI_ALIGN, 0)
        G.run_multi([1, 2], 16, out)
        assert np.array_equal(a, out[:2].cpu().numpy())


def test_multi_source_u32_overflow_reported(sssp):
    import torch

    big = 0x7FFFFFFF
    row, col, w = csr_from_arcs(4, [(0, 1, big), (1, 0, big), (1, 2, big), (2, 1, big), (2, 3, 5), (3, 2, 5)])
    with sssp.Graph(row, col, w) as G:
        out = torch.empty((1, 4), dtype=torch.int32, device="cuda")
        with pytest.raises(sssp.SSSPError) as e:
            G.run_multi([0], 16, out)
        assert e.value.status == sssp.SSSP_ERR_OVERFLOW


def test_distances_async_pipeline(sssp):
    """sssp_distances_async overlaps step k's output with step k+1's run: every
    pinned buffer ends with its own source's distances (oracle), errors of all
    pageable memory is rejected."""
    import torch

    g = gen.kronecker(12, 16, seed=12)
    srcs = [int(s) for s in gen.sample_sources(g, 6, seed=3)]
    exp = [oracle.dijkstra(g.row, g.col, g.w, s) for s in srcs]
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        with pytest.raises(sssp.SSSPError) as e:
            G.distances_async(torch.empty(g.V, dtype=torch.int32).pin_memory())
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
        bufs = [torch.empty(g.V, dtype=torch.int32).pin_memory() for _ in srcs]
        dev = torch.empty(g.V, dtype=torch.int32, device="cuda")
        for s, b in zip(srcs, bufs):
            G.run(s, 16)
            G.distances_async(b)
        G.run(srcs[0], 16)
        G.distances_async(dev)
        G.wait()
        for i, b in enumerate(bufs):
            assert_same(b.numpy().view(np.uint32), exp[i], f"async src={srcs[i]}")
        assert_same(dev.cpu().numpy().view(np.uint32), exp[0], "async device")
        assert_same(G.distances(), exp[0], "sync after async")
        with pytest.raises(sssp.SSSPError) as e:
            G.distances_async(np.empty(g.V, dtype=np.uint32))
        assert e.value.status == sssp.SSSP_ERR_INVALID_ARGUMENT


def test_determinism_1000_runs_c1_and_multi(sssp):
    """SURVEY §4 stress: 1000 repeated runs on a skewed RMAT graph are bit-identical
    (the fixpoint is unique whatever the asynchronous schedule), and so are 50
    repeated 32-source multi runs."""
    import torch

    g = gen.make_config("C1")
    s = int(gen.sample_sources(g, 1, seed=9)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        dev = torch.empty(g.V, dtype=torch.int32, device="cuda")
        acc = torch.zeros(g.V, dtype=torch.int64, device="cuda")
        first = None
        for k in range(1000):
            G.run(s, 64)
            G.distances_async(dev)
            if first is None:
                torch.cuda.synchronize()
                first = dev.clone()
            acc += (dev != first).to(torch.int64)
        torch.cuda.synchronize()
        assert int(acc.sum()) == 0, "runs differ"
        assert_same(first.cpu().numpy().view(np.uint32), exp, "C1 x1000")
        srcs = [int(x) for x in gen.sample_sources(g, 32, seed=10)]
        out = torch.empty((32, g.V), dtype=torch.int32, device="cuda")
        G.run_multi(srcs, 64, out)
        ref = out.clone()
        for _ in range(50):
            G.run_multi(srcs, 64, out)
            assert torch.equal(out, ref), "multi runs differ"
        assert_same(ref[7].cpu().numpy().view(np.uint32), oracle.dijkstra(g.row, g.col, g.w, srcs[7]), "multi lane 7")


@pytest.mark.parametrize("scale,deltas", [(12, (1, 4, 16, 64, 200)), (14, (8, 16, 32))])
@pytest.mark.parametrize("flags", [3, 2])
def test_pull_phase2_parity(sssp, scale, deltas, flags):
    """SSSP_PARAM_PULL_SYMMETRIC: large buckets run phases 2&3 as a pull over the
    unsettled vertices (symmetric generator graphs); distances unchanged."""
    g = gen.kronecker(scale, 16, seed=60 + scale)
    srcs = gen.sample_sources(g, 3, seed=5)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder(flags)
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        for s in srcs:
            exp = oracle.dijkstra(g.row, g.col, g.w, int(s))
            for d in deltas:
                assert_same(G.sssp(int(s), d), exp, f"pull s{scale} flags={flags} delta={d} src={s}")
    gg = gen.grid(300, 200, p=0.2, seed=5)
    s = int(gen.sample_sources(gg, 1, seed=1)[0])
    exp = oracle.dijkstra(gg.row, gg.col, gg.w, s)
    with sssp.Graph(gg.row, gg.col, gg.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        for d in (50, 1600, 100000):
            assert_same(G.sssp(s, d), exp, f"pull grid delta={d}")


@pytest.mark.parametrize("deltas", [(0.01, 0.05, 0.1, 0.3, float("inf"))])
def test_pull_phase2_parity_f32(sssp, deltas):
    """The f32 pull: membership by bucket_of, the early stop by the lower bound
    fl(lo_f + w) (lo_f <= every distance of the bucket); bit-exact."""
    g = gen.kronecker(13, 16, seed=71, weights="f32")
    srcs = gen.sample_sources(g, 3, seed=6)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        for s in srcs:
            exp = oracle.dijkstra(g.row, g.col, g.w, int(s))
            for d in deltas:
                assert_same(G.sssp(int(s), d), exp, f"pull f32 delta={d} src={s}")


@pytest.mark.gpu
def test_local_chase_parity(sssp):
    """SSSP_PARAM_LOCAL_CHASE (2 forced, 1 auto on sparse graphs, while max w < Delta):
    in-bucket phase-1 pushes stay in the pushing CTA's shared memory. Distances
    bit-exact with it on and off: grids (hundreds of buckets), Kronecker hubs that
    overflow the one-batch local list (Delta = inf: one bucket, Bellman-Ford mode),
    f32 weights, unreordered graphs; valid updates = reachable - 1 either way."""
    cases = [(gen.grid(300, 200, p=0.2, seed=5), (101, 400, 1600, float("inf")), (True, False)),
             (gen.kronecker(14, 16, seed=71), (101, 300, float("inf")), (True, False)),
             (gen.kronecker(13, 16, seed=72, weights="f32"), (1.5, 4.0, float("inf")), (True,))]
    for g, deltas, reorders in cases:
        srcs = gen.sample_sources(g, 2, seed=3)
        exp = {int(s): oracle.dijkstra(g.row, g.col, g.w, int(s)) for s in srcs}
        for reorder in reorders:
            with sssp.Graph(g.row, g.col, g.w) as G:
                if reorder:
                    G.reorder()
                for local, lim in ((2, 512), (2, 8), (1, 64), (0, 512)):
                    G.set_param(sssp.SSSP_PARAM_LOCAL_CHASE, local)
                    G.set_param(sssp.SSSP_PARAM_LOCAL_LIMIT, lim)
                    for d in deltas:
                        for s in srcs:
                            e = exp[int(s)]
                            what = f"local={local} lim={lim} reorder={reorder} {g.wtype} V={g.V} delta={d} src={s}"
                            assert_same(G.sssp(int(s), d), e, what)
                            st = G.stats()
                            reach = int(np.count_nonzero(e != (INF if g.wtype == "u32" else np.float32(np.inf))))
                            assert st["reachable"] == reach, what
                            assert st["updates"] >= reach - 1, what


# ------------------------------------------- run-error contract (§8(b)) ----
def _overflow_graph():
    """Symmetric graph whose shortest distance to vertex 38 overflows u32:
    0 -(1)- leaves 1..16 (light at Delta = 2^31), leaf 1 -(0xC0000000)- 20
    vertices 17..36 (heavy), 17 -(0xC0000000)- 37 -(1)- 38. Buckets 0 and 1
    hold >= V/16 entries, so with PULL_SYMMETRIC the pull phases 2&3 see the
    overflowing candidate; with push phases 2&3 the push relaxation does.
    Vertices 39 -(2)- 40 form a separate component with no overflow."""
    big = 0xC0000000
    e = [(0, i, 1) for i in range(1, 17)] + [(1, 16 + j, big) for j in range(1, 21)]
    e += [(17, 37, big), (37, 38, 1), (39, 40, 2)]
    arcs = [(u, v, w) for u, v, w in e] + [(v, u, w) for u, v, w in e]
    return csr_from_arcs(41, arcs)


@pytest.mark.parametrize("pull", [0, 1])
@pytest.mark.parametrize("path", ["sync", "async", "batch"])
def test_overflow_reported_on_every_path(sssp, pull, path):
    """u32 overflow (R12) is reported by sssp_distances, by sssp_wait after
    sssp_distances_async, and by sssp_run_batch -- with push and with pull
    phases 2&3 -- and a later clean run reports OK again."""
    import torch

    row, col, w = _overflow_graph()
    delta = 2.0 ** 31
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, pull)
        with pytest.raises(sssp.SSSPError) as e:
            if path == "sync":
                G.sssp(0, delta)
            elif path == "async":
                G.run(0, delta)
                G.distances_async(torch.empty(41, dtype=torch.int32).pin_memory())
                G.wait()
            else:
                out = torch.empty((2, 41), dtype=torch.int32, device="cuda")
                G.run_batch([5, 0], delta, out)
        assert e.value.status == sssp.SSSP_ERR_OVERFLOW, path
        # the error was reported once and cleared: a clean run (the other component) is OK
        d = G.sssp(39, 1)
        assert d[40] == 2 and d[39] == 0 and d[0] == INF
        G.run(39, 1)
        G.distances_async(torch.empty(41, dtype=torch.int32).pin_memory())
        G.wait()


def test_overflow_of_unreported_run_surfaces_at_wait(sssp):
    """Errors accumulate per handle: an overflowing run followed by a clean run
    (neither reported) still makes the next sssp_wait fail."""
    row, col, w = _overflow_graph()
    with sssp.Graph(row, col, w) as G:
        G.run(0, 2.0 ** 31)
        G.run(39, 1)
        with pytest.raises(sssp.SSSPError) as e:
            G.wait()
        assert e.value.status == sssp.SSSP_ERR_OVERFLOW
        G.wait()  # cleared


def test_multi_source_overflow_in_first_group(sssp):
    """sssp_run_multi with 64 sources: the overflow happens only in group 0
    (source 0); group 1's clean run must not wipe it."""
    import torch

    row, col, w = _overflow_graph()
    g2 = gen.kronecker(8, 8, seed=3)  # second component, small weights
    V1 = 41
    row2 = np.concatenate([row, g2.row[1:] + row[-1]]).astype(np.int64)
    col2 = np.concatenate([col, g2.col + V1]).astype(np.uint32)
    w2 = np.concatenate([w, g2.w]).astype(np.uint32)
    V = V1 + g2.V
    other = [V1 + int(s) for s in gen.sample_sources(g2, 63, seed=1)]
    srcs = [0] + other
    with sssp.Graph(row2, col2, w2) as G:
        out = torch.empty((64, V), dtype=torch.int32, device="cuda")
        with pytest.raises(sssp.SSSPError) as e:
            G.run_multi(srcs, 2.0 ** 31, out)
        assert e.value.status == sssp.SSSP_ERR_OVERFLOW
        G.run_multi(other, 16, out[:63])  # clean


def test_pull_symmetric_is_checked(sssp):
    """SSSP_PARAM_PULL_SYMMETRIC is verified, not trusted: a directed
    Kronecker graph (one arc per edge, R13) is reported asymmetric and the
    pull cannot be enabled; the generators' symmetrised graphs pass."""
    gd = gen.kronecker(11, 16, seed=5, symmetrize=False)
    gs = gen.kronecker(11, 16, seed=5)
    s = int(gen.sample_sources(gd, 1, seed=1)[0])
    exp = oracle.dijkstra(gd.row, gd.col, gd.w, s)
    with sssp.Graph(gd.row, gd.col, gd.w) as G:
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)  # not reordered yet: checked at run
        G.reorder()
        assert not G.is_symmetric()
        with pytest.raises(sssp.SSSPError) as e:
            G.run(s, 16)
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 0)
        assert_same(G.sssp(s, 16), exp, "directed graph, push phases 2&3")
        with pytest.raises(sssp.SSSPError) as e:
            G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        assert e.value.status == sssp.SSSP_ERR_INVALID_STATE
    with sssp.Graph(gs.row, gs.col, gs.w) as G:
        with pytest.raises(sssp.SSSPError):
            G.is_symmetric()  # needs the weight-sorted layout
        G.reorder()
        assert G.is_symmetric()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
    # one reverse arc with a different weight breaks symmetry
    row, col, w = csr_from_arcs(3, [(0, 1, 4), (1, 0, 5), (1, 2, 1), (2, 1, 1)])
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        assert not G.is_symmetric()
    # multiplicities must match: (0,1,4) twice one way, once the other
    row, col, w = csr_from_arcs(2, [(0, 1, 4), (0, 1, 4), (1, 0, 4)])
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        assert not G.is_symmetric()
    row, col, w = csr_from_arcs(2, [(0, 1, 4), (0, 1, 4), (1, 0, 4), (1, 0, 4), (0, 0, 3)])
    with sssp.Graph(row, col, w) as G:
        G.reorder()
        assert G.is_symmetric()


def test_allocator_hook_torch(sssp):
    """sssp_set_allocator: with PyTorch's caching allocator behind the hook the
    handle's buffers are torch allocations (memory_allocated grows by them and returns after
    destroy), every hooked buffer is freed exactly once, and the SSSP is unchanged."""
    import torch

    g = gen.kronecker(12, 16, seed=21)
    s = int(gen.sample_sources(g, 1, seed=2)[0])
    exp = oracle.dijkstra(g.row, g.col, g.w, s)
    log = {"alloc": 0, "free": 0, "live": {}}

    def alloc(n, dev, stream):
        p = torch.cuda.caching_allocator_alloc(n, dev, stream if stream else None)
        log["alloc"] += 1
        log["live"][p] = n
        return p

    def free(ptr, n, dev, stream):
        assert log["live"].pop(ptr) == n
        log["free"] += 1
        torch.cuda.caching_allocator_delete(ptr)

    torch.cuda.synchronize()
    base = torch.cuda.memory_allocated()
    sssp.sssp_set_allocator(alloc, free)
    try:
        with sssp.Graph(g.row, g.col, g.w) as G:
            G.reorder()
            G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
            assert_same(G.sssp(s, 16), exp, "torch allocator")
            held = sum(log["live"].values())
            assert log["alloc"] > 8 and held > 8 * g.A  # the arc array at least
            assert torch.cuda.memory_allocated() - base >= held
    finally:
        sssp.sssp_set_allocator(None, None)
    torch.cuda.synchronize()
    assert log["free"] == log["alloc"] and not log["live"]
    assert torch.cuda.memory_allocated() == base
    with pytest.raises(sssp.SSSPError):  # one of the pair only
        sssp._check(sssp._lib.sssp_set_allocator(sssp._ALLOC_FN(lambda *a: None), sssp._FREE_FN(), None), "x")


# ------------------------------------------------- Bellman-Ford end ----
@pytest.mark.parametrize("case", ["kron-pull", "kron-push", "kron-noreorder", "grid", "kron-f32"])
def test_bf_tail_parity(sssp, case):
    """SSSP_PARAM_BF_TAIL: once the ring holds <= threshold entries, the rest of the run is
    one bucket [cur, inf) relaxing every arc (Delta = inf is Bellman-Ford).
    Bit-exact with the oracle for thresholds 0 (never), small (the last buckets), the
    default, and 2^30 (never reached: the wave's peak must hold 8x the threshold), with the
    merge of non-empty ring slots, and with a tiny queue capacity (dropped pushes -> rescans);
    the end phase must actually run in the small-threshold case (fewer buckets)."""
    if case == "grid":
        g, deltas = gen.grid(200, 150, p=0.2, seed=9), (50, 400)
    elif case == "kron-f32":
        g, deltas = gen.kronecker(13, 16, seed=77, weights="f32"), (0.02, 0.1)
    else:
        g, deltas = gen.kronecker(13, 16, seed=76), (4, 16, 64)
    srcs = [int(x) for x in gen.sample_sources(g, 2, seed=11)]
    exp = {s: oracle.dijkstra(g.row, g.col, g.w, s) for s in srcs}
    with sssp.Graph(g.row, g.col, g.w) as G:
        if case != "kron-noreorder":
            G.reorder()
        if case in ("kron-pull", "kron-f32"):
            G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        if case == "grid":  # the CTA-local chase keeps the buckets' queues short: no peak to pass
            for s in srcs:
                G.set_param(sssp.SSSP_PARAM_BF_TAIL, 256)
                assert_same(G.sssp(s, deltas[0]), exp[s], f"grid local chase bf_tail=256 src={s}")
            G.set_param(sssp.SSSP_PARAM_LOCAL_CHASE, 0)
        nb = {}
        for t in (0, 64, 256, -1, sssp.SSSP_BF_TAIL_DEFAULT, 1 << 30):
            G.set_param(sssp.SSSP_PARAM_BF_TAIL, t)
            for d in deltas:
                for s in srcs:
                    assert_same(G.sssp(s, d), exp[s], f"{case} bf_tail={t} delta={d} src={s}")
                    nb[(t, d, s)] = G.stats()["buckets"]
        ran = sum(nb[(256, d, s)] < nb[(0, d, s)] for d in deltas for s in srcs)
        assert ran > 0, f"{case}: the Bellman-Ford end never ran at threshold 256"
        G.set_param(sssp.SSSP_PARAM_SLOT_CAPACITY, 4096)  # pushes dropped: rescans inside the end phase
        G.set_param(sssp.SSSP_PARAM_BF_TAIL, 256)
        for s in srcs:
            assert_same(G.sssp(s, deltas[0]), exp[s], f"{case} bf_tail=256 capacity=4096 src={s}")
        with pytest.raises(sssp.SSSPError):
            G.set_param(sssp.SSSP_PARAM_BF_TAIL, -2)


@pytest.mark.parametrize("wt,scale", [("u32", 12), ("f32", 12), ("f32", 17)])
def test_symmetry_check_paths(sssp, wt, scale):
    """sssp_is_symmetric has two exact paths: the sort-based one (transposed keys radix-sorted
    and compared with the arcs, when (dst, w, src) packs into 64 bits: u32 s12, f32 s12) and the
    per-run binary searches (f32 s17: 17 + 32 + 17 bits do not pack). Both must accept the
    symmetrised graph and reject it after one arc's weight changes by one ulp/unit."""
    g = gen.kronecker(scale, 8, seed=91, weights=wt)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        assert G.is_symmetric()
    w = g.w.copy()
    k = len(w) // 3
    w[k] = np.nextafter(w[k], np.float32(np.inf)) if wt == "f32" else w[k] + 1
    with sssp.Graph(g.row, g.col, w) as G:
        G.reorder()
        assert not G.is_symmetric()
    # a self-loop-free directed copy: drop one arc of a symmetric pair
    keep = np.ones(len(g.col), bool)
    keep[k] = False
    u = np.repeat(np.arange(g.V), np.diff(g.row))[keep]
    row = np.zeros(g.V + 1, np.int64)
    np.add.at(row, u + 1, 1)
    row = np.cumsum(row)
    with sssp.Graph(row, g.col[keep].copy(), g.w[keep].copy()) as G:
        G.reorder()
        assert not G.is_symmetric()
