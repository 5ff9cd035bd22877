"""Small end-to-end cases through every kernel path, for compute-sanitizer
(memcheck / racecheck / synccheck): python tools/sanitize_cases.py
Each case is checked against the oracle, so a sanitizer-clean run is also a
parity run. Uses 1 persistent CTA per SM to keep the sanitizer runs short."""
import os
import sys

sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icppw_zhangczsdhay23_b200 as sssp  # noqa: E402


def same(a, b, what):
    assert np.array_equal(np.ascontiguousarray(a).view(np.uint32), np.ascontiguousarray(b).view(np.uint32)), what


def main():
    for wt, d in (("u32", 16), ("f32", 0.1)):
        g = gen.kronecker(10, 16, seed=5, weights=wt)
        s = int(gen.sample_sources(g, 1, seed=2)[0])
        exp = oracle.dijkstra(g.row, g.col, g.w, s)
        for flags in (3, 0):
            with sssp.Graph(g.row, g.col, g.w) as G:
                G.set_param(sssp.SSSP_PARAM_CTAS_PER_SM, 1)
                if flags:
                    G.reorder(flags)
                same(G.sssp(s, d), exp, f"{wt} flags={flags}")
                for param, val in ((sssp.SSSP_PARAM_P2_EDGE_BALANCED, 0), (sssp.SSSP_PARAM_ADAPTIVE_DELTA, 1),
                                   (sssp.SSSP_PARAM_SLOT_CAPACITY, 4096)):
                    G.set_param(param, val)
                    same(G.sssp(s, d), exp, f"{wt} flags={flags} param {param}={val}")
                srcs = [int(x) for x in gen.sample_sources(g, 5, seed=4)]
                out = torch.empty((5, g.V), dtype=torch.float32 if wt == "f32" else torch.int32, device="cuda")
                G.run_multi(srcs, d, out)
                rows = out.cpu().numpy()
                for i, x in enumerate(srcs):
                    same(rows[i], oracle.dijkstra(g.row, g.col, g.w, x), f"{wt} multi lane {i}")
                G.run(s, d)
                pin = torch.empty(g.V, dtype=torch.float32 if wt == "f32" else torch.int32).pin_memory()
                G.distances_async(pin)
                G.wait()
                same(pin.numpy(), exp, f"{wt} async")
        print(f"sanitize cases {wt}: OK", flush=True)
    # CTA-local chase (SSSP_PARAM_LOCAL_CHASE): a grid in auto mode, a Kronecker graph forced
    # (hubs overflow the one-batch local list), Delta above the max weight so no arc is heavy
    for g, d in ((gen.grid(60, 40, p=0.2, seed=3), 400), (gen.kronecker(10, 16, seed=5), 101)):
        s = int(gen.sample_sources(g, 1, seed=2)[0])
        exp = oracle.dijkstra(g.row, g.col, g.w, s)
        with sssp.Graph(g.row, g.col, g.w) as G:
            G.set_param(sssp.SSSP_PARAM_CTAS_PER_SM, 1)
            G.reorder()
            for local in (1, 2):
                G.set_param(sssp.SSSP_PARAM_LOCAL_CHASE, local)
                same(G.sssp(s, d), exp, f"local chase {local} V={g.V}")
    print("sanitize cases local chase: OK", flush=True)
    # Bellman-Ford end (SSSP_PARAM_BF_TAIL): the merge of non-empty ring slots, the all-arc phase 1,
    # the final clear, and the rescan inside the end phase (tiny queue capacity); pull phases on
    g = gen.kronecker(11, 16, seed=76)
    srcs = [int(x) for x in gen.sample_sources(g, 2, seed=11)]
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.set_param(sssp.SSSP_PARAM_CTAS_PER_SM, 1)
        G.reorder()
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
        for t, cap in ((16, 0), (64, 0), (64, 4096)):
            G.set_param(sssp.SSSP_PARAM_BF_TAIL, t)
            G.set_param(sssp.SSSP_PARAM_SLOT_CAPACITY, cap)
            for s in srcs:
                for d in (4, 16):
                    same(G.sssp(s, d), oracle.dijkstra(g.row, g.col, g.w, s), f"bf_tail={t} cap={cap} d={d}")
    print("sanitize cases Bellman-Ford end: OK", flush=True)


if __name__ == "__main__":
    main()
