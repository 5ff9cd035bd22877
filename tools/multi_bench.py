"""NEXT-4 timing: sssp_run_multi (32 sources per persistent launch) vs sssp_run_batch
(one persistent launch per source) on one config. python tools/multi_bench.py C4 [n_sources] [delta...]"""
import os
import sys
import time

sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import gen  # noqa: E402
import paper_conf_icppw_zhangczsdhay23_b200 as sssp  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 64
g = gen.make_config(cfg)
d0 = gen.CONFIGS[cfg]["delta"]
deltas = [float(x) for x in sys.argv[3:]] or [d0]
srcs = gen.sample_sources(g, n, seed=7)
m = g.m
with sssp.Graph(g.row, g.col, g.w) as G:
    G.reorder()
    if os.environ.get("MULTI_ALIGN") is not None:
        G.set_param(sssp.SSSP_PARAM_MULTI_ALIGN, int(os.environ["MULTI_ALIGN"]))
    if os.environ.get("MULTI_HUB_DELAY") is not None:
        G.set_param(sssp.SSSP_PARAM_MULTI_HUB_DELAY, int(os.environ["MULTI_HUB_DELAY"]))
    out = torch.empty((n, g.V), dtype=torch.int32, device="cuda")
    out2 = torch.empty_like(out)
    for d in deltas:
        G.run_multi(srcs[:32], d, out)  # warm-up + allocation
        torch.cuda.synchronize()
        G.kernel_time(reset=True)
        t0 = time.perf_counter()
        G.run_multi(srcs, d, out)
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        kt, nl = G.kernel_time(reset=True)
        st = G.multi_stats()
        print(f"{cfg} multi  delta={d:g}: {kt / n:.3f} ms/source kernel ({kt:.1f} ms, {nl} launches), "
              f"wall {wall * 1e3 / n:.3f} ms/source, {n * m / (kt * 1e-3) / 1e9:.1f} GTEPS; last group {st}", flush=True)
    G.run_batch(srcs[:2], d0, out2)
    torch.cuda.synchronize()
    G.kernel_time(reset=True)
    G.run_batch(srcs[:16], d0, out2)
    torch.cuda.synchronize()
    kt, nl = G.kernel_time(reset=True)
    print(f"{cfg} batch  delta={d0:g}: {kt / nl:.3f} ms/source kernel, {m / (kt / nl * 1e-3) / 1e9:.1f} GTEPS", flush=True)
    a = out[:16].cpu().numpy()
    b = out2[:16].cpu().numpy()
    print("multi == batch on 16 sources:", bool(np.array_equal(a, b)))
