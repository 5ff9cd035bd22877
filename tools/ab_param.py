"""A/B of one libsssp over set_param values (interleaved): python tools/ab_param.py CONFIG PARAM v1 v2 ..."""
import sys, os
sys.path.insert(0, "/root/repo" if not os.environ.get("GRAFT_REPO_ROOT") else os.environ["GRAFT_REPO_ROOT"])
import numpy as np, torch
import gen
import paper_conf_icppw_zhangczsdhay23_b200 as sssp
cfg, param = sys.argv[1], int(sys.argv[2]); vals = [int(x) for x in sys.argv[3:]]
g = gen.make_config(cfg); delta = gen.CONFIGS[cfg]["delta"]
srcs = gen.sample_sources(g, 8, seed=7)
with sssp.Graph(g.row, g.col, g.w) as G:
    G.reorder()
    for r in range(2):
        for v in vals:
            G.set_param(param, v)
            G.run(int(srcs[0]), delta); G.kernel_time(reset=True)
            for s in srcs: G.run(int(s), delta)
            t, n = G.kernel_time(reset=True)
            st = G.stats()
            print(f"{cfg} param{param}={v:7d}: {t/n:.3f} ms  buckets={st['buckets']} heavy={st['heavy_arcs']/1e6:.1f}M", flush=True)
