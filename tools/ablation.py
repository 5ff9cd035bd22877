"""Ablation ladder on synthetic k-n21-16 (PAPER Fig. 8):
BL (level-synchronous push, static thread-per-vertex) -> BASYN -> +PRO / +ADWL ->
BASYN+PRO+ADWL, with the work-efficiency ratio total/valid updates (Fig. 9,
P:1530-1538). Prints one JSON line per variant and a summary table.

python tools/ablation.py [--scale 21] [--sources 8] [--delta 32]"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import gen  # noqa: E402

VARIANTS = [  # name, sync, adwl, PRO flags
    ("BL", 1, 0, 0),
    ("BASYN", 0, 0, 0),
    ("BASYN+PRO", 0, 0, 3),
    ("BASYN+ADWL", 0, 1, 0),
    ("BASYN+PRO+ADWL", 0, 1, 3),
]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=21)
    ap.add_argument("--edgefactor", type=int, default=16)
    ap.add_argument("--sources", type=int, default=8)
    ap.add_argument("--delta", type=float, default=32)
    ap.add_argument("--seed", type=int, default=21)
    a = ap.parse_args()
    import torch

    import paper_conf_icppw_zhangczsdhay23_b200 as sssp

    g = gen.kronecker(a.scale, a.edgefactor, a.seed)
    srcs = gen.sample_sources(g, a.sources, seed=7)
    rows = []
    for name, sync, adwl, flags in VARIANTS:
        G = sssp.Graph(g.row, g.col, g.w)
        if flags:
            G.reorder(flags)
        G.set_param(sssp.SSSP_PARAM_SYNC, sync)
        G.set_param(sssp.SSSP_PARAM_ADWL, adwl)
        G.run(int(srcs[0]), a.delta)  # warm-up (heavy offsets, buffers)
        torch.cuda.synchronize()
        G.kernel_time(reset=True)
        upd = val = 0
        times = []
        for s in srcs:
            G.run(int(s), a.delta)
            st = G.stats()
            times.append(st["run_ms"])
            upd += st["updates"]
            val += st["reachable"] - 1  # valid updates = reachable - 1
        ms = float(np.mean(times))
        r = dict(variant=name, ms=round(ms, 4), gteps=round(g.m / ms / 1e6, 3),
                 work_ratio=round(upd / max(val, 1), 3), graph=f"k-n{a.scale}-{a.edgefactor}",
                 delta=a.delta, sources=len(srcs))
        print(json.dumps(r), flush=True)
        rows.append(r)
        G.close()
    bl = rows[0]["ms"]
    print(f"{'variant':18s} {'ms':>9s} {'GTEPS':>8s} {'speedup/BL':>11s} {'total/valid':>12s}")
    for r in rows:
        print(f"{r['variant']:18s} {r['ms']:9.3f} {r['gteps']:8.2f} {bl / r['ms']:11.2f} {r['work_ratio']:12.3f}")


if __name__ == "__main__":
    main()
