"""A/B timing of libsssp builds on one graph using only stable ABI calls.

python tools/ab.py --config C4 --runs 8 lib1.so lib2.so ...   (interleaved rounds)"""
import argparse
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--runs", type=int, default=8)
    ap.add_argument("--rounds", type=int, default=3)
    ap.add_argument("--deltas", type=float, nargs="*", default=None)
    ap.add_argument("--param", action="append", default=[], help="PARAM_ID=VALUE (sssp_set_param)")
    ap.add_argument("libs", nargs="+")
    a = ap.parse_args()
    import torch  # noqa: F401  (CUDA context)

    g = gen.make_config(a.config)
    delta = gen.CONFIGS[a.config]["delta"]
    deltas = a.deltas or [delta]
    srcs = gen.sample_sources(g, a.runs, seed=7)
    P, I64, I, D = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
    handles = []
    for path in a.libs:
        L = ctypes.CDLL(os.path.abspath(path))
        L.sssp_graph_create.argtypes = [ctypes.POINTER(P), I, I64, I64, P, P, P, I, I, P]
        L.sssp_reorder.argtypes = [P]
        L.sssp_run.argtypes = [P, I64, D]
        L.sssp_kernel_time.argtypes = [P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64), I]
        h = P()
        wt = 1 if g.wtype == "f32" else 0
        assert L.sssp_graph_create(ctypes.byref(h), 0, g.V, g.A, g.row.ctypes.data, g.col.ctypes.data,
                                   g.w.ctypes.data, wt, 0, None) == 0
        assert L.sssp_reorder(h) == 0
        L.sssp_set_param.argtypes = [P, I, I64]
        for kv in a.param:
            k, v = kv.split("=")
            assert L.sssp_set_param(h, int(k), int(v)) == 0
        assert L.sssp_run(h, int(srcs[0]), float(delta)) == 0
        t, n = ctypes.c_double(), ctypes.c_int64()
        L.sssp_kernel_time(h, ctypes.byref(t), ctypes.byref(n), 1)
        handles.append((path, L, h))
    res = {(p, d): [] for p in a.libs for d in deltas}
    for r in range(a.rounds):
        for path, L, h in handles:
            for d in deltas:
                for s in srcs:
                    assert L.sssp_run(h, int(s), float(d)) == 0
                t, n = ctypes.c_double(), ctypes.c_int64()
                L.sssp_kernel_time(h, ctypes.byref(t), ctypes.byref(n), 1)
                res[(path, d)].append(t.value / n.value)
    for (path, d), v in res.items():
        print(f"{os.path.basename(path):20s} delta={d:<8g} mean/round ms: " + " ".join(f"{x:.3f}" for x in v)
              + f"  | best {min(v):.3f}")


if __name__ == "__main__":
    main()
