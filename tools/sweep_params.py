"""Sweep sssp_set_param combinations x Delta on one graph loaded once (stable ABI calls only).

python tools/sweep_params.py --config C2 --deltas 1600 3200 --grid 1=0,2 --grid 3=64,512
Each --grid PARAM_ID=v1,v2,... adds one axis; --param PARAM_ID=V is applied to every run."""
import argparse
import ctypes
import itertools
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import gen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--runs", type=int, default=4)
    ap.add_argument("--rounds", type=int, default=2)
    ap.add_argument("--deltas", type=float, nargs="*", default=None)
    ap.add_argument("--param", action="append", default=[])
    ap.add_argument("--grid", action="append", default=[])
    ap.add_argument("--lib", default="paper_conf_icppw_zhangczsdhay23_b200/libsssp.so")
    a = ap.parse_args()
    import torch  # noqa: F401  (CUDA context)

    g = gen.make_config(a.config)
    deltas = a.deltas or [gen.CONFIGS[a.config]["delta"]]
    srcs = gen.sample_sources(g, a.runs, seed=7)
    P, I64, I, D = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int, ctypes.c_double
    L = ctypes.CDLL(os.path.abspath(a.lib))
    L.sssp_graph_create.argtypes = [ctypes.POINTER(P), I, I64, I64, P, P, P, I, I, P]
    L.sssp_reorder.argtypes = [P]
    L.sssp_run.argtypes = [P, I64, D]
    L.sssp_set_param.argtypes = [P, I, I64]
    L.sssp_kernel_time.argtypes = [P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64), I]
    h = P()
    assert L.sssp_graph_create(ctypes.byref(h), 0, g.V, g.A, g.row.ctypes.data, g.col.ctypes.data,
                               g.w.ctypes.data, 1 if g.wtype == "f32" else 0, 0, None) == 0
    assert L.sssp_reorder(h) == 0
    for kv in a.param:
        k, v = kv.split("=")
        assert L.sssp_set_param(h, int(k), int(v)) == 0
    axes = []
    for spec in a.grid:
        k, vs = spec.split("=")
        axes.append([(int(k), int(v)) for v in vs.split(",")])
    for combo in itertools.product(*axes) if axes else [()]:
        for k, v in combo:
            assert L.sssp_set_param(h, k, v) == 0
        for d in deltas:
            assert L.sssp_run(h, int(srcs[0]), float(d)) == 0  # warm-up (re-allocation)
            t, n = ctypes.c_double(), ctypes.c_int64()
            L.sssp_kernel_time(h, ctypes.byref(t), ctypes.byref(n), 1)
            best = []
            for _ in range(a.rounds):
                for s in srcs:
                    assert L.sssp_run(h, int(s), float(d)) == 0
                L.sssp_kernel_time(h, ctypes.byref(t), ctypes.byref(n), 1)
                best.append(t.value / n.value)
            tag = " ".join(f"p{k}={v}" for k, v in combo)
            print(f"{a.config} {tag:24s} delta={d:<8g} ms: " + " ".join(f"{x:.3f}" for x in best)
                  + f" | best {min(best):.3f}", flush=True)


if __name__ == "__main__":
    main()
