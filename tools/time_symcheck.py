"""Wall time of sssp_is_symmetric (one-off per reorder) on a config: python tools/time_symcheck.py [C4]"""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import gen  # noqa: E402


def main():
    import torch
    import paper_conf_icppw_zhangczsdhay23_b200 as sssp

    cfg = sys.argv[1] if len(sys.argv) > 1 else "C4"
    g = gen.make_config(cfg)
    with sssp.Graph(g.row, g.col, g.w) as G:
        G.reorder()
        torch.cuda.synchronize()
        t = time.perf_counter()
        sym = G.is_symmetric()
        dt = time.perf_counter() - t
    print(f"{cfg}: symmetric={sym} sssp_is_symmetric {dt * 1e3:.1f} ms ({os.path.basename(sssp.LIB_PATH)})", flush=True)


if __name__ == "__main__":
    main()
