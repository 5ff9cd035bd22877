"""Run one SSSP on a config and print the device-side scheduler timeline.

python tools/trace_run.py --config C4 [--delta 32] [--runs 3] [--param k=v]"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import gen  # noqa: E402

NAMES = {0: "P1", 1: "P2", 2: "RC", 3: "RF", 4: "SL", 5: "SH", 6: "P2C", 7: "MG", 8: "ADAPT", 9: "PL", 10: "F", 99: "start"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--scale", type=int, default=None)
    ap.add_argument("--delta", type=float, nargs="*", default=None)
    ap.add_argument("--runs", type=int, default=3)
    ap.add_argument("--no-reorder", action="store_true")
    ap.add_argument("--param", action="append", default=[])
    ap.add_argument("--quiet", action="store_true")
    ap.add_argument("--samples", action="store_true", help="phase-1 claim samples of the last run per bucket")
    a = ap.parse_args()
    import torch
    import paper_conf_icppw_zhangczsdhay23_b200 as sssp

    over = {"scale": a.scale} if a.scale else {}
    t = time.time()
    c = dict(gen.CONFIGS[a.config])
    c.update(over)
    g = gen.kronecker(c["scale"], c["edgefactor"], c["seed"], c["weights"]) if c["kind"] == "kron" else gen.make_config(a.config)
    print(f"gen {time.time()-t:.1f}s V={g.V} A={g.A}", flush=True)
    G = sssp.Graph(g.row, g.col, g.w)
    for kv in a.param:
        k, v = kv.split("=")
        G.set_param(getattr(sssp, "SSSP_PARAM_" + k.upper()), int(v))
    if not a.no_reorder:
        G.reorder()
        print("reorder_ms", G.stats()["reorder_ms"])
    srcs = gen.sample_sources(g, 8, seed=7)
    for delta in (a.delta or [c["delta"]]):
        for r in range(a.runs):
            G.run(int(srcs[r % len(srcs)]), delta)
            torch.cuda.synchronize()
            st = G.stats()
            print(f"delta={delta} run {r}: {st['run_ms']:.3f} ms  GTEPS={g.m/st['run_ms']/1e6:.2f}  "
                  f"upd={st['updates']} light={st['light_arcs']} heavy={st['heavy_arcs']} "
                  f"settled={st['vertices_settled']} stale={st['stale_items']} chunks={st['hub_chunks']} "
                  f"bins t/w/c={st['bin_thread']}/{st['bin_warp']}/{st['bin_cta']} buckets={st['buckets']} "
                  f"rescans={st['rescans']} reach={st['reachable']}", flush=True)
            pr = G.profile()
            cyc = sum(pr[k] for k in ("claim", "stage", "task", "tail", "barrier"))
            print("    profile %: " + " ".join(f"{k}={100*pr[k]/max(cyc,1):.1f}" for k in ("claim", "stage", "task", "tail", "barrier"))
                  + f" batches={pr['batches']} tasks={pr['tasks']} avg_task_cyc(w0)={pr['task']/max(pr['tasks'],1)*1.0:.0f}", flush=True)
            if pr["lat_n"]:
                n = pr["lat_n"]
                print(f"    task latency (cycles, warp 0): arc={pr['lat_arc']/n:.0f} probe={pr['lat_probe']/n:.0f} "
                      f"atom={pr['lat_atom']/n:.0f} stage={pr['lat_stage']/n:.0f} atomics_issued={pr['atoms']}", flush=True)
        if a.samples:
            smp = G.samples()
            tr0 = G.trace()
            t0 = tr0[0]["t_us"] if tr0 else 0.0
            import collections
            byb = collections.defaultdict(list)
            bat = collections.defaultdict(list)
            for x in smp:
                (byb if x.get("kind", "claim") == "claim" else bat)[x["cur"]].append(x)
            print("  batches per bucket (sampled CTAs): n  tasks/batch  stage/task/tail kcycles per batch"
                  "  [LAT builds: warp-0 probe / staging kcycles per batch]")
            for b in sorted(bat):
                xs = bat[b]
                n = len(xs)
                print(f"   bucket {b}: {n:5d}  {sum(x['tasks'] for x in xs)/n:7.1f}  "
                      f"{sum(x['cyc_stage'] for x in xs)/n/1e3:6.2f} {sum(x['cyc_task'] for x in xs)/n/1e3:6.2f} "
                      f"{sum(x['cyc_tail'] for x in xs)/n/1e3:6.2f}   "
                      f"[{sum(x['tb_tasks'] for x in xs)/n/1e3:6.2f} {sum(x['ranges'] for x in xs)/n/1e3:6.2f}]")
            # claim latency per sampled CTA: end of its previous batch -> end of this claim
            # (diagnostics builds), with the unclaimed backlog (tail - claim position) it saw
            per = collections.defaultdict(list)
            for x in smp:
                per[x["cta"]].append(x)
            gaps = collections.defaultdict(list)
            for xs in per.values():
                xs.sort(key=lambda x: x["t_ns"])
                for a_, b_ in zip(xs, xs[1:]):
                    if a_.get("kind") == "batch" and b_.get("kind", "claim") == "claim" and b_["claimed"]:
                        gaps[b_["cur"]].append(((b_["t_ns"] - a_["t_ns"]) / 1e3, b_["tail"] - b_["pos"], b_["claimed"]))
            print("  claim latency (us, sampled CTAs: previous batch end -> claim end): bucket n  p50 p90 max"
                  "  | backlog tail-pos at the claim p10 p50  | items p50")
            for b in sorted(gaps):
                g = sorted(x[0] for x in gaps[b])
                bl = sorted(x[1] for x in gaps[b])
                it = sorted(x[2] for x in gaps[b])
                q = lambda v, f: v[min(len(v) - 1, int(f * len(v)))]
                print(f"   bucket {b}: {len(g):5d}  {q(g,.5):7.2f} {q(g,.9):7.2f} {g[-1]:7.2f}  | {q(bl,.1):9d} {q(bl,.5):9d}"
                      f"  | {q(it,.5):5d}")
            base = min((x["t_ns"] for x in smp), default=0)
            print(f"  samples: {len(smp)} (every 37th CTA's phase-1 claims); per bucket, 50 us windows: "
                  "t_us  claims  items  tail(max)  pend(max)")
            for b in sorted(byb):
                xs = sorted(byb[b], key=lambda x: x["t_ns"])
                tb = xs[0]["t_ns"]
                win = collections.defaultdict(list)
                for x in xs:
                    win[int((x["t_ns"] - tb) / 50e3)].append(x)
                print(f"   bucket {b}: {len(xs)} claims over {(xs[-1]['t_ns']-tb)/1e3:.1f} us "
                      f"(from +{(tb-base)/1e3:.1f} us)")
                if len(xs) > 20:
                    for w in sorted(win):
                        ys = win[w]
                        print(f"      {w*50:6d}  {len(ys):5d}  {sum(y['claimed'] for y in ys):7d}  "
                              f"{max(y['tail'] for y in ys):9d}  {max(y['pend'] for y in ys):9d}")
        if not a.quiet:
            tr = G.trace()
            prev = 0.0
            prev_rel = 0.0
            print("  columns: t(last arrival)  (+since previous)  kind ... | work = first arrival - previous "
                  "release, drain = last - first arrival, step = release - last arrival")
            for e in tr:
                if "t_first_us" in e and e["which"] != 8:
                    print(f"      | work {e['t_first_us']-prev_rel:8.1f}  drain {e['t_us']-e['t_first_us']:7.1f}  "
                          f"step {e['t_rel_us']-e['t_us']:5.1f} us")
                    prev_rel = e["t_rel_us"]
                print(f"  {e['t_us']:10.1f} us (+{e['t_us']-prev:8.1f})  {NAMES.get(e['which'], e['which']):5s} "
                      f"cur={e['cur']} tail={e['tail']} mode={e['mode']}"
                      + (f"  closed b{e['closed_b']} C={e['closed_c']}" if e.get("closed_b", 0xFFFFFFFF) != 0xFFFFFFFF else ""))
                prev = e["t_us"]


if __name__ == "__main__":
    main()
