#!/usr/bin/env python3
"""Benchmark: single-source SSSP GTEPS on a B200 (BASELINE.json metric).

A "step" is one whole bucket-aware asynchronous Delta-stepping SSSP (all
SURVEY §8(a) rows a5-a7: init, phase 1, phases 2&3) from one seeded source on
the resident, PRO-reordered graph. Default workload: C4 = Kronecker scale-24
edgefactor-16, u32 weights U{1..100}, Delta=32 (the north star's ">= 50% of
HBM on scale-24 RMAT" config). GTEPS = m / time with m = EF * 2^SCALE input
edges.

Multi-GPU (torchrun): the graph is replicated, the 64 sources are sharded
round-robin (sources[rank::N]), each rank runs K steps; value = N*K*m / max
rank time ("scaling": "weak"). `--impl reference` times the CPU oracle
(plain Dijkstra, oracle/) on a bounded sample of the same workload.

Prints ONE JSON line on rank 0.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PAPER_V100 = {"C3": 16.78, "C4": 20.16}  # GTEPS, PAPER Fig. 11, context only
MULTI_DELTA = {"C1": 64, "C3": 0.1, "C4": 4, "C5": 2}  # sssp_run_multi default Delta (profiles/r01c/multi_delta_sweep.txt)
METRIC = "SSSP GTEPS (m/time) at 1 GPU; multi-source GTEPS at 1/2/4/8 B200; HBM GB/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C4", choices=["C1", "C2", "C3", "C4", "C5"])
    ap.add_argument("--delta", type=float, default=None)
    ap.add_argument("--no-reorder", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--sources", type=int, default=64)
    ap.add_argument("--ctas-per-sm", type=int, default=0)
    ap.add_argument("--profile", action="store_true", help="short run for ncu (no clocks/cpu/e2e)")
    ap.add_argument("--no-pull", action="store_true", help="push-style phases 2&3 in every bucket")
    ap.add_argument("--multi", action="store_true",
                    help="NEXT-4: a step is one group of up to 32 of the rank's sources through sssp_run_multi")
    return ap.parse_args()


def workload_desc(name, cfg, delta, reorder):
    import gen

    c = dict(gen.CONFIGS[name])
    if c["kind"] == "kron":
        d = (f"{name}: Kronecker scale-{c['scale']} edgefactor-{c['edgefactor']} (Graph500 A=.57 B=.19 C=.19 "
             f"D=.05, scrambled, symmetrised), {c['weights']} weights, delta={delta}, reorder={'on' if reorder else 'off'}")
    else:
        d = (f"{name}: road-like grid {c['W']}x{c['H']} (horizontal + p={c['p']} vertical), {c['weights']} "
             f"weights, delta={delta}, reorder={'on' if reorder else 'off'}")
    return d, c


class ClockSampler:
    """NVML samples of SM clock + throttle reasons during the timed region."""

    REASONS = {
        0x0000000000000004: "sw_power_cap",
        0x0000000000000008: "hw_slowdown",
        0x0000000000000020: "sw_thermal_slowdown",
        0x0000000000000040: "hw_thermal_slowdown",
        0x0000000000000080: "hw_power_brake_slowdown",
        0x0000000000000002: "applications_clocks_setting",
    }

    def __init__(self, dev_index):
        self.ok = False
        self.samples = []
        self.reasons = set()
        try:
            import pynvml

            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None
        self._stop = threading.Event()

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def algorithmic_bytes(g, dist_bits, inf):
    """SURVEY §8(d) B_alg per SSSP: 8*A_r (arc stream) + 48*V_r (row pair, dist,
    queue push/pop, settle list, atomic) + 12*V (init + output)."""
    reach = dist_bits != inf
    deg = np.diff(g.row)
    A_r = int(deg[reach].sum())
    V_r = int(reach.sum())
    return 8 * A_r + 48 * V_r + 12 * g.V, A_r, V_r


def load_traffic(config):
    """ncu dram bytes per launch of the persistent kernel, from the committed summary."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(path) as f:
            d = json.load(f)
        return d.get(config, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def measured_peak():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def host_info():
    """Host cores and CPU model (cpu_baseline context)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def cpu_baseline(g, sources, budget_s=30.0, parallel=False):
    """The oracle as it stands (binary-heap Dijkstra, oracle/) on a bounded sample.
    parallel=False: single-threaded, sources one after another until ~budget_s/2
    (C1-C4 protocol). parallel=True (multi-source batches, C5 protocol of
    BASELINE.md §3): one wave of min(nproc, len(sources)) sources, one per
    thread (the C oracle runs without the GIL), wall time."""
    import oracle

    info = host_info()
    if parallel:
        from concurrent.futures import ThreadPoolExecutor

        nt = max(1, min(info["nproc"] or 1, len(sources), 32))  # <= 32: ~1.6 GB of oracle state each at s26
        t0 = time.perf_counter()
        with ThreadPoolExecutor(nt) as ex:
            list(ex.map(lambda s: oracle.dijkstra(g.row, g.col, g.w, int(s)), list(sources[:nt])))
        dt = time.perf_counter() - t0
        return {"value": round(nt * g.m / dt / 1e9, 6), "unit": "GTEPS", "cores": nt, "kind": "oracle",
                "sample": f"{nt} source(s) of the full {g.name} graph in parallel, one binary-heap Dijkstra "
                          f"per thread ({dt:.1f} s wall)", **info}
    t0 = time.perf_counter()
    n = 0
    for s in sources:
        oracle.dijkstra(g.row, g.col, g.w, int(s))
        n += 1
        if time.perf_counter() - t0 > budget_s * 0.5:
            break
    dt = time.perf_counter() - t0
    return {"value": round(n * g.m / dt / 1e9, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"{n} source(s) of the full {g.name} graph, single-threaded binary-heap Dijkstra "
                      f"({dt:.1f} s)", **info}


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    import gen

    cfg = gen.CONFIGS[args.config]
    delta = args.delta if args.delta is not None else cfg["delta"]
    reorder = not args.no_reorder
    desc, c = workload_desc(args.config, cfg, delta, reorder)

    if args.impl == "reference":
        if rank != 0:
            return
        g = gen.make_config(args.config)
        srcs = gen.sample_sources(g, args.sources, seed=7)
        import oracle

        steps = []
        for k in range(args.warmup + args.steps):
            t0 = time.perf_counter()
            oracle.dijkstra(g.row, g.col, g.w, int(srcs[k % len(srcs)]))
            dt = time.perf_counter() - t0
            if k >= args.warmup:
                steps.append(dt)
            if sum(steps) > 150:  # bounded: keep the reference arm within minutes
                break
        t = sum(steps)
        val = len(steps) * g.m / t / 1e9
        line = {"impl": "reference", "metric": METRIC, "value": round(val, 6), "unit": "GTEPS", "n_gpus": args.gpus,
                "steps": len(steps), "steps_requested": args.steps,
                "steps_note": "the oracle arm is bounded to ~150 s of CPU work, so it may run fewer steps "
                              "than requested; value is per step it ran",
                "warmup": args.warmup, "ms_per_step": round(1e3 * t / len(steps), 3),
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": cfg["weights"],
                "data": "synthetic",
                "config": {"workload": desc, "parallelism": "cpu oracle, rank 0 only"},
                "cpu_baseline": {"value": round(val, 6), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                                 "sample": f"{len(steps)} source(s) of the full graph, single-threaded Dijkstra",
                                 **host_info()},
                "e2e": {"value": round(val, 6), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
        print(json.dumps(line), flush=True)
        return

    import torch

    # SSSP_DIST_BACKEND=gloo (test only): exercise the multi-rank logic with
    # several ranks sharing fewer GPUs; the product path is NCCL, one GPU per rank.
    backend = os.environ.get("SSSP_DIST_BACKEND", "nccl")
    dev = (local % torch.cuda.device_count()) if world > 1 else 0
    if world > 1:
        import torch.distributed as dist

        torch.cuda.set_device(dev)
        if backend == "nccl":
            # communicator setup lines (nranks, NVLS / P2P transport) on stderr, so the one JSON
            # line stays alone on stdout and the driver can check the communicator size
            os.environ.setdefault("NCCL_DEBUG", "INFO")
            os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
            os.environ.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
    tdev = f"cuda:{dev}" if backend == "nccl" else "cpu"
    torch.cuda.set_device(dev)
    import paper_conf_icppw_zhangczsdhay23_b200 as sssp

    t_gen = time.perf_counter()
    g = gen.make_config(args.config)
    t_gen = time.perf_counter() - t_gen
    sources = gen.sample_sources(g, args.sources, seed=7)
    from paper_conf_icppw_zhangczsdhay23_b200 import batch

    mine = batch.shard_sources(sources, rank, world)  # contiguous blocks (batch.py)
    stream = torch.cuda.Stream(device=dev)
    G = sssp.Graph(g.row, g.col, g.w, device=dev, stream=stream)
    if gen.CONFIGS[args.config].get("symmetric", True) and not args.no_pull:
        # the generators symmetrise every config (reading R13): large buckets may pull
        G.set_param(sssp.SSSP_PARAM_PULL_SYMMETRIC, 1)
    if args.ctas_per_sm:
        G.set_param(sssp.SSSP_PARAM_CTAS_PER_SM, args.ctas_per_sm)
    reorder_ms = None
    if reorder:
        G.reorder()
        torch.cuda.synchronize(dev)
        reorder_ms = G.stats()["reorder_ms"]
    inf = 0x7F800000 if g.wtype == "f32" else 0xFFFFFFFF
    if args.multi:
        # swept on B200 (profiles/r01c/multi_delta_sweep.txt): the batched kernel prefers wide buckets
        if args.delta is None:
            delta = MULTI_DELTA.get(args.config, delta)
            desc, _ = workload_desc(args.config, cfg, delta, reorder)
        return bench_multi(args, G, g, sources, mine, delta, desc, world, rank, dev, tdev, stream,
                           reorder, reorder_ms, t_gen, inf)

    def step(k):
        G.run(int(mine[k % len(mine)]), delta)

    for k in range(args.warmup):
        step(k)
    stream.synchronize()
    G.kernel_time(reset=True)

    # ---------------- timed region (device events on the library's stream)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize(dev)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev)
    with sampler if not args.profile else _Null():
        ev0.record(stream)
        for k in range(args.steps):
            step(args.warmup + k)
        ev1.record(stream)
        ev1.synchronize()
    torch.cuda.synchronize(dev)
    t_ms = ev0.elapsed_time(ev1)
    kt_total, kt_n = G.kernel_time(reset=True)
    if world > 1:
        tt = torch.tensor([t_ms], device=tdev)
        torch.distributed.all_reduce(tt, op=torch.distributed.ReduceOp.MAX)
        torch.distributed.barrier()
        t_ms = float(tt.item())
    st = G.stats()
    value = world * args.steps * g.m / (t_ms * 1e-3) / 1e9

    # ---------------- multi-GPU end to end: every step each rank runs one source,
    # the N distance rows are gathered to rank 0 over NCCL and copied to pinned host
    e2e_multi = None
    if world > 1 and not args.no_e2e and not args.profile:
        ne = min(args.steps, 16)
        # rank 0 copies step k's gathered rows to pinned host memory on a copy stream while
        # step k+1 runs (double-buffered); every copy finishes inside the timed region
        pinned = [torch.empty((world, g.V), dtype=torch.int32).pin_memory() for _ in range(2)] \
            if rank == 0 else None
        cs = torch.cuda.Stream(device=dev) if rank == 0 else None
        keep = [None, None]
        torch.distributed.barrier()
        t0 = time.perf_counter()
        for k in range(ne):
            step_src = sources[(k * world) % len(sources):][:world]
            rows = batch.run_sharded(G, step_src, delta, dst=0, kernel="per_source")
            if rank == 0:
                b = k % 2
                if keep[b] is not None:
                    cs.synchronize()  # pinned[b] / keep[b] are free again
                ev = torch.cuda.Event()
                ev.record(torch.cuda.current_stream(dev))
                cs.wait_event(ev)
                with torch.cuda.stream(cs):
                    src_rows = rows.view(torch.int32) if rows.dtype != torch.int32 else rows
                    pinned[b].copy_(src_rows, non_blocking=rows.is_cuda)
                keep[b] = rows  # keep the device rows alive until their copy is done
        if rank == 0:
            cs.synchronize()
        torch.distributed.barrier()
        te = torch.tensor([time.perf_counter() - t0], device=tdev)
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
        e2e_multi = {"value": round(world * ne * g.m / float(te.item()) / 1e9, 4), "unit": "GTEPS",
                     "h2d_bytes_per_step": 8 * world, "d2h_bytes_per_step": 4 * g.V * world,
                     "note": "per step: one source per rank, NCCL gather of the N distance rows to rank 0, "
                             "rank 0 copies them to pinned host (overlapped with the next step); wall "
                             "clock, max over ranks"}

    if rank != 0:
        if world > 1:
            torch.distributed.barrier()
            torch.distributed.destroy_process_group()
        return

    # ---------------- roofline of the dominant kernel (persistent Delta-stepping kernel)
    used = [int(mine[(args.warmup + k) % len(mine)]) for k in range(args.steps)]
    distinct = sorted(set(used))
    balg = {}
    out = np.empty(g.V, dtype=np.uint32 if g.wtype == "u32" else np.float32)
    for s in distinct[:16]:
        G.run(s, delta)
        G.distances(out)
        balg[s] = algorithmic_bytes(g, out.view(np.uint32), inf)
    mean_b = float(np.mean([balg.get(s, balg[distinct[0]])[0] for s in used]))
    kt_avg_ms = kt_total / max(kt_n, 1)
    peak, peak_kind = measured_peak()
    achieved = mean_b / (kt_avg_ms * 1e-3) / 1e9
    roof = {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
            "frac": round(achieved / peak, 4), "traffic": load_traffic(args.config),
            "peak_kind": peak_kind, "kernel": "k_delta_step (persistent)",
            "kernel_ms_avg": round(kt_avg_ms, 4), "kernel_share_of_step": round(kt_total / t_ms, 4),
            "alg_bytes_per_launch": int(mean_b)}

    # ---------------- end-to-end through the public API, host buffers
    e2e = None
    if not args.no_e2e and not args.profile and world > 1:
        e2e = e2e_multi  # measured collectively above (all ranks)
    elif not args.no_e2e and not args.profile:
        # two pinned result buffers: step k's distances stream to the host (sssp_distances_async,
        # the library's output stream) while step k+1 runs; one sssp_wait ends the timed region
        pinned = [torch.empty(g.V, dtype=torch.int32).pin_memory() for _ in range(2)]
        ne = args.steps  # the device-timed loop's steps and sources (run time varies by source)
        for k in range(2):
            G.run(int(mine[k % len(mine)]), delta)
            G.distances_async(pinned[k % 2])
        G.wait()
        t0 = time.perf_counter()
        for k in range(ne):
            G.run(int(mine[(args.warmup + k) % len(mine)]), delta)  # source id host -> device (launch argument)
            G.distances_async(pinned[k % 2])  # D2H of the result, overlapped with the next run
        G.wait()
        te = time.perf_counter() - t0
        e2e = {"value": round(ne * g.m / te / 1e9, 4), "unit": "GTEPS", "h2d_bytes_per_step": 8,
               "d2h_bytes_per_step": 4 * g.V,
               "note": "graph resident (uploaded+reordered once, like weights); per step: source id in, "
                       "V distances out to pinned host memory (overlapped with the next step via "
                       "sssp_distances_async; all copies complete inside the timed region); wall clock"}

    cpu = None
    if not args.no_cpu_baseline and not args.profile and world == 1:
        cpu = cpu_baseline(g, sources)

    line = {
        "metric": METRIC, "value": round(value, 4), "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(t_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32" if g.wtype == "u32" else "f32",
        "data": "synthetic",
        "config": {"workload": desc, "V": g.V, "m_edges": g.m, "arcs": g.A, "delta": delta,
                   "reorder": reorder, "reorder_ms": reorder_ms, "sources": len(sources),
                   "pull_phase2": not args.no_pull,
                   "parallelism": f"replicas x{world} (sources sharded, graph replicated)",
                   "l2": "inputs larger than L2 (arc array %.2f GB > 126 MB L2); dist re-initialised every step" % (8 * g.A / 1e9),
                   "gen_s": round(t_gen, 1), "grid_ctas": st["grid_ctas"], "ring_slots": st["ring_slots"],
                   "paper_v100_gteps_context": PAPER_V100.get(args.config)},
        "roofline": roof,
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": 3 * args.steps,
        "clocks": sampler.summary() if not args.profile else None,
        "last_run_stats": {k: st[k] for k in ("updates", "light_arcs", "heavy_arcs", "vertices_settled",
                                              "stale_items", "hub_chunks", "buckets", "rescans", "reachable")},
    }
    print(json.dumps(line), flush=True)
    G.close()
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


def multi_alg_bytes(g, dist_bits, inf, lanes):
    """Algorithmic bytes of one sssp_run_multi group (NEXT-4 design):
    every reachable vertex expanded once -> its arcs streamed once (8 B) and one
    128-byte D row probed per arc; one row read per expansion + 16 B of queue
    traffic; init of D and Q (132 B per vertex) and the output gather (128 B row
    read + 4 B per source per vertex)."""
    reach = dist_bits != inf
    deg = np.diff(g.row)
    A_r, V_r = int(deg[reach].sum()), int(reach.sum())
    return 136 * A_r + 144 * V_r + (132 + 128 + 4 * lanes) * g.V, A_r, V_r


def bench_multi(args, G, g, sources, mine, delta, desc, world, rank, dev, tdev, stream, reorder, reorder_ms,
                t_gen, inf):
    """NEXT-4 bench: each step runs one group of <= 32 of this rank's sources
    through sssp_run_multi (one persistent launch); value = sources*m / time."""
    import torch

    L = 32
    groups = [list(mine[i:i + L]) for i in range(0, len(mine), L)] or [[]]
    out = torch.empty((L, g.V), dtype=torch.int32, device=f"cuda:{dev}")

    def step(k):
        G.run_multi(groups[k % len(groups)], delta, out)

    for k in range(args.warmup):
        step(k)
    torch.cuda.synchronize(dev)
    G.kernel_time(reset=True)
    if world > 1:
        torch.distributed.barrier()
    torch.cuda.synchronize(dev)
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    sampler = ClockSampler(dev)
    with sampler if not args.profile else _Null():
        ev0.record(stream)
        for k in range(args.steps):
            step(args.warmup + k)
        ev1.record(stream)
        ev1.synchronize()
    torch.cuda.synchronize(dev)
    t_ms = ev0.elapsed_time(ev1)
    kt_total, kt_n = G.kernel_time(reset=True)
    n_src = sum(len(groups[(args.warmup + k) % len(groups)]) for k in range(args.steps))
    tot = torch.tensor([t_ms, float(n_src)], device=tdev)
    if world > 1:
        t_max = tot[:1].clone()
        torch.distributed.all_reduce(t_max, op=torch.distributed.ReduceOp.MAX)
        torch.distributed.all_reduce(tot, op=torch.distributed.ReduceOp.SUM)
        t_ms, n_all = float(t_max.item()), float(tot[1].item())
    else:
        n_all = float(n_src)
    value = n_all * g.m / (t_ms * 1e-3) / 1e9
    ms = G.multi_stats()
    e2e = None
    if not args.no_e2e and not args.profile:
        # SURVEY §8(e) end to end: one step = the whole source batch through batch.run_sharded --
        # each rank computes its block of sources 32 per sssp_run_multi launch; after each group
        # its rows go to rank 0 (NCCL gather, async, overlapped with the next group; no gather
        # at N = 1) and rank 0 streams them to pinned host memory on a copy stream, also
        # overlapped with the next group. Every copy completes inside the timed region.
        from paper_conf_icppw_zhangczsdhay23_b200 import batch

        n = len(sources)
        k = batch.shard_bounds(n, 0, world)[2]
        out_all = torch.empty((world * k, g.V), dtype=torch.int32, device=f"cuda:{dev}") \
            if rank == 0 or world == 1 else None
        pinned = torch.empty((world * k, g.V), dtype=torch.int32).pin_memory() if rank == 0 else None
        cs = torch.cuda.Stream(device=dev)

        def d2h(first, cnt, work):
            if work is not None:
                work.wait()  # the current stream waits for this group's gather (no host sync)
            ev = torch.cuda.Event()
            ev.record(torch.cuda.current_stream(dev))
            cs.wait_event(ev)
            with torch.cuda.stream(cs):
                for r in range(world):
                    a = r * k + first
                    pinned[a:a + cnt].copy_(out_all[a:a + cnt], non_blocking=True)

        if world > 1:
            torch.distributed.barrier()
        t0 = time.perf_counter()
        batch.run_sharded(G, sources, delta, dst=0, kernel="multi", out=out_all,
                          on_group=d2h if rank == 0 else None)
        cs.synchronize()
        torch.cuda.synchronize(dev)
        if world > 1:
            torch.distributed.barrier()
        te = torch.tensor([time.perf_counter() - t0], device=tdev)
        if world > 1:
            torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
        e2e = {"value": round(n * g.m / float(te.item()) / 1e9, 4), "unit": "GTEPS",
               "h2d_bytes_per_step": 8 * n, "d2h_bytes_per_step": 4 * g.V * n,
               "note": "one step = the whole %d-source batch through batch.run_sharded: block-sharded "
                       "sources, 32 per sssp_run_multi launch; each group's rows gathered to rank 0 "
                       "(NCCL, async; none at N=1) and copied to pinned host on a copy stream while the "
                       "next group computes; wall clock, max over ranks" % n}
    if rank != 0:
        if world > 1:
            torch.distributed.barrier()
            torch.distributed.destroy_process_group()
        return
    row0 = out[0].cpu().numpy().view(np.uint32)
    b_alg, A_r, V_r = multi_alg_bytes(g, row0, inf, len(groups[0]))
    kt_avg = kt_total / max(kt_n, 1)
    peak, peak_kind = measured_peak()
    achieved = b_alg / (kt_avg * 1e-3) / 1e9
    cpu = None
    if not args.no_cpu_baseline and not args.profile and world == 1:
        cpu = cpu_baseline(g, sources, parallel=True)
    line = {
        "metric": METRIC, "value": round(value, 4), "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(t_ms / args.steps, 4), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "u32" if g.wtype == "u32" else "f32",
        "data": "synthetic",
        "config": {"workload": desc + f"; multi-source batch ({len(sources)} sources, <= 32 per persistent "
                                      "launch, sssp_run_multi, NEXT-4)",
                   "V": g.V, "m_edges": g.m, "arcs": g.A, "delta": delta, "reorder": reorder,
                   "reorder_ms": reorder_ms, "sources": len(sources), "sources_per_step": len(groups[0]),
                   "parallelism": f"replicas x{world} (sources sharded, graph replicated)",
                   "l2": "inputs larger than L2 (D rows %.2f GB, arcs %.2f GB > 126 MB L2); D re-initialised "
                         "every step" % (128 * g.V / 1e9, 8 * g.A / 1e9), "gen_s": round(t_gen, 1)},
        "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                     "frac": round(achieved / peak, 4), "traffic": load_traffic(args.config + "_multi"),
                     "peak_kind": peak_kind, "kernel": "k_ms_step (persistent, 32 sources)", "kernel_ms_avg": round(kt_avg, 4),
                     "kernel_share_of_step": round(kt_total / t_ms, 4), "alg_bytes_per_launch": int(b_alg)},
        "cpu_baseline": cpu,
        "e2e": e2e,
        "gpu_launches": 4 * args.steps,
        "clocks": sampler.summary() if not args.profile else None,
        "last_group_stats": ms,
    }
    print(json.dumps(line), flush=True)
    G.close()
    if world > 1:
        torch.distributed.barrier()
        torch.distributed.destroy_process_group()


class _Null:
    def __enter__(self):
        return self

    def __exit__(self, *a):
        pass

    def summary(self):
        return None


if __name__ == "__main__":
    main()
