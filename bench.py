#!/usr/bin/env python
"""bench.py -- PHAST multi-tree sweep throughput on B200 (driver contract).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--k 64] [--impl phast|reference]

A step is one pass of the whole hot path (source intake,
upward CH searches, seeding, the level-ordered downward sweep, result left in HBM)
over one batch of k synthetic sources on the Europe-scale synthetic road graph
(BASELINE.json metric: "SSSP trees/sec on 18M-vertex road-like graph"; configs[2]).
value = trees/s over all ranks (weak scaling: every rank sweeps its own sources on
its own replica of the graph; no collective on the data path).  Rank 0 prints ONE
JSON line.  `--impl reference` times the oracle (binary-heap Dijkstra on the
original graph, oracle/) on the host cores instead -- the reference arm of this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import phastgen  # noqa: E402

METRIC = "SSSP trees/sec on 18M-vertex road-like graph at 1/2/4/8 B200; sweep HBM GB/s"
THROTTLE_BITS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
                 0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
                 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown",
                 0x100: "display_clock_setting"}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class Clocks:
    """nvidia-smi sampler during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, dev):
        self.dev = dev
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.dev), "--query-gpu=clocks.sm,clocks.max.sm,clocks_event_reasons.active",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None
        time.sleep(0.25)
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        for r in self.rows:
            try:
                a, b, c = [x.strip() for x in r.split(",")]
                sm.append(float(a))
                mx = max(mx, float(b))
                bits = int(c, 16)
                for bit, name in THROTTLE_BITS.items():
                    if bits & bit and name != "gpu_idle":
                        reasons.add(name)
            except Exception:
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


def build_graph(cfg_name):
    cfg = phastgen.CONFIGS[cfg_name]
    t = time.time()
    g = cfg["graph"]()
    log(f"[bench] {cfg_name}: generated n={g.n} m={g.m} in {time.time() - t:.1f}s")
    return g, cfg


def source_table(n, cfg, rank, batches, k):
    """Seeded sources: batch b of rank r draws k uniform sources."""
    return [phastgen.sources(n, k, seed=cfg["src_seed"] * 1_000_003 + rank * 100_003 + b) for b in range(batches)]


def oracle_sample(g, cfg, threads, count):
    import oracle
    src = phastgen.sources(g.n, count, seed=cfg["src_seed"] + 777)
    t = time.perf_counter()
    oracle.tree_maxima(g, src, threads=threads)
    dt = time.perf_counter() - t
    return count / dt, dt, src


def run_reference(args):
    """Reference arm: the oracle as it stands, on the host cores, same metric/config."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    g, cfg = build_graph(args.config)
    threads = os.cpu_count() or 1
    per_step = threads
    for _ in range(args.warmup):
        oracle_sample(g, cfg, threads, per_step)
    t = time.perf_counter()
    for s in range(args.steps):
        oracle_sample(g, cfg, threads, per_step)
    dt = time.perf_counter() - t
    value = per_step * args.steps / dt
    sample = f"{per_step} uniform sources per step (one per thread), full {args.config} graph, {args.steps} steps"
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "trees/s", "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg['desc']}", "n": g.n, "m": g.m, "sources_per_step": per_step},
        "cpu_baseline": {"value": value, "unit": "trees/s", "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "trees/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--impl", default="phast", choices=["phast", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cache", default="", help="hierarchy file to reuse/create (optional)")
    ap.add_argument("--layout", default="levels-bfs", choices=["wavefront", "levels", "levels-bfs", "diagonal"],
                    help="vertex order: wavefront, the paper's level layout (DFS within a level), or level "
                         "layout with BFS order within a level (default)")
    ap.add_argument("--delta", type=int, default=0, help="wavefront skew (0 = library default)")
    ap.add_argument("--parents", action="store_true",
                    help="also time the parent-pointer pass (phast_parents, NEXT-1) on the last batch")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_dellinggnw11_b200 as P

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def barrier():
        if world > 1:
            dist.barrier()

    g, cfg = build_graph(args.config)
    k = args.k
    bopts = dict(layout=args.layout, delta=args.delta)
    # hierarchy: rank 0 builds (host CH, not the timed target) and shares it via a file
    path = args.cache or f"/tmp/phast_{args.config}_{os.getpid() if world == 1 else 'dist'}.phast"
    if world > 1:
        from paper_conf_ipps_dellinggnw11_b200.parallel import share_hierarchy
        t = time.time()
        h = share_hierarchy(lambda: P.Phast.from_graph(g, **bopts), P.Phast.load, path, rank, barrier)
        log(f"[bench] rank {rank}: hierarchy ready in {time.time() - t:.1f}s")
    elif args.cache and os.path.exists(args.cache):
        h = P.Phast.load(args.cache)
    else:
        t = time.time()
        h = P.Phast.from_graph(g, **bopts)
        log(f"[bench] CH build {time.time() - t:.1f}s")
        if args.cache:
            h.save(args.cache)
    info = h.info()
    lsz = h.level_sizes()
    log(f"[bench] n={info.n} m={info.m} m_up={info.m_up} m_down={info.m_down} n_tail={info.n_tail} "
        f"levels={info.levels} L0={lsz[0] / info.n:.3f} CH={info.build_seconds:.1f}s")

    stream = torch.cuda.current_stream()
    sptr = stream.cuda_stream
    dist_buf = torch.empty((g.n, k), dtype=torch.int32, device="cuda")
    srcs = source_table(g.n, cfg, rank, args.warmup + args.steps, k)

    for b in range(args.warmup):
        h.trees_into(srcs[b], dist_buf.data_ptr(), sptr)
    h.sync(stream)

    # ---------------------------------------------------------------- timed region
    # working set: the n*k*4-byte label array (4.6 GB at C3, k=64) >> 126 MB L2: no flush needed
    # small configs (C1, C2: labels + graph fit in L2): every timed step starts from a
    # flushed L2 (a 512 MB write between steps, outside the step's events)
    flush = 4 * k * info.n + 16 * info.m_down < 256e6
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if flush:
        scrub = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(local) as clk:
        barrier()
        torch.cuda.synchronize()
        h.timing(True)
        l0 = P.launch_count()
        t0.record(stream)
        for i, b in enumerate(range(args.warmup, args.warmup + args.steps)):
            if flush:
                scrub.fill_(i & 0xFF)
                torch.cuda.synchronize()   # the step's upward search (side stream) starts after ev[i][0]
                ev[i][0].record(stream)
            h.trees_into(srcs[b], dist_buf.data_ptr(), sptr)
            if flush:
                ev[i][1].record(stream)
        t1.record(stream)
        torch.cuda.synchronize()
        launches = P.launch_count() - l0
        barrier()
    h.timing(False)
    h.sync(stream)
    ms = sum(a.elapsed_time(b) for a, b in ev) if flush else t0.elapsed_time(t1)
    ms_up, ms_sweep, nb = h.timing_read()
    if world > 1:
        tt = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    trees = world * args.steps * k
    value = trees / (ms / 1e3)

    # roofline of the dominant kernel (the level sweep; one "launch" = one whole sweep)
    B_alg = 8 * info.m_down + 4 * (info.n + 1) + 4 * k * info.n + 4 * k * info.n_tail + info.n / 8
    sweep_ms = ms_sweep / max(nb, 1)
    achieved = B_alg / (sweep_ms / 1e3) / 1e9
    peak, peak_src = peaks()
    traffic = None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "sweep_traffic.json")))
        key = f"{args.config}_k{k}"
        e = prof.get(key, {})
        default_path = not any(os.environ.get(v) for v in ("PHAST_SWEEP", "PHAST_ARC_BATCH", "PHAST_TOP",
                                                            "PHAST_FUSED", "PHAST_TOP_MAXV"))
        if e.get("layout") == P.LAYOUT_NAMES[info.layout] and default_path and e.get("arc_batch") == "ell":
            traffic = e["dram_bytes_per_sweep"]   # ncu launch list of this configuration (warm L2)
    except Exception:
        pass

    # NEXT-1: parent pointers of the last timed batch (a separate pass, not in `value`)
    parents = None
    if args.parents:
        par_buf = torch.empty((g.n, k), dtype=torch.int32, device="cuda")
        last = srcs[args.warmup + args.steps - 1]
        h.parents(last, dist_buf, out=par_buf, stream=stream)
        h.sync(stream)
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = max(1, min(args.steps, 10))
        p0.record(stream)
        for _ in range(reps):
            h.parents(last, dist_buf, out=par_buf, stream=stream)
        p1.record(stream)
        h.sync(stream)
        pms = p0.elapsed_time(p1) / reps
        m_in = g.m   # original arcs (self-loops, if any, are dropped by the library)
        B_par = 8 * m_in + 4 * (g.n + 1) + 12 * k * g.n
        parents = {"ms_per_pass": pms, "alg_bytes": B_par, "achieved_GBps": B_par / (pms / 1e3) / 1e9,
                   "frac": B_par / (pms / 1e3) / 1e9 / peaks()[0],
                   "note": "B = 8m + 4(n+1) + 12kn: in-arcs, offsets, own row read, in-neighbour rows read "
                           "at least once, parent row written"}
        del par_buf

    # end to end through the public host entry point (sources in, all labels out)
    e2e = None
    if args.e2e_steps > 0:
        host_out = torch.empty((g.n, k), dtype=torch.int32, pin_memory=True).numpy().view(np.uint32)
        h.trees_host(srcs[0], host_out, stream)
        barrier()
        te = time.perf_counter()
        for b in range(args.e2e_steps):
            h.trees_host(srcs[args.warmup + b % args.steps], host_out, stream)
        te = time.perf_counter() - te
        if world > 1:
            tt = torch.tensor([te], dtype=torch.float64, device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            te = float(tt.item())
        e2e = {"value": world * args.e2e_steps * k / te, "unit": "trees/s", "h2d_bytes_per_step": 4 * k,
               "d2h_bytes_per_step": 4 * k * g.n,
               "note": "phast_trees_host: sources in as kernel parameters, all n*k labels copied to pinned host memory"}
        del host_out

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        threads = os.cpu_count() or 1
        v, dt, s = oracle_sample(g, cfg, threads, threads)
        cpu = {"value": v, "unit": "trees/s", "cores": threads, "kind": "oracle",
               "sample": f"{threads} uniform sources of the full {args.config} graph, one per thread, "
                         f"binary-heap Dijkstra, {dt:.1f}s wall"}
        if k == 1:   # latency configs (C1): one tree on one core, against the GPU's us/tree
            v1, dt1, _ = oracle_sample(g, cfg, 1, 8)
            cpu["us_per_tree_1thread"] = dt1 / 8 * 1e6

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "trees/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": f"{args.config}: {cfg['desc']}", "k": k, "trees_per_step_per_gpu": k,
                       "n": info.n, "m": info.m, "m_down": info.m_down, "m_up": info.m_up, "n_tail": info.n_tail,
                       "levels": info.levels, "layout": P.LAYOUT_NAMES[info.layout],
                       "delta": info.delta, "sweep": os.environ.get("PHAST_SWEEP", "levels" if info.layout else "warp"), "parallelism": f"sources sharded over {world} GPU(s), graph replicated",
                       "l2": ("L2 flushed before every timed step (512 MB write outside the step's events); "
                              "value = steps * k / sum of per-step times") if flush else
                             f"label array {4 * k * info.n / 1e9:.2f} GB >> 126 MB L2 (no flush needed)",
                       "us_per_tree": ms * 1e3 / (args.steps * k),
                       "ch_build_s": round(info.build_seconds, 1)},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": traffic, "kernel": "sweep_top_kernel + sweep_kernel (all levels of one sweep)",
                         "alg_bytes_per_sweep": B_alg, "sweep_ms": sweep_ms, "upward_ms": ms_up / max(nb, 1),
                         "peak_source": peak_src},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clk.summary(),
            **({"parents": parents} if parents else {}),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    h.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
