#!/usr/bin/env python
"""bench.py -- PHAST multi-tree sweep throughput on B200 (driver contract).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--k 64]
                  [--inflight S] [--total-sources T] [--steady] [--impl phast|reference]

A step is one pass of the whole hot path (source intake,
upward CH searches, seeding, the level-ordered downward sweep, result left in HBM)
over one batch of k synthetic sources on the Europe-scale synthetic road graph
(BASELINE.json metric: "SSSP trees/sec on 18M-vertex road-like graph"; configs[2]).
Batches are issued round robin on S streams (`--inflight`, the library keeps
PHAST_SLOTS queries in flight), each stream with its own label buffer.
value = trees/s over all ranks.  Weak scaling (default): every rank sweeps `--steps`
batches of its own sources on its own replica of the graph; strong scaling
(`--total-sources T`, BASELINE configs[3] "8192 sources sharded at 1/2/4/8 B200"):
T sources split into contiguous per-rank shards.  No collective on the data path.
`--gpus N` without a torchrun environment re-launches itself under
torch.distributed.run with N ranks (one per GPU, NCCL).  Rank 0 prints ONE JSON line.
`--impl reference` times the oracle (binary-heap Dijkstra on the original graph,
oracle/) on the host cores instead -- the reference arm of this tier.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
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
L2_BYTES = 126 << 20


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


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch_distributed(args):
    """`--gpus N` (N > 1) outside torchrun: run this script under
    torch.distributed.run with N ranks on this node, NCCL communicator init logged."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    log("[bench] relaunch: " + " ".join(cmd))
    return subprocess.call(cmd, env=env)


def rank_batches(n, cfg, k, world, rank, steps, warmup, total_sources=0):
    """This rank's batches of k sources: (warm-up batches, timed batches, trees counted).
    Weak scaling: `steps` batches of its own seeded sources per rank.  Strong scaling
    (total_sources = T): one seeded list of T sources split into contiguous per-rank
    shards (parallel.shard); a ragged last batch is padded with duplicates of its first
    source, whose extra trees are not counted."""
    from paper_conf_ipps_dellinggnw11_b200.parallel import shard
    warm = source_table(n, cfg, rank + 7919, warmup, k)
    if not total_sources:
        return warm, source_table(n, cfg, rank, steps, k), steps * k
    lo, hi = shard(total_sources, world, rank)
    mine = phastgen.sources(n, total_sources, seed=cfg["src_seed"] * 7919 + 1)[lo:hi]
    timed = [mine[i:i + k] for i in range(0, mine.size, k)]
    timed = [b if b.size == k else np.concatenate([b, np.repeat(b[:1], k - b.size)]).astype(np.uint32)
             for b in timed]
    return warm, timed, int(hi - lo)


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
        "higher_is_better": True, "scaling": "strong" if args.total_sources else "weak", "vs_baseline": None,
        "dtype": "u32", "data": "synthetic",
        "config": {"workload": f"{args.config}: {cfg['desc']}", "n": g.n, "m": g.m, "sources_per_step": per_step},
        "cpu_baseline": {"value": value, "unit": "trees/s", "cores": threads, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": "trees/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def try_load(P, path):
    """A cached hierarchy, or None if the file is stale (another format version) or unreadable."""
    try:
        return P.Phast.load(path)
    except P.PhastError as e:
        log(f"[bench] cache {path} not loaded ({e}); rebuilding")
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--inflight", type=int, default=0,
                    help="streams with a batch in flight (1..8; 0 = auto: 8 on small graphs whose labels fit L2, "
                         "1 on large ones, where overlapping sweeps thrash L2: measured slower, DESIGN.md §6)")
    ap.add_argument("--total-sources", type=int, default=0,
                    help="strong scaling: this many sources split over the ranks (C4: 8192); steps is derived")
    ap.add_argument("--steady", action="store_true",
                    help="small configs: no L2 flush between steps (steady state; label buffers rotate)")
    ap.add_argument("--impl", default="phast", choices=["phast", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-probes", action="store_true")
    ap.add_argument("--cache", default="", help="hierarchy file to reuse/create (optional)")
    ap.add_argument("--layout", default="levels-bands", choices=["levels", "levels-bfs", "levels-bands"],
                    help="vertex order: the paper's level layout (DFS within a level), BFS within a level, or "
                         "BFS with the bottom levels in bands of closed groups (default)")
    ap.add_argument("--band-unit", type=int, default=0,
                    help="vertices per work unit of a band launch (phast_query_opts band_unit; 0 = 8192/k)")
    ap.add_argument("--band-threads", type=int, default=0, help="CTA size of a band launch (128/256; 0 = 128)")
    ap.add_argument("--band-variant", type=int, default=0, help="band kernel variant (phast_query_opts band_variant)")
    ap.add_argument("--top-max-vertices", type=int, default=0,
                    help="cap on the vertices of the shared-memory top launch (phast_query_opts top_max_vertices)")
    ap.add_argument("--query-flags", type=int, default=0,
                    help="phast_configure flags (schedule experiments: 1 no fused single-launch query, 2 no shared-memory top launch)")
    ap.add_argument("--parents", action="store_true",
                    help="also time the parent-pointer pass (phast_parents, NEXT-1) on the last batch")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    args.inflight = max(0, min(8, args.inflight))
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch_distributed(args)

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_dellinggnw11_b200 as P

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        log(f"[bench] WARNING: --gpus {args.gpus} but WORLD_SIZE={world}; using {world} rank(s)")
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(x):
        if world == 1:
            return x
        tt = torch.tensor([x], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        return float(tt.item())

    cfg = phastgen.CONFIGS[args.config]
    k = args.k
    bopts = dict(layout=args.layout)
    # hierarchy: rank 0 generates the graph and builds (host CH, not the timed target),
    # the other ranks load it from a file (graph replicated per GPU)
    g = None
    if rank == 0:
        g, _ = build_graph(args.config)
    path = args.cache or f"/tmp/phast_{args.config}_{os.getpid() if world == 1 else 'dist'}.phast"
    if world > 1:
        from paper_conf_ipps_dellinggnw11_b200.parallel import share_hierarchy
        t = time.time()
        h = share_hierarchy(lambda: P.Phast.from_graph(g, **bopts), P.Phast.load, path, rank, barrier)
        log(f"[bench] rank {rank}: hierarchy ready in {time.time() - t:.1f}s")
    elif args.cache and os.path.exists(args.cache) and (h := try_load(P, args.cache)) is not None:
        pass
    else:
        t = time.time()
        h = P.Phast.from_graph(g, **bopts)
        log(f"[bench] CH build {time.time() - t:.1f}s")
        if args.cache:
            h.save(args.cache)
    if args.query_flags or args.band_unit or args.band_threads or args.band_variant or args.top_max_vertices:
        h.configure(flags=args.query_flags, band_unit=args.band_unit, band_threads=args.band_threads,
                    band_variant=args.band_variant, top_max_vertices=args.top_max_vertices)
    n = h.n
    info = h.info()
    lsz = h.level_sizes()
    sched = h.schedule(k)
    if rank == 0:
        log(f"[bench] n={info.n} m={info.m} m_up={info.m_up} m_down={info.m_down} n_tail={info.n_tail} "
            f"levels={info.levels} L0={lsz[0] / info.n:.3f} CH={info.build_seconds:.1f}s "
            f"upward search space mean={info.mean_up_space:.1f} max={info.max_up_space} "
            f"({info.up_space_samples} sampled sources)")
        log("[bench] level histogram (level: vertices, 0 = lowest): " +
            " ".join(f"{i}:{int(c)}" for i, c in enumerate(lsz)))
        log(f"[bench] schedule k={k}: {sched}")

    warm, timed, trees_here = rank_batches(n, cfg, k, world, rank, args.steps, args.warmup, args.total_sources)
    args.steps = len(timed)

    small = 4 * k * n + 16 * info.m_down < 256e6
    S = args.inflight or (8 if small else 1)
    stream = torch.cuda.current_stream()
    streams = [torch.cuda.Stream() for _ in range(S)]
    # L2 protocol: the C3/C4 label arrays (>= 1 GB) are far beyond the 126 MB L2; small
    # configs (labels + graph fit in L2) flush L2 before every step, or with --steady
    # rotate over enough label buffers that the labels alone exceed 2x L2
    flush = small and not args.steady
    nbuf = S
    if small and args.steady:
        nbuf = max(S, -(-2 * L2_BYTES // (4 * k * n)))
    bufs = [torch.empty(n * k, dtype=torch.int32, device="cuda") for _ in range(nbuf)]

    def issue(batches, ev0=None):
        """batches round robin over the S streams (each waits for ev0 first)."""
        if ev0 is not None:
            for st in streams:
                st.wait_event(ev0)
        for i, b in enumerate(batches):
            h.trees_into(b, bufs[i % nbuf].data_ptr(), streams[i % S].cuda_stream)

    def join():
        for st in streams:
            e = torch.cuda.Event()
            e.record(st)
            stream.wait_event(e)

    issue(warm)
    join()
    h.sync(stream)

    # ---------------------------------------------------------------- timed region
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    if flush:
        scrub = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
        groups = [timed[i:i + S] for i in range(0, len(timed), S)]   # a step of S sweeps in flight
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in groups]
    with Clocks(local) as clk:
        barrier()
        torch.cuda.synchronize()
        h.timing(True)
        l0 = P.launch_count()
        if flush:
            for i, grp in enumerate(groups):
                scrub.fill_(i & 0xFF)
                torch.cuda.synchronize()   # the step's upward searches start after ev[i][0]
                ev[i][0].record(stream)
                issue(grp, ev[i][0])
                join()
                ev[i][1].record(stream)
        else:
            t0.record(stream)
            issue(timed, t0)
            join()
            t1.record(stream)
        torch.cuda.synchronize()
        launches = P.launch_count() - l0
        barrier()
    h.timing(False)
    h.sync(stream)
    ms_local = sum(a.elapsed_time(b) for a, b in ev) if flush else t0.elapsed_time(t1)
    ms_up, ms_sweep, nb = h.timing_read()
    ms = max_over_ranks(ms_local)
    total_trees = args.total_sources if args.total_sources else world * trees_here
    value = total_trees / (ms / 1e3)

    # roofline of the dominant kernel: the level sweep of one batch (sweep_top_kernel +
    # one sweep_kernel per level), algorithmic bytes B_alg
    B_alg = 8 * info.m_down + 4 * (info.n + 1) + 4 * k * info.n + 4 * k * info.n_tail + info.n / 8
    sweeps = len(timed)
    sweep_ms_events = ms_sweep / max(nb, 1)            # per-batch events (a3 + flag clear), stream-local
    if S == 1:
        sweep_ms = sweep_ms_events
        how = "per-batch CUDA events around the sweep launches (a3 + flag clear) on the query stream"
    else:   # overlapping sweeps: the whole timed region per sweep (upward searches and seeding included)
        sweep_ms = ms_local / sweeps
        how = (f"timed region / sweeps with {S} sweeps in flight (includes upward searches and seeding; "
               "a lower bound of the sweep kernels' rate)")
    achieved = B_alg / (sweep_ms / 1e3) / 1e9
    peak, peak_src = peaks()
    traffic = None
    try:
        prof = json.load(open(os.path.join(ROOT, "profiles", "sweep_traffic.json")))
        e = prof.get(f"{args.config}_k{k}", {})
        if e.get("layout") == P.LAYOUT_NAMES[info.layout]:
            traffic = e["dram_bytes_per_sweep"]   # warm-L2 ncu launch list of this configuration
    except Exception:
        pass

    # probes A33 / A34 on the same arrays: ceilings for the sweep
    ceiling = None
    if not args.no_probes:
        def timed_probe(kind, reps=5):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            h.probe(kind, k, bufs[0], sources=timed[0], stream=stream)
            h.sync(stream)
            a.record(stream)
            for _ in range(reps):
                h.probe(kind, k, bufs[0], sources=timed[0], stream=stream)
            b.record(stream)
            h.sync(stream)
            return a.elapsed_time(b) / reps
        a33 = timed_probe(0)
        a34 = timed_probe(1)
        B33 = 16 * n + 8 * k * n
        ceiling = {"a33_stream_ms": a33, "a33_bytes": B33, "a33_GBps": B33 / (a33 / 1e3) / 1e9,
                   "a34_nogather_ms": a34, "sweep_over_a33": sweep_ms / a33, "sweep_over_a34": sweep_ms / a34,
                   "note": "A33: one sequential launch reading every ELL record and label row and writing "
                           "every row (PAPER.md:22 §VIII-B 'PHAST is only 2.6 times slower than this'); A34: the "
                           "query's launches with every tail-row gather replaced by the arc length "
                           "('it takes 153 ms to traverse the graph exactly as PHAST does'); ratios are sweep "
                           "time over probe time (L2 warm, back to back)"}

    # NEXT-1: parent pointers of the last timed batch (a separate pass, not in `value`)
    parents = None
    if args.parents:
        par_buf = torch.empty(n * k, dtype=torch.int32, device="cuda")
        last = timed[-1]
        dist_t = bufs[0]
        h.trees_into(last, dist_t.data_ptr(), stream.cuda_stream)   # the probes above overwrote the buffers
        h.parents(last, dist_t, out=par_buf, stream=stream)
        h.sync(stream)
        p0, p1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        reps = max(1, min(args.steps, 10))
        p0.record(stream)
        for _ in range(reps):
            h.parents(last, dist_t, out=par_buf, stream=stream)
        p1.record(stream)
        h.sync(stream)
        pms = p0.elapsed_time(p1) / reps
        B_par = 8 * info.m + 4 * (n + 1) + 12 * k * n
        h.parents_ch(last, dist_t, out=par_buf, stream=stream)   # first use uploads the A-up in-arcs
        h.sync(stream)
        p0.record(stream)
        for _ in range(reps):
            h.parents_ch(last, dist_t, out=par_buf, stream=stream)
        p1.record(stream)
        h.sync(stream)
        cms = p0.elapsed_time(p1) / reps
        parents = {"ms_per_pass": pms, "alg_bytes": B_par, "achieved_GBps": B_par / (pms / 1e3) / 1e9,
                   "frac": B_par / (pms / 1e3) / 1e9 / peak,
                   "note": "B = 8m + 4(n+1) + 12kn: in-arcs, offsets, own row read, in-neighbour rows read "
                           "at least once, parent row written",
                   "hierarchy_ms_per_pass": cms,
                   "hierarchy_note": "phast_parents_ch (G+ parents, reading R19): the same pass over the "
                                     "A-down in-arcs, then the A-up in-arcs for trees still without a parent"}
        del par_buf

    # end to end through the public host entry point (sources in, all labels out)
    e2e = None
    if args.e2e_steps > 0:
        host_out = torch.empty((n, k), dtype=torch.int32, pin_memory=True).numpy().view(np.uint32)
        h.trees_host(timed[0], host_out, stream)
        barrier()
        te = time.perf_counter()
        for b in range(args.e2e_steps):
            h.trees_host(timed[b % len(timed)], host_out, stream)
        te = max_over_ranks(time.perf_counter() - te)
        e2e = {"value": world * args.e2e_steps * k / te, "unit": "trees/s", "h2d_bytes_per_step": 4 * k,
               "d2h_bytes_per_step": 4 * k * n,
               "note": "phast_trees_host: sources in as kernel parameters, all n*k labels copied to pinned host "
                       "memory (PCIe-bound at large n*k)"}
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
        if flush:
            l2 = (f"L2 flushed before every timed step (512 MB write outside the step's events); a step = "
                  f"{S} sweep(s) of k={k} in flight; value = trees / sum of per-step times")
        elif small:
            l2 = f"steady state: no flush, {nbuf} label buffers of {4 * k * n / 1e6:.0f} MB rotate (> 2x L2)"
        else:
            l2 = f"label array {4 * k * n / 1e9:.2f} GB per buffer >> 126 MB L2 (no flush needed)"
        line = {
            "metric": METRIC, "value": value, "unit": "trees/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / max(args.steps, 1), "higher_is_better": True,
            "scaling": "strong" if args.total_sources else "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": f"{args.config}: {cfg['desc']}", "k": k, "sweeps_in_flight": S,
                       "trees_total": total_trees, "n": info.n, "m": info.m, "m_down": info.m_down,
                       "m_up": info.m_up, "n_tail": info.n_tail, "levels": info.levels,
                       "level_sizes": [int(c) for c in lsz],
                       "up_space": {"mean": round(info.mean_up_space, 1), "max": info.max_up_space,
                                    "samples": info.up_space_samples},
                       "schedule": sched, "layout": P.LAYOUT_NAMES[info.layout],
                       "parallelism": (f"{args.total_sources} sources sharded over {world} GPU(s)"
                                       if args.total_sources else f"{args.steps} batches per GPU on {world} GPU(s)")
                                      + ", graph replicated",
                       "l2": l2, "us_per_tree": ms * 1e3 / total_trees * world if args.total_sources
                       else ms * 1e3 / trees_here,
                       "ch_build_s": round(info.build_seconds, 1)},
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                         "traffic": traffic, "kernel": "sweep_top_kernel + sweep_band_kernel + sweep_kernel (all levels of one sweep)",
                         "alg_bytes_per_sweep": B_alg, "sweep_ms": sweep_ms, "sweep_ms_events": sweep_ms_events,
                         "upward_ms": ms_up / max(nb, 1), "how": how, "peak_source": peak_src},
            "ceiling": ceiling, "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches,
            "clocks": clk.summary(),
            **({"parents": parents} if parents else {}),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    h.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
