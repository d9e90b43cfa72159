#!/usr/bin/env python
"""bench_betweenness.py -- SURVEY.md §8(f) NEXT-3: exact (partial) betweenness on top
of PHAST trees (§VII-B "Computing exact betweenness relies on n shortest
path tree computations ... replacing Dijkstra's algorithm by PHAST makes exact
betweenness tractable"), sources sharded over the ranks, one NCCL SUM all-reduce of
the per-GPU partial sums.

  python bench_betweenness.py [--config C2] [--count 2048] [--k 64]
  torchrun --nproc-per-node N --master-addr 127.0.0.1 bench_betweenness.py

Prints one JSON line on rank 0: sources/s (device time, max over ranks) and a
full-size parity check: the GPU partial betweenness of `--check` sources against the
oracle on the same sources (the oracle is timed for cpu_baseline).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import phastgen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--count", type=int, default=2048, help="sources (over all ranks)")
    ap.add_argument("--reach", action="store_true", help="exact reach instead of betweenness")
    ap.add_argument("--check", type=int, default=2, help="sources cross-checked against the oracle (0 = none)")
    args = ap.parse_args()

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_dellinggnw11_b200 as P
    from paper_conf_ipps_dellinggnw11_b200.parallel import combine_centrality, shard, share_hierarchy

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    barrier = dist.barrier if world > 1 else (lambda: None)

    cfg = phastgen.CONFIGS[args.config]
    g = cfg["graph"]()
    h = share_hierarchy(lambda: P.Phast.from_graph(g), P.Phast.load, f"/tmp/phast_bc_{args.config}.phast", rank,
                        barrier) if world > 1 else P.Phast.from_graph(g)
    sources = phastgen.sources(g.n, args.count, seed=cfg["src_seed"])
    lo, hi = shard(sources.size, world, rank)
    mine = sources[lo:hi]
    cb = torch.empty(g.n, dtype=torch.int32 if args.reach else torch.float64, device="cuda")
    run = h.reach if args.reach else h.betweenness
    run(mine, k_batch=args.k, out=cb)      # warm-up: uploads, scratch, plans, CUDA graphs
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches0 = P.launch_count()
    barrier()
    torch.cuda.synchronize()
    t0.record()
    run(mine, k_batch=args.k, out=cb)
    t1.record()
    torch.cuda.synchronize()
    ms = t0.elapsed_time(t1)
    launches = P.launch_count() - launches0
    if world > 1:
        combine_centrality(cb, args.reach)
        tt = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    if rank == 0:
        check = cpu = None
        if args.check:
            import oracle
            pick = sources[: args.check]
            got = h.vertex_to_original(run(pick, k_batch=args.k).cpu().numpy())
            c0 = time.perf_counter()
            want = (oracle.reach if args.reach else oracle.betweenness)(g, pick)
            sec = time.perf_counter() - c0
            cpu = {"value": args.check / sec, "unit": "sources/s", "cores": 1, "kind": "oracle",
                   "sample": f"{args.check} sources of {args.config}, pure-Python oracle over the C Dijkstra"}
            if args.reach:
                got, want = got.view(np.uint32).astype(np.float64), want.astype(np.float64)
            err = float(np.max(np.abs(got - want)) / max(1.0, float(np.abs(want).max())))
            check = {"sources": args.check, "k_batch": args.k, "max_rel_err": err, "ok": bool(err < 1e-9)}
        print(json.dumps({
            "metric": "exact partial reach (NEXT-3)" if args.reach else "exact partial betweenness (NEXT-3)", "value": sources.size / (ms / 1e3),
            "unit": "sources/s", "config": {"workload": args.config, "n": g.n, "m": g.m, "sources": int(sources.size),
                                            "k_batch": args.k}, "n_gpus": world, "ms": ms,
            "ms_per_source": ms / sources.size, "gpu_launches": launches, "dtype": "u32" if args.reach else "f64",
            "check": check, "cpu_baseline": cpu,
        }), flush=True)
    if world > 1:
        dist.destroy_process_group()
    h.close()


if __name__ == "__main__":
    main()
