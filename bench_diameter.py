#!/usr/bin/env python
"""bench_diameter.py -- BASELINE.json configs[4] (C5): exact graph diameter over ALL
sources of a 1M-vertex road-like graph (§VII-B "Its exact value can be
computed by building n shortest path trees"), sources sharded over the ranks, per-GPU
max fused into the sweep, then one NCCL MAX all-reduce.

  python bench_diameter.py [--config C5] [--k 64] [--limit N]
  torchrun --nproc-per-node 8 --master-addr 127.0.0.1 bench_diameter.py

Prints one JSON line on rank 0: diameter D, device time (max over ranks), trees/s.
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
    ap.add_argument("--config", default="C5")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--limit", type=int, default=0, help="use only the first N sources (0 = all n)")
    ap.add_argument("--check", type=int, default=8, help="oracle trees to cross-check on rank 0")
    args = ap.parse_args()

    import torch
    import torch.distributed as dist

    import paper_conf_ipps_dellinggnw11_b200 as P
    from paper_conf_ipps_dellinggnw11_b200.parallel import allreduce_max_u32, shard, share_hierarchy

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    barrier = dist.barrier if world > 1 else (lambda: None)

    cfg = phastgen.CONFIGS[args.config]
    g = cfg["graph"]()
    h = share_hierarchy(lambda: P.Phast.from_graph(g), P.Phast.load, f"/tmp/phast_diam_{args.config}.phast", rank,
                        barrier) if world > 1 else P.Phast.from_graph(g)
    count = args.limit or g.n
    sources = np.arange(count, dtype=np.uint32)
    lo, hi = shard(count, world, rank)
    mine = sources[lo:hi]
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    # warm-up: one batch (plan build, first-touch)
    h.diameter_async(mine[: args.k], args.k, out)
    h.sync()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    torch.cuda.synchronize()
    t0.record()
    h.diameter_async(mine, args.k, out)
    t1.record()
    h.sync()
    ms = t0.elapsed_time(t1)
    local_max = int(out.cpu().numpy().view(np.uint32)[0])
    D = allreduce_max_u32(local_max, device="cuda")
    ms_all = ms
    if world > 1:
        tt = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_all = float(tt.item())
    if rank == 0:
        check = None
        if args.check:
            import oracle
            pick = phastgen.sources(count, args.check, seed=5)
            tm = oracle.tree_maxima(g, pick)
            check = {"sources": int(args.check), "oracle_max_of_sample": int(tm.max()),
                     "sample_le_D": bool(int(tm.max()) <= D)}
        print(json.dumps({
            "metric": "exact diameter over all sources (C5)", "config": args.config, "n": g.n, "m": g.m,
            "sources": count, "k_batch": args.k, "n_gpus": world, "diameter": D, "ms": ms_all,
            "trees_per_s": count / (ms_all / 1e3), "check": check,
        }), flush=True)
    if world > 1:
        dist.destroy_process_group()
    h.close()


if __name__ == "__main__":
    main()
