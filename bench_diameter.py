#!/usr/bin/env python
"""bench_diameter.py -- BASELINE.json configs[4] (C5): exact graph diameter over ALL
sources of a 1M-vertex road-like graph (§VII-B "Its exact value can be
computed by building n shortest path trees"), sources sharded over the ranks, per-GPU
max fused into the sweep (batches on up to PHAST_SLOTS library streams), then one NCCL
MAX all-reduce.

  python bench_diameter.py [--gpus N] [--config C5] [--k 64] [--limit N] [--check 1024]

`--gpus N` outside torchrun relaunches under torch.distributed.run with N ranks.
After the timed pass each rank computes its shard's witness (phast_diameter_witness,
outside the timed region); the global (D, s*, t*) is checked on rank 0 against the
oracle: dist(s*, t*) = D, and the oracle's maximum over `--check` sampled sources <= D.
Prints one JSON line on rank 0.
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
from bench import Clocks, free_port, log  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--config", default="C5")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--limit", type=int, default=0, help="use only the first N sources (0 = all n)")
    ap.add_argument("--check", type=int, default=1024, help="oracle trees sampled on rank 0 (<= D)")
    ap.add_argument("--no-witness", action="store_true")
    ap.add_argument("--query-flags", type=int, default=0, help="phast_configure flags (64: no band launches)")
    ap.add_argument("--band-unit", type=int, default=0, help="vertices per band work unit (0 = library default)")
    args = ap.parse_args()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        import subprocess
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={free_port()}", os.path.abspath(__file__)] + sys.argv[1:]
        env = dict(os.environ)
        env.setdefault("NCCL_DEBUG", "INFO")
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        return subprocess.call(cmd, env=env)

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
    g = cfg["graph"]() if rank == 0 else None
    if world > 1:
        h = share_hierarchy(lambda: P.Phast.from_graph(g), P.Phast.load, f"/tmp/phast_diam_{args.config}.phast",
                            rank, barrier)
    else:
        h = P.Phast.from_graph(g)
    if args.query_flags or args.band_unit:
        h.configure(flags=args.query_flags, band_unit=args.band_unit)
    n = h.n
    count = args.limit or n
    sources = np.arange(count, dtype=np.uint32)
    lo, hi = shard(count, world, rank)
    mine = sources[lo:hi]
    out = torch.zeros(1, dtype=torch.int32, device="cuda")
    h.diameter_async(mine[: args.k], args.k, out)      # warm-up: plans, first-touch
    h.sync()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with Clocks(local) as clk:
        barrier()
        torch.cuda.synchronize()
        t0.record()
        h.diameter_async(mine, args.k, out)
        t1.record()
        h.sync()
        barrier()
    ms = t0.elapsed_time(t1)
    local_max = int(out.cpu().numpy().view(np.uint32)[0])
    D = allreduce_max_u32(local_max, device="cuda")
    ms_all = ms
    if world > 1:
        tt = torch.tensor([ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_all = float(tt.item())
    witness = None
    if not args.no_witness:
        w = h.diameter_witness(mine, k_batch=args.k)
        if world > 1:
            allw = [None] * world
            dist.all_gather_object(allw, w)
        else:
            allw = [w]
        witness = max(allw)                             # (D, s*, t*) of the rank holding the max
    if rank == 0:
        check = None
        if args.check or witness:
            import oracle
            check = {}
            if witness:
                Dw, s, t = witness
                check["witness"] = {"D": Dw, "s": s, "t": t, "oracle_dist_s_t": int(oracle.sssp(g, s)[t])}
                check["witness_ok"] = Dw == D and check["witness"]["oracle_dist_s_t"] == D
            if args.check:
                pick = phastgen.sources(count, min(args.check, count), seed=cfg["src_seed"] + 9)
                t = time.time()
                tm = oracle.tree_maxima(g, pick)
                check.update({"sources": int(pick.size), "oracle_max_of_sample": int(tm.max()),
                              "sample_le_D": bool(int(tm.max()) <= D), "oracle_s": round(time.time() - t, 1)})
        print(json.dumps({
            "metric": "exact diameter over all sources (C5)", "config": args.config, "n": n, "m": h.info().m,
            "sources": count, "k_batch": args.k, "n_gpus": world, "diameter": D, "ms": ms_all,
            "trees_per_s": count / (ms_all / 1e3), "check": check, "clocks": clk.summary(),
            "lanes": "batches on up to 4 library streams per GPU (phast_diameter)",
        }), flush=True)
    if world > 1:
        dist.destroy_process_group()
    h.close()
    log("[bench_diameter] done")


if __name__ == "__main__":
    sys.exit(main())
