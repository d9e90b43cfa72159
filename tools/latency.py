"""Single-query latency (NEXT-2): one k-tree query at a time on one
stream, CUDA events around each query; with an L2 flush (512 MB write) before every
query (cold) and back to back (warm).  One JSON line per schedule flag set.

  python tools/latency.py --config C1 --k 1 --flags 0 32 1
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import phastgen  # noqa: E402


def main():
    import torch
    import paper_conf_ipps_dellinggnw11_b200 as P
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C1")
    ap.add_argument("--k", type=int, default=1)
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--flags", type=int, nargs="+", default=[0])
    a = ap.parse_args()
    cfg = phastgen.CONFIGS[a.config]
    g = cfg["graph"]()
    h = P.Phast.from_graph(g)
    srcs = [phastgen.sources(g.n, a.k, seed=cfg["src_seed"] + i) for i in range(a.reps)]
    out = torch.empty(g.n * a.k, dtype=torch.int32, device="cuda")
    scrub = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    st = torch.cuda.current_stream()
    for fl in a.flags:
        h.configure(flags=fl)
        for s in srcs[:5]:
            h.trees(s, out=out)
        h.sync()
        res = {}
        for mode in ("cold", "warm"):
            ts = []
            for i, s in enumerate(srcs):
                if mode == "cold":
                    scrub.fill_(i & 0xFF)
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                torch.cuda.synchronize()
                e0.record(st)
                h.trees(s, out=out)
                e1.record(st)
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e3)
            res[mode] = {"us_median": float(np.median(ts)), "us_min": float(np.min(ts))}
        print(json.dumps({"config": a.config, "k": a.k, "flags": fl, "schedule": h.schedule(a.k), **res}), flush=True)


if __name__ == "__main__":
    main()
