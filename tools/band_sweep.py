"""Parameter sweep of the band dataflow launch (instrumentation, one GPU):

  python tools/band_sweep.py --config C3 --k 64 --cache /tmp/c3.phast \
      --grid "levels=12,bands=512,lag=2,chunk=1024" "levels=8,lag=1" ...

For each setting: phast_configure, 3 warm-up sweeps, 10 timed sweeps back to back (CUDA
events on the query stream), the sweep's labels compared bit for bit with the
one-launch-per-level schedule on the same sources (a consistency check; the parity
tests against the oracle are tests/test_gpu.py).  One JSON line per setting."""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import phastgen  # noqa: E402


def main():
    import torch
    import paper_conf_ipps_dellinggnw11_b200 as P
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--k", type=int, default=64)
    ap.add_argument("--cache", default="")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--grid", nargs="+", default=["default"])
    a = ap.parse_args()
    cfg = phastgen.CONFIGS[a.config]
    if a.cache and os.path.exists(a.cache):
        h = P.Phast.load(a.cache)
    else:
        h = P.Phast.from_graph(cfg["graph"]())
        if a.cache:
            h.save(a.cache)
    inf = h.info()
    k = a.k
    B_alg = 8 * inf.m_down + 4 * (inf.n + 1) + 4 * k * inf.n + 4 * k * inf.n_tail + inf.n / 8
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    srcs = [phastgen.sources(h.n, k, seed=500 + i) for i in range(a.reps + 3)]
    out = torch.empty(h.n * k, dtype=torch.int32, device="cuda")
    ref = torch.empty(h.n * k, dtype=torch.int32, device="cuda")
    st = torch.cuda.current_stream()
    h.configure(flags=P.Q_NO_BAND)
    h.trees(srcs[0], out=ref)
    h.sync()
    for spec in a.grid:
        kw = {}
        flags = 0
        if spec != "default":
            for item in spec.split(","):
                key, val = item.split("=")
                if key == "flags":
                    flags = int(val)
                else:
                    kw[{"levels": "band_levels", "bands": "bands", "lag": "band_lag", "chunk": "band_chunk"}[key]] = int(val)
        t = time.time()
        h.configure(flags=flags, **kw)
        sched = h.schedule(k)
        plan_s = time.time() - t
        h.trees(srcs[0], out=out)
        h.sync()
        same = bool(torch.equal(out, ref))
        for s in srcs[1:3]:
            h.trees(s, out=out)
        h.sync()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st)
        for s in srcs[3:]:
            h.trees(s, out=out)
        e1.record(st)
        h.sync()
        ms = e0.elapsed_time(e1) / a.reps
        print(json.dumps({"spec": spec, "k": k, "ms_per_sweep": ms, "trees_per_s": k / ms * 1e3,
                          "frac": B_alg / (ms / 1e3) / 1e9 / peak, "same_as_per_level": same, "schedule": sched,
                          "plan_s": round(plan_s, 2)}), flush=True)


if __name__ == "__main__":
    main()
