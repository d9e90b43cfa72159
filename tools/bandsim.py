"""L2 model of the band dataflow order (profiles/r2_bandsim.md).

Replays the sweep's label-row accesses (per vertex: read every G-down tail row, then
write the vertex's row) through tools/l2sim.c (LRU, 16-way, one row per line) in two
processing orders over an exported hierarchy:
  - level by level (the per-level launches), and
  - the band dataflow sequence of capi.cu: the levels below the top `--top` levels cut
    into aligned quantile bands (B_l = min(B, size/32)), tasks in Kahn order, smallest
    quantile first.

  python tools/bandsim.py HIERARCHY.phast [--rows 400000] [--top 25] [--bands 512]
(build the .phast with bench.py --cache or Phast.save; gcc builds l2sim.so on the fly)
"""
import argparse
import ctypes
import heapq
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def l2sim():
    so = "/tmp/l2sim_tools.so"
    subprocess.run(["gcc", "-O2", "-shared", "-fPIC", "-o", so, os.path.join(ROOT, "tools", "l2sim.c")], check=True)
    lib = ctypes.CDLL(so)
    lib.sim.restype = ctypes.c_uint64
    lib.sim.argtypes = [ctypes.c_uint32, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_uint64,
                        ctypes.c_int, ctypes.POINTER(ctypes.c_uint64), ctypes.POINTER(ctypes.c_uint64)]
    return lib


def band_order(lev, df, dt, top, bands, min_v=32):
    n = lev.size
    L = int(lev.max()) + 1
    off = np.concatenate([[0], np.cumsum([(lev == L - 1 - j).sum() for j in range(L)])]).astype(np.int64)
    top_end = off[top]
    tasks, task_of = [], np.full(n, -1, np.int64)
    for j in range(top, L):
        lv = L - 1 - j
        a, b = off[j], off[j + 1]
        size = b - a
        nb = max(1, min(bands, size // min_v))
        for q in range(nb):
            p0, p1 = size * q // nb, size * (q + 1) // nb
            if p0 == p1:
                continue
            lo, hi = (b - p1, b - p0) if lv & 1 else (a + p0, a + p1)
            task_of[lo:hi] = len(tasks)
            tasks.append((lv, q / nb, lo, hi))
    heads = np.repeat(np.arange(n, dtype=np.int64), np.diff(df.astype(np.int64)))
    sel = (heads >= top_end) & (dt.astype(np.int64) >= top_end)
    pairs = np.unique(task_of[heads[sel]] * (1 << 32) + task_of[dt[sel].astype(np.int64)])
    T = len(tasks)
    indeg = np.zeros(T, np.int64)
    users = [[] for _ in range(T)]
    for x in pairs.tolist():
        t, u = divmod(x, 1 << 32)
        indeg[t] += 1
        users[u].append(t)
    ready = [(tasks[t][1], -tasks[t][0], t) for t in range(T) if indeg[t] == 0]
    heapq.heapify(ready)
    seq = []
    while ready:
        _, _, t = heapq.heappop(ready)
        seq.append(t)
        for u in users[t]:
            indeg[u] -= 1
            if indeg[u] == 0:
                heapq.heappush(ready, (tasks[u][1], -tasks[u][0], u))
    assert len(seq) == T
    parts = [np.arange(top_end, dtype=np.uint32)] + [np.arange(tasks[t][2], tasks[t][3], dtype=np.uint32)
                                                      for t in seq]
    return np.concatenate(parts), T


def main():
    import paper_conf_ipps_dellinggnw11_b200 as P
    ap = argparse.ArgumentParser()
    ap.add_argument("hierarchy")
    ap.add_argument("--rows", type=int, nargs="+", default=[400_000, 200_000])
    ap.add_argument("--top", type=int, default=25)
    ap.add_argument("--bands", type=int, nargs="+", default=[512])
    a = ap.parse_args()
    h = P.Phast.load(a.hierarchy, host_only=True)
    ex = h.export()
    lev, df, dt = ex["level"], ex["dn_first"], ex["dn_tail"]
    lib = l2sim()

    def run(order, rows):
        r, w = ctypes.c_uint64(), ctypes.c_uint64()
        order = np.ascontiguousarray(order, np.uint32)
        m = lib.sim(lev.size, df.ctypes.data, dt.ctypes.data, order.ctypes.data, rows, 16, ctypes.byref(r),
                    ctypes.byref(w))
        return m, r.value
    base = np.arange(lev.size, dtype=np.uint32)
    for rows in a.rows:
        m, r = run(base, rows)
        print(f"level by level, cache {rows} rows: tail reads {r / 1e6:.1f} M, misses {m / 1e6:.2f} M")
    for B in a.bands:
        order, T = band_order(lev, df, dt, a.top, B)
        assert np.unique(order).size == lev.size
        for rows in a.rows:
            m, r = run(order, rows)
            print(f"band order (top {a.top} levels apart, B = {B}, {T} tasks), cache {rows} rows: "
                  f"misses {m / 1e6:.2f} M")


if __name__ == "__main__":
    main()
