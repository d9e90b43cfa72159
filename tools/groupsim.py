"""L2 model of the band/group sweep order (profiles/r2_groupsim.md).

Replays the sweep's label-row accesses (per vertex: read every G-down tail row, then
write its row) through tools/l2sim.c (LRU, 16-way, one row per line) over an exported
hierarchy, in three orders:
  - level by level (one launch per level);
  - bands of closed groups (components of the band's own arcs, packed by BFS
    position), groups dealt to W concurrent CTAs in order (the band kernel), each
    batch of W groups swept level by level (pessimistic: all in the same phase);
  - the same groups, but each of C CTAs walking one contiguous 1/C of the band.

  python tools/groupsim.py EXPORT.npz   (np.savez of Phast.export() of a levels-bfs build)
"""
import ctypes
import os
import subprocess
import sys

import numpy as np
import scipy.sparse as sp
from scipy.sparse.csgraph import connected_components

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(path):
    so = "/tmp/l2sim_tools.so"
    subprocess.run(["gcc", "-O2", "-shared", "-fPIC", "-o", so, os.path.join(ROOT, "tools", "l2sim.c")], check=True)
    lib = ctypes.CDLL(so)
    lib.sim.restype = ctypes.c_uint64
    lib.sim.argtypes = [ctypes.c_uint32] + [ctypes.c_void_p] * 3 + [ctypes.c_uint64, ctypes.c_int,
                                                                    ctypes.POINTER(ctypes.c_uint64),
                                                                    ctypes.POINTER(ctypes.c_uint64)]
    a = np.load(path)
    lev = a["level"]
    df = np.ascontiguousarray(a["dn_first"])
    dtt = np.ascontiguousarray(a["dn_tail"])
    dt = dtt.astype(np.int64)
    n, L = lev.size, int(lev.max()) + 1
    heads = np.repeat(np.arange(n), np.diff(df.astype(np.int64)))
    off = np.zeros(L + 1, np.int64)
    for j in range(L):
        off[j + 1] = off[j] + (lev == L - 1 - j).sum()
    pos = np.arange(n) - off[(L - 1 - lev)]
    size = (off[1:] - off[:-1])[(L - 1 - lev)]
    q = (pos + 0.5) / size
    q = np.where(lev & 1, 1 - q, q)   # serpentine-corrected position within the level

    def run(order, rows=400_000):
        r, w = ctypes.c_uint64(), ctypes.c_uint64()
        order = np.ascontiguousarray(order, np.uint32)
        return lib.sim(n, df.ctypes.data, dtt.ctypes.data, order.ctypes.data, rows, 16, ctypes.byref(r),
                       ctypes.byref(w)) / 1e6

    def band_groups(lo, hi, G):
        inr = (lev >= lo) & (lev < hi)
        sel = inr[heads] & inr[dt]
        idx = np.nonzero(inr)[0]
        loc = -np.ones(n, np.int64)
        loc[idx] = np.arange(idx.size)
        A = sp.coo_matrix((np.ones(sel.sum()), (loc[heads[sel]], loc[dt[sel]])), shape=(idx.size, idx.size))
        nc, lab = connected_components(A, directed=False)
        key = np.full(nc, 2.0)
        np.minimum.at(key, lab, q[idx])
        csz = np.bincount(lab, minlength=nc)
        gid = np.empty(nc, np.int64)
        g = acc = 0
        for c in np.argsort(key, kind="stable"):
            if acc + csz[c] > G and acc > 0:
                g, acc = g + 1, 0
            gid[c] = g
            acc += csz[c]
        return idx, gid[lab]

    bands = [(0, 5), (5, 8), (8, 11), (11, 14), (14, 17), (17, 20), (20, 23)]

    def order_batches(G, W):
        parts = [np.arange(off[L - bands[-1][1]])]
        for lo, hi in reversed(bands):
            idx, gv = band_groups(lo, hi, G)
            parts.append(idx[np.lexsort((idx, gv, -lev[idx], gv // W))])
        return np.concatenate(parts)

    def order_parts(G, C):
        parts = [np.arange(off[L - bands[-1][1]])]
        for lo, hi in reversed(bands):
            idx, gv = band_groups(lo, hi, G)
            s = idx[np.lexsort((idx, -lev[idx], gv))]
            N = s.size
            c = (np.arange(N) * C) // N
            i = np.arange(N) - np.searchsorted(c, np.arange(C))[c]
            parts.append(s[np.lexsort((c, i))])
        return np.concatenate(parts)

    base = np.arange(n)
    print(f"level by level: tail-row misses {run(base):.2f} M (400 k rows), {run(base, 200_000):.2f} M (200 k)")
    for G, W in ((128, 1), (128, 1024), (256, 1024), (1024, 1024)):
        o = order_batches(G, W)
        print(f"groups of {G}, {W} in flight: {run(o):.2f} M / {run(o, 200_000):.2f} M")
    for G in (128, 512):
        o = order_parts(G, 1184)
        print(f"groups of {G}, 1184 contiguous parts: {run(o):.2f} M / {run(o, 200_000):.2f} M")


if __name__ == "__main__":
    main(sys.argv[1])
