"""Test helper (NOT the oracle, NOT product code): a numpy re-execution of PHAST's
two subphases over an exported hierarchy, used to check the host CH build and the
layout on CPU without a GPU.  Results are compared against the oracle."""
import numpy as np

INF = 0xFFFFFFFF


def upward_labels(ex, s_int, n):
    """Exact G-up distances from internal id s_int.  G-up arcs go from a lower level
    to a higher one, i.e. from a larger internal id to a smaller one, so decreasing
    internal id is a topological order (§IV-A, Lemma 4.1)."""
    big = np.int64(1) << 60
    d = np.full(n, big, np.int64)
    d[s_int] = 0
    uf, uh, ul = ex["up_first"], ex["up_head"], ex["up_len"].astype(np.int64)
    for r in range(s_int, -1, -1):
        if d[r] >= big:
            continue
        a, b = int(uf[r]), int(uf[r + 1])
        if a == b:
            continue
        hs = uh[a:b]
        np.minimum.at(d, hs, d[r] + ul[a:b])
    return d


def sweep(ex, d_init, n):
    """Level by level: d(v) = min(d(v), min over in-arcs d(u) + l(u,v)) (§III)."""
    big = np.int64(1) << 60
    d = d_init.copy()
    lo, df, dt, dl = ex["lvl_off"], ex["dn_first"], ex["dn_tail"], ex["dn_len"].astype(np.int64)
    for j in range(len(lo) - 1):
        a, b = int(lo[j]), int(lo[j + 1])
        ea, eb = int(df[a]), int(df[b])
        if ea == eb:
            continue
        cand = d[dt[ea:eb]] + dl[ea:eb]
        heads = np.repeat(np.arange(a, b), np.diff(df[a:b + 1]).astype(np.int64))
        np.minimum.at(d, heads, cand)
    return np.where(d >= INF, INF, np.minimum(d, big)).astype(np.uint32)


def phast_cpu(h, ex, sources):
    perm = h.order()
    inv = np.empty_like(perm)
    inv[perm] = np.arange(perm.size, dtype=perm.dtype)
    out = []
    for s in sources:
        d = sweep(ex, upward_labels(ex, int(perm[s]), h.n), h.n)
        out.append(d[perm])
    return np.array(out, dtype=np.uint32)
