"""Test helper (NOT the oracle, NOT product code): a numpy re-execution of PHAST's
two subphases over an exported hierarchy, used to check the host CH build and the
layout on CPU without a GPU.  Results are compared against the oracle."""
import numpy as np

INF = 0xFFFFFFFF
BIG = np.int64(1) << 60


def _by_level(level):
    """Internal ids grouped by CH level, highest level first."""
    order = np.argsort(-level.astype(np.int64), kind="stable")
    lv = level[order]
    cuts = np.flatnonzero(np.diff(lv)) + 1
    return np.split(order, cuts)


def upward_labels(ex, s_int, n):
    """Exact G-up distances from internal id s_int.  Every G-up arc goes to a strictly
    higher CH level (§IV-A level rule), so ascending level is a
    topological order of G-up."""
    d = np.full(n, BIG, np.int64)
    d[s_int] = 0
    uf, uh, ul = ex["up_first"].astype(np.int64), ex["up_head"], ex["up_len"].astype(np.int64)
    for grp in reversed(_by_level(ex["level"])):          # lowest level first
        live = grp[d[grp] < BIG]
        for r in live:
            a, b = uf[r], uf[r + 1]
            if a != b:
                np.minimum.at(d, uh[a:b], d[r] + ul[a:b])
    return d


def sweep(ex, d_init, n):
    """Highest level first: d(v) = min(d(v), min over in-arcs d(u) + l(u,v))
    (§III); all tails of a level are on higher levels (Lemma 4.1)."""
    d = d_init.copy()
    df = ex["dn_first"].astype(np.int64)
    dt, dl = ex["dn_tail"], ex["dn_len"].astype(np.int64)
    for grp in _by_level(ex["level"]):
        cnt = df[grp + 1] - df[grp]
        sel = grp[cnt > 0]
        if sel.size == 0:
            continue
        idx = np.concatenate([np.arange(df[v], df[v + 1]) for v in sel])
        heads = np.repeat(sel, (df[sel + 1] - df[sel]))
        np.minimum.at(d, heads, d[dt[idx]] + dl[idx])
    return np.where(d >= INF, INF, d).astype(np.uint32)


def sweep_in_order(ex, d_init, order):
    """The same relaxation, one vertex at a time in the given processing order (which
    must see every tail before its head)."""
    d = [int(x) for x in d_init]
    df = ex["dn_first"].tolist()
    dt, dl = ex["dn_tail"].tolist(), ex["dn_len"].tolist()
    for v in order.tolist():
        best = d[v]
        for e in range(df[v], df[v + 1]):
            c = d[dt[e]] + dl[e]
            if c < best:
                best = c
        d[v] = best
    d = np.array(d, dtype=np.int64)
    return np.where(d >= INF, INF, d).astype(np.uint32)


def phast_cpu(h, ex, sources, order=None):
    perm = h.order()
    out = []
    for s in sources:
        up = upward_labels(ex, int(perm[s]), h.n)
        d = sweep(ex, up, h.n) if order is None else sweep_in_order(ex, up, order)
        out.append(d[perm])
    return np.array(out, dtype=np.uint32)
