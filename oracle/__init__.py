"""THE ORACLE -- test infrastructure only.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl
reference` legs may import this package.  The product path
(paper_conf_ipps_dellinggnw11_b200/) never imports it, and the two share no code.

Plain binary-heap Dijkstra on the ORIGINAL graph (§II-A), exact by
Theorem 3.1 (§III) for what PHAST computes; diameter (PAPER.md:20
§VII-B); O(n+m) optimality certificate; canonical parent
pointers by the tight-arc identity (§VII-A, reading R14) and in the hierarchy
G+ (reading R19); exact betweenness
and reach (§VII-B, readings R16/R17, plain Python below).  See oracle.c for the
passage each function follows.  Pins: tests/test_oracle.py.  Parity status of
every function: pinned.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

INF = 0xFFFFFFFF
_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def _load():
    global _lib
    if _lib is None:
        if not os.path.exists(_LIB_PATH):
            raise RuntimeError(f"{_LIB_PATH} missing: run __graft_entry__.build()")
        lib = ctypes.CDLL(_LIB_PATH)
        u32, u64, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_void_p
        lib.oracle_sssp.argtypes = [u32, vp, vp, vp, u32, vp]
        lib.oracle_sssp_many.argtypes = [u32, vp, vp, vp, vp, u64, vp, vp, u32]
        lib.oracle_diameter.argtypes = [u32, vp, vp, vp, vp, u64, u32, vp]
        lib.oracle_certify.argtypes = [u32, vp, vp, vp, u32, vp]
        lib.oracle_parents.argtypes = [u32, vp, vp, vp, u32, vp, vp]
        for f in (lib.oracle_sssp, lib.oracle_sssp_many, lib.oracle_diameter, lib.oracle_certify,
                  lib.oracle_parents):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _csr(g):
    first = np.ascontiguousarray(g.first, dtype=np.uint64)
    head = np.ascontiguousarray(g.head, dtype=np.uint32)
    ln = np.ascontiguousarray(g.len, dtype=np.uint32)
    if head.size == 0:
        head = np.zeros(1, np.uint32)
        ln = np.zeros(1, np.uint32)
    return first, head, ln


def _threads(threads):
    return int(threads) if threads else (os.cpu_count() or 1)


def sssp(g, s: int) -> np.ndarray:
    """uint32[n]: min(dist(s, v), INF) on the original graph."""
    first, head, ln = _csr(g)
    out = np.empty(g.n, dtype=np.uint32)
    rc = _load().oracle_sssp(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data, int(s),
                             out.ctypes.data)
    if rc:
        raise ValueError(f"oracle_sssp: {rc}")
    return out


def sssp_many(g, sources, threads: int | None = None) -> np.ndarray:
    """uint32[count, n]: one tree per source, one source per worker thread."""
    first, head, ln = _csr(g)
    src = np.ascontiguousarray(sources, dtype=np.uint32)
    out = np.empty((src.size, g.n), dtype=np.uint32)
    rc = _load().oracle_sssp_many(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data,
                                  src.ctypes.data, src.size, out.ctypes.data, None,
                                  _threads(threads))
    if rc:
        raise ValueError(f"oracle_sssp_many: {rc}")
    return out


def tree_maxima(g, sources, threads: int | None = None) -> np.ndarray:
    """uint32[count]: max finite label of each tree (no trees stored)."""
    first, head, ln = _csr(g)
    src = np.ascontiguousarray(sources, dtype=np.uint32)
    maxs = np.empty(max(src.size, 1), dtype=np.uint32)
    rc = _load().oracle_sssp_many(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data,
                                  src.ctypes.data, src.size, None, maxs.ctypes.data,
                                  _threads(threads))
    if rc:
        raise ValueError(f"oracle_sssp_many: {rc}")
    return maxs[: src.size]


def diameter(g, sources, threads: int | None = None) -> int:
    """max over sources s and vertices v with dist(s,v) != INF of dist(s,v)."""
    first, head, ln = _csr(g)
    src = np.ascontiguousarray(sources, dtype=np.uint32)
    out = np.zeros(1, dtype=np.uint32)
    rc = _load().oracle_diameter(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data,
                                 src.ctypes.data, src.size, _threads(threads), out.ctypes.data)
    if rc:
        raise ValueError(f"oracle_diameter: {rc}")
    return int(out[0])


def certify(g, s: int, d) -> int:
    """0 iff d == min(dist(s, .), INF); else 1/2/3 = which optimality condition fails."""
    first, head, ln = _csr(g)
    d = np.ascontiguousarray(d, dtype=np.uint32)
    if d.size != g.n:
        raise ValueError("label vector has wrong length")
    rc = _load().oracle_certify(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data, int(s),
                                d.ctypes.data)
    if rc < 0:
        raise ValueError(f"oracle_certify: {rc}")
    return rc


def parents(g, s: int, d=None) -> np.ndarray:
    """uint32[n]: canonical parent of every vertex in the tree of s (oracle.c:
    oracle_parents; d defaults to the oracle's own labels sssp(g, s))."""
    first, head, ln = _csr(g)
    d = sssp(g, s) if d is None else np.ascontiguousarray(d, dtype=np.uint32)
    out = np.empty(g.n, dtype=np.uint32)
    rc = _load().oracle_parents(g.n, first.ctypes.data, head.ctypes.data, ln.ctypes.data, int(s),
                                d.ctypes.data, out.ctypes.data)
    if rc:
        raise ValueError(f"oracle_parents: {rc}")
    return out


def parents_ch(ex: dict, d_int, s_int: int) -> np.ndarray:
    """uint32[n]: parent pointers in the contraction hierarchy G+ = A-down U A-up
    (shortcuts included) -- "it suffices to remember the arc (u, v) responsible for
    d(v)" (§VII-A) and "some of the parent pointers in this case will be
    shortcuts" (§VII-A), reading R19.

    Inputs are in INTERNAL ids: `ex` = the exported hierarchy (Phast.export(): dn_first /
    dn_tail / dn_len = A-down in-arcs by head, up_first / up_head / up_len = A-up out-arcs
    by tail), `d_int` = the TRUE distances from the source (oracle sssp, permuted to
    internal ids), `s_int` = the source.  The definition written out: parent(s) = s;
    parent(v) = INF where d(v) = INF; else the tail of v's first tight A-down in-arc
    (d(u) + l = d(v), export order), and if there is none the tail of its first tight
    A-up in-arc (tails in increasing id, each tail's arcs in export order).  A tight arc
    always exists (a shortest up-down path reaches v either down an A-down arc or, at its
    peak, up an A-up arc; §III) -- the pins check it.  Plain Python: small
    graphs only."""
    d = np.asarray(d_int, dtype=np.int64)
    n = d.size
    dn_first = ex["dn_first"].astype(np.int64)
    dn_tail, dn_len = ex["dn_tail"].astype(np.int64), ex["dn_len"].astype(np.int64)
    up_first = ex["up_first"].astype(np.int64)
    up_head, up_len = ex["up_head"].astype(np.int64), ex["up_len"].astype(np.int64)
    par = np.full(n, INF, dtype=np.int64)
    for v in range(n):
        if d[v] == INF or v == s_int:
            continue
        for e in range(dn_first[v], dn_first[v + 1]):
            u = dn_tail[e]
            if d[u] != INF and d[u] + dn_len[e] == d[v]:
                par[v] = u
                break
    for u in range(n):                 # A-up in-arcs: tails in increasing id
        if d[u] == INF:
            continue
        for e in range(up_first[u], up_first[u + 1]):
            v = up_head[e]
            if par[v] == INF and v != s_int and d[v] != INF and d[u] + up_len[e] == d[v]:
                par[v] = u
    par[s_int] = s_int
    return par.astype(np.uint32)


def betweenness(g, sources) -> np.ndarray:
    """float64[n]: partial betweenness c_B(v) = sum over s in `sources`, t in V,
    s != v != t, of sigma_st(v) / sigma_st (§VII-B "c_B(v) = sum_{s != v
    != t in V} sigma_st(v)/sigma_st, where sigma_st is the number of shortest paths
    between two vertices s and t"); with sources = V it is the exact betweenness.

    SURVEY.md §8(f) NEXT-3.  Readings (R16): directed graph, ordered pairs;
    a path is a sequence of arcs, so parallel tight arcs are distinct paths; all
    lengths must be > 0 (zero-length cycles make sigma unbounded; §VII-A
    "As long as all original arc lengths are strictly positive").

    Written step by step after Brandes' accumulation, the method PAPER.md:20 cites
    for "Computing exact betweenness relies on n shortest path tree computations
    [28]": per source, the tree of `sssp` (pinned Dijkstra); sigma in nondecreasing
    distance order over tight arcs d(u) + l = d(w); then
    delta(u) = sum over tight (u, w) of sigma(u)/sigma(w) * (1 + delta(w)) in
    nonincreasing distance order; c_B(w) += delta(w) for w != s.  Plain Python
    loops: small graphs only.  Pins: tests/test_oracle.py (brute-force path
    enumeration, closed forms on paths and stars)."""
    n = g.n
    first = np.asarray(g.first, dtype=np.int64).tolist()
    head = np.asarray(g.head, dtype=np.int64).tolist()
    ln = np.asarray(g.len, dtype=np.int64).tolist()
    if head and min(ln) == 0:
        raise ValueError("betweenness needs all arc lengths > 0")
    cb = np.zeros(n, dtype=np.float64)
    for s in np.asarray(sources, dtype=np.int64).ravel():
        d = sssp(g, int(s)).astype(np.int64)
        order = [int(v) for v in np.argsort(d, kind="stable") if d[v] != INF]
        d = d.tolist()
        sigma = [0.0] * n
        sigma[s] = 1.0
        for u in order:                               # nondecreasing d(u)
            for e in range(first[u], first[u + 1]):
                w = head[e]
                if w != u and d[w] != INF and d[u] + ln[e] == d[w]:
                    sigma[w] += sigma[u]
        delta = [0.0] * n
        for w in reversed(order):                      # nonincreasing d(w)
            for e in range(first[w], first[w + 1]):
                x = head[e]
                if x != w and d[x] != INF and d[w] + ln[e] == d[x]:
                    delta[w] += sigma[w] / sigma[x] * (1.0 + delta[x])
            if w != s:
                cb[w] += delta[w]
    return cb


def reach(g, sources) -> np.ndarray:
    """uint32[n]: partial exact reach r(v) = max over s in `sources`, t in V and shortest
    s-t paths P containing v of min(dist(s, v), dist(v, t)) (§VII-B "The
    reach of v is defined as the maximum, over all shortest s t paths containing v, of
    min{dist(s, v), dist(v, t)}"); 0 where v lies on no such path.  With sources = V
    it is the exact reach.  Readings (R17): every shortest path counts (ties
    included); dist(v, t) along P equals dist(s, t) - dist(s, v); lengths > 0.

    Per source: the tree of `sssp`; v lies on a shortest s-t path iff t is reachable
    from v over tight arcs, so the largest dist(v, t) is the height
    h(v) = max(0, max over tight (v, w) of l + h(w)), taken in nonincreasing distance
    order; r(v) = max over s of min(d_s(v), h_s(v)).  Plain Python loops: small
    graphs only.  Pins: tests/test_oracle.py (brute-force path enumeration, path
    closed form)."""
    n = g.n
    first = np.asarray(g.first, dtype=np.int64).tolist()
    head = np.asarray(g.head, dtype=np.int64).tolist()
    ln = np.asarray(g.len, dtype=np.int64).tolist()
    if head and min(ln) == 0:
        raise ValueError("reach needs all arc lengths > 0")
    r = [0] * n
    for s in np.asarray(sources, dtype=np.int64).ravel():
        d = sssp(g, int(s)).astype(np.int64)
        order = [int(v) for v in np.argsort(d, kind="stable") if d[v] != INF]
        d = d.tolist()
        h = [0] * n
        for v in reversed(order):                      # nonincreasing d(v)
            for e in range(first[v], first[v + 1]):
                w = head[e]
                if w != v and d[w] != INF and d[v] + ln[e] == d[w]:
                    h[v] = max(h[v], ln[e] + h[w])
            r[v] = max(r[v], min(d[v], h[v]))
    return np.array(r, dtype=np.uint32)
