"""Pins for the oracle (-m "not gpu").  The oracle is pinned to things other than
itself: Floyd-Warshall and Bellman-Ford brute force (written here, independently),
scipy's csgraph Dijkstra (a library routine), closed forms, and hand-derived golden
fixtures (tests/golden/).  Each pin is chosen so that a plausible oracle mistake (a
dropped length term, a reversed arc direction, a wrong clamp, a missing parallel-arc
min, a stale heap entry accepted) fails at least one of them."""
import os

import numpy as np
import pytest

import oracle
import phastgen
from phastgen import Graph

INF = oracle.INF
GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def csr_from_arcs(n, arcs):
    """Graph from a list of (tail, head, len)."""
    arcs = sorted(arcs, key=lambda a: a[0])  # stable: keeps per-tail order
    first = np.zeros(n + 1, np.uint64)
    for t, _, _ in arcs:
        first[t + 1] += 1
    first = np.cumsum(first).astype(np.uint64)
    head = np.array([a[1] for a in arcs], np.uint32)
    ln = np.array([a[2] for a in arcs], np.uint32)
    return Graph(n, first, head, ln)


def floyd_warshall(g):
    """All-pairs, exact in Python-int-safe int64 (n*(2^32-1) < 2^63), clamped."""
    BIG = np.int64(1) << np.int64(60)
    D = np.full((g.n, g.n), BIG, dtype=np.int64)
    tails = g.tails()
    for t, h, l in zip(tails, g.head, g.len):
        D[t, h] = min(D[t, h], int(l))
    np.fill_diagonal(D, 0)
    for k in range(g.n):
        D = np.minimum(D, D[:, k:k + 1] + D[k:k + 1, :])
    return np.where(D >= INF, INF, D).astype(np.uint32)


def bellman_ford(g, s):
    """Single source, vectorised relaxation of every arc until a fixed point."""
    BIG = np.int64(1) << np.int64(60)
    d = np.full(g.n, BIG, dtype=np.int64)
    d[s] = 0
    tails = g.tails().astype(np.int64)
    heads = g.head.astype(np.int64)
    lens = g.len.astype(np.int64)
    for _ in range(g.n):
        cand = d[tails] + lens
        nd = d.copy()
        np.minimum.at(nd, heads, cand)
        if np.array_equal(nd, d):
            break
        d = nd
    return np.where(d >= INF, INF, d).astype(np.uint32)


# ---------------------------------------------------------------- brute force
@pytest.mark.parametrize("lenrange", [(0, 3), (0, 1000), (1, 1 << 20), (1 << 30, INF), (0, INF)])
def test_vs_floyd_warshall(lenrange):
    lo, hi = lenrange
    rng = np.random.default_rng(lo ^ hi)
    for trial in range(400):
        n = int(rng.integers(1, 24))
        m = int(rng.integers(0, 4 * n + 1))
        g = phastgen.random_digraph(n, m, lo, hi, seed=trial * 7919 + lo)
        fw = floyd_warshall(g)
        got = oracle.sssp_many(g, np.arange(n), threads=2)
        assert np.array_equal(got, fw), (trial, n, m)


def test_vs_bellman_ford_medium():
    for trial in range(20):
        n = 200 + 90 * trial
        m = 3 * n
        lo, hi = [(0, 5), (1, 100), (0, INF), (1 << 31, INF)][trial % 4]
        g = phastgen.random_digraph(n, m, lo, hi, seed=1000 + trial)
        for s in (0, n // 2, n - 1):
            assert np.array_equal(oracle.sssp(g, s), bellman_ford(g, s)), (trial, s)


def test_vs_scipy_csgraph_road():
    """Library routine pin at scale: scipy's Dijkstra on a 1M-vertex road-like graph
    (no zero lengths, no parallel arcs: scipy would sum duplicates)."""
    sp = pytest.importorskip("scipy.sparse")
    csgraph = pytest.importorskip("scipy.sparse.csgraph")
    g = phastgen.road(200_000, seed=11)
    A = sp.csr_matrix((g.len.astype(np.float64), g.head.astype(np.int64), g.first.astype(np.int64)),
                      shape=(g.n, g.n))
    srcs = phastgen.sources(g.n, 4, seed=12)
    ref = csgraph.dijkstra(A, directed=True, indices=srcs)
    ref = np.where(np.isinf(ref), INF, ref).astype(np.uint64)
    got = oracle.sssp_many(g, srcs)
    assert np.array_equal(got.astype(np.uint64), ref)


def test_vs_scipy_csgraph_grid_all_sources():
    sp = pytest.importorskip("scipy.sparse")
    csgraph = pytest.importorskip("scipy.sparse.csgraph")
    g = phastgen.grid(30, 20, 1, 1 << 20, seed=3)
    A = sp.csr_matrix((g.len.astype(np.float64), g.head.astype(np.int64), g.first.astype(np.int64)),
                      shape=(g.n, g.n))
    ref = csgraph.dijkstra(A, directed=True).astype(np.uint64)
    got = oracle.sssp_many(g, np.arange(g.n)).astype(np.uint64)
    assert np.array_equal(got, ref)


# ---------------------------------------------------------------- closed forms
def test_unit_grid_manhattan():
    W, H = 37, 23
    g = phastgen.grid(W, H, 1, 2, seed=5)   # every length 1
    assert (g.len == 1).all()
    for s in (0, W * H - 1, (H // 2) * W + W // 2, 5 * W + 30):
        sx, sy = s % W, s // W
        v = np.arange(W * H)
        want = np.abs(v % W - sx) + np.abs(v // W - sy)
        assert np.array_equal(oracle.sssp(g, s), want.astype(np.uint32))


def test_directed_path_prefix_sums():
    rng = np.random.default_rng(3)
    L = rng.integers(0, 1 << 28, size=40)
    g = csr_from_arcs(41, [(i, i + 1, int(L[i])) for i in range(40)])
    d = oracle.sssp(g, 0)
    pref = np.concatenate([[0], np.cumsum(L)])
    assert np.array_equal(d, np.where(pref >= INF, INF, pref).astype(np.uint32))
    d5 = oracle.sssp(g, 5)   # directed: nothing before 5 is reachable
    assert (d5[:5] == INF).all() and d5[5] == 0
    rest = pref[5:] - pref[5]
    assert np.array_equal(d5[5:], np.where(rest >= INF, INF, rest).astype(np.uint32))
    assert (d == INF).any() and (d != INF).sum() > 5    # the clamp is exercised


def test_bidirectional_cycle():
    n = 31
    fw_len = [3 + (i % 5) for i in range(n)]      # i -> i+1
    bw_len = [2 + (i % 7) for i in range(n)]      # i+1 -> i
    arcs = [(i, (i + 1) % n, fw_len[i]) for i in range(n)] + [((i + 1) % n, i, bw_len[i]) for i in range(n)]
    g = csr_from_arcs(n, arcs)
    for s in range(n):
        d = oracle.sssp(g, s)
        for t in range(n):
            cw = sum(fw_len[(s + j) % n] for j in range((t - s) % n))
            ccw = sum(bw_len[(s - j - 1) % n] for j in range((s - t) % n))
            assert d[t] == min(cw, ccw)


def test_star_and_metric_complete_graph():
    # star: centre 0, spokes both ways
    L = [5, 9, 0, 1 << 31]
    g = csr_from_arcs(5, [(0, i + 1, L[i]) for i in range(4)] + [(i + 1, 0, 1) for i in range(4)])
    assert list(oracle.sssp(g, 0)) == [0] + L
    # leaf 1 -> 0 -> j
    assert list(oracle.sssp(g, 1)) == [1, 0] + [1 + x for x in L[1:]]
    # complete digraph on points of a line, l(i,j) = |x_i - x_j|: direct arc is shortest
    x = np.array([0, 3, 4, 10, 11, 25, 40])
    n = len(x)
    g = csr_from_arcs(n, [(i, j, abs(int(x[i] - x[j]))) for i in range(n) for j in range(n) if i != j])
    for s in range(n):
        assert np.array_equal(oracle.sssp(g, s), np.abs(x - x[s]).astype(np.uint32))


# ---------------------------------------------------------------- golden
def load_golden(path, parents=None):
    n, arcs, dists, diam = None, [], {}, None
    for line in open(path):
        line = line.split("#")[0].split()
        if not line:
            continue
        if line[0] == "n":
            n = int(line[1])
        elif line[0] == "arc":
            arcs.append(tuple(int(x) for x in line[1:4]))
        elif line[0] == "dist":
            dists[int(line[1])] = [INF if x == "INF" else int(x) for x in line[2:]]
        elif line[0] == "diameter":
            diam = int(line[1])
        elif line[0] == "parent" and parents is not None:
            parents[int(line[1])] = [INF if x == "INF" else int(x) for x in line[2:]]
    return csr_from_arcs(n, arcs), dists, diam


GOLDEN_FILES = sorted(f for f in os.listdir(GOLDEN) if f.endswith(".txt"))


@pytest.mark.parametrize("name", GOLDEN_FILES)
def test_golden(name):
    g, dists, diam = load_golden(os.path.join(GOLDEN, name))
    for s, want in dists.items():
        assert list(oracle.sssp(g, s)) == want, (name, s)
        assert oracle.certify(g, s, np.array(want, np.uint32)) == 0
    assert oracle.diameter(g, list(dists)) == diam


@pytest.mark.parametrize("name", GOLDEN_FILES)
def test_golden_parents(name):
    want = {}
    g, dists, _ = load_golden(os.path.join(GOLDEN, name), want)
    for s, p in want.items():
        assert list(oracle.parents(g, s)) == p, (name, s)


# ---------------------------------------------------------------- parents
def _random_graph(rng, n, lo, hi, density=3):
    m = int(rng.integers(0, density * n + 1))
    arcs = [(int(rng.integers(n)), int(rng.integers(n)), int(rng.integers(lo, hi))) for _ in range(m)]
    return csr_from_arcs(n, arcs)


@pytest.mark.parametrize("lenrange", [(1, 4), (1, 1000), (0, 3)])
def test_parents_vs_floyd_warshall(lenrange):
    """Parents computed from Floyd-Warshall labels (independent of the oracle's
    Dijkstra): every parent arc exists and is tight; unreached <-> INF; with
    positive lengths, following parents from any reached vertex ends at s after
    < n steps with total length d(v) (a shortest-path tree, §VII-A)."""
    rng = np.random.default_rng(77 + lenrange[1])
    for trial in range(150):
        n = int(rng.integers(1, 24))
        g = _random_graph(rng, n, *lenrange)
        D = floyd_warshall(g)
        tails = g.tails()
        arcs = {}
        for e, (t, h, l) in enumerate(zip(tails, g.head, g.len)):
            arcs.setdefault((int(t), int(h)), []).append(int(l))
        for s in range(n):
            d = D[s]
            p = oracle.parents(g, s, d)
            assert np.array_equal(oracle.parents(g, s), p)      # same labels from the oracle's own sssp
            assert p[s] == s
            for v in range(n):
                if v == s:
                    continue
                if d[v] == INF:
                    assert p[v] == INF
                    continue
                u = int(p[v])
                assert u != v and (u, v) in arcs
                assert any(int(d[u]) + l == int(d[v]) for l in arcs[(u, v)])
                if lenrange[0] > 0:
                    x, tot, steps = v, 0, 0
                    while x != s:
                        y = int(p[x])
                        tot += min(l for l in arcs[(y, x)] if int(d[y]) + l == int(d[x]))
                        x, steps = y, steps + 1
                        assert steps < n
                    assert tot == int(d[v])


# ---------------------------------------------------------------- diameter
def test_diameter_vs_floyd_warshall():
    for trial in range(200):
        rng = np.random.default_rng(trial)
        n = int(rng.integers(1, 20))
        g = phastgen.random_digraph(n, int(rng.integers(0, 3 * n + 1)), 0, 50, seed=trial + 99)
        fw = floyd_warshall(g)
        fin = fw[fw != INF]
        assert oracle.diameter(g, np.arange(n)) == (int(fin.max()) if fin.size else 0)
        sub = np.arange(0, n, 2)
        fs = fw[sub]
        fs = fs[fs != INF]
        assert oracle.diameter(g, sub) == (int(fs.max()) if fs.size else 0)


# ---------------------------------------------------------------- certificate
def test_certificate_accepts_exact_and_rejects_perturbed():
    rng = np.random.default_rng(17)
    checked = 0
    for trial in range(300):
        n = int(rng.integers(2, 30))
        g = phastgen.random_digraph(n, int(rng.integers(n, 4 * n)), 0, 20, seed=5000 + trial)
        s = int(rng.integers(0, n))
        d = oracle.sssp(g, s)
        assert oracle.certify(g, s, d) == 0
        fin = np.flatnonzero((d != INF) & (np.arange(n) != s))
        if fin.size:
            v = int(rng.choice(fin))
            bad = d.copy(); bad[v] += 1                # too long: some arc is violated (ii)
            assert oracle.certify(g, s, bad) != 0
            if d[v] > 0:
                bad = d.copy(); bad[v] -= 1            # too short: no tight path (iii) or (ii)
                assert oracle.certify(g, s, bad) != 0
            bad = d.copy(); bad[v] = INF               # reachable marked unreachable (ii)
            assert oracle.certify(g, s, bad) == 2
            checked += 1
        bad = d.copy(); bad[s] = 1
        assert oracle.certify(g, s, bad) != 0
    assert checked > 200


def test_certificate_zero_length_cycle_counterexample():
    """s->a (10), a<->b (0,0), labels d(a)=d(b)=5 satisfy 'every
    reached v != s has a tight incoming arc' but are wrong; condition (iii) rejects."""
    g = csr_from_arcs(3, [(0, 1, 10), (1, 2, 0), (2, 1, 0)])
    assert oracle.certify(g, 0, np.array([0, 10, 10], np.uint32)) == 0
    assert oracle.certify(g, 0, np.array([0, 5, 5], np.uint32)) == 3


def test_oracle_rejects_bad_input():
    g = csr_from_arcs(3, [(0, 1, 1)])
    with pytest.raises(ValueError):
        oracle.sssp(g, 3)
    bad = Graph(3, g.first, np.array([7], np.uint32), g.len)
    with pytest.raises(ValueError):
        oracle.sssp(bad, 0)


# ---------------------------------------------------------------- NEXT-3 betweenness
def brute_shortest_paths(n, arcs, s):
    """{t: (shortest length, [list of prefix lengths along each shortest path, one
    (vertex, length from s) pair per vertex after s])} by enumerating every simple arc
    path from s (lengths > 0, so shortest paths are simple)."""
    out = [[] for _ in range(n)]
    for t, h, l in arcs:
        if t != h:
            out[t].append((h, l))
    paths = {}

    def dfs(v, length, seen, pre):
        for h, l in out[v]:
            if h in seen:
                continue
            paths.setdefault(h, []).append((length + l, pre + [(h, length + l)]))
            dfs(h, length + l, seen | {h}, pre + [(h, length + l)])
    dfs(s, 0, {s}, [])
    res = {}
    for t, ps in paths.items():
        best = min(p[0] for p in ps)
        res[t] = (best, [p[1] for p in ps if p[0] == best])
    return res


def brute_reach(n, arcs, sources):
    """reach by definition (§VII-B): over every shortest s-t path and every
    vertex v on it (s and t included, where the min is 0), min(len to v, len from v)."""
    r = np.zeros(n, np.int64)
    for s in sources:
        for t, (best, sp) in brute_shortest_paths(n, arcs, s).items():
            for p in sp:
                for v, dv in p:
                    r[v] = max(r[v], min(dv, best - dv))
    return r


def brute_betweenness(n, arcs, sources):
    """c_B by definition (§VII-B): enumerate every simple arc path s -> t
    by DFS (with lengths > 0 every shortest path is simple), keep the shortest ones
    per (s, t), and add sigma_st(v)/sigma_st for each interior v.  Parallel arcs are
    distinct arcs, so distinct paths (reading R16).  Independent of Brandes."""
    out = [[] for _ in range(n)]
    for t, h, l in arcs:
        if t != h:
            out[t].append((h, l))
    cb = np.zeros(n)
    for s in sources:
        paths = {}                     # t -> list of (length, interior vertex list)

        def dfs(v, length, seen, interior):
            for h, l in out[v]:
                if h in seen:
                    continue
                paths.setdefault(h, []).append((length + l, list(interior)))
                dfs(h, length + l, seen | {h}, interior + [h])
        dfs(s, 0, {s}, [])
        for t, ps in paths.items():
            best = min(p[0] for p in ps)
            sp = [p[1] for p in ps if p[0] == best]
            for inter in sp:
                for v in inter:            # the vertices strictly between s and t
                    cb[v] += 1.0 / len(sp)
    return cb


@pytest.mark.parametrize("seed", range(6))
def test_betweenness_vs_brute_force(seed):
    rng = np.random.default_rng(100 + seed)
    n = 6
    arcs = []
    for _ in range(14):
        t, h = rng.integers(0, n, 2)
        arcs.append((int(t), int(h), int(rng.integers(1, 4))))   # small lengths: many ties
    arcs.append((0, 1, 2))
    arcs.append((0, 1, 2))            # a parallel pair
    g = csr_from_arcs(n, arcs)
    src = list(range(n))
    np.testing.assert_allclose(oracle.betweenness(g, src), brute_betweenness(n, arcs, src),
                               rtol=1e-12, atol=1e-12)
    # partial sums over a source subset add up (the batching reading)
    a = oracle.betweenness(g, [0, 2, 4]) + oracle.betweenness(g, [1, 3, 5])
    np.testing.assert_allclose(a, oracle.betweenness(g, src), rtol=1e-12)


def test_betweenness_unit_grid_vs_brute_force():
    """3x3 bidirected unit grid: many equal-length paths (sigma up to 6)."""
    W = 3
    arcs = []
    for y in range(W):
        for x in range(W):
            v = y * W + x
            if x + 1 < W:
                arcs += [(v, v + 1, 1), (v + 1, v, 1)]
            if y + 1 < W:
                arcs += [(v, v + W, 1), (v + W, v, 1)]
    g = csr_from_arcs(W * W, arcs)
    cb = oracle.betweenness(g, range(W * W))
    np.testing.assert_allclose(cb, brute_betweenness(W * W, arcs, range(W * W)), rtol=1e-12)
    assert cb[4] == max(cb)           # the centre is the most central


def test_betweenness_closed_forms():
    # bidirected path v0 - ... - v(n-1): c_B(v_i) = 2 i (n-1-i) over ordered pairs
    n = 9
    arcs = [(i, i + 1, 3) for i in range(n - 1)] + [(i + 1, i, 3) for i in range(n - 1)]
    cb = oracle.betweenness(csr_from_arcs(n, arcs), range(n))
    np.testing.assert_array_equal(cb, [2.0 * i * (n - 1 - i) for i in range(n)])
    # bidirected star: centre (n-1)(n-2), leaves 0
    arcs = [(0, j, 5) for j in range(1, n)] + [(j, 0, 7) for j in range(1, n)]
    cb = oracle.betweenness(csr_from_arcs(n, arcs), range(n))
    np.testing.assert_array_equal(cb, [float((n - 1) * (n - 2))] + [0.0] * (n - 1))
    # a diamond with doubled middle: 0->1->3, 0->2->3, plus a parallel 0->1:
    # sigma_03 = 3, of which 2 pass through 1 and 1 through 2
    arcs = [(0, 1, 1), (0, 1, 1), (0, 2, 1), (1, 3, 1), (2, 3, 1)]
    cb = oracle.betweenness(csr_from_arcs(4, arcs), [0])
    np.testing.assert_allclose(cb, [0.0, 2.0 / 3.0, 1.0 / 3.0, 0.0], rtol=1e-15)


def test_betweenness_rejects_zero_length():
    with pytest.raises(ValueError):
        oracle.betweenness(csr_from_arcs(2, [(0, 1, 0)]), [0])


@pytest.mark.parametrize("seed", range(6))
def test_reach_vs_brute_force(seed):
    rng = np.random.default_rng(200 + seed)
    n = 7
    arcs = [(int(t), int(h), int(rng.integers(1, 5))) for t, h in rng.integers(0, n, (16, 2))]
    g = csr_from_arcs(n, arcs)
    src = list(range(n))
    np.testing.assert_array_equal(oracle.reach(g, src), brute_reach(n, arcs, src))
    np.testing.assert_array_equal(np.maximum(oracle.reach(g, [0, 1, 2]), oracle.reach(g, [3, 4, 5, 6])),
                                  oracle.reach(g, src))


def test_reach_closed_forms():
    # bidirected path with length-c arcs: r(v_i) = c * min(i, n-1-i)
    n, c = 10, 7
    arcs = [(i, i + 1, c) for i in range(n - 1)] + [(i + 1, i, c) for i in range(n - 1)]
    np.testing.assert_array_equal(oracle.reach(csr_from_arcs(n, arcs), range(n)),
                                  [c * min(i, n - 1 - i) for i in range(n)])
    # a tie: 0->1->3 and 0->2->3 both shortest (length 2+3 = 4+1); reach counts every
    # shortest path: r(1) = min(2, 3), r(2) = min(4, 1)
    arcs = [(0, 1, 2), (1, 3, 3), (0, 2, 4), (2, 3, 1)]
    np.testing.assert_array_equal(oracle.reach(csr_from_arcs(4, arcs), [0]), [0, 2, 1, 0])
