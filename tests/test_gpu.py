"""GPU parity tests (-m gpu): the CUDA path, called through the C ABI, against the
oracle, element by element, bit-exact (all lengths and labels are uint32; Theorem
3.1, §III makes PHAST exact, so the bar is equality)."""
import numpy as np
import pytest

import oracle
import phastgen

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_dellinggnw11_b200 as P  # noqa: E402

INF = 0xFFFFFFFF


def gpu_trees(h, src, stream=None):
    d = h.trees(np.asarray(src, np.uint32), stream=stream)
    h.sync(stream)
    return h.to_original(d.cpu().numpy())


@pytest.fixture(scope="module")
def c1():
    g = phastgen.CONFIGS["C1"]["graph"]()
    return g, P.Phast.from_graph(g)


@pytest.fixture(scope="module")
def road():
    g = phastgen.road(150_000, seed=31)
    return g, P.Phast.from_graph(g)


def test_library_is_the_cuda_path():
    # the package imports libphast.so (no CPU fallback exists); kernels count up
    before = P.launch_count()
    g = phastgen.grid(8, 8)
    with P.Phast.from_graph(g) as h:
        gpu_trees(h, [0])
    assert P.launch_count() > before


def test_c1_all_sources(c1):
    """C1: 100x100 grid, every one of the 10 000 sources, k=64 batches (+ k=1 on a
    sample), bit-exact."""
    g, h = c1
    want = oracle.sssp_many(g, np.arange(g.n))
    for b in range(0, g.n, 64):
        src = np.arange(b, b + 64) % g.n
        got = gpu_trees(h, src)
        assert np.array_equal(got, want[src]), b
    for s in (0, 5050, 9999, 123):
        assert np.array_equal(gpu_trees(h, [s])[0], want[s])


@pytest.mark.parametrize("k", P.K_ALLOWED)
def test_every_k_with_duplicates(road, k):
    g, h = road
    src = phastgen.sources(g.n, k, seed=100 + k, distinct=False)
    if k >= 4:
        src[1] = src[0]                      # duplicate sources are allowed
    got = gpu_trees(h, src)
    assert np.array_equal(got, oracle.sssp_many(g, src))


def test_repeated_calls_no_stale_state(road):
    """Visited bits and seeded rows must not leak between calls (§IV-C
    "After scanning v we unmark the vertex")."""
    g, h = road
    out = torch.empty((g.n, 16), dtype=torch.int32, device="cuda")
    for rep in range(4):
        src = phastgen.sources(g.n, 16, seed=200 + rep)
        h.trees(src, out=out)
        h.sync()
        assert np.array_equal(h.to_original(out.cpu().numpy()), oracle.sssp_many(g, src)), rep
    # same buffer, alternating k
    for k in (64, 1, 32, 4):
        src = phastgen.sources(g.n, k, seed=300 + k)
        assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src))


EDGE_GRAPHS = {
    "zero_lengths": lambda: phastgen.random_digraph(500, 1800, 0, 3, seed=41),
    "grid_zero": lambda: phastgen.grid(80, 40, 0, 4, seed=46),
    "saturating": lambda: phastgen.random_digraph(1500, 6000, 1 << 30, 0xFFFFFFFF, seed=42),
    "unreachable": lambda: phastgen.random_digraph(4000, 3000, 1, 1000, seed=43),
    "unit_grid": lambda: phastgen.grid(70, 30, 1, 2, seed=44),
}


@pytest.mark.parametrize("name", sorted(EDGE_GRAPHS))
def test_edge_case_graphs(name):
    g = EDGE_GRAPHS[name]()
    with P.Phast.from_graph(g) as h:
        for k in (1, 16, 64):
            src = phastgen.sources(g.n, k, seed=7 + k)
            assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), k


def gpu_parents(h, src):
    src = np.asarray(src, np.uint32)
    d = h.trees(src)
    p = h.parents(src, d)
    h.sync()
    return h.to_original(d.cpu().numpy()), h.parents_to_original(p.cpu().numpy())


@pytest.mark.parametrize("k", (1, 4, 16, 64))
def test_parents_bit_exact(c1, road, k):
    """NEXT-1 parent pointers (§VII-A tight-arc identity, reading R14):
    bit-exact with the oracle's canonical parents, C1 and a road graph."""
    for g, h in (c1, road):
        src = phastgen.sources(g.n, k, seed=600 + k, distinct=False)
        d, par = gpu_parents(h, src)
        for i, s in enumerate(src):
            assert np.array_equal(d[i], oracle.sssp(g, s)), (k, i)
            assert np.array_equal(par[i], oracle.parents(g, s)), (k, i)


@pytest.mark.parametrize("name", sorted(EDGE_GRAPHS))
def test_parents_edge_case_graphs(name):
    """Zero lengths (ties, zero cycles), saturating lengths, unreachable parts."""
    g = EDGE_GRAPHS[name]()
    with P.Phast.from_graph(g) as h:
        for k in (2, 64):
            src = phastgen.sources(g.n, k, seed=17 + k)
            _, par = gpu_parents(h, src)
            for i, s in enumerate(src):
                assert np.array_equal(par[i], oracle.parents(g, s)), (k, i)


def test_upward_global_fallback_and_overflow(monkeypatch):
    """A shared-memory table too small for the search space falls back to the global
    table (same labels); a per-source capacity too small is reported as ERANGE by
    phast_sync (never silently wrong labels)."""
    g = phastgen.grid(100, 100, 1, 1 << 20, seed=1)   # upward spaces ~200-300 vertices
    src = phastgen.sources(g.n, 16, seed=3)
    want = oracle.sssp_many(g, src)
    monkeypatch.setenv("PHAST_FUSED", "0")             # the upward-search kernel, not the fused pull sweep
    monkeypatch.setenv("PHAST_UP_HYBRID", "0")         # full searches (the hybrid stops below the top levels)
    monkeypatch.setenv("PHAST_UP_SMEM_CAP", "32")
    with P.Phast.from_graph(g) as h:
        assert np.array_equal(gpu_trees(h, src), want)
    monkeypatch.setenv("PHAST_SEED_CAP", "32")
    with P.Phast.from_graph(g) as h:
        h.trees(src)
        with pytest.raises(P.PhastError) as e:
            h.sync()
        assert e.value.status == -4
        h.sync()                                       # error word is cleared


@pytest.mark.parametrize("mode,level_layout,delta", [("levels", True, 0), ("levels", "bfs", 0),
                                                     ("levels-hybrid", True, 0), ("levels-flat", "bfs", 0),
                                                     ("levels-hybrid", "bfs", 0), ("levels-hybrid", "diagonal", 0),
                                                     ("levels-ab1", "bfs", 0), ("levels-ab3", "bfs", 0),
                                                     ("levels-ab4", "bfs", 0), ("levels-ab8", "bfs", 0),
                                                     ("levels-ab8", "diagonal", 0), ("levels-ab16", "bfs", 0),
                                                     ("levels-ab17", "bfs", 0), ("levels-ab17", True, 0),
                                                     ("bottomseg2-2", "diagonal", 0), ("bottomseg2-2", "diagonal", 3000),
                                                     ("bottomseg3-2", "diagonal", 0), ("bottomsegauto-3", "diagonal", 500),
                                                     ("bottomseg2-1", "diagonal", 2000),
                                                     ("warp", True, 0), ("staged", True, 0),
                                                     ("warp", False, 0), ("persistent", False, 0),
                                                     ("wpipe", False, 0), ("wpipe", False, 300), ("wpipe", True, 0),
                                                     ("pipe", False, 0), ("pipe", False, 300), ("pipe", True, 0),
                                                     ("staged", False, 0), ("warp", False, 300),
                                                     ("staged", False, 300), ("wave", False, 0),
                                                     ("wave", False, 300), ("wave", True, 0), ("wave", "bfs", 0),
                                                     ("levels", "diagonal", 0), ("levels", "diagonal", 500),
                                                     ("segments", True, 0), ("segments", "bfs", 0),
                                                     ("segments", "diagonal", 0), ("segments", "diagonal", 500)])
def test_sweep_modes(monkeypatch, mode, level_layout, delta):
    """Every schedule is bit-exact: one launch per level on the paper's level layout
    (§VI); the single persistent launch as warp dataflow (default) or CTA
    waves (with and without bulk-staged arcs), on both layouts, including a small
    wavefront skew (many short dependencies)."""
    if mode.startswith("bottomseg"):            # diagonal layout, bottom diagonals in one lagged launch
        cut, lag = mode[len("bottomseg"):].split("-")
        monkeypatch.setenv("PHAST_BOTTOM_SEG", "1")
        monkeypatch.setenv("PHAST_DIAG_LAG", lag)
        if cut != "auto":
            monkeypatch.setenv("PHAST_DIAG_CUT", cut)
        mode = "levels"
    elif mode.startswith("levels-ab"):            # per-level launches, other arc batch (1-4, 8 = cp.async staged,
                                                 # 16 = ELL-2 records, 17 = ELL-2 with the next record loaded ahead)
        monkeypatch.setenv("PHAST_ARC_BATCH", mode[len("levels-ab"):])
        mode = "levels"
    elif mode == "levels-hybrid":                # a few small top levels fused, the rest one launch each
        monkeypatch.setenv("PHAST_TOP_THRESH", "3000")
        mode = "levels"
    elif mode == "levels-flat":                  # one launch per level, no fusion
        monkeypatch.setenv("PHAST_TOP_THRESH", "0")
        mode = "levels"
    monkeypatch.setenv("PHAST_SWEEP", mode)
    g = phastgen.road(120_000, seed=33)
    layout = {True: "levels", "bfs": "levels-bfs", False: "wavefront"}.get(level_layout, level_layout)
    with P.Phast.from_graph(g, layout=layout, delta=delta) as h:
        for k in (1, 2, 16, 64):
            src = phastgen.sources(g.n, k, seed=900 + k)
            assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), k
        src = phastgen.sources(g.n, 200, seed=901)
        assert h.diameter(src, k_batch=64) == oracle.diameter(g, src)


@pytest.mark.parametrize("top", ["off", "default", "nofused", "nohybrid", "40", "700", "3000", "cluster-only", "cl4"])
def test_top_levels_kernel(monkeypatch, top):
    """The shared-memory sweep (sweep_top_kernel: rows in shared memory, cp.async-
    staged arc chunks) and the cluster sweep of the mid levels (sweep_cluster_kernel):
    off (one launch per level), cluster only, a 4-CTA cluster, default (C1 at k <= 4: the whole query
    fused in one launch, G-up as a pull sweep; larger k / the road graph: the top
    levels), top levels only ("nofused"), and top levels capped at V <= 40 / 700 /
    3000 vertices (the prefix ends inside the hierarchy, chunks split long levels);
    every k, bit-exact; plus the diameter (fused max over the final rows)."""
    if top == "off":
        monkeypatch.setenv("PHAST_TOP", "0")
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_CL_SIZE", "0")
    elif top == "cluster-only":                  # no shared-memory launch: mid levels in a 16-CTA cluster
        monkeypatch.setenv("PHAST_TOP", "0")
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_CL_SIZE", "16")
    elif top == "cl4":                           # a 4-CTA cluster, one pass per level: long levels excluded
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_CL_SIZE", "4")
        monkeypatch.setenv("PHAST_CL_PASSES", "1")
    elif top == "nofused":                       # top levels; the hybrid upward search forced on
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_UP_HYBRID", "1")
    elif top == "nohybrid":                      # full upward searches, the top kernel only sweeps G-down
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_UP_HYBRID", "0")
    elif top != "default":
        monkeypatch.setenv("PHAST_FUSED", "0")
        monkeypatch.setenv("PHAST_TOP_MAXV", top)
    for g in (phastgen.CONFIGS["C1"]["graph"](), phastgen.road(40_000, seed=35), phastgen.road(9_000, seed=36)):
        with P.Phast.from_graph(g) as h:
            for k in (1, 2, 4, 16, 64):
                src = phastgen.sources(g.n, k, seed=950 + k)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (k, top)
            for kb in (1, 4, 16):
                src = phastgen.sources(g.n, 130, seed=951)
                assert h.diameter(src, k_batch=kb) == oracle.diameter(g, src), kb


def test_fused_query_edge_cases(monkeypatch):
    """The fused single-launch query on graphs with unreachable parts, one-way arcs,
    zero and near-2^32 lengths (random digraphs), duplicate sources; bit-exact, and
    again with the per-level path for comparison."""
    for seed in range(6):
        g = phastgen.random_digraph(400 + 50 * seed, 1500 + 300 * seed, 0 if seed % 2 else 1,
                                    (1 << 32) - 1 if seed == 5 else 1 << 20, seed=70 + seed)
        for fused in ("1", "0"):
            monkeypatch.setenv("PHAST_FUSED", fused)
            with P.Phast.from_graph(g) as h:
                for k in (1, 4, 16):
                    src = phastgen.sources(g.n, k, seed=seed, distinct=False)
                    assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (seed, fused, k)


def test_top_levels_hub_vertex():
    """A sink hub with more in-arcs than a chunk holds (small chunks: 1 024 arcs, big:
    4 096): a grid plus one extra vertex that every grid vertex points to.  The hub
    has no out-arcs, so it is contracted first and keeps all its in-arcs in G-down.
    With 3 000 in-arcs, the fused query takes it in a big chunk (k = 1) and the top
    plan stops before its level (k = 16).  With 4 500 in-arcs no chunk holds it, and
    the fused plan falls back.  Bit-exact."""
    for W, H in ((60, 50), (75, 60)):
        base = phastgen.grid(W, H, 1, 1000, seed=W)
        n = base.n + 1
        hub = base.n
        rng = np.random.default_rng(W)
        deg = np.diff(base.first).astype(np.int64) + 1          # every grid vertex: one more arc, to the hub
        first = np.zeros(n + 1, np.uint64)
        first[1:base.n + 1] = np.cumsum(deg)
        first[n] = first[base.n]
        head = np.empty(int(first[n]), np.uint32)
        length = np.empty(int(first[n]), np.uint32)
        for_v = np.repeat(np.arange(base.n), np.diff(base.first).astype(np.int64))
        pos = first[:-2].astype(np.int64)[for_v] + (np.arange(base.m) - base.first[:-1].astype(np.int64)[for_v])
        head[pos] = base.head
        length[pos] = base.len
        last = first[1:base.n + 1].astype(np.int64) - 1
        head[last] = hub
        length[last] = rng.integers(1, 1000, base.n).astype(np.uint32)
        g = phastgen.Graph(n, first, head, length)
        with P.Phast.from_graph(g) as h:
            for k in (1, 16):
                src = phastgen.sources(n, k, seed=960 + k)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (n, k)


def test_l2_persistence_window(monkeypatch):
    """The per-level sweep with an L2 persistence window over the top levels' rows
    (PHAST_L2_PERSIST_MB) is bit-exact; the setting is process-wide, so the test
    switches it off again at the end."""
    g = phastgen.road(120_000, seed=39)
    try:
        monkeypatch.setenv("PHAST_L2_PERSIST_MB", "8")
        with P.Phast.from_graph(g) as h:
            for k in (1, 16, 64):
                src = phastgen.sources(g.n, k, seed=980 + k)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), k
    finally:
        monkeypatch.setenv("PHAST_L2_PERSIST_MB", "0")
        with P.Phast.from_graph(phastgen.grid(8, 8)):
            pass


@pytest.mark.parametrize("window", ["0", "1", "64"])
def test_wave_sweep_every_k(monkeypatch, window):
    """The warp-wave sweep (plan_waves + sweep_wave_kernel) at every k (each k has its
    own chunk geometry) and several placement windows, bit-exact, repeated calls
    (epoch-monotone completion counters)."""
    monkeypatch.setenv("PHAST_SWEEP", "wave")
    monkeypatch.setenv("PHAST_WAVE_WINDOW", window)
    g = phastgen.road(60_000, seed=35)
    with P.Phast.from_graph(g, layout="wavefront", delta=2000) as h:
        for k in (1, 2, 4, 8, 16, 32, 64):
            for rep in range(2):
                src = phastgen.sources(g.n, k, seed=950 + k + rep)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (k, rep)


def test_tiny_and_degenerate():
    for g in (phastgen.Graph(1, np.array([0, 0], np.uint64), np.zeros(0, np.uint32), np.zeros(0, np.uint32)),
              phastgen.grid(1, 2), phastgen.grid(3, 1, 0, 1)):
        with P.Phast.from_graph(g) as h:
            src = np.zeros(4, np.uint32)
            src[1::2] = g.n - 1
            assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src))


def test_source_out_of_range(road):
    g, h = road
    with pytest.raises(P.PhastError) as e:
        h.trees(np.array([g.n], np.uint32))
    assert e.value.status == -4
    with pytest.raises(ValueError):
        h.trees(np.zeros(3, np.uint32))


def test_host_entry_point(road):
    g, h = road
    src = phastgen.sources(g.n, 8, seed=77)
    out = np.empty((g.n, 8), np.uint32)
    h.trees_host(src, out)
    assert np.array_equal(h.to_original(out), oracle.sssp_many(g, src))


def test_diameter_c1_all_sources(c1):
    """Exact diameter (§VII-B) of C1 over all 10 000 sources; per-batch
    maxima against the oracle's per-tree maxima; count not divisible by k_batch."""
    g, h = c1
    allsrc = np.arange(g.n, dtype=np.uint32)
    tm = oracle.tree_maxima(g, allsrc)
    assert h.diameter(allsrc, k_batch=64) == int(tm.max())
    sub = allsrc[:1000]                      # 1000 = 15*64 + 40: ragged last batch
    bm = torch.zeros(16, dtype=torch.int32, device="cuda")
    d = h.diameter(sub, k_batch=64, batch_max=bm)
    assert d == int(tm[:1000].max())
    bmv = bm.cpu().numpy().view(np.uint32)
    for b in range(16):
        assert bmv[b] == tm[b * 64:(b + 1) * 64].max(), b
    for kb in (1, 16):
        assert h.diameter(sub[:37], k_batch=kb) == int(tm[:37].max())


def test_diameter_road_and_unreachable(road):
    g, h = road
    src = phastgen.sources(g.n, 100, seed=5)
    assert h.diameter(src, k_batch=32) == oracle.diameter(g, src)
    g2 = EDGE_GRAPHS["unreachable"]()
    with P.Phast.from_graph(g2) as h2:
        src = np.arange(0, g2.n, 7, dtype=np.uint32)
        assert h2.diameter(src, k_batch=64) == oracle.diameter(g2, src)


def test_distance_metric_deep_hierarchy():
    """NEXT-4: the travel-distance metric (§VIII-G: 410 levels instead of
    140 on Europe) gives a much deeper hierarchy; every schedule stays bit-exact."""
    g = phastgen.road(40_000, seed=37, metric="distance")
    with P.Phast.from_graph(g) as h:
        assert h.levels >= 50
        for k in (1, 16, 64):
            src = phastgen.sources(g.n, k, seed=970 + k)
            assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), k
        src = phastgen.sources(g.n, 100, seed=971)
        assert h.diameter(src, k_batch=16) == oracle.diameter(g, src)


def test_c2_1m_k16():
    """C2: ~1M-vertex road-like graph, k=16 (BASELINE.json configs[1]), all 16
    trees bit-exact, then a 64-tree batch certified by the O(n+m) certificate."""
    cfg = phastgen.CONFIGS["C2"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        src = phastgen.sources(g.n, 16, seed=cfg["src_seed"])
        assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src))
        src64 = phastgen.sources(g.n, 64, seed=cfg["src_seed"] + 1)
        got = gpu_trees(h, src64)
        for i in range(64):
            assert oracle.certify(g, int(src64[i]), got[i]) == 0, i


@pytest.mark.slow
def test_c3_europe_scale_bench_config():
    """C3 at full size (~18M vertices, ~42M arcs) in the bench's launch configuration
    (k=64): 4 sampled trees bit-exact against the oracle, 16 more certified."""
    cfg = phastgen.CONFIGS["C3"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        src = phastgen.sources(g.n, 64, seed=cfg["src_seed"])
        got = gpu_trees(h, src)
        pick = [0, 17, 40, 63]
        want = oracle.sssp_many(g, src[pick])
        assert np.array_equal(got[pick], want)
        for i in range(1, 64, 4):
            assert oracle.certify(g, int(src[i]), got[i]) == 0, i


@pytest.mark.slow
def test_c4_usa_scale_bench_config():
    """C4 at full size (~24M vertices, ~58M arcs, USA shape) in the bench's launch
    configuration (k=64): 3 sampled trees bit-exact against the oracle, 8 more
    certified; plus the diameter path on the same hierarchy for 64 sources against
    the oracle's maxima of those trees."""
    cfg = phastgen.CONFIGS["C4"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        src = phastgen.sources(g.n, 64, seed=cfg["src_seed"])
        got = gpu_trees(h, src)
        pick = [3, 31, 62]
        want = oracle.sssp_many(g, src[pick])
        assert np.array_equal(got[pick], want)
        for i in range(0, 64, 8):
            assert oracle.certify(g, int(src[i]), got[i]) == 0, i
        fin = np.where(got == INF, 0, got).max()
        assert h.diameter(src, k_batch=64) == int(fin)


@pytest.mark.slow
def test_c2d_distance_metric_config():
    """C2D (travel-distance metric, 167 levels) at full size, k=16, bit-exact."""
    cfg = phastgen.CONFIGS["C2D"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        src = phastgen.sources(g.n, 16, seed=cfg["src_seed"])
        assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src))


# ---------------------------------------------------------------- NEXT-3 betweenness
BC_GRAPHS = {
    "grid": lambda: phastgen.grid(40, 30, 1, 100, seed=81),
    "unit_grid": lambda: phastgen.grid(30, 20, 1, 2, seed=82),      # sigma ~ binomials: many ties
    "small_lengths": lambda: phastgen.random_digraph(900, 3600, 1, 4, seed=83),
    "unreachable": lambda: phastgen.random_digraph(1200, 1000, 1, 50, seed=84),
    "road": lambda: phastgen.road(3000, seed=85),
}


def bc_close(got, want):
    scale = max(1.0, float(np.abs(want).max()))
    np.testing.assert_allclose(got, want, rtol=1e-9, atol=1e-12 * scale)


@pytest.mark.parametrize("name", sorted(BC_GRAPHS))
@pytest.mark.parametrize("k_batch", (1, 16, 64))
def test_betweenness_vs_oracle(name, k_batch):
    """Partial betweenness over 37 sources (ragged last batch, one duplicate) against
    the oracle (§VII-B; fp64, tolerance: summation order only)."""
    g = BC_GRAPHS[name]()
    src = phastgen.sources(g.n, 37, seed=90 + k_batch, distinct=False)
    src[5] = src[4]
    want = oracle.betweenness(g, src)
    with P.Phast.from_graph(g) as h:
        got = h.vertex_to_original(h.betweenness(src, k_batch=k_batch).cpu().numpy())
    bc_close(got, want)


def test_betweenness_exact_all_sources_and_additivity():
    """count = n: the exact betweenness; disjoint source shards add up (the multi-GPU
    all_reduce(SUM) reading)."""
    g = phastgen.grid(12, 10, 1, 6, seed=86)
    allv = np.arange(g.n, dtype=np.uint32)
    want = oracle.betweenness(g, allv)
    with P.Phast.from_graph(g) as h:
        got = h.vertex_to_original(h.betweenness(allv, k_batch=64).cpu().numpy())
        a = h.vertex_to_original(h.betweenness(allv[::2], k_batch=32).cpu().numpy())
        b = h.vertex_to_original(h.betweenness(allv[1::2], k_batch=8).cpu().numpy())
    bc_close(got, want)
    bc_close(a + b, want)


def test_betweenness_rejects_zero_lengths():
    g = phastgen.grid(10, 10, 0, 3, seed=87)
    assert int(np.asarray(g.len).min()) == 0
    with P.Phast.from_graph(g) as h:
        with pytest.raises(P.PhastError) as e:
            h.betweenness([0, 1])
        assert e.value.status == -1


@pytest.mark.parametrize("name", sorted(BC_GRAPHS))
@pytest.mark.parametrize("k_batch", (1, 16, 64))
def test_reach_bit_exact(name, k_batch):
    """NEXT-3 exact reach (§VII-B, reading R17) over 37 sources with a
    ragged last batch and a duplicate: integer, bit-exact with the oracle."""
    g = BC_GRAPHS[name]()
    src = phastgen.sources(g.n, 37, seed=190 + k_batch, distinct=False)
    src[5] = src[4]
    want = oracle.reach(g, src)
    with P.Phast.from_graph(g) as h:
        got = h.vertex_to_original(h.reach(src, k_batch=k_batch).cpu().numpy().view(np.uint32))
    assert np.array_equal(got, want)


def test_reach_exact_all_sources_and_max_shards():
    g = phastgen.grid(12, 10, 1, 6, seed=186)
    allv = np.arange(g.n, dtype=np.uint32)
    want = oracle.reach(g, allv)
    with P.Phast.from_graph(g) as h:
        got = h.vertex_to_original(h.reach(allv, k_batch=64).cpu().numpy().view(np.uint32))
        a = h.vertex_to_original(h.reach(allv[:50], k_batch=4).cpu().numpy().view(np.uint32))
        b = h.vertex_to_original(h.reach(allv[50:], k_batch=32).cpu().numpy().view(np.uint32))
        # betweenness and reach share scratch: interleaving them must not leak state
        cb = h.vertex_to_original(h.betweenness(allv[:20], k_batch=16).cpu().numpy())
    assert np.array_equal(got, want)
    assert np.array_equal(np.maximum(a, b), want)
    bc_close(cb, oracle.betweenness(g, allv[:20]))


@pytest.mark.parametrize("persist", ("0", "1"))
def test_centrality_both_pass_drivers(monkeypatch, persist):
    """The graph-captured pass chunks (default) and the persistent cooperative Kahn
    kernel (PHAST_BC_PERSIST=1) give the oracle's values."""
    monkeypatch.setenv("PHAST_BC_PERSIST", persist)
    g = BC_GRAPHS["unit_grid"]()
    src = phastgen.sources(g.n, 21, seed=77)
    with P.Phast.from_graph(g) as h:
        cb = h.vertex_to_original(h.betweenness(src, k_batch=8).cpu().numpy())
        r = h.vertex_to_original(h.reach(src, k_batch=16).cpu().numpy().view(np.uint32))
    bc_close(cb, oracle.betweenness(g, src))
    assert np.array_equal(r, oracle.reach(g, src))
