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


@pytest.mark.parametrize("k", (1, 2, 3, 4, 5, 7, 8, 12, 16, 17, 31, 32, 33, 48, 63, 64))
def test_every_k_with_duplicates(road, k):
    """Every k of the boundary (1 <= k <= 64): the vector widths
    directly, the others padded to the next width and compacted into the caller's
    n*k buffer."""
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
    for k in (64, 1, 32, 4, 9, 64):
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
        for k in (1, 13, 16, 64):
            src = phastgen.sources(g.n, k, seed=7 + k)
            assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), k


def gpu_parents(h, src):
    src = np.asarray(src, np.uint32)
    d = h.trees(src)
    p = h.parents(src, d)
    h.sync()
    return h.to_original(d.cpu().numpy()), h.parents_to_original(p.cpu().numpy())


@pytest.mark.parametrize("k", (1, 4, 5, 16, 24, 64))
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


def test_upward_global_fallback_and_overflow():
    """A shared-memory table too small for the search space falls back to the global
    table (same labels); a per-source capacity too small is reported as ERANGE by
    phast_sync (never silently wrong labels)."""
    g = phastgen.grid(100, 100, 1, 1 << 20, seed=1)   # upward spaces ~200-300 vertices
    src = phastgen.sources(g.n, 16, seed=3)
    want = oracle.sssp_many(g, src)
    full_searches = P.Q_NO_FUSED | P.Q_HYBRID_OFF       # the upward kernel, whole searches
    with P.Phast.from_graph(g) as h:
        h.configure(flags=full_searches, up_smem_cap=32)
        assert np.array_equal(gpu_trees(h, src), want)
        h.configure(flags=full_searches, seed_cap=32)
        h.trees(src)
        with pytest.raises(P.PhastError) as e:
            h.sync()
        assert e.value.status == -4
        h.sync()                                       # error word is cleared
        h.configure()                                  # defaults again: exact
        assert np.array_equal(gpu_trees(h, src), want)


SCHEDULES = {
    "default": {},
    "per_level": dict(flags=P.Q_NO_TOP | P.Q_NO_FUSED),          # the paper's: one launch per level
    "top_hybrid": dict(flags=P.Q_NO_FUSED | P.Q_HYBRID_ON),
    "top_full_searches": dict(flags=P.Q_NO_FUSED | P.Q_HYBRID_OFF),
    "top_40": dict(flags=P.Q_NO_FUSED, top_max_vertices=40),    # the prefix ends inside the hierarchy
    "top_700": dict(flags=P.Q_NO_FUSED, top_max_vertices=700),
    "top_3000_hybrid": dict(flags=P.Q_NO_FUSED | P.Q_HYBRID_ON, top_max_vertices=3000),
    "no_bands": dict(flags=P.Q_NO_FUSED | P.Q_NO_BANDS),        # band levels one launch per level
    "bands_unit_32": dict(flags=P.Q_NO_FUSED, band_unit=32),   # one closed group per work unit
    "bands_unit_big": dict(flags=P.Q_NO_FUSED | P.Q_NO_TOP, band_unit=1 << 20),   # few units, no top launch
    "bands_v1_256": dict(flags=P.Q_NO_FUSED, band_variant=1, band_threads=256),   # records one item ahead
    "bands_v4": dict(flags=P.Q_NO_FUSED | P.Q_NO_TOP, band_variant=4, band_threads=128),   # tails through the L1
    "bands_lpt2": dict(flags=P.Q_NO_FUSED, band_variant=13),                   # two 16-byte lanes per thread
    "bands_v5_k32": dict(flags=P.Q_NO_FUSED | P.Q_NO_TOP, band_variant=5, band_threads=256),
}


@pytest.mark.parametrize("layout", ["levels-bands", "levels-bfs", "levels"])
@pytest.mark.parametrize("sched", sorted(SCHEDULES))
def test_schedules(layout, sched):
    """Every launch schedule (phast_configure) on both vertex orders is bit-exact:
    one launch per level (§VI), the shared-memory top launch with and
    without the hybrid upward search, capped top prefixes, and (default, small graphs)
    the single fused launch; every k including padded ones; plus the diameter."""
    for g in (phastgen.CONFIGS["C1"]["graph"](), phastgen.road(40_000, seed=35), phastgen.road(9_000, seed=36)):
        with P.Phast.from_graph(g, layout=layout) as h:
            h.configure(**SCHEDULES[sched])
            for k in (1, 2, 4, 6, 16, 64):
                src = phastgen.sources(g.n, k, seed=950 + k)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (k, sched)
            for kb in (1, 4, 16):
                src = phastgen.sources(g.n, 130, seed=951)
                assert h.diameter(src, k_batch=kb) == oracle.diameter(g, src), kb


def test_schedule_reports_launch_shape():
    """phast_schedule: C1 at k <= 4 is one fused launch; a road graph gets a top launch,
    band launches for the bottom levels and per-level launches between; NO_TOP|NO_BANDS
    gives one launch per level."""
    g = phastgen.CONFIGS["C1"]["graph"]()
    with P.Phast.from_graph(g) as h:
        s = h.schedule(1)
        assert s["fused"] and s["level_launches"] == 0 and s["top_vertices"] == g.n
    g = phastgen.road(120_000, seed=33)
    with P.Phast.from_graph(g) as h:
        s = h.schedule(64)
        assert not s["fused"] and s["top_levels"] >= 2 and s["band_launches"] >= 1
        assert s["top_levels"] + s["level_launches"] + s["band_levels"] == h.levels
        h.configure(flags=P.Q_NO_TOP | P.Q_NO_FUSED | P.Q_NO_BANDS)
        assert h.schedule(64) == dict(fused=False, top_levels=0, top_vertices=0, level_launches=h.levels,
                                      band_launches=0, band_levels=0)
        h.configure(flags=P.Q_NO_TOP | P.Q_NO_FUSED)
        s = h.schedule(64)
        assert s["band_levels"] == sum(b["seg_hi"] - b["seg_lo"] for b in h.bands())
        assert s["band_launches"] == len(h.bands()) and s["level_launches"] + s["band_levels"] == h.levels


def test_fused_query_edge_cases():
    """The fused single-launch query on graphs with unreachable parts, one-way arcs,
    zero and near-2^32 lengths (random digraphs), duplicate sources; bit-exact, and
    again with the per-level path for comparison."""
    for seed in range(6):
        g = phastgen.random_digraph(400 + 50 * seed, 1500 + 300 * seed, 0 if seed % 2 else 1,
                                    (1 << 32) - 1 if seed == 5 else 1 << 20, seed=70 + seed)
        with P.Phast.from_graph(g) as h:
            for flags in (0, P.Q_NO_FUSED):
                h.configure(flags=flags)
                for k in (1, 3, 4, 16):
                    src = phastgen.sources(g.n, k, seed=seed, distinct=False)
                    assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (seed, flags, k)


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


def test_queries_in_flight_on_several_streams(road):
    """PHAST_SLOTS queries in flight: 11 queries issued round robin on 3 streams into 3
    label buffers (each buffer reused by its own stream), mixed k (padded k too), no
    host synchronisation in between; every result bit-exact.  Exercises the slot
    rotation (visited bits, search spaces, padded scratch) across streams."""
    g, h = road
    streams = [torch.cuda.Stream() for _ in range(3)]
    ks = [64, 16, 5, 64, 1, 33, 16, 64, 7, 2, 64]
    srcs = [phastgen.sources(g.n, k, seed=1200 + i) for i, k in enumerate(ks)]
    bufs = [torch.empty(g.n * 64, dtype=torch.int32, device="cuda") for _ in range(3)]
    got = []
    for i, (k, src) in enumerate(zip(ks, srcs)):
        st = streams[i % 3]
        out = bufs[i % 3][:g.n * k]
        h.trees(src, out=out, stream=st)
        host = torch.empty(g.n * k, dtype=torch.int32, pin_memory=True)
        with torch.cuda.stream(st):
            host.copy_(out, non_blocking=True)
        got.append((host, st))
    for (host, st), src in zip(got, srcs):
        st.synchronize()
        assert np.array_equal(h.to_original(host.numpy()), oracle.sssp_many(g, src))
    h.sync()


def test_probes_leave_state_clean(road):
    """Probes A33 (stream) and A34 (no-gather traversal) run through the C ABI; a query
    after them is still exact (A34 seeds and clears its slot like a query)."""
    g, h = road
    buf = torch.zeros(g.n * 16, dtype=torch.int32, device="cuda")
    src = phastgen.sources(g.n, 16, seed=1300)
    h.probe(0, 16, buf)
    h.probe(1, 16, buf, sources=src)
    h.sync()
    with pytest.raises(P.PhastError):
        h.probe(1, 16, buf)                 # A34 needs sources
    with pytest.raises(P.PhastError):
        h.probe(0, 12, buf[:g.n * 12])      # probes take the vector widths only
    assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src))


def test_binding_rejects_bad_output_tensors(road):
    """The binding checks what the library will write: dtype, element
    count, device, contiguity -- before any pointer reaches the C ABI."""
    g, h = road
    src = phastgen.sources(g.n, 4, seed=1)
    with pytest.raises(TypeError):
        h.trees(src, out=torch.empty(g.n * 4, dtype=torch.int64, device="cuda"))
    with pytest.raises(ValueError):
        h.trees(src, out=torch.empty(g.n * 4 - 1, dtype=torch.int32, device="cuda"))
    with pytest.raises(ValueError):
        h.trees(src, out=torch.empty(g.n * 4, dtype=torch.int32))
    with pytest.raises(ValueError):
        h.trees(src, out=torch.empty(g.n * 8, dtype=torch.int32, device="cuda")[::2])
    with pytest.raises(TypeError):
        h.betweenness([0, 1], out=torch.empty(g.n, dtype=torch.int32, device="cuda"))
    with pytest.raises(ValueError):
        h.reach([0, 1], out=torch.empty(g.n + 1, dtype=torch.int32, device="cuda"))
    d = h.trees(src)
    with pytest.raises(ValueError):
        h.parents(src, d, out=torch.empty(g.n, dtype=torch.int32, device="cuda"))


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs two GPUs")
def test_two_devices_in_one_process():
    """Handles on two devices (per-device kernel attributes and SM counts)."""
    g = phastgen.road(30_000, seed=41)
    src = phastgen.sources(g.n, 16, seed=2)
    want = oracle.sssp_many(g, src)
    hs = []
    for dev in (0, 1):
        torch.cuda.set_device(dev)
        hs.append(P.Phast.from_graph(g))
    for dev, h in enumerate(hs):
        torch.cuda.set_device(dev)
        assert np.array_equal(gpu_trees(h, src), want), dev
        h.close()
    torch.cuda.set_device(0)


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
        h.trees(np.zeros(65, np.uint32))       # k > PHAST_KMAX
    with pytest.raises(ValueError):
        h.trees(np.zeros(0, np.uint32))


@pytest.mark.parametrize("k", (8, 11))
def test_host_entry_point(road, k):
    g, h = road
    src = phastgen.sources(g.n, k, seed=77)
    out = np.empty((g.n, k), np.uint32)
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
    for kb in (1, 5, 16):
        assert h.diameter(sub[:37], k_batch=kb) == int(tm[:37].max())


def test_diameter_road_and_unreachable(road):
    g, h = road
    src = phastgen.sources(g.n, 100, seed=5)
    assert h.diameter(src, k_batch=32) == oracle.diameter(g, src)
    g2 = EDGE_GRAPHS["unreachable"]()
    with P.Phast.from_graph(g2) as h2:
        src = np.arange(0, g2.n, 7, dtype=np.uint32)
        assert h2.diameter(src, k_batch=64) == oracle.diameter(g2, src)


def witness_ok(g, src, D, s, t):
    """(D, s*, t*) from phast_diameter_witness: D is the oracle's diameter over src, s*
    is one of the sources, and the oracle's dist(s*, t*) = D."""
    assert s in set(int(x) for x in src)
    assert int(oracle.sssp(g, s)[t]) == D


def test_diameter_witness(c1, road):
    for g, h in (c1, road):
        src = phastgen.sources(g.n, 300, seed=12)
        for kb in (64, 7):
            D, s, t = h.diameter_witness(src, k_batch=kb)
            assert D == oracle.diameter(g, src), kb
            witness_ok(g, src, D, s, t)
    g1 = phastgen.Graph(2, np.array([0, 0, 0], np.uint64), np.zeros(0, np.uint32), np.zeros(0, np.uint32))
    with P.Phast.from_graph(g1) as h1:
        assert h1.diameter_witness([1, 0]) == (0, 1, 1)     # no finite nonzero label


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
def test_c3_europe_scale_bench_configs():
    """C3 at full size (~18M vertices, ~42M arcs) in the bench's launch configurations
    (BASELINE.json configs[2]: k = 16, 32, 64; labels left in HBM): per k, 4 sampled
    trees bit-exact against the oracle and 12 more certified by the O(n+m)
    certificate."""
    cfg = phastgen.CONFIGS["C3"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        for k in (16, 32, 64):
            src = phastgen.sources(g.n, k, seed=cfg["src_seed"] + k)
            got = gpu_trees(h, src)
            pick = [0, k // 3, (2 * k) // 3, k - 1]
            assert np.array_equal(got[pick], oracle.sssp_many(g, src[pick])), k
            for i in range(1, k, max(1, k // 12)):
                assert oracle.certify(g, int(src[i]), got[i]) == 0, (k, i)


@pytest.mark.slow
def test_c4_usa_scale_bench_config():
    """C4 at full size (~24M vertices, ~58M arcs, USA shape) in the bench's launch
    configuration (k=64): 3 sampled trees bit-exact against the oracle, 8 more
    certified; plus the diameter over the same 64 sources against the ORACLE's
    maxima of those 64 trees (oracle.tree_maxima, independent of the GPU rows)."""
    cfg = phastgen.CONFIGS["C4"]
    g = cfg["graph"]()
    with P.Phast.from_graph(g) as h:
        src = phastgen.sources(g.n, 64, seed=cfg["src_seed"])
        got = gpu_trees(h, src)
        pick = [3, 31, 62]
        assert np.array_equal(got[pick], oracle.sssp_many(g, src[pick]))
        for i in range(0, 64, 8):
            assert oracle.certify(g, int(src[i]), got[i]) == 0, i
        del got
        assert h.diameter(src, k_batch=64) == int(oracle.tree_maxima(g, src).max())


@pytest.mark.slow
def test_c5_exact_diameter_with_witness():
    """C5 (BASELINE.json configs[4]): the exact diameter over ALL sources of the 1M
    road graph, with its witness (SURVEY.md §8(c) diameter row): the oracle confirms
    dist(s*, t*) = D, and the oracle's maximum over 1 024 sampled sources is <= D.
    The per-rank form (sources sharded, MAX all-reduce) is covered on CPU by
    tests/test_parallel.py."""
    cfg = phastgen.CONFIGS["C5"]
    g = cfg["graph"]()
    allsrc = np.arange(g.n, dtype=np.uint32)
    with P.Phast.from_graph(g) as h:
        D, s, t = h.diameter_witness(allsrc, k_batch=64)
        assert h.diameter(allsrc, k_batch=64) == D
    witness_ok(g, allsrc, D, s, t)
    sample = phastgen.sources(g.n, 1024, seed=cfg["src_seed"] + 9)
    assert int(oracle.tree_maxima(g, sample).max()) <= D
    assert int(oracle.tree_maxima(g, [s]).max()) == D        # s* is an eccentricity-D source


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


def test_centrality_padded_batches():
    """k_batch not a power of two (rounded up internally): same values."""
    g = BC_GRAPHS["unit_grid"]()
    src = phastgen.sources(g.n, 21, seed=77)
    with P.Phast.from_graph(g) as h:
        cb = h.vertex_to_original(h.betweenness(src, k_batch=5).cpu().numpy())
        r = h.vertex_to_original(h.reach(src, k_batch=11).cpu().numpy().view(np.uint32))
    bc_close(cb, oracle.betweenness(g, src))
    assert np.array_equal(r, oracle.reach(g, src))


@pytest.mark.parametrize("name", ["c1", "road", "unit_grid", "unreachable", "zero_lengths"])
def test_parents_ch_bit_exact(c1, road, name):
    """NEXT-1 in the hierarchy (phast_parents_ch, reading R19): bit-exact with
    oracle.parents_ch on the exported hierarchy and the oracle's distances, for k in
    {1, 5, 16, 64}; parents are internal ids, shortcut tails included."""
    if name == "c1":
        g, h = c1
    elif name == "road":
        g, h = road
    else:
        g = EDGE_GRAPHS[name]()
        h = P.Phast.from_graph(g)
    ex = h.export()
    perm = h.order()
    for k in (1, 5, 16, 64):
        src = phastgen.sources(g.n, k, seed=700 + k, distinct=False)
        d = h.trees(src)
        p = h.parents_ch(src, d)
        h.sync()
        rows = p.cpu().numpy().view(np.uint32).reshape(h.n, k)
        for i in (0, k // 2, k - 1):
            dint = np.empty(h.n, np.int64)
            dint[perm] = oracle.sssp(g, int(src[i])).astype(np.int64)
            want = oracle.parents_ch(ex, dint, int(perm[src[i]]))
            assert np.array_equal(rows[:, i], want), (name, k, i)


@pytest.mark.gpu
def test_band_layout_save_load_device(tmp_path):
    """The band layout (R20) survives phast_save / phast_load onto the device: same
    bands, same schedule, bit-exact trees and diameter against the oracle, with the
    band launches on (default) and off."""
    g = phastgen.road(60_000, seed=45)
    p = str(tmp_path / "bands.phast")
    with P.Phast.from_graph(g) as h:
        h.save(p)
        b1, s1 = h.bands(), h.schedule(64)
    with P.Phast.load(p) as h:
        b2 = h.bands()
        assert len(b1) == len(b2) > 0 and h.schedule(64) == s1
        for x, y in zip(b1, b2):
            assert np.array_equal(x["goff"], y["goff"])
        assert s1["band_launches"] > 0
        for flags in (P.Q_NO_FUSED, P.Q_NO_FUSED | P.Q_NO_BANDS):
            h.configure(flags=flags)
            for k in (16, 64):
                src = phastgen.sources(g.n, k, seed=460 + k)
                assert np.array_equal(gpu_trees(h, src), oracle.sssp_many(g, src)), (flags, k)
            src = phastgen.sources(g.n, 200, seed=461)
            assert h.diameter(src, k_batch=64) == oracle.diameter(g, src)
