"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
every kernel of libphast on small graphs, results checked against the oracle.

  compute-sanitizer --tool racecheck python tools/sanitize_driver.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import phastgen  # noqa: E402
import paper_conf_ipps_dellinggnw11_b200 as P  # noqa: E402


def check(h, g, src):
    d = h.trees(src)
    h.sync()
    got = h.to_original(d.cpu().numpy())
    assert np.array_equal(got, oracle.sssp_many(g, src)), "labels differ"
    return d


def main():
    import torch
    g1 = phastgen.grid(40, 30, 1, 1 << 20, seed=1)          # fused single-launch query (k <= 4)
    g2 = phastgen.road(20_000, seed=35)                      # upward kernel, seeds, top launch, level and band launches
    for g in (g1, g2):
        with P.Phast.from_graph(g) as h:
            for k in (1, 4, 16, 5):
                check(h, g, phastgen.sources(g.n, k, seed=k))
            h.configure(flags=P.Q_NO_FUSED | P.Q_HYBRID_ON)   # hybrid upward + top pull pass
            check(h, g, phastgen.sources(g.n, 16, seed=3))
            h.configure(flags=P.Q_NO_FUSED | P.Q_HYBRID_OFF, up_smem_cap=32)   # global-table fallback
            check(h, g, phastgen.sources(g.n, 8, seed=4))
            for v in (1, 4, 5):                               # band kernel variants (k >= 16), k = 64
                h.configure(flags=P.Q_NO_FUSED, band_variant=v)
                check(h, g, phastgen.sources(g.n, 64, seed=6 + v))
            h.configure(flags=P.Q_NO_FUSED | P.Q_NO_TOP, band_unit=32)   # one group per unit, no top launch
            check(h, g, phastgen.sources(g.n, 16, seed=9))
            h.configure()
            src = phastgen.sources(g.n, 16, seed=5)
            d = check(h, g, src)
            p = h.parents(src, d)
            h.sync()
            par = h.parents_to_original(p.cpu().numpy())
            for i, s in enumerate(src[:4]):
                assert np.array_equal(par[i], oracle.parents(g, s))
            allv = np.arange(min(g.n, 200), dtype=np.uint32)
            D, s, t = h.diameter_witness(allv, k_batch=16)
            assert D == oracle.diameter(g, allv) and int(oracle.sssp(g, s)[t]) == D
            buf = torch.zeros(g.n * 16, dtype=torch.int32, device="cuda")
            h.probe(0, 16, buf)
            h.probe(1, 16, buf, sources=src)
            h.sync()
    g3 = phastgen.grid(12, 10, 1, 6, seed=86)                # betweenness / reach passes
    with P.Phast.from_graph(g3) as h:
        allv = np.arange(g3.n, dtype=np.uint32)
        cb = h.vertex_to_original(h.betweenness(allv, k_batch=16).cpu().numpy())
        np.testing.assert_allclose(cb, oracle.betweenness(g3, allv), rtol=1e-9)
        r = h.vertex_to_original(h.reach(allv, k_batch=16).cpu().numpy().view(np.uint32))
        assert np.array_equal(r, oracle.reach(g3, allv))
    print("sanitize_driver ok")


if __name__ == "__main__":
    main()
