"""Debug: band launches vs the oracle on small graphs; prints where labels differ."""
import sys, os
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ipps_dellinggnw11_b200 as P, phastgen, oracle
import torch

def run(g, name, flags, unit, k):
    with P.Phast.from_graph(g) as h:
        h.configure(flags=flags, band_unit=unit)
        src = phastgen.sources(g.n, k, seed=950 + k)
        d = h.trees(src); h.sync()
        got = h.to_original(d.cpu().numpy())
        want = oracle.sssp_many(g, src)
        bad = np.nonzero((got != want).any(axis=0))[0]
        sched = h.schedule(k)
        ex = h.export(); perm = h.order()
        msg = f"{name} flags={flags} unit={unit} k={k}: bad={bad.size} sched={sched}"
        if bad.size:
            bi = perm[bad]
            lev = ex["level"][bi]
            msg += f"\n   bad internal ids min {bi.min()} max {bi.max()} levels {np.bincount(lev)[:12]}"
            bands = h.bands()
            msg += f"\n   bands {[(b['seg_lo'], b['seg_hi'], b['ngroups']) for b in bands]} levels {h.levels}"
            lo = np.concatenate([[0], np.cumsum(h.level_sizes()[::-1])])
            msg += f"\n   seg offsets {lo.tolist()}"
        print(msg, flush=True)

C1 = phastgen.CONFIGS["C1"]["graph"]()
R = phastgen.road(40_000, seed=35)
for g, name in ((C1, "C1"), (R, "road40k")):
    for flags, unit in ((P.Q_NO_FUSED | P.Q_NO_TOP, 0), (P.Q_NO_FUSED | P.Q_NO_TOP, 1 << 20), (P.Q_NO_FUSED, 0),
                        (0, 0), (P.Q_NO_FUSED | P.Q_NO_TOP | P.Q_NO_BANDS, 0)):
        for k in (1, 16, 64):
            run(g, name, flags, unit, k)
