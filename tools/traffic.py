"""Per-sweep DRAM bytes of the default path from an ncu launch list (tools/launches.py
format) -> profiles/sweep_traffic.json entry used as bench.py's roofline.traffic.

  python tools/traffic.py LAUNCHES.csv KEY LAYOUT [--cache-control none|all]
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from launches import load  # noqa: E402


def main(path, key, layout, cache="all"):
    L = load(path)
    starts = [j for j, x in enumerate(L) if 'upward' in x['name']] + [len(L)]
    rd, wr, t, n = 0.0, 0.0, 0.0, 0
    for a, b in zip(starts[:-1], starts[1:]):
        sw = [x for x in L[a:b] if 'sweep' in x['name']]
        if not sw:
            continue
        rd += sum(x.get('dram__bytes_read.sum', 0) for x in sw)
        wr += sum(x.get('dram__bytes_write.sum', 0) for x in sw)
        t += sum(x.get('gpu__time_duration.sum', 0) for x in sw)
        n += 1
    out = os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", "profiles", "sweep_traffic.json")
    prof = json.load(open(out)) if os.path.exists(out) else {}
    prof[key] = {"dram_bytes_per_sweep": (rd + wr) / n, "dram_read": rd / n, "dram_write": wr / n,
                 "ncu_sweep_s": t / n, "sweeps_averaged": n, "cache_control": cache,
                 "source": f"{os.path.relpath(path)} (ncu launch list, dram__bytes per sweep launch "
                           f"(sweep_top_kernel + sweep_band_kernel + sweep_kernel), summed per sweep, averaged)",
                 "layout": layout, "sweep": "levels", "arc_batch": "ell", "top": True}
    json.dump(prof, open(out, "w"), indent=1)
    print(key, prof[key])


if __name__ == "__main__":
    a = sys.argv[1:]
    cache = "all"
    if "--cache-control" in a:
        i = a.index("--cache-control")
        cache = a[i + 1]
        del a[i:i + 2]
    main(*a, cache=cache)
