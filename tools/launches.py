"""Summarise an ncu --csv launch list (gpu__time_duration, dram bytes) per sweep."""
import collections
import csv
import sys

SC = {'Gbyte': 1e9, 'Mbyte': 1e6, 'Kbyte': 1e3, 'byte': 1, 'Tbyte': 1e12, 'GB': 1e9, 'MB': 1e6, 'KB': 1e3, 'B': 1}
TS = {'nsecond': 1e-9, 'usecond': 1e-6, 'msecond': 1e-3, 'ns': 1e-9, 'us': 1e-6, 'ms': 1e-3, 'second': 1, 's': 1}


def load(path):
    hdr, by = None, collections.OrderedDict()
    for r in csv.reader(open(path)):
        if r and r[0] == 'ID':
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            e = by.setdefault(d['ID'], {'name': d['Kernel Name']})
            v = float(d['Metric Value'].replace(',', ''))
            u = d['Metric Unit']
            e[d['Metric Name']] = v * (TS.get(u) or SC.get(u) or 1)
    return list(by.values())


def main(path, verbose=False):
    L = load(path)
    starts = [j for j, x in enumerate(L) if 'upward' in x['name']]
    if not starts:   # fused single-launch queries: one launch per step
        starts = [j for j, x in enumerate(L) if 'sweep_top' in x['name']]
    starts.append(len(L))
    for a, b in zip(starts[:-1], starts[1:]):
        grp = L[a:b]
        tot = sum(x.get('gpu__time_duration.sum', 0) for x in grp)
        rd = sum(x.get('dram__bytes_read.sum', 0) for x in grp)
        wr = sum(x.get('dram__bytes_write.sum', 0) for x in grp)
        sw = [x for x in grp if 'sweep' in x['name']]
        st = sum(x.get('gpu__time_duration.sum', 0) for x in sw)
        print(f"step: {len(grp)} launches, total {tot*1e3:.3f} ms, sweep {st*1e3:.3f} ms over {len(sw)} launches "
              f"({st/tot*100:.1f}%), DRAM read {rd/1e9:.2f} GB write {wr/1e9:.2f} GB")
    if verbose:
        for x in L[starts[-2]:]:
            print(f"{x['name'][:50]:50s} {x.get('gpu__time_duration.sum',0)*1e6:9.1f} us "
                  f"R {x.get('dram__bytes_read.sum',0)/1e6:9.1f} MB W {x.get('dram__bytes_write.sum',0)/1e6:9.1f} MB")


if __name__ == '__main__':
    main(sys.argv[1], len(sys.argv) > 2)
