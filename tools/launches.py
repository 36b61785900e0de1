"""Summarise an ncu --metrics gpu__time_duration.sum launch list: per-kernel average us."""
import collections
import csv
import sys


def summarise(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
    h = rows[hi]
    ki, mi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
    d = collections.defaultdict(list)
    for r in rows[hi + 1:]:
        if len(r) <= mi:
            continue
        v = float(r[mi].replace(',', ''))
        u = r[ui]
        v = v / 1000 if u in ('nsecond', 'ns') else (v * 1000 if u in ('msecond', 'ms') else v)
        name = r[ki].split('(')[0].replace('void ', '').replace('dp::<unnamed>::', '').replace('unnamed>::', '')[:48]
        d[name].append(v)
    return d


if __name__ == "__main__":
    d = summarise(sys.argv[1])
    tot = 0.0
    for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1]) / len(kv[1])):
        avg = sum(v) / len(v)
        if 'Fill' not in k:
            tot += avg
        print(f"{k:50s} n={len(v):3d} avg={avg:9.2f} us")
    print(f"{'sum of libdp kernel averages':50s}       {tot:9.2f} us")
