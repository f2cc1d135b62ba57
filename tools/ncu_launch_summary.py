"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list: per-kernel count, total
ms and share (cold-cache, serialised: compare SHARES, not absolute times)."""
import collections, csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]
scale = {'ns': 1e-6, 'us': 1e-3, 'usecond': 1e-3, 'nsecond': 1e-6, 'ms': 1.0, 'msecond': 1.0}
agg = collections.defaultdict(lambda: [0, 0.0])
for r in rows[hi + 1:]:
    if len(r) != len(h):
        continue
    d = dict(zip(h, r))
    if d.get('Metric Name') != 'gpu__time_duration.sum':
        continue
    name = d['Kernel Name'].split('(')[0].replace('void ', '')
    a = agg[name]
    a[0] += 1
    a[1] += float(d['Metric Value']) * scale.get(d['Metric Unit'], 1e-6)
skip = [k for k in agg if k.startswith('<unnamed>') or k.startswith('cub::')]
tot = sum(v[1] for k, v in agg.items() if k not in skip)
print(f"{'kernel':45s} {'n':>5s} {'ms':>9s} {'share':>6s}   (generator / cub kernels excluded from the share)")
for k, (n, ms) in sorted(agg.items(), key=lambda x: -x[1][1]):
    share = f"{ms / tot * 100:5.1f}%" if k not in skip else "  gen "
    print(f"{k[:45]:45s} {n:5d} {ms:9.2f} {share}")
