"""Instruction mix + per-source-line summary of one ncu report (SASS page with -lineinfo):
python tools/ncu_ops.py report.ncu-rep [groups]   (groups: 32-record groups, for per-group counts)"""
import collections, csv, io, subprocess, sys
rep = sys.argv[1]
groups = float(sys.argv[2]) if len(sys.argv) > 2 else 0
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
data = [dict(zip(h, r)) for r in rows[2:] if len(r) == len(h)]
f = lambda x: float(x) if x not in ('', '-') else 0.0
tot = sum(f(d["Instructions Executed"]) for d in data)
ts = sum(f(d["Warp Stall Sampling (All Samples)"]) for d in data)
op = collections.Counter()
for d in data:
    src = d["Source"].strip()
    if src.startswith('@'):
        src = src.split(None, 1)[1]
    op[(src.split() or ['?'])[0].split('.')[0]] += f(d["Instructions Executed"])
print(f"total warp instructions {tot/1e9:.3f} G" + (f" = {tot/groups:.1f} per group" if groups else ""))
for o, c in op.most_common(25):
    print(f"  {o:12s} {c/1e9:7.3f} G {100*c/tot:5.1f}%" + (f" {c/groups:6.1f}/group" if groups else ""))
stalls = [x for x in h if x.startswith("stall_") and "Not Issued" not in x]
agg = {s: sum(f(d[s]) for d in data) for s in stalls}
print("stall reasons (share of samples):", ", ".join(f"{k[6:]} {100*v/ts:.1f}%" for k, v in sorted(agg.items(), key=lambda x: -x[1])[:8]))
