"""Summarise an ncu --page source --csv (SASS) dump: top instructions by stall samples and by
executed instructions, with nearby context. Usage: python tools/ncu_sass_top.py file.csv [N]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
data = [dict(zip(hdr, r)) for r in rows[2:] if len(r) == len(hdr)]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
def f(x):
    try: return float(x)
    except: return 0.0
tot_s = sum(f(d["Warp Stall Sampling (All Samples)"]) for d in data)
tot_i = sum(f(d["Instructions Executed"]) for d in data)
print("total samples", tot_s, "total warp instr", tot_i)
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
for key in ("Warp Stall Sampling (All Samples)", "Instructions Executed"):
    print("=== top by", key)
    idx = sorted(range(len(data)), key=lambda i: -f(data[i][key]))[:N]
    for i in sorted(idx):
        d = data[i]
        st = sorted(((f(d[s]), s) for s in stalls), reverse=True)[:2]
        print(f"{i:5d} {d['Source'][:60]:60s} samp={f(d['Warp Stall Sampling (All Samples)'])/tot_s*100:5.1f}% inst={f(d['Instructions Executed'])/tot_i*100:5.2f}% thr={d['Avg. Threads Executed']:>5s} {st}")
