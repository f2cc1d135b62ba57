"""Per-CUDA-source-line summary of an ncu report (needs -lineinfo):
python tools/ncu_lines.py report.ncu-rep [N]  -> top lines by executed instructions / stall samples."""
import csv, subprocess, sys, io
rep = sys.argv[1]
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
lines, fname, hdr = [], None, None
for r in rows:
    if len(r) >= 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
    elif r and r[0] == "Line No":
        hdr = r
    elif hdr and r and r[0] not in ("", "Function Name") and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        d["_file"] = fname
        lines.append(d)
f = lambda x: float(x) if x.replace('.', '', 1).isdigit() else 0.0
ti = sum(f(d["Instructions Executed"]) for d in lines) or 1
ts = sum(f(d["Warp Stall Sampling (All Samples)"]) for d in lines) or 1
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
for key in ("Instructions Executed", "Warp Stall Sampling (All Samples)"):
    print("=== top lines by", key)
    for d in sorted(lines, key=lambda d: -f(d[key]))[:N]:
        st = sorted(((f(d[s]), s[6:]) for s in stalls), reverse=True)[:2]
        print(f"{d['_file'][:16]:16s}:{d['Line No']:>4s} inst {f(d['Instructions Executed'])/ti*100:5.1f}% samp {f(d['Warp Stall Sampling (All Samples)'])/ts*100:5.1f}% thr {d['Avg. Threads Executed']:>3s} {[(s, round(v/ts*100,1)) for v, s in st]} | {d['Source'].strip()[:70]}")
