"""Top CUDA source lines of an ncu report by executed instructions / stall samples, with the
local source text: python tools/ncu_srclines.py report.ncu-rep [groups] [N]"""
import csv, io, subprocess, sys, os
rep = sys.argv[1]
G = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
N = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = {}
for fn in ["paper_conf_ipps_mokhtaris17_b200/csrc/sepo_kernels.cu", "paper_conf_ipps_mokhtaris17_b200/csrc/sepo_dev.cuh"]:
    src[os.path.basename(fn)] = open(os.path.join(os.environ.get("SRC_DIR", ""), os.path.basename(fn)) if os.environ.get("SRC_DIR") else os.path.join(ROOT, fn)).read().split('\n')
fname = hdr = None
lines = []
for r in rows:
    if len(r) >= 2 and r[0] in ("File Path", "File Name"):
        fname = os.path.basename(r[1])
    elif r and r[0] == "Line No":
        hdr = r
    elif hdr and r and len(r) == len(hdr) and r[0].isdigit():
        d = dict(zip(hdr, r)); d['_f'] = fname; lines.append(d)
f = lambda x: float(x) if x.replace('.', '', 1).isdigit() else 0.0
ik = "Instructions Executed"; sk = "Warp Stall Sampling (All Samples)"
ts = sum(f(d.get(sk, '0')) for d in lines) or 1
for key in (ik, sk):
    print("=== top by", key)
    top = sorted(lines, key=lambda d: -f(d.get(key, '0')))[:N]
    for d in sorted(top, key=lambda d: (d['_f'], int(d['Line No']))):
        ln = int(d['Line No']); fn = d['_f']
        t = src[fn][ln - 1].strip()[:78] if fn in src and ln - 1 < len(src[fn]) else '?'
        print(f"{fn[:14]:14s}:{ln:5d} {f(d.get(ik,'0'))/G:6.1f}/grp samp {100*f(d.get(sk,'0'))/ts:4.1f}%  {t}")
