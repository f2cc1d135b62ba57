"""Summarise one-kernel ncu --set full captures into the traffic JSON bench.py reads:
  python tools/ncu_extract.py REPORT.ncu-rep OUT.json "launch description" ALG_BYTES"""
import csv, io, json, subprocess, sys
rep, out, desc, alg = sys.argv[1], sys.argv[2], sys.argv[3], int(float(sys.argv[4]))
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, u, v = rows[0], rows[1], rows[2]
def get(name, scale=1.0):
    i = h.index(name)
    x = float(v[i].replace(",", ""))
    unit = u[i]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "msecond": 1, "usecond": 1e-3, "nsecond": 1e-6,
            "ms": 1, "us": 1e-3, "ns": 1e-6}.get(unit, 1)
    return x * mult
d = {"kernel": v[h.index("Kernel Name")][:120], "launch": desc,
     "dram_read_bytes": int(get("dram__bytes_read.sum")), "dram_write_bytes": int(get("dram__bytes_write.sum")),
     "alg_bytes": alg, "duration_ms_cold": get("gpu__time_duration.sum"),
     "warp_instructions": int(get("smsp__inst_executed.sum")),
     "issue_active_pct": get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
     "l2_hit_pct": get("lts__t_sector_hit_rate.pct")}
d["traffic_over_alg"] = (d["dram_read_bytes"] + d["dram_write_bytes"]) / alg
json.dump(d, open(out, "w"), indent=1)
print(json.dumps(d))
