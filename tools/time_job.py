"""Time one SEPO job configuration (no ncu): python tools/time_job.py CFG RATIO [SCALE] -> phase times"""
import sys, json; sys.path.insert(0, '.')
import torch, bench
cfg = sys.argv[1]; ratio = float(sys.argv[2]); scale = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
job = bench.Job(cfg, ratio, scale=scale)
t = job.table()
k, o, v = job.inputs()
for _ in range(2):
    t.reset(); t.run(k, o, v)
torch.cuda.synchronize()
ms, info = bench.timed_steps(job, t, 3, torch.cuda.current_stream())
st = info["last"]
print(json.dumps({"cfg": cfg, "ratio": ratio, "ms_per_job": ms / 3, "passes": st["passes"],
                  "insert_ms": st["t_insert_ms"], "reprobe_ms": st["t_reprobe_ms"], "compact_ms": st["t_compact_ms"],
                  "evict_ms": st["t_evict_ms"], "post": st["postponed_per_pass"],
                  "insert_ms_per_pass": [round(x, 3) for x in st["t_insert_ms_per_pass"]], "p1_ms": info["p1_ms"] / 3}))
