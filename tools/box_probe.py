"""Box measurement: host cores/RAM, device props, pinned host-link
bandwidth, read-only HBM bandwidth. Writes gpurun_out/box_probe.json. Test/bench tooling."""
import json, os, subprocess, time
import torch

out = {}
out["nproc"] = os.cpu_count()
try:
    out["sched_affinity"] = len(os.sched_getaffinity(0))
except Exception:
    pass
try:
    out["lscpu_model"] = [l for l in subprocess.check_output(["lscpu"], text=True).splitlines() if "Model name" in l]
except Exception as e:
    out["lscpu_model"] = str(e)
with open("/proc/meminfo") as f:
    out["meminfo"] = [l.strip() for l in f.readlines()[:3]]
p = torch.cuda.get_device_properties(0)
out["device"] = {"name": p.name, "sms": p.multi_processor_count, "total_mem": p.total_memory,
                 "l2": getattr(p, "L2_cache_size", None), "cc": [p.major, p.minor]}
out["n_gpus"] = torch.cuda.device_count()

def ev_time(fn, reps=10):
    best = 1e9
    for _ in range(reps):
        s = torch.cuda.Event(enable_timing=True); e = torch.cuda.Event(enable_timing=True)
        s.record(); fn(); e.record(); torch.cuda.synchronize()
        best = min(best, s.elapsed_time(e) / 1e3)
    return best

nb = 1 << 30
h = torch.empty(nb, dtype=torch.uint8, pin_memory=True)
d = torch.empty(nb, dtype=torch.uint8, device="cuda")
h.fill_(1)
t = ev_time(lambda: d.copy_(h, non_blocking=True)); out["h2d_GBps"] = nb / t / 1e9
t = ev_time(lambda: h.copy_(d, non_blocking=True)); out["d2h_GBps"] = nb / t / 1e9
t0 = time.time(); hh = torch.empty(nb, dtype=torch.uint8, pin_memory=True); out["pin_alloc_1GiB_s"] = time.time() - t0
x = torch.empty(4 << 30, dtype=torch.uint8, device="cuda").view(torch.int64)
x.fill_(1)
t = ev_time(lambda: x.sum()); out["read_sum_GBps"] = x.numel() * 8 / t / 1e9
y = torch.empty_like(x)
t = ev_time(lambda: y.copy_(x)); out["copy_GBps_rw"] = 2 * x.numel() * 8 / t / 1e9
try:
    out["topo"] = subprocess.check_output(["nvidia-smi", "topo", "-m"], text=True)
except Exception as e:
    out["topo"] = str(e)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(out, open("gpurun_out/box_probe.json", "w"), indent=1)
print(json.dumps({k: v for k, v in out.items() if k != "topo"}, indent=1))
