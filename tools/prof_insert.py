"""Profiling driver: one in-budget C2 job at a given scale (insert kernel dominant)."""
import sys; sys.path.insert(0, '.')
import torch, bench
scale = float(sys.argv[1]) if len(sys.argv) > 1 else 0.125
ratio = float(sys.argv[2]) if len(sys.argv) > 2 else 0.5
job = bench.Job("C2", ratio, scale=scale)
t = job.table()
k, o, v = job.inputs()
for _ in range(2):
    t.reset(); t.run(k, o, v)
torch.cuda.synchronize()
print(t.stats())
