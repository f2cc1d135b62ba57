import sys, time, json, os
sys.path.insert(0, '.')
import torch, gen
from paper_conf_ipps_mokhtaris17_b200 import shard
import paper_conf_ipps_mokhtaris17_b200 as sepo
s = gen.config("C5z", scale=1 / 32)
k, _, v = s.device()
wire, counts = shard.route_combine(k, None, v, 1, route_seed=9, fixed_key_width=8, fixed_val_width=8)
t = sepo.Table(sepo.budget_for(1 << 18, 16384, 336), 1 << 18, 16384, fixed_key_width=8, fixed_val_width=8)
torch.cuda.synchronize(); t0 = time.perf_counter()
p = t.run_wire(wire)
torch.cuda.synchronize(); t1 = time.perf_counter()
st = t.stats()
print(json.dumps({"ms": (t1 - t0) * 1e3, "passes": p, "ins": [round(x, 2) for x in st["t_insert_ms_per_pass"][:p]], "post": st["postponed_per_pass"][:p]}), flush=True)
