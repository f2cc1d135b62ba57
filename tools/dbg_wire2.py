import sys, time, json, os
sys.path.insert(0, '.')
import torch, gen
from paper_conf_ipps_mokhtaris17_b200 import shard
import paper_conf_ipps_mokhtaris17_b200 as sepo
s = gen.config("C5z", scale=0.125)
k, _, v = s.device()
wire, counts = shard.route_combine(k, None, v, 1, route_seed=9, fixed_key_width=8, fixed_val_width=8)
def rep(name, fn):
    t = sepo.Table(sepo.budget_for(1 << 20, 16384, 1344), 1 << 20, 16384, fixed_key_width=8, fixed_val_width=8)
    torch.cuda.synchronize(); t0 = time.perf_counter()
    p = fn(t)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    st = t.stats()
    print(json.dumps({"case": name, "ms": (t1 - t0) * 1e3, "passes": p, "ins": [round(x, 2) for x in st["t_insert_ms_per_pass"][:p]],
                      "post": st["postponed_per_pass"][:p], "dead": st["dead_bytes"], "recs": st["records_inserted"]}), flush=True)
    t.close()
rep("csr", lambda t: t.run(k, None, v))
rep("wire", lambda t: t.run_wire(wire))
# the wire records as CSR-less fixed keys: keys = w0 column, values = v column
import numpy as np
a = wire.view(torch.int64).reshape(-1, 4)
k2 = a[:, 0].contiguous().view(torch.uint8)
v2 = a[:, 2].contiguous().view(torch.uint8)
rep("wire_as_fixed", lambda t: t.run(k2, None, v2))
