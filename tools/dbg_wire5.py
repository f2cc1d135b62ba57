import sys, time, json
sys.path.insert(0, '.')
import torch, gen, numpy as np
from paper_conf_ipps_mokhtaris17_b200 import shard
import paper_conf_ipps_mokhtaris17_b200 as sepo
from tests.util import oracle_expected
s = gen.config("C5z", scale=1 / 256)
exp = oracle_expected(s)
k, _, v = s.device()
wire, counts = shard.route_combine(k, None, v, 1, route_seed=9, fixed_key_width=8, fixed_val_width=8)
a = wire.cpu().numpy().view(np.uint64).reshape(-1, 4)
print("wire recs", len(a), "lens", np.unique(a[:, 3], return_counts=True), "w1 nonzero", int((a[:, 1] != 0).sum()), flush=True)
t = sepo.Table(sepo.budget_for(1 << 16, 16384, 80), 1 << 16, 16384, fixed_key_width=8, fixed_val_width=8)
t0 = time.perf_counter(); p = t.run_wire(wire); t1 = time.perf_counter()
res = t.export()
st = t.stats()
ko = res["key_offsets"]; kb = res["keys"].tobytes()
keys = [kb[ko[i]:ko[i + 1]] for i in range(res["n_keys"])]
print("passes", p, "ms", (t1 - t0) * 1e3, "n_keys", res["n_keys"], "distinct", len(set(keys)), "expected", len(exp), "post", st["postponed_per_pass"][:p], flush=True)
got = {}
for key, val in zip(keys, res["values"].tolist()):
    got.setdefault(key, []).append(val)
dups = {kk: vv for kk, vv in got.items() if len(vv) > 1}
print("dup keys", len(dups), list(dups.items())[:3])
bad = [kk for kk in exp if sum(got.get(kk, [0])) % (1 << 64) != exp[kk]]
print("bad sums", len(bad))
