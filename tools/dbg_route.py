"""debug: route_combine owners vs partition owners vs a Python re-statement of the route hash; timing of C5z steps"""
import sys, time, json
sys.path.insert(0, '.')
import numpy as np, torch
import gen, oracle
from paper_conf_ipps_mokhtaris17_b200 import shard
import paper_conf_ipps_mokhtaris17_b200 as sepo
M = (1 << 64) - 1
def fmix(k):
    k ^= k >> 33; k = (k * 0xff51afd7ed558ccd) & M; k ^= k >> 33; k = (k * 0xc4ceb9fe1a85ec53) & M; k ^= k >> 33; return k
def hw(h, w): return ((h ^ w) * 0x9e3779b97f4a7c15) & M
def h16(key, seed):
    L = len(key); b = key.ljust(16, b"\0")
    w0 = int.from_bytes(b[:8], "little"); w1 = int.from_bytes(b[8:16], "little")
    x = seed ^ ((L * 0x87c37b91114253d5) & M)
    return fmix(hw(hw(x, w0), w1))
P = 4
s = gen.config("C2", scale=1 / 1024)
k, o, v = s.device()
wire, counts = shard.route_combine(k, o, None, P, route_seed=5)
a = wire.cpu().numpy().view(np.uint64).reshape(-1, 4)
bad = 0
for p in range(P):
    for w0, w1, val, ln in a[int(counts[p]):int(counts[p + 1])][:2000]:
        key = (int(w0).to_bytes(8, "little") + int(w1).to_bytes(8, "little"))[:int(ln)]
        own = ((h16(key, 5) >> 32) * P) >> 32
        if own != p:
            bad += 1
            if bad < 5: print("combine part", p, "key", key, "py owner", own)
ok, oko, _, starts = shard.partition(k, o, None, P, route_seed=5)
kb = ok.cpu().numpy().tobytes(); ko = oko.cpu().numpy()
bad2 = 0
for p in range(P):
    r0, r1 = int(starts[p][0]), int(starts[p + 1][0]); b0 = int(starts[p][1])
    for j in range(r0, min(r1, r0 + 2000)):
        e = int(ko[j + 1]) if j + 1 < r1 else int(starts[p + 1][1]) - b0
        key = kb[b0 + int(ko[j]): b0 + e]
        own = ((h16(key, 5) >> 32) * P) >> 32
        if own != p:
            bad2 += 1
            if bad2 < 5: print("partition part", p, "key", key, "py owner", own)
print(json.dumps({"combine_bad": bad, "partition_bad": bad2, "counts": counts.tolist()}))
# C5z timing breakdown
s = gen.config("C5z", scale=0.125)
k, _, v = s.device()
torch.cuda.synchronize(); t0 = time.perf_counter()
wire, counts = shard.route_combine(k, None, v, 1, route_seed=9, fixed_key_width=8, fixed_val_width=8)
torch.cuda.synchronize(); t1 = time.perf_counter()
print(json.dumps({"c5z_route_ms": (t1 - t0) * 1e3, "n_out": int(counts[-1])}), flush=True)
t = sepo.Table(sepo.budget_for(1 << 22, 16384, 8192), 1 << 22, 16384)
torch.cuda.synchronize(); t0 = time.perf_counter()
p = t.run_wire(wire)
torch.cuda.synchronize(); t1 = time.perf_counter()
st = t.stats()
print(json.dumps({"c5z_run_wire_ms": (t1 - t0) * 1e3, "passes": p, "ins": st["t_insert_ms_per_pass"][:p], "evict": st["t_evict_ms"], "hot": st["hot_keys"]}), flush=True)
