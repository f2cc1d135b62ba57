"""Round-2 paths at small sizes with forced options (compute-sanitizer is closed on this GPU pool, so this
runs them plainly and checks parity): the hot-key router (hot set forced on a small batch), the CSR
partition's aligned key copy, sepo_compact on URL keys, GROUP with the overlapped gather eviction, and
sepo_run_sharded on a one-rank NCCL communicator (peer-memory window and CSR).
Exits non-zero on a parity failure."""
import os
import sys
sys.path.insert(0, '.')
os.environ["SEPO_HOT_MIN"] = "20000"      # the hot set on these small batches
os.environ["SEPO_EVICT_OVERLAP"] = "1"    # overlapped evictions (gather with per-warp progress for GROUP)
os.environ["SEPO_SHARD_CHUNK"] = "16384"  # several chunks
import numpy as np
import gen
import oracle
import paper_conf_ipps_mokhtaris17_b200 as sepo
from paper_conf_ipps_mokhtaris17_b200 import shard
from tests.util import oracle_expected

s = gen.config("C5z", scale=2 ** -14)
k, _, v = s.device()
wire, counts = shard.route_combine(k, None, v, 3, route_seed=7, fixed_key_width=8, fixed_val_width=8)
print("route_combine ok", int(counts[-1]), "of", s.n)

s = gen.config("C3", scale=1e-5)
k, o, _ = s.device()
ok_, oko, _, st = shard.partition(k, o, None, 3, route_seed=5)
print("partition ok", st[-1].tolist())
t = sepo.Table(sepo.budget_for(1 << 10, 65536, 4), 1 << 10, 65536)
c, bm = t.insert_batch(k, o, n=s.n)
rem, kb, _ = t.reprobe(k, o, None, bm, n=s.n)
if rem:
    okk, okko, _, m = t.compact(k, o, None, bm, n=s.n)
    hk, ho, _ = s.host()
    ek, eo, _, _, em = oracle.compact(hk, np.asarray(ho).view(np.uint64), bm.cpu().numpy().view(np.uint32))
    assert okk.cpu().numpy().tobytes() == ek.tobytes(), "compact parity"
print("compact ok", rem)
t.close()

s = gen.config("C4", scale=2e-5)
k, o, v = s.device()
t = sepo.Table(sepo.budget_for(1 << 12, 4096, 24), 1 << 12, 4096, mode=sepo.GROUP, fixed_val_width=4, check_dups=True)
p = t.run(k, o, v)
assert sepo.result_dict(t.export(), sepo.GROUP) == oracle_expected(s), "group parity"
print("group (overlapped gather) ok, passes", p)
t.close()

for name, scale in (("C1", 0.02), ("C3", 1e-5)):
    s = gen.config(name, scale=scale)
    k, o, _ = s.device()
    pb = 65536 if name == "C3" else 4096
    t = sepo.Table(sepo.budget_for(1 << 12, pb, 8), 1 << 12, pb, check_dups=True)
    t.attach_nccl(sepo.nccl_unique_id(), 1, 0)
    p = t.run_sharded(k, o)
    st = t.stats()
    assert sepo.result_dict(t.export()) == oracle_expected(s), "sharded parity " + name
    print("run_sharded ok", name, "passes", p, "p2p chunks", st["p2p_chunks"])
    t.close()
