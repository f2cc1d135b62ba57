"""Small SEPO jobs for compute-sanitizer: COMBINE (C1, 2x over budget, words) and GROUP (C4 small,
3x over), plus the router. Exits non-zero on a parity failure."""
import sys; sys.path.insert(0, '.')
import gen, oracle
import paper_conf_ipps_mokhtaris17_b200 as sepo
from paper_conf_ipps_mokhtaris17_b200 import shard
from tests.util import oracle_expected

s = gen.config("C1", scale=0.05)
k, o, _ = s.device()
t = sepo.Table(sepo.budget_for(1 << 12, 4096, 16), 1 << 12, 4096, check_dups=True)
p = t.run(k, o)
assert sepo.result_dict(t.export()) == oracle_expected(s), "combine parity"
print("combine ok, passes", p)
t.close()
s = gen.config("C4", scale=2e-5)
k, o, v = s.device()
t = sepo.Table(sepo.budget_for(1 << 12, 4096, 24), 1 << 12, 4096, mode=sepo.GROUP, fixed_val_width=4, check_dups=True)
p = t.run(k, o, v)
assert sepo.result_dict(t.export(), sepo.GROUP) == oracle_expected(s), "group parity"
print("group ok, passes", p)
t.close()
s = gen.config("C3", scale=1e-5)
k, o, _ = s.device()
ok_, oko, _, st = shard.partition(k, o, None, 3, route_seed=5)
print("partition ok", st[-1].tolist())
