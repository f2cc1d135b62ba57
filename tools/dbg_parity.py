import sys; sys.path.insert(0, '.')
import numpy as np, torch, gen
import paper_conf_ipps_mokhtaris17_b200 as sepo
from tests.util import oracle_expected, device_inputs
s = gen.config("C1", scale=0.2)
exp = oracle_expected(s)
inp = device_inputs(s)
for pb, nb, grid, pages in [(65536, 3, 296, 128), (65536, 3, 148, 128), (65536, 1024, 296, 128), (65536, 3, 296, 4096), (65536, 1 << 16, 148, 16)]:
    t = sepo.Table(sepo.budget_for(nb, pb, pages), nb, pb, grid_ctas=grid, hash_seed=3, check_dups=True)
    passes = t.run(*inp)
    got = sepo.result_dict(t.export())
    st = t.stats()
    missing = [k for k in exp if k not in got]
    wrong = [k for k in exp if k in got and got[k] != exp[k]]
    extra = [k for k in got if k not in exp]
    print(pb, nb, grid, pages, "passes", passes, "keys", len(got), len(exp), "missing", len(missing), "wrong", len(wrong), "extra", len(extra),
          "sum", sum(got.values()), sum(exp.values()), "dead", st["dead_bytes"], "post", st["postponed_per_pass"][:6], "dups", st["cross_gen_dups"])
    if wrong[:3]: print("  wrong", [(k, got[k], exp[k]) for k in wrong[:3]])
    t.close()
