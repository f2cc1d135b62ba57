"""GPU parity of the basic organization: every pair
is its own entry; a pass halts once basic_halt_pct % of the allocator slots (the paper's bucket
groups) failed, the heap is evicted and the job restarts from the postponed records. Result = the
oracle's multiset of pairs exactly, in and over budget, for halt thresholds 50 % (the paper's) and
100 %, with values implicit (Word Count) or u64 (pairs), and under allocation fault injection."""
import numpy as np
import pytest

import gen
import oracle
from tests.util import device_inputs, run_job

pytestmark = pytest.mark.gpu


def expected_basic(s):
    k, o, v = s.host()
    return oracle.basic(k, o, v, 8) if s.val == "u64" else oracle.basic(k, o)


def kw(s, **extra):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    d = dict(mode=sepo.BASIC)
    if s.val == "u64":
        d.update(fixed_key_width=8, fixed_val_width=8)
    d.update(extra)
    return d


def basic_footprint(s, inp, nb, pb):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    _, passes, st = run_job(s, sepo.budget_for(nb, pb, 1 << 14), nb, pb, inputs=inp, **kw(s))
    assert passes == 1
    return st["pages_used_max"]


@pytest.mark.parametrize("cfg", ["C1", "C5z"])
@pytest.mark.parametrize("ratio,halt", [(0.5, 50), (2, 50), (4, 50), (4, 100)])
def test_basic_parity(cuda, cfg, ratio, halt):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    s = gen.config(cfg, scale=0.1 if cfg == "C1" else 2e-4)
    inp = device_inputs(s)
    exp = expected_basic(s)
    nb, pb = 1 << 14, 4096
    F = basic_footprint(s, inp, nb, pb)
    pages = int(np.ceil(F / ratio)) + (2 * 148 if ratio < 1 else 0)
    got, passes, st = run_job(s, sepo.budget_for(nb, pb, max(8, pages)), nb, pb, inputs=inp,
                              **kw(s, basic_halt_pct=halt))
    assert got == exp
    assert sum(len(v) for v in got.values()) == s.n
    if ratio > 1:
        assert passes >= 2
        post = st["postponed_per_pass"]
        assert all(post[i] > post[i + 1] for i in range(len(post) - 1)) and post[-1] == 0, post


def test_basic_fault_injection(cuda):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    s = gen.config("C1", scale=0.05)
    inp = device_inputs(s)
    exp = expected_basic(s)
    got, passes, st = run_job(s, sepo.budget_for(1 << 14, 4096, 4096), 1 << 14, 4096, inputs=inp,
                              **kw(s, fail_alloc_ppm=200000, fail_mode=1, fail_until_pass=3))
    assert got == exp and passes >= 3


def test_basic_insert_batch_api(cuda):
    """the fine-grained API: insert_batch returns the postponed count; the bitmap marks exactly the
    records not stored (stored pairs + postponed pairs = the input multiset)"""
    import torch
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    s = gen.config("C1", scale=0.05)
    k, o, _ = device_inputs(s)
    exp = expected_basic(s)
    F = basic_footprint(s, (k, o, None), 1 << 14, 4096)
    t = sepo.Table(sepo.budget_for(1 << 14, 4096, max(8, F // 3)), 1 << 14, 4096, **kw(s))
    bm = torch.zeros((s.n + 31) // 32, dtype=torch.int32, device="cuda")
    c, _ = t.insert_batch(k, o, None, bitmap=bm)
    assert 0 < c < s.n
    bits = np.unpackbits(bm.cpu().numpy().view(np.uint8), bitorder="little")[: s.n]
    assert int(bits.sum()) == c
    got = sepo.result_dict(t.export(), sepo.BASIC)
    t.close()
    hk, ho, _ = s.host()
    post = oracle.basic(*oracle.compact(hk, ho, bm.cpu().numpy().view(np.uint32))[:2])
    merged = {kk: sorted(got.get(kk, []) + post.get(kk, [])) for kk in set(got) | set(post)}
    assert merged == exp
