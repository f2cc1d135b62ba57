"""GPU parity of SEPO lookups on the larger-than-memory table (sepo_lookup; SURVEY §8(f) NEXT-4;
P:L147): after a multi-generation COMBINE job, every key of the oracle's result is found with
exactly the oracle's value, absent keys are not found, whatever generation a key was evicted in;
lookups work before and after export, and inserts are refused until sepo_reset."""
import numpy as np
import pytest
import torch

import gen
import oracle
from tests.util import device_inputs, footprint_pages

pytestmark = pytest.mark.gpu


def sepo():
    import paper_conf_ipps_mokhtaris17_b200 as m
    return m


def csr_device(keys):
    offs = np.cumsum([0] + [len(k) for k in keys]).astype(np.int64)
    kb = b"".join(keys)
    kt = torch.empty(max(len(kb), 1) + 16, dtype=torch.uint8, device="cuda")
    if kb:
        kt[:len(kb)].copy_(torch.frombuffer(bytearray(kb), dtype=torch.uint8))
    return kt, torch.from_numpy(offs).cuda()


@pytest.mark.parametrize("cfg,ratio", [("C1", 1), ("C1", 4), ("C5z", 4)])
def test_lookup_parity(cuda, cfg, ratio):
    S = sepo()
    s = gen.config(cfg, scale=0.25 if cfg == "C1" else 1e-4)
    k, o, v = device_inputs(s)
    hk, ho, hv = s.host()
    exp = oracle.combine(hk, ho, hv, 8).as_dict() if s.val == "u64" else oracle.combine(hk, ho).as_dict()
    kw = dict(fixed_key_width=8, fixed_val_width=8) if s.val == "u64" else {}
    F = footprint_pages(s, 1 << 14, 4096, inputs=(k, o, v), **kw)
    P = F + 600 if ratio == 1 else max(8, F // ratio)
    t = S.Table(S.budget_for(1 << 14, 4096, P), 1 << 14, 4096, **kw)
    passes = t.run(k, o, v)
    assert passes >= (1 if ratio == 1 else 2)
    present = sorted(exp)
    rng = np.random.default_rng(3)
    absent = [b"\x00absent%d" % i for i in range(500)] + [b""]
    if s.val == "u64":
        absent = [int(x).to_bytes(8, "little") for x in rng.integers(1, 2**63, 500)]
        absent = [a for a in absent if a not in exp]
    queries = present + absent
    order = rng.permutation(len(queries))
    queries = [queries[i] for i in order]
    if s.val == "u64":
        qk = torch.from_numpy(np.frombuffer(b"".join(queries), dtype=np.uint8).copy()).cuda()
        found, vals, bm = t.lookup(qk, None, n=len(queries))
    else:
        qk, qo = csr_device(queries)
        found, vals, bm = t.lookup(qk, qo)
    assert found == len(present)
    vals = vals.cpu().numpy().view(np.uint64)
    bits = np.unpackbits(bm.cpu().numpy().view(np.uint8), bitorder="little")[: len(queries)]
    for i, q in enumerate(queries):
        if q in exp:
            assert bits[i] == 1 and int(vals[i]) == exp[q], q
        else:
            assert bits[i] == 0 and int(vals[i]) == 0, q
    # export after the lookups still returns the whole table; inserts are refused until reset
    got = S.result_dict(t.export())
    assert got == exp
    with pytest.raises(S.SepoError):
        t.run(k, o, v)
    t.reset()
    assert t.run(k, o, v) >= 1
    t.close()


def test_lookup_empty_table(cuda):
    S = sepo()
    t = S.Table(S.budget_for(1 << 10, 4096, 64), 1 << 10, 4096)
    qk, qo = csr_device([b"a", b"bb"])
    found, vals, bm = t.lookup(qk, qo)
    assert found == 0 and int(bm[0].item()) == 0
    t.close()
