"""GPU checks of the key-hash router (row a12) on one device: the partition kernel's properties
and a P-way sharded SEPO job run as P loopback "ranks" (one table each) against the oracle."""
import numpy as np
import pytest
import torch

import gen
import oracle
from tests.util import oracle_expected

pytestmark = pytest.mark.gpu


def sepo():
    import paper_conf_ipps_mokhtaris17_b200 as m
    return m


def segment(ok, oko, starts, p):
    r0, r1 = int(starts[p][0]), int(starts[p + 1][0])
    b0, b1 = int(starts[p][1]), int(starts[p + 1][1])
    ko = torch.empty(r1 - r0 + 1, dtype=torch.int64, device=ok.device)
    ko[:-1] = oko[r0:r1]
    ko[-1] = b1 - b0
    return ok[b0:b1], ko


@pytest.mark.parametrize("P", [1, 2, 5, 8])
def test_partition_properties(cuda, P):
    from paper_conf_ipps_mokhtaris17_b200 import shard
    s = gen.config("C3", scale=1 / 4000)
    k, o, _ = s.device()
    ok, oko, _, starts = shard.partition(k, o, None, P, route_seed=7)
    assert int(starts[P][0]) == s.n and int(starts[P][1]) == k.numel()
    keysets, all_counts = [], oracle.Combine()
    for p in range(P):
        sk, so = segment(ok, oko, starts, p)
        # purity: partitioning a part again keeps every record in the same part
        _, _, _, st2 = shard.partition(sk, so, None, P, route_seed=7)
        n_p = so.numel() - 1
        assert int(st2[p + 1][0] - st2[p][0]) == n_p
        hk, ho = sk.cpu().numpy(), so.cpu().numpy().view(np.uint64)
        d = oracle.combine(hk, ho).as_dict()
        keysets.append(set(d))
        all_counts.add(hk, ho)
    # disjoint key sets, and the records are a permutation of the input
    for a in range(P):
        for b in range(a + 1, P):
            assert not (keysets[a] & keysets[b])
    assert all_counts.as_dict() == oracle_expected(s)


def test_partition_carries_values(cuda):
    """fixed-width keys with values: every (key, value) pair of the input appears exactly once, in the
    part of its key's owner (the order within a part is unspecified)"""
    from paper_conf_ipps_mokhtaris17_b200 import shard
    s = gen.config("C5u", scale=2 ** -14)  # fixed 8-byte keys, 8-byte values
    k, _, v = s.device()
    P = 4
    ok, oko, ov, starts = shard.partition(k, None, v, P, route_seed=3, fixed_key_width=8, fixed_val_width=8)
    assert oko is None
    pairs_in = sorted(zip(k.cpu().numpy().view(np.uint64).tolist(), v.cpu().numpy().view(np.uint64).tolist()))
    pk = ok.cpu().numpy().view(np.uint64)
    pv = ov.cpu().numpy().view(np.uint64)
    assert sorted(zip(pk.tolist(), pv.tolist())) == pairs_in
    owner = {}
    for p in range(P):
        for x in range(int(starts[p][0]), int(starts[p + 1][0])):
            assert owner.setdefault(int(pk[x]), p) == p  # a key lives in one part only


@pytest.mark.parametrize("name,P", [("C3", 4), ("C5z", 3), ("C2", 8)])
def test_sharded_job_loopback(cuda, name, P):
    """P loopback ranks: partition, one SEPO table per part (budget 2x over), union == oracle."""
    from paper_conf_ipps_mokhtaris17_b200 import shard
    scale = {"C3": 1 / 4000, "C5z": 2 ** -12, "C2": 1 / 512}[name]
    s = gen.config(name, scale=scale)
    exp = oracle_expected(s)
    k, o, v = s.device()
    fixed = s.family == gen.GEN_PAIRS
    ok, oko, ov, starts = shard.partition(k, None if fixed else o, v, P, route_seed=11,
                                          fixed_key_width=8 if fixed else 0, fixed_val_width=8 if v is not None else 0)
    got = {}
    for p in range(P):
        r0, r1 = int(starts[p][0]), int(starts[p + 1][0])
        kw = dict(mode=sepo().COMBINE)
        if fixed:
            sk, so = ok[int(starts[p][1]):int(starts[p + 1][1])], None
            sv = ov[int(starts[p][2]):int(starts[p + 1][2])]
            kw.update(fixed_key_width=8, fixed_val_width=8)
        else:
            sk, so = segment(ok, oko, starts, p)
            sv = None
        t = sepo().Table(sepo().budget_for(1 << 14, 16384, 64), 1 << 14, 16384, check_dups=True, **kw)
        t.run(sk, so, sv, n=r1 - r0)
        part = sepo().result_dict(t.export())
        assert t.stats()["cross_gen_dups"] == 0
        t.close()
        assert not (set(part) & set(got))  # shards own disjoint keys
        got.update(part)
    assert got == exp


# ---- router with hot-key pre-combine (sepo_route_combine) + wire records
def top_key(s, exp):
    """the most frequent key of a stream (pairs: by record count; words: the counts are the values)"""
    if s.family != gen.GEN_PAIRS:
        return max(exp, key=lambda x: exp[x])
    keys, _, _ = s.host()
    u, c = np.unique(np.asarray(keys).view(np.uint64), return_counts=True)
    return int(u[np.argmax(c)]).to_bytes(8, "little")


def wire_count(wire, key):
    """records of `key` among 32-byte wire records"""
    a = wire.cpu().numpy().view(np.uint64).reshape(-1, 4)
    kb = key + bytes(16 - len(key))
    w0, w1 = int.from_bytes(kb[:8], "little"), int.from_bytes(kb[8:], "little")
    return int(((a[:, 0] == w0) & (a[:, 1] == w1) & (a[:, 3] == len(key))).sum())


def wire_dict(wire):
    """32-byte wire records -> {key bytes: summed value} (test-side decode; records of one key may repeat)"""
    a = wire.cpu().numpy().view(np.uint64).reshape(-1, 4)
    out = {}
    for w0, w1, v, ln in a:
        key = (int(w0).to_bytes(8, "little") + int(w1).to_bytes(8, "little"))[: int(ln)]
        out[key] = (out.get(key, 0) + int(v)) % (1 << 64)
    return out


@pytest.mark.parametrize("name,P,hot_min", [("C2", 1, None), ("C2", 4, None), ("C5z", 3, None), ("C5u", 2, None),
                                             ("C2", 4, 1 << 16), ("C5z", 8, 1 << 16)])
def test_route_combine_parts(cuda, monkeypatch, name, P, hot_min):
    """every part's pre-combined records sum to the oracle's values of exactly the keys it owns, the
    parts own disjoint key sets, and each hot key left the batch as ONE record (Zipf: far fewer records
    than the batch; the hot set runs from SEPO_HOT_MIN records, 2^21 by default)"""
    from paper_conf_ipps_mokhtaris17_b200 import shard
    if hot_min:
        monkeypatch.setenv("SEPO_HOT_MIN", str(hot_min))
    scale = {"C2": 1 / 1024, "C5z": 2 ** -12, "C5u": 2 ** -14}[name]
    s = gen.config(name, scale=scale)
    exp = oracle_expected(s)
    k, o, v = s.device()
    fixed = s.family == gen.GEN_PAIRS
    wire, counts = shard.route_combine(k, None if fixed else o, v, P, route_seed=5, fixed_key_width=8 if fixed else 0,
                                       fixed_val_width=8 if v is not None else 0)
    assert counts[0] == 0 and int(counts[-1]) == wire.numel() // 32
    got, owners = {}, []
    for p in range(P):
        part = wire_dict(wire[int(counts[p]) * 32:int(counts[p + 1]) * 32])
        owners.append(set(part))
        for key, val in part.items():
            got[key] = (got.get(key, 0) + val) % (1 << 64)
    for a in range(P):
        for b in range(a + 1, P):
            assert not (owners[a] & owners[b])
    assert got == exp
    if hot_min:  # Zipf: the hot keys leave the batch once
        assert int(counts[-1]) < 0.7 * s.n
        top = top_key(s, exp)  # the batch's most frequent key is hot: exactly one record
        assert wire_count(wire[:int(counts[-1]) * 32], top) == 1
    # the owners agree with the CSR partition's (same route hash)
    if P > 1 and not fixed:
        ok, oko, _, starts = shard.partition(k, o, None, P, route_seed=5)
        for p in range(P):
            sk, so = segment(ok, oko, starts, p)
            keys_p = set(oracle.combine(sk.cpu().numpy(), so.cpu().numpy().view(np.uint64)).as_dict())
            assert keys_p == owners[p]


def test_route_hot_set_active_large(cuda):
    """a C5z batch above the hot-set threshold (2^21 records): the top keys leave once, the parts still sum
    to the oracle"""
    from paper_conf_ipps_mokhtaris17_b200 import shard
    s = gen.config("C5z", scale=2 ** -9)
    assert s.n >= (1 << 21)
    exp = oracle_expected(s)
    k, _, v = s.device()
    wire, counts = shard.route_combine(k, None, v, 4, route_seed=9, fixed_key_width=8, fixed_val_width=8)
    got = {}
    for p in range(4):
        for key, val in wire_dict(wire[int(counts[p]) * 32:int(counts[p + 1]) * 32]).items():
            got[key] = (got.get(key, 0) + val) % (1 << 64)
    assert got == exp
    assert int(counts[-1]) < 0.5 * s.n
    top = top_key(s, exp)
    assert wire_count(wire[:int(counts[-1]) * 32], top) == 1


def test_route_combine_rejects_long_keys(cuda):
    from paper_conf_ipps_mokhtaris17_b200 import shard
    s = gen.config("C3", scale=1 / 8000)  # URLs: longer than 16 bytes
    k, o, _ = s.device()
    assert shard.route_combine(k, o, None, 2, route_seed=1) is None


@pytest.mark.parametrize("name,ratio", [("C5z", 4), ("C2", 4), ("C2", 0.5)])
def test_run_wire_vs_oracle(cuda, name, ratio):
    """the SEPO job on routed (pre-combined) wire records, one rank (loopback), in and over budget:
    == the oracle on the original records (hot set active at these sizes)"""
    from paper_conf_ipps_mokhtaris17_b200 import shard
    scale = {"C2": 1 / 256, "C5z": 1 / 128}[name]
    s = gen.config(name, scale=scale)
    exp = oracle_expected(s)
    k, o, v = s.device()
    fixed = s.family == gen.GEN_PAIRS
    wire, counts = shard.route_combine(k, None if fixed else o, v, 1, route_seed=9, fixed_key_width=8 if fixed else 0,
                                       fixed_val_width=8 if v is not None else 0)
    n = wire.numel() // 32
    assert n >= 2_097_152 or name == "C2"
    big = sepo().budget_for(1 << 18, 16384, 1 << 14)
    t = sepo().Table(big, 1 << 18, 16384)
    assert t.run_wire(wire) == 1
    F = t.stats()["pages_used_max"]
    t.close()
    P = int(np.ceil(F / ratio)) + 2
    t = sepo().Table(sepo().budget_for(1 << 18, 16384, P), 1 << 18, 16384, check_dups=True)
    passes = t.run_wire(wire)
    got = sepo().result_dict(t.export())
    st = t.stats()
    t.close()
    assert got == exp
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2


# ---- the in-library NCCL data plane (sepo_attach_nccl / sepo_insert_batch_sharded / sepo_drain)
@pytest.mark.parametrize("name,ratio", [("C2", 4), ("C5z", 4), ("C3", 2)])
def test_nccl_sharded_one_rank(cuda, name, ratio):
    """a one-rank NCCL communicator (the box has one GPU): the batch, split in 3 sharded calls, is
    routed (wire records for words / pairs, a CSR partition for URLs), exchanged through NCCL
    send/recv to itself and drained: the export equals the oracle"""
    scale = {"C2": 1 / 512, "C5z": 2 ** -12, "C3": 1 / 8000}[name]
    s = gen.config(name, scale=scale)
    exp = oracle_expected(s)
    k, o, v = s.device()
    fixed = s.family == gen.GEN_PAIRS
    kw = dict(fixed_key_width=8, fixed_val_width=8) if fixed else {}
    pb = 65536 if name == "C3" else 16384
    t = sepo().Table(sepo().budget_for(1 << 16, pb, 1 << 12), 1 << 16, pb, **kw)
    t.attach_nccl(sepo().nccl_unique_id(), 1, 0)
    n = s.n
    cuts = [0, n // 3, 2 * n // 3, n]
    held = 0
    for a, b in zip(cuts[:-1], cuts[1:]):
        if fixed:
            held = t.insert_batch_sharded(k[8 * a:8 * b], None, v[8 * a:8 * b], n=b - a)
        else:
            held = t.insert_batch_sharded(k, o[a:b + 1].contiguous(), None, n=b - a)
    assert held > 0
    passes = t.drain()
    got = sepo().result_dict(t.export())
    t.close()
    assert passes >= 1
    assert got == exp


# ---- the pipelined sharded job (sepo_run_sharded): chunk c+1 routed / exchanged beside chunk c's insert
@pytest.mark.parametrize("name,ratio,chunk,p2p", [("C2", 4, 1 << 17, "1"), ("C5z", 4, 1 << 16, "1"), ("C5u", 2, 1 << 16, "1"),
                                                  ("C3", 2, 1 << 15, "1"), ("C1", 1, 10_000, "1"),
                                                  ("C2", 4, 1 << 17, "0"), ("C5z", 4, 1 << 16, "0")])
def test_nccl_run_sharded_one_rank(cuda, monkeypatch, name, ratio, chunk, p2p):
    """sepo_run_sharded over a one-rank NCCL communicator, many chunks (SEPO_SHARD_CHUNK), the table
    `ratio` times its budget so chunks decline records into the prepared list: the export equals the
    oracle (wire records for words / pairs — stored by the route kernel into the owner's symmetric
    window, or sent with NCCL send/recv — and a CSR partition for URLs, whose held buffers grow)"""
    monkeypatch.setenv("SEPO_SHARD_CHUNK", str(chunk))
    monkeypatch.setenv("SEPO_SHARD_P2P", p2p)  # 0: NCCL send/recv of the routed parts
    scale = {"C1": 0.25, "C2": 1 / 512, "C5z": 2 ** -12, "C5u": 2 ** -12, "C3": 1 / 2000}[name]
    s = gen.config(name, scale=scale)
    exp = oracle_expected(s)
    k, o, v = s.device()
    fixed = s.family == gen.GEN_PAIRS
    kw = dict(fixed_key_width=8, fixed_val_width=8) if fixed else {}
    pb = 65536 if name == "C3" else 16384
    t = sepo().Table(sepo().budget_for(1 << 16, pb, 1 << 14), 1 << 16, pb, **kw)
    if fixed:
        t.run(k, None, v)
    else:
        t.run(k, o)
    need = t.stats()["pages_used_max"]
    t.close()
    t = sepo().Table(sepo().budget_for(1 << 16, pb, max(8, need // (2 * ratio if name == "C3" else ratio))), 1 << 16, pb,
                     check_dups=True, **kw)
    t.attach_nccl(sepo().nccl_unique_id(), 1, 0)
    passes = t.run_sharded(k, None, v) if fixed else t.run_sharded(k, o)
    st = t.stats()
    got = sepo().result_dict(t.export())
    t.close()
    assert got == exp
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2
    # keys <= 16 bytes go as wire records, routed straight into the owner's window over peer memory
    assert (st["p2p_chunks"] > 0) == (name != "C3" and p2p == "1")


def test_nccl_run_sharded_csr_words(cuda, monkeypatch):
    """SEPO_SHARD_WIRE=0: a CSR batch of words (all <= 16 bytes, wire records by default) goes as a CSR
    partition appended to the records held"""
    monkeypatch.setenv("SEPO_SHARD_CHUNK", str(1 << 16))
    monkeypatch.setenv("SEPO_SHARD_WIRE", "0")
    s = gen.config("C2", scale=1 / 1024)
    exp = oracle_expected(s)
    k, o, _ = s.device()
    t = sepo().Table(sepo().budget_for(1 << 16, 16384, 96), 1 << 16, 16384, check_dups=True)
    t.attach_nccl(sepo().nccl_unique_id(), 1, 0)
    assert t.run_sharded(k, o) >= 1
    assert sepo().result_dict(t.export()) == exp
    t.close()


@pytest.mark.parametrize("wire", ["1", "0"], ids=["wire", "csr"])
def test_nccl_run_sharded_hot_and_empty(cuda, monkeypatch, wire):
    """chunks large enough for the hot set (>= 2^21 records: the router folds the hot words out of
    wire chunks, the insert kernel folds them in CSR chunks), a trailing short chunk, and a second job
    with an empty batch on the same communicator (the rank still takes part in the agreement)"""
    monkeypatch.setenv("SEPO_SHARD_CHUNK", str(3 << 20))
    monkeypatch.setenv("SEPO_SHARD_WIRE", wire)
    s = gen.config("C2", scale=1 / 200)
    exp = oracle_expected(s)
    k, o, _ = s.device()
    t = sepo().Table(sepo().budget_for(1 << 20, 65536, 4096), 1 << 20, 65536, check_dups=True)
    t.attach_nccl(sepo().nccl_unique_id(), 1, 0)
    assert t.run_sharded(k, o) >= 1
    st = t.stats()
    got = sepo().result_dict(t.export())
    assert got == exp
    if wire == "0":
        assert st["hot_keys"] > 0
    t.reset()
    assert t.run_sharded(None, None, n=0) >= 0
    assert sepo().result_dict(t.export()) == {}
    t.close()
