"""Full-size correctness: every BASELINE config at the size and in the launch configuration bench.py
times (bench.Job: same inputs, budget, n_buckets, page size, grid), checked KEY BY KEY against the
generators' closed forms — the combine result of an exact-count stream is known without a CPU
group-by (SURVEY §8(c) "What pins each part"):
  * implicit-1 streams (C2 words, C3 URLs, raw text): every exported key spells a rank r and its
    value is c_r = floor(C / r^alpha), every rank appears exactly once;
  * u64 pairs (C5u, C5z): the value of rank r's key is the sum of the values of the records that
    hold r (gen.rank_digest), mod 2^64;
  * the inverted index (C4, GROUP): each key's value list has c_r entries and the same value sum
    and multiset digest (sum of a 64-bit mix of each doc id) as the records of its rank.
North-star target: "bit-exact agreement with the CPU oracle on all five configs" — the oracle is
pinned to these same closed forms (tests/test_oracle.py), which are evaluated here at full size."""
import numpy as np
import pytest

import gen

pytestmark = pytest.mark.gpu


def _job(cfg, ratio, scale=1.0):
    import bench
    return bench.make_job(cfg, ratio=ratio, scale=scale)


def check_combine(stream, res):
    ko, kb, vals = res["key_offsets"], res["keys"], res["values"]
    n = res["n_keys"]
    assert n == stream.n_ranks, (n, stream.n_ranks)
    ranks = stream.key_ranks(kb, ko)
    assert (ranks > 0).all(), f"{int((ranks == 0).sum())} exported keys spell no rank"
    hist = np.bincount(ranks.astype(np.int64), minlength=stream.n_ranks + 1)
    assert hist[0] == 0 and (hist[1:] == 1).all(), "a rank is missing or exported twice"
    if stream.val == "one":
        exp = stream.count_of_rank(ranks.astype(np.int64))
        assert int(vals.sum(dtype=np.uint64)) == stream.n
    else:
        _, sums, _ = stream.rank_digest()
        exp = sums[ranks.astype(np.int64) - 1]
    bad = np.nonzero(vals != exp)[0]
    assert len(bad) == 0, f"{len(bad)} keys with a wrong value, e.g. rank {ranks[bad[:3]]}: {vals[bad[:3]]} vs {exp[bad[:3]]}"


def run_and_check(job, text=False):
    t = job.table()
    if text:
        passes = t.run_text(job.stream.text_device())
    else:
        k, o, v = job.inputs()
        passes = t.run(k, o, v)
    st = t.stats()
    res = t.export(copy=False)
    check_combine(job.stream, res)
    t.close()
    return passes, st


@pytest.mark.parametrize("ratio", [0.5, 4.0])
def test_c2_full(cuda, ratio):
    """C2 word count, 1.1e9 words, all 4,194,304 keys; 0.5x = the M1 in-budget configuration"""
    passes, st = run_and_check(_job("C2", ratio))
    assert (passes == 1) if ratio < 1 else (passes >= 4)
    assert st["hot_keys"] > 1000 and st["cross_gen_dups"] == 0


def test_c2_text_full(cuda):
    """the bench headline: raw 8.6 GB C2 text, tokenizer fused (sepo_run_text), table 4x the budget"""
    passes, st = run_and_check(_job("C2", 4.0), text=True)
    assert passes >= 4 and st["hot_keys"] > 1000


@pytest.mark.parametrize("ratio", [1.0, 4.0])
def test_c3_full(cuda, ratio):
    """C3 page-view count: 16 GiB click log, 2.6e8 URL records (28..256 B), 1.5e7 keys"""
    passes, st = run_and_check(_job("C3", ratio))
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 4


@pytest.mark.parametrize("cfg", ["C5u", "C5z"])
def test_c5_full(cuda, cfg):
    """C5 u64 pairs at one rank's share of the 8-GPU config (2^28 records), table 4x the budget"""
    passes, st = run_and_check(_job(cfg, 4.0, scale=0.125))
    assert passes >= 4 and st["cross_gen_dups"] == 0


def test_c4_full(cuda):
    """C4 inverted index (GROUP): 8 GiB of documents, 1.1e9 (word, doc id) records, 3x over budget"""
    job = _job("C4", 3.0)
    s = job.stream
    t = job.table()
    k, o, v = job.inputs()
    passes = t.run(k, o, v)
    res = t.export(copy=False)
    assert passes >= 3
    assert res["n_keys"] == s.n_ranks
    ranks = s.key_ranks(res["keys"], res["key_offsets"])
    assert (ranks > 0).all()
    hist = np.bincount(ranks.astype(np.int64), minlength=s.n_ranks + 1)
    assert hist[0] == 0 and (hist[1:] == 1).all()
    c, sm, mx = gen.list_digest(res["vals"], res["val_offsets"], res["list_offsets"])
    ec, es, em = s.rank_digest()
    r = ranks.astype(np.int64) - 1
    assert int(res["n_vals"]) == s.n
    assert (c == ec[r]).all(), "list lengths differ from the record counts"
    assert (sm == es[r]).all() and (mx == em[r]).all(), "a value multiset differs"
    t.close()


@pytest.mark.parametrize("cfg,scale", [("C2", 1.0), ("C5z", 0.125), ("C3", 1.0)])
def test_sharded_full(cuda, cfg, scale):
    """the routed job at full size through sepo_run_sharded on a one-rank communicator (hot-key route
    into the rank's symmetric window for words / pairs, CSR send/recv for URLs; 2^28-record chunks;
    table 4x over budget) equals the closed forms key by key"""
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    job = _job(cfg, 4.0, scale=scale)
    k, o, v = job.inputs()
    t = job.table()
    t.attach_nccl(sepo.nccl_unique_id(), 1, 0)
    passes = t.run_sharded(k, o, v)
    st = t.stats()
    res = t.export(copy=False)
    check_combine(job.stream, res)
    assert passes >= 2 and st["cross_gen_dups"] == 0
    assert (st["p2p_chunks"] > 0) == (cfg != "C3")
    t.close()
