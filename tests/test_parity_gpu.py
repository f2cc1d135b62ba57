"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, element by element after
canonical sorting (all aggregation is integer => bit-exact), plus the SEPO invariants the paper
states: multi-pass result == single-pass result, no key in two generations,
each pass makes progress, order/budget/postponement independence."""
import numpy as np
import pytest
import torch

import gen
import oracle
from tests.util import device_inputs, footprint_pages, oracle_expected, run_job

pytestmark = pytest.mark.gpu


def sepo():
    import paper_conf_ipps_mokhtaris17_b200 as m
    return m


def assert_same(got, exp):
    assert len(got) == len(exp), f"{len(got)} keys vs {len(exp)} expected"
    bad = [k for k in exp if got.get(k) != exp[k]]
    assert not bad, f"{len(bad)} mismatching keys, e.g. {bad[:3]}: got {[got.get(k) for k in bad[:3]]}, exp {[exp[k] for k in bad[:3]]}"


def budget_pages(stream, k, n_buckets, page_bytes, inputs, **kw):
    F = footprint_pages(stream, n_buckets, page_bytes, inputs=inputs, **kw)
    return F, max(4, int(np.ceil(F / k)))


# ------------------------------------------------------------------ in-budget (one pass)
def test_c1_in_budget(cuda):
    s = gen.config("C1")
    exp = oracle_expected(s)
    assert exp == s.expected_combine()  # oracle pinned to the closed form on this very input
    # 296 CTAs each own an open 64 KiB page: the pool must exceed the allocator slots to fit in one pass
    got, passes, st = run_job(s, sepo().budget_for(1 << 16, 65536, 1024), 1 << 16, 65536)
    assert passes == 1  # P:L241 "Word Count will rarely need multiple iterations"
    assert st["postponed_per_pass"][0] == 0
    assert_same(got, exp)


@pytest.mark.parametrize("ratio", [2, 4])
def test_c1_over_budget(cuda, ratio):
    s = gen.config("C1")
    inp = device_inputs(s)
    exp = oracle_expected(s)
    F, P = budget_pages(s, ratio, 1 << 14, 4096, inp)
    got, passes, st = run_job(s, sepo().budget_for(1 << 14, 4096, P), 1 << 14, 4096, inputs=inp, check_dups=True)
    assert_same(got, exp)
    assert passes >= 2
    assert st["cross_gen_dups"] == 0  # no key is needed again after its eviction
    post = st["postponed_per_pass"]
    assert all(post[i] > post[i + 1] for i in range(len(post) - 1)) and post[-1] == 0, post


@pytest.mark.parametrize("overlap", ["1", "0"])
def test_evict_overlap(cuda, monkeypatch, overlap):
    """eviction copies overlapped with the next pass (SEPO_EVICT_OVERLAP=1: the allocator waits per
    evicted page) or waited for as a whole (default): identical results, no key in two generations"""
    monkeypatch.setenv("SEPO_EVICT_OVERLAP", overlap)
    s = gen.config("C1")
    inp = device_inputs(s)
    exp = oracle_expected(s)
    F, P = budget_pages(s, 4, 1 << 14, 4096, inp)
    for _ in range(2):  # the second job reuses the table's pages while nothing is in flight
        got, passes, st = run_job(s, sepo().budget_for(1 << 14, 4096, P), 1 << 14, 4096, inputs=inp, check_dups=True)
        assert_same(got, exp)
        assert passes >= 3 and st["cross_gen_dups"] == 0


@pytest.mark.parametrize("reissue", ["prepared", "prepared_overflow", "index"])
def test_reissue_paths(cuda, monkeypatch, reissue):
    """sepo_run re-issues postponed COMBINE records as prepared records (hash + key prefix +
    offset), falls back to index lists when the first pass's prepared list overflows, or uses
    index lists only (SEPO_NO_PREP=1): same result, same per-pass postponement invariants"""
    if reissue == "prepared_overflow":
        monkeypatch.setenv("SEPO_PREP_CAP", "1000")
    if reissue == "index":
        monkeypatch.setenv("SEPO_NO_PREP", "1")
    s = gen.config("C3", scale=0.004)  # URLs: keys longer than 16 B take the tail path
    inp = device_inputs(s)
    exp = oracle_expected(s)
    F, P = budget_pages(s, 3, 1 << 14, 16384, inp)
    got, passes, st = run_job(s, sepo().budget_for(1 << 14, 16384, P), 1 << 14, 16384, inputs=inp, check_dups=True)
    assert_same(got, exp)
    assert passes >= 2
    assert st["cross_gen_dups"] == 0
    post = st["postponed_per_pass"]
    assert all(post[i] > post[i + 1] for i in range(len(post) - 1)) and post[-1] == 0, post
    assert st["records_inserted"] == s.n + sum(post[:-1])


@pytest.mark.parametrize("ppm,mode", [(10_000, 0), (500_000, 0), (500_000, 1)])
def test_fault_injection(cuda, ppm, mode):
    """postponement pattern does not change the result; key-mode failure is monotone per key"""
    s = gen.config("C1", scale=0.3)
    exp = oracle_expected(s)
    got, passes, st = run_job(s, sepo().budget_for(1 << 14, 65536, 64), 1 << 14, 65536, fail_alloc_ppm=ppm,
                              fail_mode=mode, check_dups=True)
    assert_same(got, exp)
    assert passes >= 2
    if mode == 0:
        assert st["cross_gen_dups"] == 0


@pytest.mark.parametrize("page_bytes,n_buckets,grid,seed", [(4096, 1 << 10, 1, 1), (1 << 20, 1 << 20, 37, 2),
                                                           (65536, 3, 296, 3), (16384, 12345, 148, 4)])
def test_invariant_to_table_shape(cuda, page_bytes, n_buckets, grid, seed):
    s = gen.config("C1", scale=0.2)
    exp = oracle_expected(s)
    got, _, _ = run_job(s, sepo().budget_for(n_buckets, page_bytes, max(8, (8 << 20) // page_bytes)), n_buckets,
                        page_bytes, grid_ctas=grid, hash_seed=seed)
    assert_same(got, exp)


def test_permutation_and_batches(cuda):
    """records in another order, inserted in several batches per pass"""
    s = gen.config("C1", scale=0.1)
    keys, offs, _ = s.host()
    exp = oracle.combine(keys, offs).as_dict()
    perm = np.random.default_rng(5).permutation(s.n)
    kb = keys.tobytes()
    words = [kb[offs[i]:offs[i + 1]] for i in perm]
    lens = np.array([len(w) for w in words], dtype=np.int64)
    o2 = np.zeros(s.n + 1, dtype=np.int64)
    np.cumsum(lens, out=o2[1:])
    k2 = torch.from_numpy(np.frombuffer(b"".join(words), dtype=np.uint8).copy()).cuda()
    o2t = torch.from_numpy(o2).cuda()
    t = sepo().Table(sepo().budget_for(1 << 12, 4096, 24), 1 << 12, 4096, check_dups=True)
    # requestor-driven pass loop over 3 batches: insert, re-probe, compact, evict
    cuts = [0, s.n // 3, 2 * s.n // 3, s.n]
    batches = [(k2, o2t[cuts[i]:cuts[i + 1] + 1].clone(), cuts[i + 1] - cuts[i]) for i in range(3)]
    passes = 0
    while batches:
        bms = []
        for (k, o, n) in batches:
            c, bm = t.insert_batch(k, o, n=n)
            bms.append(bm)
        nxt = []
        for (k, o, n), bm in zip(batches, bms):
            rem, kbytes, _ = t.reprobe(k, o, None, bm, n=n)
            if rem:
                # the compaction must equal the oracle's definition on this very bitmap
                ok, oko, _, m = t.compact(k, o, None, bm, n=n)
                hk = k.cpu().numpy(); ho = o.cpu().numpy().view(np.uint64)
                bmh = bm.cpu().numpy().view(np.uint32)
                ek, eo, _, _, em = oracle.compact(hk, ho - 0, bmh)
                assert m == em == rem and int(oko[-1]) == kbytes
                assert ok.cpu().numpy().tobytes() == ek.tobytes()
                assert (oko.cpu().numpy().view(np.uint64) == eo).all()
                nxt.append((ok, oko, m))
        t.evict()
        passes += 1
        batches = nxt
        assert passes < 200
    got = sepo().result_dict(t.export())
    assert_same(got, exp)
    assert t.stats()["cross_gen_dups"] == 0
    t.close()


# ------------------------------------------------------------------ other workloads
@pytest.mark.parametrize("name,ratio", [("C5u", 4), ("C5z", 4), ("C5u", 1)])
def test_pairs_fixed_width(cuda, name, ratio):
    s = gen.config(name, scale=2 ** -12)
    exp = oracle_expected(s)
    inp = device_inputs(s)
    F, P = budget_pages(s, ratio, 1 << 16, 16384, inp)
    got, passes, st = run_job(s, sepo().budget_for(1 << 16, 16384, P), 1 << 16, 16384, inputs=inp, check_dups=True)
    assert_same(got, exp)
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2


def test_urls_c3(cuda):
    s = gen.config("C3", scale=1 / 2000)
    exp = oracle_expected(s)
    inp = device_inputs(s)
    F, P = budget_pages(s, 2, 1 << 16, 65536, inp)
    got, passes, st = run_job(s, sepo().budget_for(1 << 16, 65536, P), 1 << 16, 65536, inputs=inp, check_dups=True)
    assert_same(got, exp)
    assert st["cross_gen_dups"] == 0


@pytest.mark.parametrize("ratio", [1, 3])
def test_group_c4(cuda, ratio):
    s = gen.config("C4", scale=1 / 1000)
    exp = oracle_expected(s)
    inp = device_inputs(s)
    F, P = budget_pages(s, ratio, 1 << 16, 16384, inp)
    got, passes, st = run_job(s, sepo().budget_for(1 << 16, 16384, P + 2), 1 << 16, 16384, inputs=inp, check_dups=True)
    assert_same(got, exp)
    if ratio == 3:
        assert passes >= 2


# ------------------------------------------------------------------ edge cases
def _tensors(keys):
    offs = np.zeros(len(keys) + 1, dtype=np.int64)
    offs[1:] = np.cumsum([len(k) for k in keys])
    kb = np.frombuffer(b"".join(keys) + b"\0", dtype=np.uint8).copy()
    return torch.from_numpy(kb).cuda(), torch.from_numpy(offs).cuda()


@pytest.mark.parametrize("case", ["empty", "one", "ragged33", "hot", "zero_len", "long", "adversarial"])
def test_edge_cases(cuda, case):
    rng = np.random.default_rng(1)
    if case == "empty":
        keys = []
    elif case == "one":
        keys = [b"k"]
    elif case == "ragged33":
        keys = [bytes([65 + i % 7]) * (i % 5) for i in range(33)]
    elif case == "hot":
        keys = [b"the"] * 100_000 + [b"a"] * 3
    elif case == "zero_len":
        keys = [b""] * 40 + [b"x"] * 5 + [b""]
    elif case == "long":
        keys = [rng.integers(97, 100, size=int(L)).astype(np.uint8).tobytes() for L in rng.integers(200, 3000, size=500)] * 3
    else:
        pool = [b"", b"a", b"ab", b"a" * 256, b"a" * 255 + b"b", b"\0", b"\0\0", b"\xff" * 7, b"abcdefgh", b"abcdefgi"]
        keys = [pool[i] for i in rng.integers(0, len(pool), size=5000)]
    k, o = _tensors(keys)
    t = sepo().Table(sepo().budget_for(1 << 10, 16384, 16), 1 << 10, 16384, check_dups=True)
    passes = t.run(k, o)
    got = sepo().result_dict(t.export())
    exp = {}
    for x in keys:
        exp[x] = exp.get(x, 0) + 1
    assert_same(got, exp)
    assert t.stats()["cross_gen_dups"] == 0
    t.close()


def test_toolarge(cuda):
    keys = [b"a", b"z" * 4073, b"b"]  # 24 B header + 4080 > 4096-byte page
    k, o = _tensors(keys)
    t = sepo().Table(sepo().budget_for(1 << 10, 4096, 16), 1 << 10, 4096)
    with pytest.raises(sepo().SepoError) as e:
        t.run(k, o)
    assert e.value.code == sepo().E_TOOLARGE
    t.close()


def test_host_input_equals_device_input(cuda):
    s = gen.config("C3", scale=1 / 4000)
    exp = oracle_expected(s)
    keys, offs, _ = s.host()
    t = sepo().Table(sepo().budget_for(1 << 16, 65536, 64), 1 << 16, 65536)
    t.run(keys, offs)  # numpy (host) arrays: staged by the library
    assert_same(sepo().result_dict(t.export()), exp)
    t.close()


def test_reset_and_reuse(cuda):
    s = gen.config("C1", scale=0.1)
    exp = oracle_expected(s)
    k, o, _ = device_inputs(s)
    t = sepo().Table(sepo().budget_for(1 << 12, 4096, 32), 1 << 12, 4096)
    for _ in range(3):
        t.run(k, o)
        assert_same(sepo().result_dict(t.export()), exp)
        t.reset()
    t.close()


# ------------------------------------------------------------------ variable-length GROUP values
def _csr_t(items):
    offs = np.zeros(len(items) + 1, dtype=np.int64)
    offs[1:] = np.cumsum([len(x) for x in items])
    data = np.frombuffer(b"".join(items) + b"\0" * 16, dtype=np.uint8).copy()
    return torch.from_numpy(data).cuda(), torch.from_numpy(offs).cuda()


def test_group_paper_example_variable_values(cuda):
    """http://google.com found in a.html, c.html and d.html -> one key, three paths."""
    keys = [b"http://google.com", b"http://other.org", b"http://google.com", b"http://google.com"]
    vals = [b"a.html", b"b.html", b"c.html", b"d.html"]
    k, ko = _csr_t(keys)
    v, vo = _csr_t(vals)
    t = sepo().Table(sepo().budget_for(1 << 10, 4096, 16), 1 << 10, 4096, mode=sepo().GROUP)
    t.run(k, ko, v, val_offsets=vo)
    got = sepo().result_dict(t.export(), sepo().GROUP)
    assert got == {b"http://google.com": [b"a.html", b"c.html", b"d.html"], b"http://other.org": [b"b.html"]}
    t.close()


@pytest.mark.parametrize("ratio", [1, 3])
def test_group_variable_values_vs_oracle(cuda, ratio):
    """Inverted index with variable-length page paths as values, over budget."""
    s = gen.config("C1", scale=0.02)
    hk, ho, _ = s.host()
    kb = hk.tobytes()
    words = [kb[ho[i]:ho[i + 1]] for i in range(s.n)]
    rng = np.random.default_rng(3)
    paths = [b"/site/%d/page%d.html" % (int(x) % 97, int(x)) for x in rng.integers(0, 5000, size=s.n)]
    exp = oracle.group(*[np.frombuffer(b"".join(words), dtype=np.uint8), ho],
                       np.frombuffer(b"".join(paths), dtype=np.uint8),
                       val_offs=np.concatenate([[0], np.cumsum([len(p) for p in paths])]).astype(np.uint64)).as_dict()
    k, ko = _csr_t(words)
    v, vo = _csr_t(paths)
    t = sepo().Table(sepo().budget_for(1 << 12, 4096, 4096), 1 << 12, 4096, mode=sepo().GROUP)
    t.run(k, ko, v, val_offsets=vo)
    pages = t.stats()["pages_used_max"]
    t.close()
    t = sepo().Table(sepo().budget_for(1 << 12, 4096, max(8, pages // ratio + 2)), 1 << 12, 4096, mode=sepo().GROUP,
                     check_dups=True)
    passes = t.run(k, ko, v, val_offsets=vo)
    got = sepo().result_dict(t.export(), sepo().GROUP)
    t.close()
    assert_same(got, exp)
    if ratio > 1:
        assert passes >= 2


@pytest.mark.parametrize("cfg", ["C1", "C4"])
@pytest.mark.parametrize("evk", ["0", "1"])
def test_evict_copy_paths(cuda, monkeypatch, cfg, evk):
    """evicted pages leave through cudaMemcpyAsync per run of consecutive pages (0) or through the
    gather-copy kernel into one contiguous pinned region (1): identical page images, results"""
    monkeypatch.setenv("SEPO_EVICT_KERNEL", evk)
    s = gen.config(cfg, scale=0.25 if cfg == "C1" else 2e-4)
    inp = device_inputs(s)
    exp = oracle_expected(s)
    kw = {} if cfg == "C1" else dict(mode=sepo().GROUP, fixed_val_width=4)
    F, P = budget_pages(s, 3, 1 << 14, 4096, inp, **kw)
    got, passes, st = run_job(s, sepo().budget_for(1 << 14, 4096, P), 1 << 14, 4096, inputs=inp, check_dups=True, **kw)
    assert_same(got, exp)
    assert passes >= 2


@pytest.mark.parametrize("ratio", [0.5, 4])
def test_host_input_pipelined(cuda, monkeypatch, ratio):
    """host (pinned numpy) input with the H2D copy pipelined with pass 1 in chunks of records
    (thresholds shrunk for the test): same result as the oracle, in and over budget"""
    monkeypatch.setenv("SEPO_H2D_PIPE_MIN", "1000")
    monkeypatch.setenv("SEPO_H2D_CHUNK", "40000")
    s = gen.config("C1")
    hk, ho, _ = s.host()
    exp = oracle_expected(s)
    inp = device_inputs(s)
    F, P = budget_pages(s, ratio if ratio > 1 else 1, 1 << 14, 4096, inp)
    P = P + 600 if ratio < 1 else P
    t = sepo().Table(sepo().budget_for(1 << 14, 4096, P), 1 << 14, 4096, check_dups=True)
    passes = t.run(hk, ho.astype(np.uint64))
    got = sepo().result_dict(t.export())
    st = t.stats()
    t.close()
    assert_same(got, exp)
    assert st["records_inserted"] >= s.n and st["cross_gen_dups"] == 0
    assert (passes == 1) if ratio < 1 else (passes >= 2)


def test_compact_long_keys(cuda):
    """sepo_compact on URL keys (28-256 bytes: the copy's aligned 8-byte middle, byte head and tail at
    every alignment) equals the oracle's compaction byte for byte"""
    s = gen.config("C3", scale=1 / 8000)
    hk, ho, _ = s.host()
    k, o, _ = s.device()
    n = s.n
    t = sepo().Table(sepo().budget_for(1 << 12, 65536, 6), 1 << 12, 65536)
    c, bm = t.insert_batch(k, o, n=n)
    rem, kbytes, _ = t.reprobe(k, o, None, bm, n=n)
    assert rem > 0
    ok, oko, _, m = t.compact(k, o, None, bm, n=n)
    ek, eo, _, _, em = oracle.compact(hk, np.asarray(ho).view(np.uint64), bm.cpu().numpy().view(np.uint32))
    assert m == em == rem and int(oko[-1]) == kbytes
    assert ok.cpu().numpy().tobytes() == ek.tobytes()
    assert (oko.cpu().numpy().view(np.uint64) == eo).all()
    t.close()
