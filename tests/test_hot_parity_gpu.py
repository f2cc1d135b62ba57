"""GPU parity at sizes where the sampled hot set is ACTIVE — batches of at least
2,097,152 records — element by element against the CPU oracle, with the hot set on and off
(SEPO_NO_HOT=1) on the same input. The hot-key paths (shared-memory pending sums with warp folding
in the COMBINE stream kernel; CTA-private value chunks in the GROUP stream kernel) carry about
half of the records of the Zipf configs at bench scale (Word Count's contention on a few
keys), so they are checked where they run. Passages: P:L73 (combine <url,1> n times -> <url,n>),
P:L133 (value lists), P:L239 (hot keys)."""
import numpy as np
import pytest

import gen
from tests.util import device_inputs, footprint_pages, oracle_expected, run_job

pytestmark = pytest.mark.gpu

HOT_MIN = 2_097_152  # = 8 x the 2^18-record sample (sepo_kernels.cu launchers)


def sepo():
    import paper_conf_ipps_mokhtaris17_b200 as m
    return m


def assert_same(got, exp):
    assert len(got) == len(exp), f"{len(got)} keys vs {len(exp)} expected"
    bad = [k for k in exp if got.get(k) != exp[k]]
    assert not bad, f"{len(bad)} mismatching keys, e.g. {bad[:3]}"


_EXP = {}


def expected(name, scale):
    if (name, scale) not in _EXP:
        _EXP.clear()
        _EXP[(name, scale)] = oracle_expected(gen.config(name, scale))
    return _EXP[(name, scale)]


def _job(name, scale, ratio, page_bytes, n_buckets, hot, monkeypatch):
    s = gen.config(name, scale)
    assert s.n >= HOT_MIN, s.n
    inp = device_inputs(s)
    monkeypatch.setenv("SEPO_NO_HOT", "0" if hot else "1")
    F = footprint_pages(s, n_buckets, page_bytes, inputs=inp)
    P = max(8, int(np.ceil(F / ratio))) + (2 if ratio >= 1 else 0)
    got, passes, st = run_job(s, sepo().budget_for(n_buckets, page_bytes, P), n_buckets, page_bytes, inputs=inp,
                              check_dups=True)
    if hot:
        assert st["hot_keys"] > 100, st["hot_keys"]  # the hot path really ran
    else:
        assert st["hot_keys"] == 0
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2
    return got, passes, st


@pytest.mark.parametrize("hot", [True, False], ids=["hot", "nohot"])
@pytest.mark.parametrize("ratio", [0.5, 4])
def test_c2_hot_csr(cuda, monkeypatch, ratio, hot):
    """C2 words at 1/256 (32 MiB text, ~4.3 M records): insert_stream_kernel IN_CSR, in budget and 4x"""
    got, passes, st = _job("C2", 1 / 256, ratio, 16384, 1 << 18, hot, monkeypatch)
    assert_same(got, expected("C2", 1 / 256))
    if ratio < 1:
        assert passes == 1


@pytest.mark.parametrize("hot", [True, False], ids=["hot", "nohot"])
def test_c5z_hot_fixed(cuda, monkeypatch, hot):
    """C5 Zipf(1.2) pairs at 1/128 (D = 2^21 keys, 16.7 M records): IN_FIXED with u64 values, 4x"""
    got, _, _ = _job("C5z", 1 / 128, 4, 16384, 1 << 18, hot, monkeypatch)
    assert_same(got, expected("C5z", 1 / 128))


@pytest.mark.parametrize("hot", [True, False], ids=["hot", "nohot"])
@pytest.mark.parametrize("ratio", [1, 3])
def test_c4_hot_group(cuda, monkeypatch, ratio, hot):
    """C4 inverted index at 1/256 (~4.3 M records): insert_group_stream_kernel, hot keys append into
    CTA-private value chunks; 1x and 3x over budget"""
    s = gen.config("C4", 1 / 256)
    assert s.n >= HOT_MIN
    inp = device_inputs(s)
    monkeypatch.setenv("SEPO_NO_HOT", "0" if hot else "1")
    kw = dict(mode=sepo().GROUP, fixed_val_width=4)
    F = footprint_pages(s, 1 << 18, 16384, inputs=inp, **kw)
    P = int(np.ceil(F / ratio)) + 2
    got, passes, st = run_job(s, sepo().budget_for(1 << 18, 16384, P), 1 << 18, 16384, inputs=inp, check_dups=True, **kw)
    assert (st["hot_keys"] > 100) if hot else (st["hot_keys"] == 0)
    assert_same(got, expected("C4", 1 / 256))
    if ratio > 1:
        assert passes >= 2


@pytest.mark.parametrize("hot", [True, False], ids=["hot", "nohot"])
def test_c2_hot_text(cuda, monkeypatch, hot):
    """raw text (fused tokenizer, sepo_run_text) at 1/256, 4x: the text kernel's hot set"""
    import oracle
    s = gen.config("C2", 1 / 256)
    monkeypatch.setenv("SEPO_NO_HOT", "0" if hot else "1")
    text = s.text_device()
    exp = expected("C2", 1 / 256)
    assert exp == oracle.word_count_text(s.text_host())  # same words as the CSR stream
    inp = device_inputs(s)
    F = footprint_pages(s, 1 << 18, 16384, inputs=inp)
    t = sepo().Table(sepo().budget_for(1 << 18, 16384, max(8, F // 4)), 1 << 18, 16384, check_dups=True)
    passes = t.run_text(text)
    st = t.stats()
    got = sepo().result_dict(t.export())
    t.close()
    assert (st["hot_keys"] > 100) if hot else (st["hot_keys"] == 0)
    assert passes >= 2 and st["cross_gen_dups"] == 0
    assert_same(got, exp)


def test_hot_min_small_batches(cuda, monkeypatch):
    """SEPO_HOT_MIN moves the hot-set threshold: C1 (1.35 M records) with and without a hot set,
    in budget and 4x over, equals the oracle"""
    s = gen.config("C1")
    exp = oracle_expected(s)
    inp = device_inputs(s)
    F = footprint_pages(s, 1 << 14, 4096, inputs=inp)
    for hm in ("1000", str(1 << 40)):
        monkeypatch.setenv("SEPO_HOT_MIN", hm)
        for P in (F + 64, F // 4):
            got, passes, st = run_job(s, sepo().budget_for(1 << 14, 4096, P), 1 << 14, 4096, inputs=inp, check_dups=True)
            assert (st["hot_keys"] > 0) == (hm == "1000")
            assert_same(got, exp)
            assert st["cross_gen_dups"] == 0


@pytest.mark.parametrize("name,scale,ratio", [("C2", 1 / 256, 0.5), ("C2", 1 / 256, 4), ("C3", 1 / 2000, 2),
                                              ("C5z", 1 / 128, 4), ("C1", 1.0, 4)])
def test_dir_prefetch_path(cuda, monkeypatch, name, scale, ratio):
    """SEPO_DIR_PF=1 + SEPO_LEAN=0 force the path of tables larger than L2 (insert_stream_kernel with
    queued misses' bucket lines L2-prefetched) on small tables — every config equals the oracle, in
    budget and over (C3: long keys; C5z: values, 8 keys per bucket; C1: below the hot-set threshold)"""
    monkeypatch.setenv("SEPO_DIR_PF", "1")
    monkeypatch.setenv("SEPO_LEAN", "0")
    s = gen.config(name, scale)
    inp = device_inputs(s)
    pb = 65536 if name == "C3" else 16384
    F = footprint_pages(s, 1 << 18, pb, inputs=inp)
    P = max(8, int(np.ceil(F / ratio))) + (2 if ratio >= 1 else 0)
    got, passes, st = run_job(s, sepo().budget_for(1 << 18, pb, P), 1 << 18, pb, inputs=inp, check_dups=True)
    assert_same(got, oracle_expected(s))
    assert st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2


@pytest.mark.parametrize("name,scale,ratio", [("C4", 1 / 256, 3), ("C4", 1 / 1000, 2), ("C2", 1 / 256, 4), ("C5u", 2 ** -12, 4)])
def test_evict_overlap_forced(cuda, monkeypatch, name, scale, ratio):
    """SEPO_EVICT_OVERLAP=1 (off by default for GROUP and for pools inside L2): every eviction's copies
    overlap the next pass, whose allocator waits per evicted page (progress published by the copy stream)
    before reusing it — GROUP (retained key pages between evicted ones) and COMBINE equal the oracle"""
    monkeypatch.setenv("SEPO_EVICT_OVERLAP", "1")
    s = gen.config(name, scale)
    inp = device_inputs(s)
    kw = dict(mode=sepo().GROUP, fixed_val_width=4) if name == "C4" else {}
    F = footprint_pages(s, 1 << 18, 16384, inputs=inp, **kw)
    P = max(8, int(np.ceil(F / ratio))) + 2
    got, passes, st = run_job(s, sepo().budget_for(1 << 18, 16384, P), 1 << 18, 16384, inputs=inp, check_dups=True, **kw)
    assert_same(got, oracle_expected(s))
    assert passes >= 2 and st["cross_gen_dups"] == 0
