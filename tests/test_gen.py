"""Checks of the synthetic input generators (gen/): the exact-count construction the closed-form
pins rely on, bijectivity of the shuffle, injectivity of the key spellings, and host == device."""
import numpy as np
import pytest

import gen


def test_perm_is_bijection_and_inverse():
    for n in [1, 2, 3, 5, 100, 1000, 4097]:
        s = gen.Stream("t", gen.GEN_PAIRS, seed=11, uniform=(n, 1))
        j = np.arange(n, dtype=np.uint64)
        out = np.empty(n, dtype=np.uint64)
        gen.lib().gen_perm_host(gen.ctypes.byref(s.params()), gen._ptr(j), n, gen._ptr(out))
        assert sorted(out.tolist()) == list(range(n))
        back = np.empty(n, dtype=np.uint64)
        gen.lib().gen_perm_inv_host(gen.ctypes.byref(s.params()), gen._ptr(out), n, gen._ptr(back))
        assert (back == j).all()


def test_exact_counts_by_histogram():
    """rank r appears exactly c_r times (brute-force histogram of the generated ranks)."""
    for name, sc in [("C1", 0.2), ("C3", 1e-5), ("C5z", 1e-5), ("C5u", 1e-6)]:
        s = gen.config(name, scale=sc)
        ranks = s.ranks_host()
        h = np.bincount(ranks.astype(np.int64), minlength=s.n_ranks + 1)
        assert h[0] == 0
        assert (h[1:] == s.count_of_rank(np.arange(1, s.n_ranks + 1))).all()


def test_zipf_shape():
    s = gen.config("C2")
    c = s.count_of_rank(np.arange(1, 11)).astype(np.float64)
    # c_r = floor(C / r): Zipf(1.0) to within one count
    assert np.all(np.abs(c * np.arange(1, 11) - c[0]) <= np.arange(1, 11))
    assert s.n_ranks == 1 << 22 and 1.0e9 < s.n < 1.2e9


def test_spellings_injective():
    for name, sc in [("C1", 1.0), ("C3", 1e-3)]:
        s = gen.config(name, scale=sc)
        sp = [s.spell(r) for r in range(1, s.n_ranks + 1)]
        assert len(set(sp)) == len(sp)
        lens = s.key_lens_of_ranks()
        assert [len(x) for x in sp] == lens.tolist()
    w = gen.config("C2")
    assert w.spell(1) == b"ab" and w.spell(26) == b"aaba"  # base-26 "ba", padded to L(26) = 4
    assert max(w.key_lens_of_ranks(1 << 22, 1)) <= 16


def test_host_chunks_equal_whole():
    s = gen.config("C3", scale=1e-5)
    k, o, _ = s.host()
    k1, o1, _ = s.host(0, 100)
    k2, o2, _ = s.host(100, s.n - 100)
    assert k.tobytes() == k1.tobytes() + k2.tobytes()
    assert (o[:101] == o1).all() and (o[100:] - o[100] == o2).all()


@pytest.mark.gpu
def test_device_equals_host(cuda):
    for name, sc in [("C1", 0.3), ("C3", 2e-5), ("C4", 1e-4), ("C5u", 1e-5), ("C5z", 1e-5)]:
        s = gen.config(name, scale=sc)
        hk, ho, hv = s.host(7, s.n - 7)
        dk, do, dv = s.device(7, s.n - 7)
        assert (do.cpu().numpy().view(np.uint64) == ho).all(), name
        assert dk.cpu().numpy().tobytes() == hk.tobytes(), name
        if hv is not None:
            assert dv.cpu().numpy().tobytes() == hv.tobytes(), name


# ---- the full-size check helpers (closed forms evaluated backwards), pinned on small streams
@pytest.mark.parametrize("name,sc", [("C1", 0.2), ("C3", 2e-5), ("C5u", 1e-6), ("C5z", 1e-5)])
def test_key_ranks_inverts_spelling(name, sc):
    """key_ranks(spell(r)) == r for every rank; damaged or foreign keys map to 0"""
    s = gen.config(name, scale=sc)
    rs = np.arange(1, s.n_ranks + 1)
    sp = [s.spell(int(r)) for r in rs]
    offs = np.zeros(len(sp) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(x) for x in sp])
    got = s.key_ranks(np.frombuffer(b"".join(sp), dtype=np.uint8), offs)
    assert (got == rs.astype(np.uint64)).all()
    bad = [x[:-1] for x in sp[:50]] + [x + b"a" for x in sp[:50]] + [b"", b"\xff" * 8, b"zzzzzzzzzzzzzzzzz"]
    bad += [bytes([x[0] ^ 1]) + x[1:] for x in sp[:50]]
    offs = np.zeros(len(bad) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(x) for x in bad])
    got = s.key_ranks(np.frombuffer(b"".join(bad), dtype=np.uint8), offs)
    # a truncated / extended / flipped spelling is never the spelling of the SAME rank
    for i, x in enumerate(bad):
        r = int(got[i])
        assert r == 0 or s.spell(r) == x


@pytest.mark.parametrize("name,sc", [("C5u", 1e-5), ("C5z", 1e-5), ("C4", 2e-5)])
def test_rank_digest_equals_brute_force(name, sc):
    """per-rank count / value sum / multiset digest == a brute-force pass over the generated records"""
    s = gen.config(name, scale=sc)
    ranks = s.ranks_host()
    j = np.arange(s.n, dtype=np.uint64)
    vals = s.values_of_records(j)
    cnt, sm, mx = s.rank_digest()
    bc = np.bincount(ranks.astype(np.int64), minlength=s.n_ranks + 1)[1:]
    assert (cnt == bc.astype(np.uint64)).all()
    exp_sum = np.zeros(s.n_ranks + 1, dtype=np.uint64)
    np.add.at(exp_sum, ranks.astype(np.int64), vals)
    assert (sm == exp_sum[1:]).all()
    # digest of the lists built by a plain loop
    lists = {}
    for r, v in zip(ranks.tolist(), vals.tolist()):
        lists.setdefault(r, []).append(v)
    w = 8 if name != "C4" else 4
    order = sorted(lists)
    vb = b"".join(int(v).to_bytes(w, "little") for r in order for v in lists[r])
    vo = np.arange(0, len(vb) + 1, w, dtype=np.uint64)
    lo = np.zeros(len(order) + 1, dtype=np.uint64)
    lo[1:] = np.cumsum([len(lists[r]) for r in order])
    c2, s2, m2 = gen.list_digest(np.frombuffer(vb, dtype=np.uint8), vo, lo)
    idx = np.array(order, dtype=np.int64) - 1
    assert (c2 == cnt[idx]).all() and (s2 == sm[idx]).all() and (m2 == mx[idx]).all()
    # the digest separates multisets that agree in count and sum
    a = gen.list_digest(np.frombuffer(b"".join(int(v).to_bytes(4, "little") for v in [1, 5]), dtype=np.uint8),
                        np.array([0, 4, 8], dtype=np.uint64), np.array([0, 2], dtype=np.uint64))
    b = gen.list_digest(np.frombuffer(b"".join(int(v).to_bytes(4, "little") for v in [2, 4]), dtype=np.uint8),
                        np.array([0, 4, 8], dtype=np.uint64), np.array([0, 2], dtype=np.uint64))
    assert a[0][0] == b[0][0] and a[1][0] == b[1][0] and a[2][0] != b[2][0]
