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
