"""Pins for the CPU oracle (oracle/), against things other than itself:
paper worked examples (tests/golden), brute force on tiny adversarial inputs, an independent
sort + run-length reducer, closed forms of the exact-count generators, and invariants the paper
states (order independence P:L17; SEPO multi-pass result == single-pass result P:L77-79)."""
import os
import random

import numpy as np
import pytest

import gen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "paper_examples.txt")


def csr(keys):
    offs = np.zeros(len(keys) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(k) for k in keys])
    return b"".join(keys), offs


def brute_combine(keys, vals=None):
    """O(n*d) linear-scan grouping (no hashing): list of [key, sum]."""
    acc = []
    for i, k in enumerate(keys):
        v = 1 if vals is None else vals[i]
        for e in acc:
            if e[0] == k:
                e[1] = (e[1] + v) % (1 << 64)
                break
        else:
            acc.append([k, v % (1 << 64)])
    return {k: v for k, v in acc}


def adversarial_keys(rng, n):
    pool = [b"", b"a", b"b", b"ab", b"ba", b"a" * 256, b"a" * 255 + b"b", b"\x00", b"\x00\x00", b"\xff" * 7,
            b"abcdefgh", b"abcdefgi", b"abcdefg", b"abcdefgh\x00"]
    out = []
    for _ in range(n):
        t = rng.random()
        if t < 0.5:
            out.append(rng.choice(pool))
        elif t < 0.8:
            out.append(bytes(rng.randrange(256) for _ in range(rng.randrange(0, 24))))
        else:
            out.append(bytes(rng.choice(b"ab") for _ in range(rng.randrange(0, 5))))
    return out


# ------------------------------------------------------------------ paper examples
def test_paper_worked_examples():
    rows = [l.rstrip("\n").split("\t") for l in open(GOLD) if l.strip() and not l.startswith("#")]
    assert len(rows) == 2
    for ex, mode, key, vals, expect in rows:
        key = key.encode()
        vs = vals.split(",")
        if mode == "combine":
            k, o = csr([key] * len(vs))
            v = np.array([int(x) for x in vs], dtype=np.uint64).view(np.uint8)
            assert oracle.combine(k, o, v, 8).as_dict() == {key: int(expect)}
            assert oracle.combine(k, o).as_dict() == {key: int(expect)}  # implicit value 1
        else:
            k, o = csr([key] * len(vs))
            vb, vo = csr([x.encode() for x in vs])
            assert oracle.group(k, o, vb, val_offs=vo).as_dict() == {key: [x.encode() for x in expect.split(",")]}


# ------------------------------------------------------------------ brute force
@pytest.mark.parametrize("seed", range(6))
def test_combine_vs_bruteforce(seed):
    rng = random.Random(seed)
    keys = adversarial_keys(rng, rng.randrange(0, 2000))
    k, o = csr(keys)
    assert oracle.combine(k, o).as_dict() == brute_combine(keys)
    vals = [rng.choice([0, 1, 2**63, 2**64 - 1, rng.randrange(2**64)]) for _ in keys]
    v = np.array(vals, dtype=np.uint64).view(np.uint8)
    assert oracle.combine(k, o, v, 8).as_dict() == brute_combine(keys, vals)
    v4 = np.array([x & 0xFFFFFFFF for x in vals], dtype=np.uint32).view(np.uint8)
    assert oracle.combine(k, o, v4, 4).as_dict() == brute_combine(keys, [x & 0xFFFFFFFF for x in vals])


@pytest.mark.parametrize("seed", range(4))
def test_group_vs_bruteforce(seed):
    rng = random.Random(100 + seed)
    keys = adversarial_keys(rng, rng.randrange(0, 1500))
    vals = [bytes(rng.randrange(256) for _ in range(rng.randrange(0, 6))) for _ in keys]
    k, o = csr(keys)
    vb, vo = csr(vals)
    got = oracle.group(k, o, vb, val_offs=vo).as_dict()
    exp = []
    for key, v in zip(keys, vals):
        for e in exp:
            if e[0] == key:
                e[1].append(v)
                break
        else:
            exp.append([key, [v]])
    assert got == {key: sorted(vs) for key, vs in exp}
    # canonical order of keys: unsigned-byte lexicographic, shorter prefix first
    ks, ko, *_ = oracle.group(k, o, vb, val_offs=vo).result()
    kl = [ks[ko[i]:ko[i + 1]].tobytes() for i in range(len(ko) - 1)]
    assert kl == sorted(set(keys))


def test_fixed_width_group_values():
    keys = [b"x", b"y", b"x", b"x"]
    k, o = csr(keys)
    v = np.array([7, 9, 7, 3], dtype=np.uint32).view(np.uint8)
    got = oracle.group(k, o, v, val_width=4).as_dict()
    p = lambda x: int(x).to_bytes(4, "little")
    assert got == {b"x": sorted([p(7), p(7), p(3)]), b"y": [p(9)]}


def test_empty_input():
    k, o = csr([])
    assert oracle.combine(k, o).as_dict() == {}


# ------------------------------------------------------------------ independent reducer at ~1e6
def test_combine_vs_sort_runlength_c1():
    s = gen.config("C1")
    keys, offs, _ = s.host()
    kb = keys.tobytes()
    words = [kb[offs[i]:offs[i + 1]] for i in range(s.n)]
    words.sort()
    rl = {}
    i = 0
    while i < len(words):
        j = i
        while j < len(words) and words[j] == words[i]:
            j += 1
        rl[words[i]] = j - i
        i = j
    got = oracle.combine(keys, offs).as_dict()
    assert got == rl
    assert sum(got.values()) == s.n  # sum of counts = record count


# ------------------------------------------------------------------ closed forms
def test_combine_closed_form_words():
    s = gen.config("C1", scale=0.25)
    keys, offs, _ = s.host()
    got = oracle.combine(keys, offs).as_dict()
    assert got == s.expected_combine()  # word(r) appears exactly c_r = floor(C/r) times


def test_combine_closed_form_urls():
    s = gen.config("C3", scale=2e-5)
    keys, offs, _ = s.host()
    assert oracle.combine(keys, offs).as_dict() == s.expected_combine()


def test_combine_closed_form_pairs_u64():
    for name in ("C5u", "C5z"):
        s = gen.config(name, scale=2e-5)
        keys, offs, vals = s.host()
        got = oracle.combine(keys, offs, vals, 8).as_dict()
        assert got == s.expected_combine()


def test_group_closed_form_docs():
    s = gen.config("C4", scale=1e-4)
    keys, offs, vals = s.host()
    got = oracle.group(keys, offs, vals, val_width=4).as_dict()
    assert len(got) == s.n_ranks
    for r in [1, 2, 3, 17, s.n_ranks // 2, s.n_ranks]:
        exp = [int(d).to_bytes(4, "little") for d in s.expected_group(r)]
        assert got[s.spell(r)] == sorted(exp)
    assert sum(len(v) for v in got.values()) == s.n


# ------------------------------------------------------------------ invariants
def test_order_and_batch_independence():
    """the result does not depend on processing order; streaming batches == one batch."""
    s = gen.config("C1", scale=0.05)
    keys, offs, _ = s.host()
    kb = keys.tobytes()
    words = [kb[offs[i]:offs[i + 1]] for i in range(s.n)]
    ref = oracle.combine(keys, offs).as_dict()
    rng = random.Random(7)
    rng.shuffle(words)
    k, o = csr(words)
    assert oracle.combine(k, o).as_dict() == ref
    c = oracle.Combine()
    cuts = sorted(rng.sample(range(len(words)), 5))
    prev = 0
    for cut in cuts + [len(words)]:
        k, o = csr(words[prev:cut])
        c.add(k, o)
        prev = cut
    assert c.as_dict() == ref


# ------------------------------------------------------------------ compaction (a9)
@pytest.mark.parametrize("n", [0, 1, 31, 32, 33, 1000, 4099])
def test_compact_vs_bruteforce(n):
    rng = random.Random(n)
    keys = [bytes(rng.randrange(256) for _ in range(rng.randrange(0, 9))) for _ in range(n)]
    vals = [rng.randrange(2**64) for _ in range(n)]
    k, o = csr(keys)
    for density in (0.0, 0.3, 1.0):
        bits = [rng.random() < density for _ in range(n)]
        bm = np.zeros((n + 31) // 32 + 1, dtype=np.uint32)
        for i, b in enumerate(bits):
            if b:
                bm[i >> 5] |= np.uint32(1 << (i & 31))
        ok, oo, ov, _, m = oracle.compact(k, o, bm, np.array(vals, dtype=np.uint64).view(np.uint8), val_width=8)
        sel = [i for i in range(n) if bits[i]]
        assert m == len(sel)
        got = [ok[oo[j]:oo[j + 1]].tobytes() for j in range(m)]
        assert got == [keys[i] for i in sel]
        assert ov.view(np.uint64).tolist() == [vals[i] for i in sel]


# ------------------------------------------------------------------ the paper's pass loop
@pytest.mark.parametrize("ratio", [0.5, 1.0, 2.0, 3.0, 4.0])
def test_sepo_sim_combine_exact(ratio):
    """multi-pass SEPO result == plain group-by; no key is in two generations; each
    pass makes progress; passes >= ceil(F / heap)."""
    s = gen.config("C1", scale=0.1)
    keys, offs, _ = s.host()
    ref = oracle.combine(keys, offs).as_dict()
    F = sum(24 + len(k) for k in ref)
    heap = int(F / ratio)
    passes, post, out, dups = oracle.sepo_sim_combine(keys, offs, heap, overhead=24)
    assert out.as_dict() == ref
    assert dups == 0
    assert passes >= -(-F // heap)
    assert all(post[i] > post[i + 1] for i in range(len(post) - 1)) and post[-1] == 0
    if ratio <= 1.0:
        assert passes == 1


def test_sepo_sim_combine_pairs():
    s = gen.config("C5z", scale=1e-5)
    keys, offs, vals = s.host()
    ref = oracle.combine(keys, offs, vals, 8).as_dict()
    F = sum(32 for _ in ref)
    passes, post, out, dups = oracle.sepo_sim_combine(keys, offs, F // 3, overhead=24, vals=vals, val_width=8)
    assert out.as_dict() == ref and dups == 0 and passes >= 3


@pytest.mark.parametrize("ratio", [1.0, 3.0])
def test_sepo_sim_group_exact(ratio):
    s = gen.config("C4", scale=2e-5)
    keys, offs, vals = s.host()
    ref = oracle.group(keys, offs, vals, val_width=4).as_dict()
    F = sum(24 + len(k) + 4 * len(v) for k, v in ref.items())
    passes, post, out, forced = oracle.sepo_sim_group(keys, offs, vals, int(F / ratio), val_width=4, val_overhead=0)
    assert out.as_dict() == ref
    assert passes >= 1 if ratio == 1.0 else passes >= 3


# ------------------------------------------------------------------ basic organization (NEXT-3)
def test_basic_closed_form_pairs():
    """basic stores every pair: per key, the multiset of its records' values. Pinned to
    the generator's closed form (records of rank r = perm^-1 of its multiset block, their values),
    which never looks at the input bytes the oracle reads."""
    for name in ("C5u", "C5z"):
        s = gen.config(name, scale=2e-5)
        keys, offs, vals = s.host()
        got = oracle.basic(keys, offs, vals, 8)
        assert sum(len(v) for v in got.values()) == s.n
        for r in [1, 2, 3, s.n_ranks // 2, s.n_ranks]:
            assert got[s.spell(r)] == s.expected_group(r)


def test_basic_vs_combine_and_counts():
    """per key: count = the closed-form c_r (implicit-1 values), and the u64 sum of the stored
    values = the (independent, C++) combining oracle's value"""
    s = gen.config("C1", scale=0.02)
    keys, offs, _ = s.host()
    got = oracle.basic(keys, offs)
    comb = oracle.combine(keys, offs).as_dict()
    assert got.keys() == comb.keys()
    for r in range(1, s.n_ranks + 1, 97):
        k = s.spell(r)
        if int(s.count_of_rank(r)):
            assert len(got[k]) == int(s.count_of_rank(r)) and set(got[k]) == {1}
    s = gen.config("C5z", scale=2e-5)
    keys, offs, vals = s.host()
    got = oracle.basic(keys, offs, vals, 8)
    comb = oracle.combine(keys, offs, vals, 8).as_dict()
    assert {k: sum(v) % (1 << 64) for k, v in got.items()} == comb


def test_basic_tiny_adversarial():
    """duplicates, empty keys, prefixes: every record is one pair of the result"""
    ks = [b"", b"a", b"a", b"ab", b"", b"b\x00", b"b", b"a"]
    vs = [5, 1, 1, 7, 0, 3, 3, 2]
    keys = np.frombuffer(b"".join(ks), dtype=np.uint8)
    offs = np.cumsum([0] + [len(k) for k in ks]).astype(np.uint64)
    vals = np.array(vs, dtype=np.uint64).view(np.uint8)
    got = oracle.basic(keys, offs, vals, 8)
    assert got == {b"": [0, 5], b"a": [1, 1, 2], b"ab": [7], b"b\x00": [3], b"b": [3]}


# ------------------------------------------------------------------ raw text word count (NEXT-2)
def test_word_count_text_closed_form():
    """the raw text of a word stream (each word + one separator) counts exactly the generator's
    closed-form c_r per word — independent of the oracle's own tokenizer"""
    for name, scale in (("C1", 0.05), ("C2", 2e-5)):
        s = gen.config(name, scale=scale)
        assert oracle.word_count_text(s.text_host()) == s.expected_combine()


def test_word_count_text_tokenizer_rules():
    """R20: separators are exactly ' ', '\\n', '\\t', '\\r'; runs of them, leading/trailing ones and
    an empty text yield no empty words; other bytes (\\x0b, \\x00, 0xff) belong to words"""
    t = b"  ab\tab\r\n\nc \x0bx\x0b ab\x00 \xff\xff  c"
    exp = {b"ab": 2, b"c": 2, b"\x0bx\x0b": 1, b"ab\x00": 1, b"\xff\xff": 1}
    assert oracle.word_count_text(np.frombuffer(t, dtype=np.uint8)) == exp
    assert oracle.word_count_text(np.zeros(0, dtype=np.uint8)) == {}
    assert oracle.word_count_text(np.frombuffer(b" \n\t\r", dtype=np.uint8)) == {}
    # brute force: Python's regex split on the same separator set
    import re
    rng = random.Random(7)
    for _ in range(20):
        t = bytes(rng.choice(b"ab \n\t\rc\x0b") for _ in range(rng.randrange(0, 300)))
        ref = {}
        for w in re.split(rb"[ \n\t\r]+", t):
            if w:
                ref[w] = ref.get(w, 0) + 1
        assert oracle.word_count_text(np.frombuffer(t, dtype=np.uint8)) == ref
