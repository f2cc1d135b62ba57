"""GPU parity of the fused tokenizer + insert path (sepo_run_text): raw
text in, word counts out, exactly the oracle's (tokenizer reading R20) — in one pass and over
budget, with and without the sampled hot set, through the prepared-list overflow path, from host
memory, and on adversarial texts (separator runs, words across 512-byte windows and longer than
two windows, a text not ending in a separator)."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu


def sepo():
    import paper_conf_ipps_mokhtaris17_b200 as m
    return m


def text_footprint(text, nb=1 << 14, pb=4096):
    """pages an unconstrained sepo_run_text job touches (F of SURVEY §8c reading 23, on the text path:
    the CSR kernels spread records over the CTAs differently, so their F can differ)"""
    _, passes, st = run_text(text, 1 << 14, nb=nb, pb=pb)
    assert passes == 1
    return st["pages_used_max"]


def run_text(text, budget_pages, nb=1 << 14, pb=4096, **kw):
    S = sepo()
    t = S.Table(S.budget_for(nb, pb, budget_pages), nb, pb, check_dups=True, **kw)
    passes = t.run_text(text)
    got = S.result_dict(t.export())
    st = t.stats()
    t.close()
    return got, passes, st


@pytest.mark.parametrize("cfg,scale,ratio", [("C1", 0.25, 0.5), ("C1", 0.25, 4), ("C2", 0.004, 0.5), ("C2", 0.004, 3)])
def test_text_parity(cuda, cfg, scale, ratio):
    s = gen.config(cfg, scale=scale)
    text = s.text_device()
    exp = s.expected_combine()
    assert oracle.word_count_text(s.text_host()) == exp
    pb = 4096 if cfg == "C1" else 16384
    F = text_footprint(text, pb=pb)
    P = int(np.ceil(F / ratio)) + (600 if ratio < 1 else 0)
    got, passes, st = run_text(text, P, pb=pb)
    assert got == exp
    assert st["records_inserted"] >= s.n and st["cross_gen_dups"] == 0
    if ratio > 1:
        assert passes >= 2
        post = st["postponed_per_pass"]
        assert all(post[i] > post[i + 1] for i in range(len(post) - 1)) and post[-1] == 0, post
    else:
        assert passes == 1 and st["records_inserted"] == s.n


def test_text_prepared_overflow(cuda, monkeypatch):
    """declined words beyond the prepared list's capacity go through the text bitmap"""
    monkeypatch.setenv("SEPO_PREP_CAP", "1000")
    s = gen.config("C1", scale=0.25)
    text = s.text_device()
    F = text_footprint(text)
    got, passes, st = run_text(text, max(8, F // 4))
    assert got == s.expected_combine() and passes >= 3


def test_text_from_host(cuda):
    s = gen.config("C1", scale=0.1)
    got, passes, _ = run_text(s.text_host(), 4096)
    assert got == s.expected_combine() and passes == 1


def _dev(b):
    t = torch.empty(len(b) + 64, dtype=torch.uint8, device="cuda")[:len(b)]
    if len(b):
        t.copy_(torch.frombuffer(bytearray(b), dtype=torch.uint8))
    return t


def test_text_adversarial(cuda):
    rng = np.random.default_rng(5)
    parts = [b"  ", b"a" * 15, b" ", b"b" * 17, b"\n", b"x" * 700, b"\t\r", b"\x0bq\x0b", b" "]
    parts += [b"w%d " % i for i in range(200)]
    parts += [b"L" * 1500, b" ", b"y" * 511, b"\n", b"z" * 513, b" end"]  # no final separator
    t = b"".join(parts)
    for shift in (0, 1, 7, 16, 495, 511):  # move every word across the 16- and 512-byte boundaries
        tt = b"\r" * shift + t
        exp = oracle.word_count_text(np.frombuffer(tt, dtype=np.uint8))
        got, passes, _ = run_text(_dev(tt), 256, pb=8192)
        assert got == exp, shift
    # random texts over a small alphabet, many windows, over budget
    for seed in range(3):
        r = np.random.default_rng(seed)
        tt = bytes(r.choice(np.frombuffer(b"abcd  \n\t", dtype=np.uint8), size=200_000))
        exp = oracle.word_count_text(np.frombuffer(tt, dtype=np.uint8))
        got, passes, _ = run_text(_dev(tt), 8, pb=4096, grid_ctas=8)
        assert got == exp
    got, passes, _ = run_text(_dev(b""), 16)
    assert got == {}
    got, passes, _ = run_text(_dev(b" \n \t"), 16)
    assert got == {}


@pytest.mark.parametrize("chunk", [512, 4096, 1 << 20])
def test_text_host_pipelined(cuda, monkeypatch, chunk):
    """host text copied in chunks while earlier chunks are tokenized and inserted (the hot set from
    the first chunk): same counts, including words across chunk ends and an over-budget run"""
    monkeypatch.setenv("SEPO_H2D_TEXT_CHUNK", str(chunk))
    s = gen.config("C1", scale=0.25)
    text = s.text_host()
    exp = s.expected_combine()
    got, passes, _ = run_text(text, 4096)
    assert got == exp and passes == 1
    F = text_footprint(text)  # (same chunked launches as the run below)
    got, passes, _ = run_text(text, max(8, F // 3))
    assert got == exp and passes >= 2
    t = b"".join([b"w%d " % i for i in range(3000)] + [b"L" * 1500, b" ", b"y" * 511, b"\n", b"z" * 513, b" end"])
    exp2 = oracle.word_count_text(np.frombuffer(t, dtype=np.uint8))
    got, _, _ = run_text(np.frombuffer(t, dtype=np.uint8).copy(), 256, pb=8192)
    assert got == exp2


# ---- map runtime (NEXT-4): the paper's applications from raw text (sepo_map_run)
def test_map_lines_page_view_count(cuda):
    """MAP_LINES: one URL per line -> (URL, 1) combined == the oracle's count of the lines"""
    s = gen.config("C3", scale=1 / 8000)
    keys, offs, _ = s.host()
    kb = keys.tobytes()
    lines = [kb[offs[i]:offs[i + 1]] for i in range(s.n)]
    text = b"\n".join(lines) + b"\n\n"
    exp = {}
    for ln in lines:
        exp[ln] = exp.get(ln, 0) + 1
    S = sepo()
    t = S.Table(S.budget_for(1 << 14, 65536, 256), 1 << 14, 65536, check_dups=True)
    d = torch.from_numpy(np.frombuffer(text, dtype=np.uint8).copy()).cuda()
    passes = t.map_run(S.MAP_LINES, d)
    got = S.result_dict(t.export())
    t.close()
    assert passes >= 1 and got == exp
    assert exp == s.expected_combine()


@pytest.mark.parametrize("over", [False, True])
def test_map_word_docs_inverted_index(cuda, over):
    """MAP_WORD_DOCS: documents of words -> (word, doc id) grouped == oracle.group over the same pairs,
    in one pass and over budget"""
    rng = np.random.default_rng(4)
    s = gen.config("C1", scale=0.05)
    text = s.text_host()
    n = len(text)
    cuts = np.sort(rng.choice(np.arange(1, n), size=40, replace=False))
    doc_offsets = np.concatenate([[0], cuts]).astype(np.int64)
    # oracle pairs: every word with the document holding its first byte
    tb = text.tobytes()
    words, docs = [], []
    i = 0
    seps = b" \n\t\r"
    while i < n:
        if tb[i] in seps:
            i += 1
            continue
        j = i
        while j < n and tb[j] not in seps:
            j += 1
        words.append(tb[i:j])
        docs.append(int(np.searchsorted(doc_offsets, i, side="right") - 1))
        i = j
    ko = np.zeros(len(words) + 1, dtype=np.uint64)
    ko[1:] = np.cumsum([len(w) for w in words])
    vals = np.array(docs, dtype=np.uint32).view(np.uint8)
    exp = oracle.group(np.frombuffer(b"".join(words), dtype=np.uint8), ko, vals, val_width=4).as_dict()
    S = sepo()
    dt, dd = torch.from_numpy(text.copy()).cuda(), torch.from_numpy(doc_offsets).cuda()
    t = S.Table(S.budget_for(1 << 14, 4096, 4096), 1 << 14, 4096, mode=S.GROUP, fixed_val_width=4)
    assert t.map_run(S.MAP_WORD_DOCS, dt, dd) == 1
    F = t.stats()["pages_used_max"]
    t.close()
    t = S.Table(S.budget_for(1 << 14, 4096, F // 3 + 2 if over else F + 64), 1 << 14, 4096, mode=S.GROUP,
                fixed_val_width=4, check_dups=True)
    passes = t.map_run(S.MAP_WORD_DOCS, dt, dd)
    got = S.result_dict(t.export(), S.GROUP)
    t.close()
    assert got == exp
    if over:
        assert passes >= 2
