"""Seeded synthetic input streams for the SEPO workloads (test/bench infrastructure).

Record j of a stream is a pure function of (seed, j), computed by the same C code on the host
(`gen_host.cpp`, for the oracle) and on the device (`gen_dev.cu`, for the CUDA path); see
`gen_common.h`. This module holds none of the method's arithmetic. The "exact-count" design
(rank r appears exactly c_r times, shuffled by a seeded bijection) makes the combine result
known by construction, which pins the oracle at any size ("Input recipe").

Configs follow BASELINE.json `configs` / SURVEY.md §8(d):
  C1 word count, 8 MiB text, V = 55,000, Zipf(1.0)
  C2 word count, 8 GiB text, V = 2^22, Zipf(1.0)
  C3 page-view count, 16 GiB click log, U = 2^24 URLs, Zipf(1.0)
  C4 inverted index, 8 GiB of documents (512..1536 words each), V = 2^22, values = u32 doc id
  C5 fixed 8 B keys / 8 B values, 2^31 pairs, uniform over 2^28 keys or Zipf(1.2)
"""
import ctypes
import math
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None

GEN_WORDS, GEN_URLS, GEN_PAIRS = 0, 1, 2


class _Params(ctypes.Structure):
    _fields_ = [("family", ctypes.c_int32), ("with_doc_vals", ctypes.c_int32), ("seed", ctypes.c_uint64),
                ("n", ctypes.c_uint64), ("n_ranks", ctypes.c_uint64), ("uniform_m", ctypes.c_uint64),
                ("cum", ctypes.c_void_p), ("n_docs", ctypes.c_uint64), ("doc_start", ctypes.c_void_p)]


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "libsepogen.so")
        if not os.path.exists(path):
            import importlib.util
            spec = importlib.util.spec_from_file_location("_b", os.path.join(os.path.dirname(_HERE), "tools", "build.py"))
            m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m)
            m.build_gen()
        L = ctypes.CDLL(path)
        P = ctypes.POINTER(_Params)
        u64, vp = ctypes.c_uint64, ctypes.c_void_p
        L.gen_key_lens_of_ranks_host.argtypes = [P, u64, u64, vp]
        L.gen_spell_rank_host.argtypes = [P, u64, vp]; L.gen_spell_rank_host.restype = ctypes.c_uint32
        L.gen_ranks_host.argtypes = [P, u64, u64, vp]
        L.gen_perm_inv_host.argtypes = [P, vp, u64, vp]
        L.gen_perm_host.argtypes = [P, vp, u64, vp]
        L.gen_vals_of_records_host.argtypes = [P, vp, u64, vp]
        L.gen_offsets_host.argtypes = [P, u64, u64, vp]; L.gen_offsets_host.restype = u64
        L.gen_keys_host.argtypes = [P, u64, u64, vp, vp, vp]
        L.gen_doc_lens_host.argtypes = [u64, u64, u64, vp]
        L.gen_offsets_dev.argtypes = [P, u64, u64, vp, vp, u64, vp]; L.gen_offsets_dev.restype = ctypes.c_int64
        L.gen_keys_dev.argtypes = [P, u64, u64, vp, vp, vp, vp]; L.gen_keys_dev.restype = ctypes.c_int
        L.gen_ranks_dev.argtypes = [P, u64, u64, vp, vp]; L.gen_ranks_dev.restype = ctypes.c_int
        L.gen_text_dev.argtypes = [P, u64, u64, vp, vp, vp, vp]; L.gen_text_dev.restype = ctypes.c_int
        L.gen_text_host.argtypes = [P, u64, u64, vp, vp, vp]
        L.gen_key_ranks_host.argtypes = [P, vp, vp, u64, vp]
        L.gen_rank_digest_host.argtypes = [P, u64, u64, vp, vp, vp]
        L.gen_list_digest_host.argtypes = [vp, vp, vp, u64, vp, vp, vp]
        _LIB = L
    return _LIB


def _ptr(a):
    return ctypes.c_void_p(a.ctypes.data) if a is not None else None


class Stream:
    """One synthetic record stream (see module doc). Values: 'one' (implicit 1, no value
    array), 'u64' (8 B LE per record, PAIRS), 'doc' (4 B LE u32 doc id per record)."""

    def __init__(self, name, family, seed, counts=None, uniform=None, docs=False):
        self.name, self.family, self.seed = name, family, int(seed)
        if uniform is not None:
            n_ranks, m = uniform
            self.uniform_m, self.n_ranks = int(m), int(n_ranks)
            self.cum = None
            self.n = self.n_ranks * self.uniform_m
        else:
            counts = np.asarray(counts, dtype=np.uint64)
            nz = np.nonzero(counts)[0]
            last = int(nz[-1]) + 1 if len(nz) else 0
            counts = counts[:last]
            self.uniform_m, self.n_ranks = 0, last
            self.cum = np.zeros(last + 1, dtype=np.uint64)
            np.cumsum(counts, out=self.cum[1:])
            self.n = int(self.cum[-1])
        self.docs = bool(docs)
        self.doc_start = None
        if docs:
            # documents of 512..1536 words, laid out consecutively; the last one truncated at n
            est = self.n // 1024 + 16
            lens = np.empty(est, dtype=np.uint64)
            lib().gen_doc_lens_host(self.seed, 0, est, _ptr(lens))
            starts = np.zeros(est + 1, dtype=np.uint64)
            np.cumsum(lens, out=starts[1:])
            nd = int(np.searchsorted(starts, self.n, side="left"))
            nd = max(nd, 1)
            self.doc_start = np.concatenate([starts[:nd], np.array([self.n], dtype=np.uint64)])
            self.n_docs = nd
        else:
            self.n_docs = 0
        self.val = "u64" if family == GEN_PAIRS else ("doc" if docs else "one")
        self._dev = {}

    # ---- parameter blocks ----
    def params(self, device=None):
        if device is None:
            cum, ds = self.cum, self.doc_start
            cp = cum.ctypes.data if cum is not None else None
            dp = ds.ctypes.data if ds is not None else None
        else:
            import torch
            key = str(device)
            if key not in self._dev:
                c = torch.from_numpy(self.cum.view(np.int64)).to(device) if self.cum is not None else None
                d = torch.from_numpy(self.doc_start.view(np.int64)).to(device) if self.doc_start is not None else None
                self._dev[key] = (c, d)
            c, d = self._dev[key]
            cp = c.data_ptr() if c is not None else None
            dp = d.data_ptr() if d is not None else None
        return _Params(self.family, 1 if self.docs else 0, self.seed, self.n, self.n_ranks, self.uniform_m,
                       cp, self.n_docs, dp)

    @property
    def val_width(self):
        return {"one": 0, "u64": 8, "doc": 4}[self.val]

    # ---- host generation (oracle side) ----
    def host(self, j0=0, cnt=None):
        """-> (keys u8[], offs u64[cnt+1] rebased to 0, vals u8[] or None)"""
        if cnt is None:
            cnt = self.n - j0
        assert 0 <= j0 and j0 + cnt <= self.n
        p = self.params()
        offs = np.empty(cnt + 1, dtype=np.uint64)
        total = lib().gen_offsets_host(ctypes.byref(p), j0, cnt, _ptr(offs))
        keys = np.empty(max(int(total), 1), dtype=np.uint8)[: int(total)]
        vals = np.empty(cnt * self.val_width, dtype=np.uint8) if self.val_width else None
        lib().gen_keys_host(ctypes.byref(p), j0, cnt, _ptr(offs), _ptr(keys) if total else ctypes.c_void_p(0), _ptr(vals))
        return keys, offs, vals

    # ---- device generation (CUDA side) ----
    def device(self, j0=0, cnt=None, device="cuda", stream=None):
        """-> (keys u8 tensor, offs int64 tensor [cnt+1], vals u8 tensor or None) on `device`."""
        import torch
        if cnt is None:
            cnt = self.n - j0
        L = lib()
        p = self.params(device)
        s = torch.cuda.current_stream(device) if stream is None else stream
        offs = torch.empty(cnt + 1, dtype=torch.int64, device=device)
        need = L.gen_offsets_dev(ctypes.byref(p), j0, cnt, None, None, 0, ctypes.c_void_p(s.cuda_stream))
        tmp = torch.empty(max(int(need), 1), dtype=torch.uint8, device=device)
        rc = L.gen_offsets_dev(ctypes.byref(p), j0, cnt, offs.data_ptr(), tmp.data_ptr(), int(need), ctypes.c_void_p(s.cuda_stream))
        assert rc == 0, rc
        total = int(offs[-1].item())
        keys = torch.empty(max(total, 1), dtype=torch.uint8, device=device)
        vals = torch.empty(cnt * self.val_width, dtype=torch.uint8, device=device) if self.val_width else None
        rc = L.gen_keys_dev(ctypes.byref(p), j0, cnt, offs.data_ptr(), keys.data_ptr(),
                            vals.data_ptr() if vals is not None else None, ctypes.c_void_p(s.cuda_stream))
        assert rc == 0, rc
        return keys[:total], offs, vals

    def text_host(self, j0=0, cnt=None):
        """Raw text of a word/URL stream: each key followed by one separator (' ' or '\n')."""
        keys, offs, _ = self.host(j0, cnt)
        n = len(offs) - 1
        text = np.empty(len(keys) + n, dtype=np.uint8)
        lib().gen_text_host(ctypes.byref(self.params()), j0, n, _ptr(np.ascontiguousarray(offs, dtype=np.uint64)),
                            _ptr(keys), _ptr(text))
        return text

    def text_device(self, j0=0, cnt=None, device="cuda"):
        """Raw text on the device (16-byte aligned torch allocation), same bytes as text_host."""
        import torch
        keys, offs, _ = self.device(j0, cnt, device)
        n = offs.numel() - 1
        text = torch.empty(keys.numel() + n, dtype=torch.uint8, device=device)
        s = torch.cuda.current_stream(device)
        rc = lib().gen_text_dev(ctypes.byref(self.params(device)), j0, n, offs.data_ptr(), keys.data_ptr(),
                                text.data_ptr(), ctypes.c_void_p(s.cuda_stream))
        assert rc == 0, rc
        del keys, offs
        return text

    def ranks_host(self, j0=0, cnt=None):
        if cnt is None:
            cnt = self.n - j0
        out = np.empty(cnt, dtype=np.uint64)
        lib().gen_ranks_host(ctypes.byref(self.params()), j0, cnt, _ptr(out))
        return out

    # ---- closed forms (by construction of the exact-count stream) ----
    def count_of_rank(self, r):
        r = np.asarray(r, dtype=np.int64)
        if self.uniform_m:
            return np.full(r.shape, self.uniform_m, dtype=np.uint64)
        return (self.cum[r] - self.cum[r - 1]).astype(np.uint64)

    def spell(self, r):
        buf = ctypes.create_string_buffer(256)
        L = lib().gen_spell_rank_host(ctypes.byref(self.params()), int(r), buf)
        return buf.raw[:L]

    def key_lens_of_ranks(self, r0=1, cnt=None):
        if cnt is None:
            cnt = self.n_ranks - r0 + 1
        out = np.empty(cnt, dtype=np.uint32)
        lib().gen_key_lens_of_ranks_host(ctypes.byref(self.params()), r0, cnt, _ptr(out))
        return out

    def records_of_rank(self, r):
        """Record indices j holding rank r: perm^{-1} of the multiset block of r."""
        if self.uniform_m:
            lo, hi = (r - 1) * self.uniform_m, r * self.uniform_m
        else:
            lo, hi = int(self.cum[r - 1]), int(self.cum[r])
        idx = np.arange(lo, hi, dtype=np.uint64)
        out = np.empty(len(idx), dtype=np.uint64)
        lib().gen_perm_inv_host(ctypes.byref(self.params()), _ptr(idx), len(idx), _ptr(out))
        return out

    def values_of_records(self, j):
        j = np.ascontiguousarray(j, dtype=np.uint64)
        out = np.empty(len(j), dtype=np.uint64)
        lib().gen_vals_of_records_host(ctypes.byref(self.params()), _ptr(j), len(j), _ptr(out))
        return out

    def expected_combine(self):
        """Closed-form combine result {key bytes: value}: value = c_r for implicit-1 streams,
        = sum of the record values of rank r (mod 2^64) for PAIRS. Small streams only."""
        out = {}
        for r in range(1, self.n_ranks + 1):
            if self.val == "one":
                v = int(self.count_of_rank(r))
            else:
                v = int(self.values_of_records(self.records_of_rank(r)).sum(dtype=np.uint64))
            if v or self.val != "one":
                out[self.spell(r)] = v
        return out

    def expected_group(self, r):
        """Closed-form value multiset of rank r (sorted list of doc ids / values)."""
        return sorted(int(v) for v in self.values_of_records(self.records_of_rank(r)))

    # ---- full-size checks (closed forms evaluated backwards; host C, OpenMP) ----
    def key_ranks(self, keys, offs):
        """rank spelled by each key of a CSR key set (0: no rank spells it)"""
        keys = np.ascontiguousarray(keys, dtype=np.uint8)
        offs = np.ascontiguousarray(offs, dtype=np.uint64)
        n = len(offs) - 1
        out = np.empty(n, dtype=np.uint64)
        if n:
            lib().gen_key_ranks_host(ctypes.byref(self.params()), _ptr(keys) if len(keys) else None, _ptr(offs), n, _ptr(out))
        return out

    def rank_digest(self, r0=1, cnt=None):
        """per rank r0..: (record count, sum of record values mod 2^64, sum of mix(value) mod 2^64)
        over the records that hold the rank — the exact combine sum (PAIRS) or a digest of the
        exact value multiset (doc ids)"""
        if cnt is None:
            cnt = self.n_ranks - r0 + 1
        c, sm, mx = (np.empty(cnt, dtype=np.uint64) for _ in range(3))
        lib().gen_rank_digest_host(ctypes.byref(self.params()), r0, cnt, _ptr(c), _ptr(sm), _ptr(mx))
        return c, sm, mx

    def raw_bytes(self):
        """Bytes of the raw dataset: text with one separator per word (WORDS/URLS), 16 B per pair."""
        if self.family == GEN_PAIRS:
            return 16 * self.n
        lens = self.key_lens_of_ranks().astype(np.uint64)
        cnt = self.count_of_rank(np.arange(1, self.n_ranks + 1))
        return int(((lens + 1) * cnt).sum())


# ---------------------------------------------------------------- stream constructors
def zipf_counts(V, C, alpha=1.0):
    r = np.arange(1, V + 1, dtype=np.uint64)
    if alpha == 1.0:
        return np.uint64(C) // r
    return np.floor(float(C) / np.power(r.astype(np.float64), alpha)).astype(np.uint64)


def _fit_C(V, alpha, target, lens_plus):
    """Largest C with sum_r c_r * lens_plus[r] <= target (c_r = floor(C / r^alpha))."""
    lo, hi = 1, 1
    def size(C):
        return int((zipf_counts(V, C, alpha) * lens_plus).sum())
    while size(hi) <= target:
        hi *= 2
    while lo < hi - 1:
        mid = (lo + hi) // 2
        if size(mid) <= target:
            lo = mid
        else:
            hi = mid
    return lo


def words_stream(name, V, text_bytes, seed, alpha=1.0, docs=False):
    probe = Stream("probe", GEN_WORDS, seed, counts=np.ones(V, dtype=np.uint64))
    lens_plus = probe.key_lens_of_ranks().astype(np.uint64) + 1
    C = _fit_C(V, alpha, text_bytes, lens_plus)
    return Stream(name, GEN_WORDS, seed, counts=zipf_counts(V, C, alpha), docs=docs)


def urls_stream(name, U, log_bytes, seed, alpha=1.0):
    probe = Stream("probe", GEN_URLS, seed, counts=np.ones(U, dtype=np.uint64))
    lens_plus = probe.key_lens_of_ranks().astype(np.uint64) + 1
    C = _fit_C(U, alpha, log_bytes, lens_plus)
    return Stream(name, GEN_URLS, seed, counts=zipf_counts(U, C, alpha))


def pairs_stream(name, D, n, seed, alpha=None):
    if alpha is None:
        assert n % D == 0
        return Stream(name, GEN_PAIRS, seed, uniform=(D, n // D))
    C = _fit_C(D, alpha, n, np.ones(D, dtype=np.uint64))
    return Stream(name, GEN_PAIRS, seed, counts=zipf_counts(D, C, alpha))


GiB, MiB = 1 << 30, 1 << 20


def config(name, scale=1.0):
    """BASELINE.json configs as streams. `scale` shrinks the data size (tests)."""
    if name == "C1":
        return words_stream("C1", 55_000, int(8 * MiB * scale), seed=1)
    if name == "C2":
        return words_stream("C2", 1 << 22, int(8 * GiB * scale), seed=2)
    if name == "C3":
        return urls_stream("C3", 1 << 24, int(16 * GiB * scale), seed=3)
    if name == "C4":
        return words_stream("C4", 1 << 22, int(8 * GiB * scale), seed=4, docs=True)
    if name == "C5u":
        D = max(1, int((1 << 28) * scale))
        return pairs_stream("C5u", D, 8 * D, seed=5)
    if name == "C5z":
        D = max(16, int((1 << 28) * scale))
        return pairs_stream("C5z", D, 8 * D, seed=6, alpha=1.2)
    raise KeyError(name)


def list_digest(vals, val_offs, list_offs):
    """(count, sum, sum of mix) per key of exported value lists, the same digest as
    Stream.rank_digest (values = little-endian integers of their bytes)"""
    vals = np.ascontiguousarray(vals, dtype=np.uint8)
    vo = np.ascontiguousarray(val_offs, dtype=np.uint64)
    lo = np.ascontiguousarray(list_offs, dtype=np.uint64)
    n = len(lo) - 1
    c, sm, mx = (np.empty(n, dtype=np.uint64) for _ in range(3))
    if n:
        lib().gen_list_digest_host(_ptr(vals) if len(vals) else None, _ptr(vo), _ptr(lo), n, _ptr(c), _ptr(sm), _ptr(mx))
    return c, sm, mx
