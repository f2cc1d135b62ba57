"""Python binding of the CPU oracle (oracle.cpp). TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / `--impl reference` legs may
import this. The product package (paper_conf_ipps_mokhtaris17_b200) never does. Every function
here is the plain definition the paper fixes — see the citations in oracle.cpp.
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = None
vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(_HERE, "liboracle.so")
        if not os.path.exists(path) or os.path.getmtime(path) < os.path.getmtime(os.path.join(_HERE, "oracle.cpp")):
            import importlib.util
            spec = importlib.util.spec_from_file_location("_b", os.path.join(os.path.dirname(_HERE), "tools", "build.py"))
            m = importlib.util.module_from_spec(spec); spec.loader.exec_module(m)
            m.build_oracle()
        L = ctypes.CDLL(path)
        L.oracle_combine_new.restype = vp
        L.oracle_combine_free.argtypes = [vp]
        L.oracle_combine_add.argtypes = [vp, vp, vp, vp, u32, u64]
        L.oracle_combine_add_text.argtypes = [vp, vp, u64]
        L.oracle_combine_size.argtypes = [vp, vp]; L.oracle_combine_size.restype = u64
        L.oracle_combine_result.argtypes = [vp, vp, vp, vp]
        L.oracle_group_new.restype = vp
        L.oracle_group_free.argtypes = [vp]
        L.oracle_group_add.argtypes = [vp, vp, vp, vp, vp, u32, u64]
        L.oracle_group_size.argtypes = [vp, vp, vp, vp]; L.oracle_group_size.restype = u64
        L.oracle_group_result.argtypes = [vp, vp, vp, vp, vp, vp]
        L.oracle_compact.argtypes = [vp, vp, vp, vp, u32, u64, vp, vp, vp, vp, vp]; L.oracle_compact.restype = u64
        L.oracle_sepo_sim_combine.argtypes = [vp, vp, vp, u32, u64, u64, u64, vp, u64, vp, vp]
        L.oracle_sepo_sim_combine.restype = ctypes.c_int64
        L.oracle_sepo_sim_group.argtypes = [vp, vp, vp, vp, u32, u64, u64, u64, u64, vp, u64, vp, vp]
        L.oracle_sepo_sim_group.restype = ctypes.c_int64
        _LIB = L
    return _LIB


def _p(a):
    if a is None:
        return None
    a = np.ascontiguousarray(a)
    return ctypes.c_void_p(a.ctypes.data) if a.size else ctypes.c_void_p(0)


def _u8(a):
    return np.ascontiguousarray(np.frombuffer(a, dtype=np.uint8) if isinstance(a, (bytes, bytearray)) else a, dtype=np.uint8)


class Combine:
    """Streaming combining group-by: m[key] += value (mod 2^64)."""

    def __init__(self):
        self.h = lib().oracle_combine_new()

    def __del__(self):
        if getattr(self, "h", None):
            lib().oracle_combine_free(self.h)
            self.h = None

    def add(self, keys, offs, vals=None, val_width=0):
        keys, offs = _u8(keys), np.ascontiguousarray(offs, dtype=np.uint64)
        n = len(offs) - 1
        v = _u8(vals) if vals is not None else None
        lib().oracle_combine_add(self.h, _p(keys), _p(offs), _p(v), val_width if v is not None else 0, n)
        return self

    def add_text(self, text):
        """raw text: every word (maximal run of bytes other than ' ', '\n', '\t', '\r') adds 1"""
        t = _u8(text)
        lib().oracle_combine_add_text(self.h, _p(t), len(t))
        return self

    def result(self):
        """canonical (keys u8, offs u64[k+1], values u64[k]) sorted by key bytes"""
        kb = ctypes.c_uint64()
        k = lib().oracle_combine_size(self.h, ctypes.byref(kb))
        keys = np.empty(kb.value, dtype=np.uint8)
        offs = np.empty(k + 1, dtype=np.uint64)
        vals = np.empty(k, dtype=np.uint64)
        lib().oracle_combine_result(self.h, _p(keys), _p(offs), _p(vals))
        return keys, offs, vals

    def as_dict(self):
        keys, offs, vals = self.result()
        kb = keys.tobytes()
        return {kb[offs[i]:offs[i + 1]]: int(vals[i]) for i in range(len(vals))}


class Group:
    """Streaming multi-valued group-by: m[key].append(value)."""

    def __init__(self):
        self.h = lib().oracle_group_new()

    def __del__(self):
        if getattr(self, "h", None):
            lib().oracle_group_free(self.h)
            self.h = None

    def add(self, keys, offs, vals, val_offs=None, val_width=0):
        keys, offs = _u8(keys), np.ascontiguousarray(offs, dtype=np.uint64)
        vo = np.ascontiguousarray(val_offs, dtype=np.uint64) if val_offs is not None else None
        lib().oracle_group_add(self.h, _p(keys), _p(offs), _p(_u8(vals)), _p(vo), val_width, len(offs) - 1)
        return self

    def result(self):
        kb, nv, vb = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint64()
        k = lib().oracle_group_size(self.h, ctypes.byref(kb), ctypes.byref(nv), ctypes.byref(vb))
        keys = np.empty(kb.value, dtype=np.uint8); offs = np.empty(k + 1, dtype=np.uint64)
        lo = np.empty(k + 1, dtype=np.uint64)
        vals = np.empty(vb.value, dtype=np.uint8); vo = np.empty(nv.value + 1, dtype=np.uint64)
        lib().oracle_group_result(self.h, _p(keys), _p(offs), _p(lo), _p(vals), _p(vo))
        return keys, offs, lo, vals, vo

    def as_dict(self):
        keys, offs, lo, vals, vo = self.result()
        kb, vb = keys.tobytes(), vals.tobytes()
        out = {}
        for i in range(len(offs) - 1):
            out[kb[offs[i]:offs[i + 1]]] = [vb[vo[j]:vo[j + 1]] for j in range(lo[i], lo[i + 1])]
        return out


def combine(keys, offs, vals=None, val_width=0):
    return Combine().add(keys, offs, vals, val_width)


def word_count_text(text):
    """{word bytes: occurrences} of raw text (combining method, reading R20)."""
    return Combine().add_text(text).as_dict()


def group(keys, offs, vals, val_offs=None, val_width=0):
    return Group().add(keys, offs, vals, val_offs, val_width)


def basic(keys, offs, vals=None, val_width=0):
    """Basic organization ("Two KV pairs with the same key are stored as two separate
    entries"): the table holds exactly the input multiset of (key, value) pairs. Canonical form:
    {key bytes: sorted list of values}. Values as the combining method reads them: width 0 -> 1
    (P:L73), else val_width little-endian bytes per record. Plain loop (small inputs only)."""
    keys = _u8(keys).tobytes()
    offs = np.asarray(offs, dtype=np.uint64)
    n = len(offs) - 1
    if val_width:
        v = np.frombuffer(_u8(vals).tobytes()[: n * val_width], dtype=np.uint8).reshape(n, val_width)
        vv = [int.from_bytes(v[i].tobytes(), "little") for i in range(n)]
    else:
        vv = [1] * n
    out = {}
    for i in range(n):
        out.setdefault(keys[int(offs[i]):int(offs[i + 1])], []).append(vv[i])
    return {k: sorted(x) for k, x in out.items()}


def compact(keys, offs, bitmap, vals=None, val_offs=None, val_width=0):
    """Gather the records whose bitmap bit is 1 -> (keys, offs, vals, val_offs, m)."""
    keys, offs = _u8(keys), np.ascontiguousarray(offs, dtype=np.uint64)
    n = len(offs) - 1
    bm = np.ascontiguousarray(bitmap, dtype=np.uint32)
    ok = np.empty(max(len(keys), 1), dtype=np.uint8)
    oo = np.empty(n + 1, dtype=np.uint64)
    v = _u8(vals) if vals is not None else None
    vo = np.ascontiguousarray(val_offs, dtype=np.uint64) if val_offs is not None else None
    ov = np.empty(max(len(v), 1), dtype=np.uint8) if v is not None else None
    ovo = np.empty(n + 1, dtype=np.uint64) if vo is not None else None
    m = lib().oracle_compact(_p(keys), _p(offs), _p(v), _p(vo), val_width, n, _p(bm), _p(ok), _p(oo), _p(ov), _p(ovo))
    m = int(m)
    kb = int(oo[m])
    outv = None
    if v is not None:
        outv = ov[: int(ovo[m])] if vo is not None else ov[: m * val_width]
    return ok[:kb], oo[: m + 1], outv, (ovo[: m + 1] if vo is not None else None), m


def sepo_sim_combine(keys, offs, heap_bytes, overhead=24, vals=None, val_width=0, max_passes=256):
    """Sequential SEPO combining loop. -> (passes, postponed[], Combine, dup_keys)"""
    keys, offs = _u8(keys), np.ascontiguousarray(offs, dtype=np.uint64)
    post = np.zeros(max_passes, dtype=np.uint64)
    out = Combine()
    dups = ctypes.c_uint64()
    v = _u8(vals) if vals is not None else None
    p = lib().oracle_sepo_sim_combine(_p(keys), _p(offs), _p(v), val_width if v is not None else 0, len(offs) - 1,
                                      heap_bytes, overhead, _p(post), max_passes, out.h, ctypes.byref(dups))
    return int(p), post[: max(int(p), 0)].tolist(), out, dups.value


def sepo_sim_group(keys, offs, vals, heap_bytes, val_offs=None, val_width=0, key_overhead=24, val_overhead=0,
                   max_passes=256):
    """Sequential SEPO multi-valued loop. -> (passes, postponed[], Group, forced_full)"""
    keys, offs = _u8(keys), np.ascontiguousarray(offs, dtype=np.uint64)
    post = np.zeros(max_passes, dtype=np.uint64)
    out = Group()
    ff = ctypes.c_uint64()
    vo = np.ascontiguousarray(val_offs, dtype=np.uint64) if val_offs is not None else None
    p = lib().oracle_sepo_sim_group(_p(keys), _p(offs), _p(_u8(vals)), _p(vo), val_width, len(offs) - 1, heap_bytes,
                                    key_overhead, val_overhead, _p(post), max_passes, out.h, ctypes.byref(ff))
    return int(p), post[: max(int(p), 0)].tolist(), out, ff.value
