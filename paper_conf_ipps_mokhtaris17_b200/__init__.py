"""Python binding of the B200-native SEPO hash table (C ABI in include/sepo.h).

Argument marshalling only: every step of the hot path runs in lib/libsepo.so's sm_100a kernels.
There is no fallback — if the library is missing or CUDA is unavailable, construction raises.
Tensors passed in are used in place (their data_ptr()); numpy arrays are host memory and are
streamed to the device by the library (sepo_run only).
"""
import ctypes
import os

import numpy as np

__all__ = ["Table", "SepoError", "lib", "COMBINE", "GROUP", "Stats"]

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SEPO_LIB") or os.path.join(_HERE, "lib", "libsepo.so")
COMBINE, GROUP, BASIC = 0, 1, 2  # sepo_mode (include/sepo.h)
_LIB = None

vp, u64, u32, i64 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_int64


class Options(ctypes.Structure):
    _fields_ = [("mode", ctypes.c_int32), ("fixed_key_width", u32), ("fixed_val_width", u32), ("grid_ctas", u32),
                ("hash_seed", u64), ("fail_alloc_ppm", u32), ("fail_mode", u32), ("fail_until_pass", u32),
                ("check_dups", u32), ("stream", vp), ("host_arena_bytes", u64), ("basic_halt_pct", u32),
                ("pad_", u32)]


class Result(ctypes.Structure):
    _fields_ = [("n_keys", u64), ("keys", vp), ("key_offsets", vp), ("values", vp), ("list_offsets", vp),
                ("n_vals", u64), ("vals", vp), ("val_offsets", vp)]


MAXP = 64


class Stats(ctypes.Structure):
    _fields_ = [("passes", u64), ("insert_calls", u64), ("records_inserted", u64), ("postponed_per_pass", u64 * MAXP),
                ("n_buckets", u64), ("page_bytes", u64), ("pool_pages", u64), ("grid_ctas", u64),
                ("pages_used_max", u64), ("bytes_evicted", u64), ("dead_bytes", u64), ("cross_gen_dups", u64),
                ("forced_full_evictions", u64), ("toolarge", u64),
                ("key_bytes_inserted", u64), ("val_bytes_inserted", u64), ("kernel_launches", u64), ("value_chunks", u64), ("value_slots", u64), ("t_insert_ms", ctypes.c_double),
                ("t_reprobe_ms", ctypes.c_double), ("t_compact_ms", ctypes.c_double), ("t_evict_ms", ctypes.c_double),
                ("t_export_ms", ctypes.c_double), ("t_h2d_ms", ctypes.c_double),
                ("t_insert_ms_per_pass", ctypes.c_double * MAXP), ("hot_keys", u64),
                ("p2p_chunks", u64)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_ if k not in ("postponed_per_pass", "t_insert_ms_per_pass")}
        d["postponed_per_pass"] = list(self.postponed_per_pass[: min(int(self.passes), MAXP)])
        d["t_insert_ms_per_pass"] = list(self.t_insert_ms_per_pass[: min(max(int(self.passes), 1), MAXP)])
        return d


class SepoError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"sepo error {code}: {msg}")
        self.code = code


E_INVAL, E_NOMEM, E_TOOLARGE, E_CUDA, E_STATE, E_NCCL = -1, -2, -3, -4, -5, -6
POOL_DEVICE, POOL_HOST_PINNED, POOL_MANAGED = 0, 1, 2  # sepo_create_placed (include/sepo.h)
MAP_WORDS, MAP_LINES, MAP_WORD_DOCS = 0, 1, 2  # sepo_map_run mappers (include/sepo.h)

# every entry point declared in include/sepo.h
EXPORTS = ["sepo_create", "sepo_create_placed", "sepo_configure", "sepo_run_text", "sepo_lookup", "sepo_insert_batch", "sepo_reprobe", "sepo_compact", "sepo_evict",
           "sepo_export", "sepo_run", "sepo_reset", "sepo_stats_get", "sepo_last_insert_ms", "sepo_destroy",
           "sepo_last_error", "sepo_version", "sepo_budget_for", "sepo_partition_scratch", "sepo_partition",
           "sepo_shift_offsets", "sepo_route_scratch", "sepo_route_combine", "sepo_run_wire", "sepo_nccl_unique_id",
           "sepo_attach_nccl", "sepo_insert_batch_sharded", "sepo_drain", "sepo_map_run",
           "sepo_run_sharded"]


def nccl_unique_id():
    """128-byte NCCL unique id (rank 0 creates it; broadcast it to the other ranks)"""
    buf = ctypes.create_string_buffer(128)
    rc = lib().sepo_nccl_unique_id(buf)
    if rc:
        _err(rc)
    return buf.raw


def budget_for(n_buckets, page_bytes, pool_pages):
    """device budget that gives a pool of exactly `pool_pages` pages (host arithmetic)"""
    return int(lib().sepo_budget_for(int(n_buckets), int(page_bytes), int(pool_pages)))


def lib():
    """Load lib/libsepo.so (raises if it has not been built)."""
    global _LIB
    if _LIB is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run `python tools/build.py` (no CPU fallback exists)")
        L = ctypes.CDLL(LIB_PATH)
        L.sepo_create.argtypes = [ctypes.c_size_t, u64, u32]; L.sepo_create.restype = vp
        L.sepo_create_placed.argtypes = [ctypes.c_size_t, u64, u32, ctypes.c_int]; L.sepo_create_placed.restype = vp
        L.sepo_configure.argtypes = [vp, ctypes.POINTER(Options)]; L.sepo_configure.restype = ctypes.c_int
        L.sepo_insert_batch.argtypes = [vp, vp, vp, vp, vp, u64, vp]; L.sepo_insert_batch.restype = i64
        L.sepo_reprobe.argtypes = [vp, vp, vp, vp, vp, u64, vp, vp, vp]; L.sepo_reprobe.restype = i64
        L.sepo_compact.argtypes = [vp, vp, vp, vp, vp, u64, vp, vp, vp, vp, vp]; L.sepo_compact.restype = i64
        L.sepo_evict.argtypes = [vp]; L.sepo_evict.restype = i64
        L.sepo_export.argtypes = [vp, ctypes.POINTER(Result)]; L.sepo_export.restype = ctypes.c_int
        L.sepo_run.argtypes = [vp, vp, vp, vp, vp, u64]; L.sepo_run.restype = i64
        L.sepo_run_text.argtypes = [vp, vp, u64]; L.sepo_run_text.restype = i64
        L.sepo_lookup.argtypes = [vp, vp, vp, u64, vp, vp]; L.sepo_lookup.restype = i64
        L.sepo_reset.argtypes = [vp]; L.sepo_reset.restype = ctypes.c_int
        L.sepo_stats_get.argtypes = [vp, ctypes.POINTER(Stats)]; L.sepo_stats_get.restype = ctypes.c_int
        L.sepo_last_insert_ms.argtypes = [vp]; L.sepo_last_insert_ms.restype = ctypes.c_double
        L.sepo_destroy.argtypes = [vp]; L.sepo_destroy.restype = None
        L.sepo_last_error.restype = ctypes.c_char_p
        L.sepo_version.restype = ctypes.c_char_p
        L.sepo_budget_for.argtypes = [u64, u32, u64]; L.sepo_budget_for.restype = ctypes.c_size_t
        L.sepo_run_wire.argtypes = [vp, vp, u64]; L.sepo_run_wire.restype = i64
        L.sepo_nccl_unique_id.argtypes = [vp]; L.sepo_nccl_unique_id.restype = ctypes.c_int
        L.sepo_attach_nccl.argtypes = [vp, vp, ctypes.c_int, ctypes.c_int]; L.sepo_attach_nccl.restype = ctypes.c_int
        L.sepo_insert_batch_sharded.argtypes = [vp, vp, vp, vp, vp, u64]; L.sepo_insert_batch_sharded.restype = i64
        L.sepo_drain.argtypes = [vp]; L.sepo_drain.restype = i64
        L.sepo_run_sharded.argtypes = [vp, vp, vp, vp, vp, u64]; L.sepo_run_sharded.restype = i64
        L.sepo_map_run.argtypes = [vp, ctypes.c_int, vp, u64, vp, u64]; L.sepo_map_run.restype = i64
        _LIB = L
    return _LIB


def _err(rc):
    raise SepoError(rc, lib().sepo_last_error().decode())


def _ptr(x):
    """device tensor -> data_ptr; numpy array -> host address; None -> NULL"""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        return x.ctypes.data if x.size else None
    return x.data_ptr() if x.numel() else None


class Table:
    """One SEPO hash table on the current CUDA device (one per GPU)."""

    def __init__(self, budget_bytes, n_buckets, page_bytes=65536, mode=COMBINE, fixed_key_width=0,
                 fixed_val_width=0, grid_ctas=0, hash_seed=0, fail_alloc_ppm=0, fail_mode=0, fail_until_pass=0,
                 check_dups=False, stream=None, host_arena_bytes=0, placement=0, basic_halt_pct=0):
        import torch
        if not torch.cuda.is_available():
            raise RuntimeError("paper_conf_ipps_mokhtaris17_b200 needs a CUDA device (no CPU fallback)")
        L = lib()
        self._L = L
        if placement == POOL_DEVICE:
            self.h = L.sepo_create(int(budget_bytes), int(n_buckets), int(page_bytes))
        else:  # residency ablations (NEXT-1): pool in pinned host / managed memory
            self.h = L.sepo_create_placed(int(budget_bytes), int(n_buckets), int(page_bytes), int(placement))
        if not self.h:
            raise SepoError(E_NOMEM, L.sepo_last_error().decode())
        if stream is None:
            stream = torch.cuda.current_stream()
        self.mode = mode
        self.opts = Options(mode, fixed_key_width, fixed_val_width or (8 if mode != GROUP else 0), grid_ctas,
                            hash_seed, fail_alloc_ppm, fail_mode, fail_until_pass, int(bool(check_dups)),
                            ctypes.c_void_p(stream.cuda_stream), int(host_arena_bytes), int(basic_halt_pct), 0)
        rc = L.sepo_configure(self.h, ctypes.byref(self.opts))
        if rc:
            L.sepo_destroy(self.h)
            self.h = None
            _err(rc)
        self.val_width = self.opts.fixed_val_width

    def close(self):
        if getattr(self, "h", None):
            self._L.sepo_destroy(self.h)
            self.h = None

    __del__ = close

    # ---- the fine-grained SEPO calls (the requestor drives the pass loop)
    def insert_batch(self, keys, key_offsets, vals=None, bitmap=None, n=None, val_offsets=None):
        n = self._n(key_offsets, keys, n)
        if bitmap is None:
            import torch
            bitmap = torch.empty(max((n + 31) // 32, 1), dtype=torch.int32, device="cuda")
        rc = self._L.sepo_insert_batch(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), _ptr(val_offsets), n,
                                       _ptr(bitmap))
        if rc < 0:
            _err(rc)
        return int(rc), bitmap

    def reprobe(self, keys, key_offsets, vals, bitmap, n=None):
        n = self._n(key_offsets, keys, n)
        kb, vb = ctypes.c_uint64(), ctypes.c_uint64()
        rc = self._L.sepo_reprobe(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), None, n, _ptr(bitmap),
                                  ctypes.byref(kb), ctypes.byref(vb))
        if rc < 0:
            _err(rc)
        return int(rc), kb.value, vb.value

    def compact(self, keys, key_offsets, vals, bitmap, n=None):
        """-> (keys, key_offsets or None, vals or None, m) as new device tensors"""
        import torch
        n = self._n(key_offsets, keys, n)
        # size the outputs exactly: a count-only pass is inside sepo_compact; here use upper bounds
        kcap = keys.numel()
        ok = torch.empty(max(kcap, 1), dtype=torch.uint8, device="cuda")
        oko = torch.empty(n + 1, dtype=torch.int64, device="cuda") if key_offsets is not None else None
        ov = torch.empty(max(vals.numel(), 1), dtype=torch.uint8, device="cuda") if vals is not None else None
        m = self._L.sepo_compact(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), None, n, _ptr(bitmap), _ptr(ok),
                                 _ptr(oko), _ptr(ov), None)
        if m < 0:
            _err(m)
        m = int(m)
        if oko is not None:
            kb = int(oko[m].item()) if m else 0
            oko = oko[: m + 1]
        else:
            kb = m * self.opts.fixed_key_width
        ok = ok[:kb]
        if ov is not None:
            ov = ov[: m * self.val_width]
        return ok, oko, ov, m

    def evict(self):
        rc = self._L.sepo_evict(self.h)
        if rc < 0:
            _err(rc)
        return int(rc)

    # ---- the whole job
    def run(self, keys, key_offsets, vals=None, n=None, val_offsets=None):
        n = self._n(key_offsets, keys, n)
        rc = self._L.sepo_run(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), _ptr(val_offsets), n)
        if rc < 0:
            _err(rc)
        return int(rc)

    def run_text(self, text, n=None):
        """Word count on raw text (sepo_run_text): tokenizer fused into the insert kernel."""
        n = int(n) if n is not None else (text.numel() if hasattr(text, "numel") else len(text))
        rc = self._L.sepo_run_text(self.h, _ptr(text), n)
        if rc < 0:
            _err(rc)
        return int(rc)

    def run_wire(self, wire, n=None):
        """The whole job on routed wire records (sepo_run_wire): a uint8 device tensor of 32-byte records
        {key words, value, length} as sepo_route_combine writes them."""
        n = int(n) if n is not None else wire.numel() // 32
        rc = self._L.sepo_run_wire(self.h, _ptr(wire), n)
        if rc < 0:
            _err(rc)
        return int(rc)

    # ---- map runtime (NEXT-4): built-in mappers of the paper's applications on raw text
    def map_run(self, mapper, text, doc_offsets=None):
        """sepo_map_run: MAP_WORDS / MAP_LINES (COMBINE) or MAP_WORD_DOCS (GROUP, doc_offsets device int64)"""
        nd = doc_offsets.numel() if doc_offsets is not None else 0
        rc = self._L.sepo_map_run(self.h, int(mapper), _ptr(text), text.numel(), _ptr(doc_offsets), nd)
        if rc < 0:
            _err(rc)
        return int(rc)

    # ---- the multi-GPU data plane in the library (NCCL): attach, route + exchange, drain
    def attach_nccl(self, unique_id, nranks, rank):
        buf = ctypes.create_string_buffer(bytes(unique_id), 128)
        rc = self._L.sepo_attach_nccl(self.h, buf, int(nranks), int(rank))
        if rc:
            _err(rc)

    def insert_batch_sharded(self, keys, key_offsets, vals=None, n=None):
        """collective: route by key owner + NCCL exchange; returns the records this rank holds"""
        n = self._n(key_offsets, keys, n) if (keys is not None or key_offsets is not None) else 0
        rc = self._L.sepo_insert_batch_sharded(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), None, n)
        if rc < 0:
            _err(rc)
        return int(rc)

    def drain(self):
        rc = self._L.sepo_drain(self.h)
        if rc < 0:
            _err(rc)
        return int(rc)

    def run_sharded(self, keys, key_offsets, vals=None, n=None):
        """collective: the whole SEPO job on a batch sharded by key owner, the exchange of chunk c+1
        pipelined with the insert of chunk c (sepo_run_sharded); returns the number of passes"""
        n = self._n(key_offsets, keys, n) if (keys is not None or key_offsets is not None) else 0
        rc = self._L.sepo_run_sharded(self.h, _ptr(keys), _ptr(key_offsets), _ptr(vals), None, n)
        if rc < 0:
            _err(rc)
        return int(rc)

    def lookup(self, keys, key_offsets, n=None):
        """SEPO lookups over every generation (sepo_lookup) -> (found count, values u64 tensor,
        found bitmap int32 tensor), device tensors."""
        import torch
        n = self._n(key_offsets, keys, n)
        vals = torch.empty(max(n, 1), dtype=torch.int64, device="cuda")
        bm = torch.empty(max((n + 31) // 32, 1), dtype=torch.int32, device="cuda")
        rc = self._L.sepo_lookup(self.h, _ptr(keys), _ptr(key_offsets), n, _ptr(vals), _ptr(bm))
        if rc < 0:
            _err(rc)
        return int(rc), vals[:n], bm

    def export(self, copy=True):
        """-> dict of numpy arrays (copies unless copy=False: views of table-owned memory)."""
        r = Result()
        rc = self._L.sepo_export(self.h, ctypes.byref(r))
        if rc:
            _err(rc)
        k = int(r.n_keys)

        def arr(p, n, dt):
            if n == 0 or not p:
                return np.zeros(0, dtype=dt)
            a = np.ctypeslib.as_array(ctypes.cast(p, ctypes.POINTER(np.ctypeslib.as_ctypes_type(dt))), shape=(n,))
            return a.copy() if copy else a

        ko = arr(r.key_offsets, k + 1, np.uint64)
        out = {"n_keys": k, "key_offsets": ko, "keys": arr(r.keys, int(ko[-1]) if k else 0, np.uint8)}
        if self.mode in (COMBINE, BASIC):  # BASIC: one (key, value) row per stored pair
            out["values"] = arr(r.values, k, np.uint64)
        else:
            lo = arr(r.list_offsets, k + 1, np.uint64)
            nv = int(r.n_vals)
            vo = arr(r.val_offsets, nv + 1, np.uint64)
            out.update(list_offsets=lo, n_vals=nv, val_offsets=vo,
                       vals=arr(r.vals, int(vo[-1]) if nv else 0, np.uint8))
        return out

    def reset(self):
        rc = self._L.sepo_reset(self.h)
        if rc:
            _err(rc)

    def stats(self):
        s = Stats()
        self._L.sepo_stats_get(self.h, ctypes.byref(s))
        return s.as_dict()

    def last_insert_ms(self):
        return self._L.sepo_last_insert_ms(self.h)

    def _n(self, key_offsets, keys, n):
        if n is not None:
            return int(n)
        if key_offsets is not None:
            return (key_offsets.numel() if hasattr(key_offsets, "numel") else len(key_offsets)) - 1
        w = self.opts.fixed_key_width
        return (keys.numel() if hasattr(keys, "numel") else len(keys)) // w


def result_dict(res, mode=COMBINE):
    """Exported arrays -> {key bytes: value} (COMBINE), {key: sorted list of value bytes} (GROUP) or
    {key: sorted list of u64 values} (BASIC: the multiset of stored pairs)."""
    kb = res["keys"].tobytes()
    ko = res["key_offsets"]
    if mode == BASIC:
        v = res["values"]
        out = {}
        for i in range(res["n_keys"]):
            out.setdefault(kb[ko[i]:ko[i + 1]], []).append(int(v[i]))
        return {k: sorted(x) for k, x in out.items()}
    if mode == COMBINE:
        v = res["values"]
        return {kb[ko[i]:ko[i + 1]]: int(v[i]) for i in range(res["n_keys"])}
    vb = res["vals"].tobytes()
    vo, lo = res["val_offsets"], res["list_offsets"]
    return {kb[ko[i]:ko[i + 1]]: sorted(vb[vo[j]:vo[j + 1]] for j in range(lo[i], lo[i + 1])) for i in range(res["n_keys"])}
