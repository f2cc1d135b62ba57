"""Multi-GPU key-hash sharding: partition -> all-to-all -> local SEPO job.

One process per GPU. `torch.distributed` (backend "nccl" on GPUs, "gloo" in CPU tests) carries the
all-to-all; the partition and the offset rebasing run in libsepo's kernels (sepo_partition,
sepo_shift_offsets). A key's records all land on its owner rank, so every rank's export is final
and the union over ranks is the result (no merge).
"""
import ctypes

import numpy as np
import torch
import torch.distributed as dist

from . import _err, _ptr, lib

_bound = False


def _bind():
    global _bound
    if _bound:
        return
    L = lib()
    vp, u64, u32 = ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint32
    L.sepo_partition_scratch.argtypes = [u64, u32]
    L.sepo_partition_scratch.restype = ctypes.c_size_t
    L.sepo_partition.argtypes = [vp, vp, u32, vp, u32, u64, u32, u64, vp, vp, vp, vp, vp, ctypes.c_size_t, vp]
    L.sepo_partition.restype = ctypes.c_int
    L.sepo_shift_offsets.argtypes = [vp, u64, vp, vp, u32, u64, vp]
    L.sepo_shift_offsets.restype = ctypes.c_int
    L.sepo_route_scratch.argtypes = [u32]
    L.sepo_route_scratch.restype = ctypes.c_size_t
    L.sepo_route_combine.argtypes = [vp, vp, u32, vp, u32, u64, u32, u64, vp, u64, vp, vp, ctypes.c_size_t, vp]
    L.sepo_route_combine.restype = ctypes.c_int64
    _bound = True


def partition(keys, key_offsets, vals, n_parts, route_seed=0, fixed_key_width=0, fixed_val_width=0):
    """Stable partition of a device batch by key owner. -> (keys, key_offsets or None, vals or None,
    starts) where starts[p] = (first record, first key byte, first value byte) of part p and
    starts[n_parts] = totals (numpy uint64 [n_parts + 1, 3]). Offsets are relative to each part."""
    _bind()
    L = lib()
    n = (key_offsets.numel() - 1) if key_offsets is not None else keys.numel() // fixed_key_width
    ok = torch.empty_like(keys)
    oko = torch.empty(max(n, 1), dtype=torch.int64, device=keys.device) if key_offsets is not None else None
    ov = torch.empty_like(vals) if vals is not None else None
    scratch = torch.empty(int(L.sepo_partition_scratch(n, n_parts)), dtype=torch.uint8, device=keys.device)
    starts = np.zeros(3 * (n_parts + 1), dtype=np.uint64)
    stream = torch.cuda.current_stream(keys.device).cuda_stream
    rc = L.sepo_partition(_ptr(keys), _ptr(key_offsets), fixed_key_width, _ptr(vals), fixed_val_width, n, n_parts,
                          route_seed, _ptr(ok), _ptr(oko), _ptr(ov), starts.ctypes.data, scratch.data_ptr(),
                          scratch.numel(), ctypes.c_void_p(stream))
    if rc:
        _err(rc)
    return ok, (oko[:n] if oko is not None else None), ov, starts.reshape(n_parts + 1, 3)


WIRE_BYTES = 32  # sepo_route_combine's record: key words w0, w1, value, length (u64 each)
E_TOOLARGE = -3


def route_combine(keys, key_offsets, vals, n_parts, route_seed=0, fixed_key_width=0, fixed_val_width=0, out=None):
    """Partition with CTA pre-combine (COMBINE, keys <= 16 B; sepo_route_combine) -> (wire uint8 tensor,
    part_counts numpy [n_parts + 1]): part p's 32-byte records are rows [counts[p], counts[p+1]).
    Returns None if some key is longer than 16 bytes (route the batch with partition())."""
    _bind()
    L = lib()
    n = (key_offsets.numel() - 1) if key_offsets is not None else keys.numel() // fixed_key_width
    dev = keys.device
    scratch = torch.empty(int(L.sepo_route_scratch(n_parts)), dtype=torch.uint8, device=dev)
    counts = np.zeros(n_parts + 1, dtype=np.uint64)
    stream = ctypes.c_void_p(torch.cuda.current_stream(dev).cuda_stream)
    args = (_ptr(keys), _ptr(key_offsets), fixed_key_width, _ptr(vals), fixed_val_width, n, n_parts, route_seed)
    E_NOMEM = -2
    if out is None or out.numel() < max(n, 1) * WIRE_BYTES:  # (at most one record per input record)
        out = torch.empty(max(n, 1) * WIRE_BYTES, dtype=torch.uint8, device=dev)
    for _ in range(2):
        cap = out.numel() // WIRE_BYTES if out is not None else 0
        m = L.sepo_route_combine(*args, out.data_ptr() if cap else None, cap, counts.ctypes.data, scratch.data_ptr(),
                                 scratch.numel(), stream)
        if m == E_TOOLARGE:
            return None
        if m == E_NOMEM or (m >= 0 and not cap):  # (too small / sizing call): allocate and run again
            out = torch.empty(max(int(counts[-1]), 1) * WIRE_BYTES, dtype=torch.uint8, device=dev)
            continue
        if m < 0:
            _err(m)
        return out[: int(m) * WIRE_BYTES], counts
    raise RuntimeError("sepo_route_combine: output size changed between calls")


def exchange_wire(wire, counts, group=None):
    """All-to-all of routed wire records (part p -> rank p) -> the records this rank owns."""
    world = dist.get_world_size(group)
    send = np.diff(np.asarray(counts, dtype=np.int64))
    if world == 1:
        return wire
    dev = wire.device
    send_t = torch.as_tensor(send, dtype=torch.int64, device=dev)
    recv_t = torch.empty_like(send_t)
    dist.all_to_all_single(recv_t, send_t, group=group)
    recv = recv_t.cpu().numpy()
    out = torch.empty(max(int(recv.sum()), 1) * WIRE_BYTES, dtype=torch.uint8, device=dev)
    dist.all_to_all_single(out[: int(recv.sum()) * WIRE_BYTES], wire[: int(send.sum()) * WIRE_BYTES],
                           (recv * WIRE_BYTES).tolist(), (send * WIRE_BYTES).tolist(), group=group)
    return out[: int(recv.sum()) * WIRE_BYTES]


def shift_offsets_cuda(ko, seg_rec, seg_base, total):
    """ko[j] += seg_base[s] for records of segment s; ko[n] = total (libsepo kernel)."""
    _bind()
    n = ko.numel() - 1
    dev = ko.device
    sr = torch.as_tensor(np.asarray(seg_rec, dtype=np.int64), device=dev)
    sb = torch.as_tensor(np.asarray(seg_base, dtype=np.int64), device=dev)
    rc = lib().sepo_shift_offsets(ko.data_ptr(), n, sr.data_ptr(), sb.data_ptr(), len(seg_rec), int(total),
                                  ctypes.c_void_p(torch.cuda.current_stream(dev).cuda_stream))
    if rc:
        _err(rc)
    return ko


def exchange(ok, oko, ov, starts, group=None, shift_fn=shift_offsets_cuda):
    """All-to-all of the parts (part p -> rank p). -> (keys, key_offsets [n+1] or None, vals or None)
    for the records this rank owns, in sender-rank order (sender's input order within a sender)."""
    world = dist.get_world_size(group)
    starts = np.asarray(starts, dtype=np.int64)
    send = np.diff(starts, axis=0)  # [world, 3]: records, key bytes, value bytes per destination
    dev = ok.device
    send_t = torch.as_tensor(send.reshape(-1), dtype=torch.int64, device=dev)
    recv_t = torch.empty_like(send_t)
    dist.all_to_all_single(recv_t, send_t, group=group)
    recv = recv_t.cpu().numpy().reshape(world, 3)
    nrec, nkb, nvb = (int(x) for x in recv.sum(axis=0))
    rk = torch.empty(max(nkb, 1), dtype=torch.uint8, device=dev)
    # send buffers sliced to the partition totals (the caller's arrays may carry trailing bytes)
    ok = ok[: int(starts[-1, 1])]
    oko = oko[: int(starts[-1, 0])] if oko is not None else None
    ov = ov[: int(starts[-1, 2])] if ov is not None else None
    dist.all_to_all_single(rk[:nkb], ok, recv[:, 1].tolist(), send[:, 1].tolist(), group=group)
    rko = None
    if oko is not None:
        rko = torch.empty(nrec + 1, dtype=torch.int64, device=dev)
        dist.all_to_all_single(rko[:nrec], oko, recv[:, 0].tolist(), send[:, 0].tolist(), group=group)
        seg_rec = np.concatenate([[0], np.cumsum(recv[:, 0])[:-1]])
        seg_base = np.concatenate([[0], np.cumsum(recv[:, 1])[:-1]])
        shift_fn(rko, seg_rec, seg_base, nkb)
    rv = None
    if ov is not None:
        rv = torch.empty(max(nvb, 1), dtype=torch.uint8, device=dev)
        dist.all_to_all_single(rv[:nvb], ov, recv[:, 2].tolist(), send[:, 2].tolist(), group=group)
        rv = rv[:nvb]
    return rk[:nkb], rko, rv


def route(keys, key_offsets, vals, group=None, route_seed=0, fixed_key_width=0, fixed_val_width=0):
    """partition + exchange: the records of this rank's keys."""
    world = dist.get_world_size(group)
    ok, oko, ov, starts = partition(keys, key_offsets, vals, world, route_seed, fixed_key_width, fixed_val_width)
    return exchange(ok, oko, ov, starts, group)


class Router:
    """Routes each step's batch of this rank to the key owners and keeps per-step statistics.

    combine=True (COMBINE tables, keys <= 16 B): sepo_route_combine folds the batch's hot keys into one
    record each and the exchange carries 32-byte wire records -> route() returns ("wire", tensor) for Table.run_wire;
    batches with longer keys (and combine=False) are partitioned as CSR -> ("csr", (keys, offsets,
    vals)) for Table.run."""

    def __init__(self, group=None, route_seed=0, fixed_key_width=0, fixed_val_width=0, combine=True):
        self.group, self.seed, self.kw, self.vw, self.combine = group, route_seed, fixed_key_width, fixed_val_width, combine
        self._last = {}
        self._wire_buf = None

    def route(self, keys, key_offsets, vals):
        world = dist.get_world_size(self.group)
        n_in = (key_offsets.numel() - 1) if key_offsets is not None else keys.numel() // max(self.kw, 1)
        if self.combine:
            if self._wire_buf is None or self._wire_buf.numel() < max(n_in, 1) * WIRE_BYTES:  # (reused step to step)
                self._wire_buf = None
                self._wire_buf = torch.empty(max(n_in, 1) * WIRE_BYTES, dtype=torch.uint8, device=keys.device)
            r = route_combine(keys, key_offsets, vals, world, self.seed, self.kw, self.vw, out=self._wire_buf)
            if r is not None:
                wire, counts = r
                out = exchange_wire(wire, counts, self.group)
                self._last = {"records_in": n_in, "records_sent": int(counts[-1]), "records_out": out.numel() // WIRE_BYTES,
                              "format": "wire (pre-combined)"}
                return "wire", out
        ok, oko, ov, starts = partition(keys, key_offsets, vals, world, self.seed, self.kw, self.vw)
        out = exchange(ok, oko, ov, starts, self.group)
        self._last = {"records_in": n_in, "records_out": int(out[1].numel() - 1) if out[1] is not None
                      else int(out[0].numel() // max(self.kw, 1)), "format": "csr"}
        return "csr", out

    @staticmethod
    def run(table, routed):
        """the SEPO job on what route() returned"""
        kind, data = routed
        return table.run_wire(data) if kind == "wire" else table.run(*data)

    def last_stats(self):
        return dict(self._last)
