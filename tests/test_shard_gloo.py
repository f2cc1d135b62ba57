"""Host-side logic of the multi-GPU path on CPU: the all-to-all exchange of
partitioned batches over a world_size-2 gloo group. The partition itself is a CUDA kernel (tested
in test_shard_gpu.py); here parts are built by the test with a trivial owner rule."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def cpu_shift(ko, seg_rec, seg_base, total):
    n = ko.numel() - 1
    bounds = list(seg_rec) + [n]
    for s in range(len(seg_rec)):
        ko[bounds[s]:bounds[s + 1]] += int(seg_base[s])
    ko[n] = total
    return ko


def make_rank_input(rank, n=300):
    rng = np.random.default_rng(rank)
    keys = [bytes(rng.integers(97, 123, size=int(rng.integers(0, 9))).astype(np.uint8)) for _ in range(n)]
    vals = rng.integers(0, 2**63, size=n, dtype=np.uint64)
    return keys, vals


def owner(k, world):
    return (k[0] if k else 0) % world


def build_parts(keys, vals, world):
    """stable partition on the host (test-side stand-in for sepo_partition)"""
    order = [i for p in range(world) for i in range(len(keys)) if owner(keys[i], world) == p]
    starts = np.zeros((world + 1, 3), dtype=np.uint64)
    kb, ko = bytearray(), []
    pv = []
    for p in range(world):
        starts[p] = (len(ko), len(kb), 8 * len(ko))
        base = len(kb)
        for i in order:
            if owner(keys[i], world) == p:
                ko.append(len(kb) - base)
                kb += keys[i]
                pv.append(vals[i])
    starts[world] = (len(ko), len(kb), 8 * len(ko))
    return (torch.frombuffer(bytes(kb) + b"\0", dtype=torch.uint8)[: len(kb)].clone(), torch.tensor(ko, dtype=torch.int64),
            torch.from_numpy(np.array(pv, dtype=np.uint64).view(np.uint8).copy()), starts)


def worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_mokhtaris17_b200.shard import exchange
    keys, vals = make_rank_input(rank)
    ok, oko, ov, starts = build_parts(keys, vals, world)
    rk, rko, rv = exchange(ok, oko, ov, starts, shift_fn=cpu_shift)
    kb = rk.numpy().tobytes()
    ko = rko.numpy()
    got = [(kb[ko[j]:ko[j + 1]], int(rv.numpy().view(np.uint64)[j])) for j in range(len(ko) - 1)]
    # expected: records owned by this rank from every sender, sender order then input order
    exp = []
    for src in range(world):
        k2, v2 = make_rank_input(src)
        exp += [(k2[i], int(v2[i])) for i in range(len(k2)) if owner(k2[i], world) == rank]
    q.put((rank, got == exp, len(got), int(ko[-1]) == len(kb)))
    dist.destroy_process_group()


def free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_exchange_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = free_port()
    ps = [ctx.Process(target=worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=120) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    assert sorted(r[0] for r in res) == [0, 1]
    for rank, ok, n, closed in res:
        assert ok, f"rank {rank} received the wrong records"
        assert closed and n > 0


def _wire_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_ipps_mokhtaris17_b200 import shard
    rng = np.random.default_rng(10 + rank)
    n_per = [int(x) for x in rng.integers(0, 40, size=world)]
    recs, counts = [], [0]
    for p in range(world):  # part p's records: key "r<rank>p<p>i<i>", value = rank*1000 + i
        for i in range(n_per[p]):
            key = b"r%dp%di%d" % (rank, p, i)
            w = key.ljust(16, b"\0")
            recs.append(np.frombuffer(w, dtype=np.uint64).tolist() + [rank * 1000 + i, len(key)])
        counts.append(counts[-1] + n_per[p])
    wire = torch.from_numpy(np.array(recs, dtype=np.uint64).reshape(-1).view(np.uint8).copy() if recs
                            else np.zeros(0, dtype=np.uint8))
    out = shard.exchange_wire(wire, np.array(counts, dtype=np.uint64))
    q.put((rank, out.numpy().tobytes(), n_per))
    dist.destroy_process_group()


def test_exchange_wire_gloo():
    """wire records (32 B each) of part p reach rank p, in sender-rank order, byte for byte"""
    world = 2
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_wire_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = {}
    for _ in range(world):
        r, b, n_per = q.get(timeout=120)
        res[r] = (b, n_per)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    for dst in range(world):
        got = np.frombuffer(res[dst][0], dtype=np.uint64).reshape(-1, 4)
        exp = []
        for src in range(world):
            for i in range(res[src][1][dst]):
                key = b"r%dp%di%d" % (src, dst, i)
                exp.append(np.frombuffer(key.ljust(16, b"\0"), dtype=np.uint64).tolist() + [src * 1000 + i, len(key)])
        assert got.tolist() == exp
