"""Measurement of the organizations besides the headline COMBINE job (SURVEY §8(f) NEXT-3 and the
GROUP row a4): whole SEPO jobs (all passes + evictions + final transfer to pinned host memory,
P:L227) at table/budget ratios, CUDA-event timed on the table's stream, input resident in HBM.

  python tools/time_modes.py [--out profiles/x.json]

  basic_c5z : BASIC on C5-Zipf pairs, 2^25 records (every pair is an entry)
  basic_c2  : BASIC on a 1/16 prefix of the C2 word stream (69 M words, implicit values)
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    import torch
    import gen
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()
    rows = []
    for name, cfg, scale, pb in (("basic_c5z", "C5z", 1 / 64, 65536), ("basic_c2", "C2", 1 / 16, 65536)):
        s = gen.config(cfg, scale=scale)
        k, o, v = s.device()
        kw = dict(mode=sepo.BASIC)
        if s.val == "u64":
            kw.update(fixed_key_width=8, fixed_val_width=8)
            o = None
        in_bytes = k.numel() + (8 * (o.numel() - 1) if o is not None else 0) + (v.numel() if v is not None else 0)
        nb = 1 << 22
        big = sepo.Table(sepo.budget_for(nb, pb, (48 * s.n) // pb + 1024), nb, pb, host_arena_bytes=48 * s.n + (1 << 28), **kw)
        assert big.run(k, o, v) == 1
        pages = big.stats()["pages_used_max"]
        big.close()
        F = 4 * nb + pages * pb
        for ratio in (1.0, 2.0, 4.0):
            P = pages + 2 * 148 if ratio == 1.0 else max(8, int(pages / ratio))
            t = sepo.Table(sepo.budget_for(nb, pb, P), nb, pb, host_arena_bytes=int(F * 1.3) + (1 << 28), **kw)
            t.run(k, o, v)
            ms = []
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            for _ in range(a.reps):
                torch.cuda.synchronize()
                e0.record(stream)
                t.reset()
                passes = t.run(k, o, v)
                e1.record(stream)
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            st = t.stats()
            t.close()
            r = {"name": name, "ratio": ratio, "records": s.n, "input_bytes": in_bytes, "ms": min(ms),
                 "input_gbs": in_bytes / min(ms) / 1e6, "kv_inserts_per_s": s.n / min(ms) * 1e3, "passes": passes,
                 "postponed_per_pass": st["postponed_per_pass"][:passes], "bytes_evicted": st["bytes_evicted"],
                 "table_footprint_bytes": F, "insert_ms": st["t_insert_ms"], "evict_ms": st["t_evict_ms"]}
            rows.append(r)
            print(json.dumps(r), flush=True)
    if a.out:
        json.dump(rows, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
