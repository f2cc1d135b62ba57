"""Residency ablations — both sides of the SEPO inequality
 measured on one B200 with the same kernels:

  sepo_device  : the SEPO table, pool in HBM, table k x the budget (postpone + evict + re-issue)
  device_fit   : pool in HBM holding the whole table (one pass; the "efficient service")
  host_pinned  : pool in pinned host memory mapped into the GPU (one pass; every entry access
                 crosses the host link — the paper's Fig. 7 alternative)
  managed      : pool in cudaMallocManaged memory (one pass; pages fault-migrate to the GPU on
                 first touch — hardware demand paging without oversubscription)

Each job includes the final transfer of the table to pinned host memory. Input: a
bounded prefix of the C2 stream (word count, Zipf(1.0), V = 2^22), resident in HBM.

  python tools/ablation_residency.py [--scale 0.0625] [--reps 3] [--out profiles/x.json]
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--scale", type=float, default=1 / 16)
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--ratios", default="1,2,4")
    ap.add_argument("--out", default=None)
    ap.add_argument("--oversub", default="1,2,4", help="managed pool with HBM capped to F/k (k list; '' skips)")
    a = ap.parse_args()
    import torch
    import bench
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    torch.cuda.set_device(0)
    stream = torch.cuda.current_stream()

    def timed(t, k, o, v):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t.reset()
        t.run(k, o, v)  # warm-up (first touch of managed pages happens here too; reset keeps them)
        ms = []
        for _ in range(a.reps):
            torch.cuda.synchronize()
            e0.record(stream)
            t.reset()
            t.run(k, o, v)
            e1.record(stream)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
        st = t.stats()
        return min(ms), st

    out = {"config": a.config, "scale": a.scale, "rows": []}
    base = bench.Job(a.config, 1.0, scale=a.scale)
    k, o, v = base.inputs()
    csr = base.csr_bytes()
    n = base.stream.n
    pages_F, F = base.footprint()
    out.update(records=n, input_csr_bytes=csr, table_footprint_bytes=F)

    def row(name, t, extra=None):
        ms, st = timed(t, k, o, v)
        r = {"name": name, "ms": ms, "input_gbs": csr / ms / 1e6, "kv_inserts_per_s": n / ms * 1e3,
             "passes": st["passes"], "bytes_evicted": st["bytes_evicted"]}
        r.update(extra or {})
        t.close()
        out["rows"].append(r)
        print(json.dumps(r), flush=True)

    nb_full = base.nb_full
    fit_pages = pages_F + 2 * 148 + 64  # the open pages of the allocator slots on top of F
    arena = int(F * 1.25) + 64 * (1 << 20)
    row("device_fit", sepo.Table(sepo.budget_for(nb_full, base.page_bytes, fit_pages), nb_full, base.page_bytes,
                                 host_arena_bytes=arena, **base.kw), {"ratio": 1.0})
    for r in [float(x) for x in a.ratios.split(",")]:
        job = bench.Job(a.config, r, scale=a.scale)
        job._inputs = (k, o, v)
        row(f"sepo_device_{r:g}x", job.table(), {"ratio": r})
    for name, pl in (("host_pinned", sepo.POOL_HOST_PINNED), ("managed", sepo.POOL_MANAGED)):
        t0 = time.time()
        row(name, sepo.Table(sepo.budget_for(nb_full, base.page_bytes, fit_pages), nb_full, base.page_bytes,
                             host_arena_bytes=arena, placement=pl, **base.kw), {"ratio": 1.0, "wall_s": time.time() - t0})
    # managed pool OVERSUBSCRIBED (NEXT-1 (ii), the Table III analogue): the same pool
    # with device memory capped by a balloon so that only F/k of it fits in HBM at once — the driver
    # demand-pages the table in and evicts pages back to host memory during the job
    if a.oversub:
        for kk in [float(x) for x in a.oversub.split(",")]:
            t = sepo.Table(sepo.budget_for(nb_full, base.page_bytes, fit_pages), nb_full, base.page_bytes,
                           host_arena_bytes=arena, placement=sepo.POOL_MANAGED, **base.kw)
            t.reset(); t.run(k, o, v)  # every library buffer allocated before the balloon
            torch.cuda.synchronize()
            free, _ = torch.cuda.mem_get_info()
            leave = int(F / kk) + (8 << 20)
            balloon = torch.empty(max(free - leave, 0), dtype=torch.uint8, device="cuda") if free > leave else None
            torch.cuda.synchronize()
            t0 = time.time()
            try:
                row(f"managed_oversub_{kk:g}x", t, {"ratio": kk, "device_free_for_pool": leave, "wall_s": time.time() - t0})
            except Exception as e:  # (an allocation inside the job failed under the cap)
                out["rows"].append({"name": f"managed_oversub_{kk:g}x", "error": str(e)[:200]})
                print(json.dumps(out["rows"][-1]), flush=True)
            del balloon
            torch.cuda.empty_cache()
    fit = out["rows"][0]["ms"]
    for r in out["rows"]:
        if "ms" not in r:
            continue
        r["slowdown_vs_device_fit"] = r["ms"] / fit
    print(json.dumps(out), flush=True)
    if a.out:
        json.dump(out, open(a.out, "w"), indent=1)


if __name__ == "__main__":
    main()
