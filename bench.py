"""bench.py — SEPO bulk insert-and-combine on B200 (BASELINE.json metric / configs).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--ratio 4] [--impl ours|reference]

A step = one whole SEPO job (every SURVEY §8(a) row): reset the table, insert all records of the
workload (input resident in HBM), re-probe + compact + evict + re-issue until nothing is
postponed, and transfer the final generation to pinned host memory (P:L227 timing scope).
Default workload: C2 (word count, 8 GiB Zipf(1.0) text = 1.1e9 words, V = 2^22) with the device
budget capped at F/4, i.e. the table is 4x the budget (BASELINE.json configs[1]).

Prints ONE JSON line (rank 0). `value` is input GB/s (CSR bytes the job consumes: key bytes +
8 B offsets [+ values]) over the device-timed steps; `e2e` is the same job through sepo_run with
pinned HOST buffers (H2D of the input + job + result assembly on the host). The oracle
(oracle/, test infrastructure) is run only by the cpu_baseline leg and by --impl reference.
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

BASE = json.load(open(os.path.join(ROOT, "BASELINE.json")))
METRIC = BASE["metric"]
MiB, GiB = 1 << 20, 1 << 30

CONFIG_TEXT = {
    "C1": BASE["configs"][0], "C2": BASE["configs"][1], "C3": BASE["configs"][2], "C4": BASE["configs"][3],
    "C5u": BASE["configs"][4] + " [uniform keys]", "C5z": BASE["configs"][4] + " [Zipf(1.2) keys]",
}


def next_pow2(x):
    p = 1
    while p < x:
        p <<= 1
    return p


def prev_pow2(x):
    p = 1
    while p * 2 <= x:
        p *= 2
    return p


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {"hbm_gbs": 6650.0, "_fallback": True}


class Job:
    """One workload at one budget ratio (table size / device budget)."""
    _footprint_cache = {}

    def __init__(self, cfg, ratio=4.0, page_bytes=None, scale=1.0):
        import gen
        self.cfg, self.ratio, self.scale = cfg, float(ratio), scale
        self.stream = gen.config(cfg, scale=scale)
        s = self.stream
        self.page_bytes = page_bytes or (16384 if s.family != gen.GEN_URLS else 65536)
        self.distinct = s.n_ranks
        self.nb_full = max(1 << 16, next_pow2(self.distinct))
        self._inputs = None
        self.kw = {}
        import paper_conf_ipps_mokhtaris17_b200 as sepo
        self.sepo = sepo
        if s.val == "u64":
            self.kw = dict(mode=sepo.COMBINE, fixed_key_width=8, fixed_val_width=8)
        elif s.val == "doc":
            self.kw = dict(mode=sepo.GROUP, fixed_val_width=4)
        else:
            self.kw = dict(mode=sepo.COMBINE)

    def inputs(self):
        if self._inputs is None:
            k, o, v = self.stream.device()
            if self.stream.val == "u64":
                o = None
            self._inputs = (k, o, v)
        return self._inputs

    def csr_bytes(self):
        k, o, v = self.inputs()
        b = k.numel()
        if o is not None:
            b += 8 * (o.numel() - 1)
        if v is not None:
            b += v.numel()
        return b

    def footprint(self):
        """F (SURVEY §8c reading 23): directory + pages an unconstrained run touches."""
        key = (self.cfg, self.scale, self.page_bytes)
        if key not in Job._footprint_cache:
            sepo = self.sepo
            t = sepo.Table(sepo.budget_for(self.nb_full, self.page_bytes, max(64, (self.csr_bytes() * 2) // self.page_bytes + 64)),
                           self.nb_full, self.page_bytes, **self.kw)
            k, o, v = self.inputs()
            passes = t.run(k, o, v)
            assert passes == 1
            pages = t.stats()["pages_used_max"]
            t.close()
            Job._footprint_cache[key] = (pages, 4 * self.nb_full + pages * self.page_bytes)
        return Job._footprint_cache[key]

    def table_params(self):
        pages_F, F = self.footprint()
        if self.ratio <= 1.0:
            nb = self.nb_full
            pages = int(np.ceil(pages_F / self.ratio)) if self.ratio < 1 else pages_F + 8
        else:  # directory: the largest power of two <= 2x the keys of one generation (load <= ~1)
            mult = float(os.environ.get("SEPO_BENCH_NB_MULT", "2"))
            nb = max(1 << 16, prev_pow2(int(self.distinct * mult / self.ratio)))
            pages = max(8, int((F / self.ratio - 4 * nb) // self.page_bytes))
        return nb, pages, F

    def table(self, **extra):
        sepo = self.sepo
        nb, pages, F = self.table_params()
        kw = dict(self.kw)
        kw.update(extra)
        _, F = self.footprint()
        arena = int(F * 1.25) + 64 * MiB
        return sepo.Table(sepo.budget_for(nb, self.page_bytes, pages), nb, self.page_bytes, host_arena_bytes=arena, **kw)


def make_job(cfg, ratio=4.0, **kw):
    return Job(cfg, ratio, **kw)


# ---------------------------------------------------------------- clocks during the timed region
class ClockSampler:
    """SM clock + throttle reasons sampled DURING the timed region: NVML in a thread every 5 ms
    (a bench step is ~40 ms, far shorter than nvidia-smi's start-up), nvidia-smi -lms as fallback.
    One sample is taken synchronously at start() so a short region still has one."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu_index=0):
        self.rows, self.proc = [], None
        self.gpu = gpu_index
        self.nv = None

    def _nvml_sample(self):
        nv, h = self.nv, self.handle
        sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
        mx = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
        r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
        bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]
        self.rows.append([str(self.gpu), str(sm), str(mx), "", ""] + ["Active" if r & b else "Not Active" for b in bits])

    def _nvml_loop(self):
        while not self.done.is_set():
            try:
                self._nvml_sample()
            except Exception:
                pass
            self.done.wait(0.005)

    def start(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            vis = os.environ.get("CUDA_VISIBLE_DEVICES", "")
            idx = int(vis.split(",")[self.gpu]) if vis and vis.split(",")[0].isdigit() else self.gpu
            self.handle = nv.nvmlDeviceGetHandleByIndex(idx)
            self.nv = nv
            self._nvml_sample()
            self.done = threading.Event()
            self.th = threading.Thread(target=self._nvml_loop, daemon=True)
            self.th.start()
            return
        except Exception:
            self.nv = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.nv is not None:
            self.done.set()
            self.th.join(timeout=2)
            try:
                self._nvml_sample()
            except Exception:
                pass
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        sm = [float(r[1]) for r in self.rows if len(r) >= 9 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 9 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            if len(r) >= 9:
                for nm, v in zip(names, r[5:9]):
                    if v.strip().lower() == "active":
                        reasons.add(nm)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------- the CPU oracle legs
def oracle_sample(job, max_records, budget_s=15.0):
    """Time the oracle (as it stands) on the first records of the same stream. -> (GB/s, recs/s, desc)"""
    import oracle
    s = job.stream
    chunk = min(max_records, 1 << 23)
    done, t_ins, bytes_in = 0, 0.0, 0
    h = oracle.Combine() if s.val != "doc" else oracle.Group()
    while done < max_records and t_ins < budget_s:
        cnt = min(chunk, s.n - done, max_records - done)
        if cnt <= 0:
            break
        k, o, v = s.host(done, cnt)
        t0 = time.perf_counter()
        if s.val == "doc":
            h.add(k, o, v, val_width=4)
        elif s.val == "u64":
            h.add(k, o, v, 8)
        else:
            h.add(k, o)
        t_ins += time.perf_counter() - t0
        bytes_in += len(k) + (8 * cnt if s.family != 2 else 0) + (len(v) if v is not None else 0)
        done += cnt
    return bytes_in / t_ins / 1e9, done / t_ins, done, t_ins


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    job = Job(args.config, args.ratio)
    for _ in range(args.warmup):
        oracle_sample(job, 1 << 20, budget_s=1.0)
    vals, recs, times = [], [], []
    for _ in range(args.steps):
        gbs, rps, n, t = oracle_sample(job, args.ref_records, budget_s=args.ref_seconds)
        vals.append(gbs); recs.append(n); times.append(t)
    v = float(np.median(vals))
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": float(np.median(times)) * 1e3, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
            "config": {"workload": CONFIG_TEXT[args.config], "ratio_table_over_budget": args.ratio},
            "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": f"first {int(np.median(recs))} records of {args.config} per step (oracle/oracle.cpp "
                                       f"std::unordered_map, single thread; generation excluded)"},
            "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------- our arm
def timed_steps(job, t, steps, stream, route_fn=None):
    import torch
    k, o, v = job.inputs()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ins_ms, launches, recs_ins, kb_ins, vb_ins, p1_ms = 0.0, 0, 0, 0, 0, 0.0
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(steps):
        if route_fn is not None:  # sharded: route this rank's slice by key owner every step
            k, o, v = route_fn()
            launches += 2
        t.reset()
        t.run(k, o, v)
        st = t.stats()
        ins_ms += st["t_insert_ms"]
        p1_ms += st["t_insert_ms_per_pass"][0]
        launches += st["kernel_launches"]
        recs_ins += st["records_inserted"]
        kb_ins += st["key_bytes_inserted"]
        vb_ins += st["val_bytes_inserted"]
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1), dict(insert_ms=ins_ms, p1_ms=p1_ms, launches=launches, recs=recs_ins, kb=kb_ins, vb=vb_ins,
                                     last=st)


def run_ours(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    if args.route and world == 1 and not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", local))
    job = Job(args.config, args.ratio, scale=args.scale)
    stream = torch.cuda.current_stream()
    routed = world > 1 or args.route
    fixed = job.stream.family == 2
    route_fn = None
    if routed:
        # strong scaling: rank r holds records [r*n/W, (r+1)*n/W) of the SAME global stream; each
        # step routes them by key hash (sepo_partition + NCCL all-to-all) and runs
        # the SEPO job on the records this rank owns
        from paper_conf_ipps_mokhtaris17_b200 import shard
        if not dist.is_initialized():
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        n_all = job.stream.n
        j0, j1 = rank * n_all // world, (rank + 1) * n_all // world
        sk, so, sv = job.stream.device(j0, j1 - j0)
        if fixed:
            so = None

        def route_fn():
            return shard.route(sk, so, sv, route_seed=0x5eed, fixed_key_width=8 if fixed else 0,
                               fixed_val_width=job.stream.val_width if sv is not None else 0)
        job.distinct = max(1, job.distinct // world)  # keys per rank (sizes the directory)
        job._inputs = route_fn()
        job.slice_bytes = sk.numel() + (8 * (so.numel() - 1) if so is not None else 0) + (sv.numel() if sv is not None else 0)
        job.slice_records = j1 - j0
    job.inputs()
    nb, pages, F = job.table_params()
    t = job.table()
    k, o, v = job.inputs()
    for _ in range(max(args.warmup, 3)):
        t.reset()
        t.run(k, o, v)
    sampler = ClockSampler(local)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    ms, info = timed_steps(job, t, args.steps, stream, route_fn)
    clocks = sampler.stop()
    st = info["last"]
    if world > 1:
        tt = torch.tensor([ms], device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms = float(tt.item())
    if routed:  # strong scaling: the whole stream is split over the ranks
        csr_all = job.slice_bytes
        tt = torch.tensor([csr_all], device="cuda", dtype=torch.float64)
        if world > 1:
            dist.all_reduce(tt)
        csr, n = float(tt.item()), job.stream.n
        value = csr * args.steps / (ms / 1e3) / 1e9
        recs_per_s = n * args.steps / (ms / 1e3)
    else:
        csr = job.csr_bytes()
        n = job.stream.n
        value = world * csr * args.steps / (ms / 1e3) / 1e9
        recs_per_s = world * n * args.steps / (ms / 1e3)

    # roofline of the dominant kernel: the pass-1 insert (insert_stream_kernel, rows a1..a7, plus
    # its hot-set sampling kernels) handed every record of the step. Algorithmic bytes = the
    # step's CSR input (key bytes + 8 B offset [+ value bytes] per record) over the
    # CUDA-event time of that insert call (on the table's stream), summed over the timed steps.
    pk = peaks()
    alg = job.csr_bytes() if not routed else job.slice_bytes
    achieved = alg * args.steps / (info["p1_ms"] / 1e3) / 1e9
    traffic, traffic_note, issue = args.traffic, None, None
    tj = os.path.join(ROOT, "profiles", "r01_traffic.json")
    if traffic is None and os.path.exists(tj) and args.config == "C2" and args.scale == 1.0:
        tr = json.load(open(tj))
        traffic = tr["dram_read_bytes"] + tr["dram_write_bytes"]
        traffic_note = (f"dram read+write of one launch ({tr['launch']}); that launch's algorithmic bytes: "
                        f"{tr['alg_bytes']}")
        if "warp_instructions" in tr:
            # the kernel is issue-bound, not HBM-bound: its instruction roofline from the same capture
            # (peak = 148 SMs x 4 schedulers x 1 warp instruction / cycle at the sampled SM clock)
            peak_wi = 148 * 4 * (clocks.get("sm_mhz") or 1965.0) * 1e6
            wi_per_s = tr["warp_instructions"] / (info["p1_ms"] / args.steps / 1e3)
            issue = {"warp_instructions_per_launch": tr["warp_instructions"],
                     "warp_instructions_per_record": tr["warp_instructions"] / n,
                     "achieved_warp_instr_per_s": wi_per_s, "peak_warp_instr_per_s": peak_wi,
                     "frac": wi_per_s / peak_wi, "ncu_issue_active": tr.get("issue_active_pct", 0) / 100.0}
    roof = {"bound": "hbm", "achieved": achieved, "peak": pk["hbm_gbs"], "unit": "GB/s",
            "frac": achieved / pk["hbm_gbs"], "traffic": traffic, "traffic_note": traffic_note,
            "kernel": "sepo::insert_stream_kernel (COMBINE, pass 1) / sepo::insert_group_stream_kernel (GROUP)",
            "alg_bytes_per_launch": alg, "launch_ms": info["p1_ms"] / args.steps,
            "share_of_step": info["p1_ms"] / ms, "all_insert_passes_share_of_step": info["insert_ms"] / ms,
            "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy)" if not pk.get("_fallback") else "fallback 6.65 TB/s",
            "issue": issue}

    # host link: page bytes evicted (intermediate generations + the final one)
    # over the eviction phase time, against the measured pinned D2H bandwidth (PEAKS_EXTRA.json)
    host_link = None
    try:
        d2h_peak = json.load(open(os.path.join(ROOT, "PEAKS_EXTRA.json"))).get("d2h_GBps")
    except Exception:
        d2h_peak = None
    if st["t_evict_ms"] > 0:
        gbs = st["bytes_evicted"] / (st["t_evict_ms"] / 1e3) / 1e9
        host_link = {"bytes_evicted_per_step": st["bytes_evicted"], "evict_ms_per_step": st["t_evict_ms"],
                     "achieved": gbs, "unit": "GB/s", "peak": d2h_peak,
                     "frac": (gbs / d2h_peak) if d2h_peak else None,
                     "note": "evict phase includes seal/classify kernels and the directory reset; peak = "
                             "measured pinned D2H (PEAKS_EXTRA.json)"}

    # end to end through sepo_run with pinned HOST buffers (H2D + job + host result assembly)
    e2e = None
    if args.e2e_steps > 0 and not routed:
        hk = torch.empty(k.numel(), dtype=torch.uint8, pin_memory=True); hk.copy_(k)
        ho = torch.empty(o.numel(), dtype=torch.int64, pin_memory=True).copy_(o) if o is not None else None
        hv = torch.empty(v.numel(), dtype=torch.uint8, pin_memory=True).copy_(v) if v is not None else None
        # warm (staging buffers are allocated once)
        t.reset(); t.run(hk, ho, hv); t.export(copy=False)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        d2h = 0
        for _ in range(args.e2e_steps):
            t.reset()
            t.run(hk, ho, hv)
            res = t.export(copy=False)
            d2h += t.stats()["bytes_evicted"]
        el = time.perf_counter() - t0
        if world > 1:
            tt = torch.tensor([el], device="cuda")
            dist.all_reduce(tt, op=dist.ReduceOp.MAX)
            el = float(tt.item())
        e2e = {"value": world * csr * args.e2e_steps / el / 1e9, "unit": "GB/s",
               "h2d_bytes_per_step": csr, "d2h_bytes_per_step": d2h // args.e2e_steps,
               "kv_inserts_per_s": world * n * args.e2e_steps / el,
               "note": "sepo_run on pinned host buffers; includes H2D, all passes, page D2H, host result assembly"}

    # slowdown curve (M3): job time at table/budget = 0.5 .. 4 relative to 0.5
    curve = None
    if args.curve and rank == 0 and not routed:
        curve = {}
        base = None
        for r in (0.5, 1.0, 2.0, 3.0, 4.0):
            j2 = Job(args.config, r, scale=args.scale)
            j2._inputs = job._inputs
            t2 = j2.table()
            for _ in range(2):
                t2.reset(); t2.run(k, o, v)
            m2, i2 = timed_steps(j2, t2, 2, stream)
            ms2 = m2 / 2
            if base is None:
                base = ms2
            curve[str(r)] = {"ms": ms2, "slowdown": ms2 / base, "passes": i2["last"]["passes"]}
            t2.close()

    # raw-text job (NEXT-2 (i), sepo_run_text): the same word stream as the 8 GB text the config
    # names (each word + one separator), tokenized inside the insert kernel; device-resident
    # input timed like the main line, plus e2e from pinned host text (H2D inside the timed region)
    raw_text = None
    if args.text and rank == 0 and not routed and job.stream.family == 0 and job.stream.val == "one":
        text = job.stream.text_device()
        tb = text.numel()
        for _ in range(2):
            t.reset(); t.run_text(text)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.steps):
            t.reset(); t.run_text(text)
        e1.record(stream)
        torch.cuda.synchronize()
        tms = e0.elapsed_time(e1) / args.steps
        stt = t.stats()
        raw_text = {"text_bytes": tb, "ms_per_step": tms, "value": tb / tms / 1e6, "unit": "GB/s of raw text",
                    "words_per_s": n / tms * 1e3, "passes": stt["passes"],
                    "pass1_ms": stt["t_insert_ms_per_pass"][0]}
        if args.e2e_steps > 0:
            ht = torch.empty(tb, dtype=torch.uint8, pin_memory=True)
            ht.copy_(text)
            del text
            t.reset(); t.run_text(ht); t.export(copy=False)
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            d2h = 0
            for _ in range(args.e2e_steps):
                t.reset(); t.run_text(ht); t.export(copy=False)
                d2h += t.stats()["bytes_evicted"]
            el = (time.perf_counter() - t0) / args.e2e_steps
            raw_text["e2e"] = {"value": tb / el / 1e9, "unit": "GB/s of raw text", "words_per_s": n / el,
                               "h2d_bytes_per_step": tb, "d2h_bytes_per_step": d2h // args.e2e_steps,
                               "note": "sepo_run_text on pinned host text; includes H2D, all passes, page D2H, host result assembly"}
            del ht
        else:
            del text
        torch.cuda.empty_cache()

    cpu = None
    if rank == 0 and args.cpu_baseline:
        gbs, rps, nrec, tsec = oracle_sample(job, args.ref_records, budget_s=args.ref_seconds)
        cpu = {"value": gbs, "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"first {nrec} records of {args.config} ({tsec:.1f} s, oracle/oracle.cpp std::unordered_map, "
                         f"single thread pinned by construction; generation excluded)", "kv_inserts_per_s": rps}

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
                "warmup": max(args.warmup, 3), "ms_per_step": ms / args.steps, "higher_is_better": True,
                "scaling": "strong" if routed else "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
                "kv_inserts_per_s": recs_per_s,
                "config": {"workload": CONFIG_TEXT[args.config], "records": n, "input_csr_bytes": csr,
                           "distinct_keys": job.distinct, "ratio_table_over_budget": args.ratio,
                           "table_footprint_bytes": F, "device_budget_bytes": job.sepo.budget_for(nb, job.page_bytes, pages),
                           "n_buckets": nb, "page_bytes": job.page_bytes, "pool_pages": pages,
                           "passes": st["passes"], "postponed_per_pass": st["postponed_per_pass"],
                           "bytes_evicted": st["bytes_evicted"], "l2": "inputs (>= 15 GiB) far larger than L2 (126 MB)",
                           "parallelism": (f"key-hash sharded x{world} (sepo_partition + NCCL all-to-all)" if routed
                                           else "1 GPU"),
                           "phase_ms": {kk: st[kk] for kk in ("t_insert_ms", "t_reprobe_ms", "t_compact_ms", "t_evict_ms")}},
                "roofline": roof, "host_link": host_link, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
                "gpu_launches": info["launches"], "slowdown_curve": curve, "raw_text": raw_text}
        print(json.dumps(line), flush=True)
    t.close()
    if dist.is_initialized():
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--ratio", type=float, default=4.0)
    ap.add_argument("--scale", type=float, default=1.0, help="shrink the workload (profiling only; not a bench value)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-curve", dest="curve", action="store_false")
    ap.add_argument("--no-cpu", dest="cpu_baseline", action="store_false")
    ap.add_argument("--no-text", dest="text", action="store_false", help="skip the raw-text (fused tokenizer) line")
    ap.add_argument("--ref-records", type=int, default=120_000_000)
    ap.add_argument("--ref-seconds", type=float, default=15.0)
    ap.add_argument("--route", action="store_true", help="run the sharded (router) path even at N=1")
    ap.add_argument("--traffic", type=float, default=None, help="dram bytes/launch from an ncu --set full capture")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
