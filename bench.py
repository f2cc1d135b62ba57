"""bench.py — SEPO bulk insert-and-combine on B200 (BASELINE.json metric / configs).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2] [--ratio 4] [--impl ours|reference]

A step = one whole SEPO job (every SURVEY §8(a) row): reset the table, insert all records of the
workload (input resident in HBM), re-probe + compact + evict + re-issue until nothing is
postponed, and transfer the final generation to pinned host memory (P:L227 timing scope).
Default workload: C2 (word count, 8 GiB Zipf(1.0) text = 1.1e9 words, V = 2^22) with the device
budget capped at F/4, i.e. the table is 4x the budget (BASELINE.json configs[1]).

Prints ONE JSON line (rank 0). For word counts (C1/C2) the headline is SURVEY §8(d) M2 on the RAW
text: `value` = GB/s of raw text (each word + one separator, 8.6 GB for C2) over the device-timed
sepo_run_text jobs — the tokenizer is fused into the insert kernel, so it is inside the job;
`e2e` = the same job from pinned HOST text through the public API (H2D + job + sepo_export).
`csr_job` is the same workload from a pre-tokenised CSR (sepo_run). `roofline` is M1: the pass-1
insert kernel of the IN-BUDGET job (C2 at 0.5x, one pass), CUDA events on the table's stream;
`roofline_m1_c3` the same for C3 at P = 1; `roofline_headline_kernel` the headline step's own
pass-1 kernel. The oracle (oracle/, test infrastructure) is run only by the cpu_baseline leg and
by --impl reference.
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
        self.run_fn = None  # routed jobs: runs the SEPO job on this rank's routed records
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

    def run_job(self, t):
        if self.run_fn is not None:
            return self.run_fn(t)
        k, o, v = self.inputs()
        return t.run(k, o, v)

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
            nbytes = self.bytes_hint if self.run_fn is not None else self.csr_bytes()
            t = sepo.Table(sepo.budget_for(self.nb_full, self.page_bytes, max(64, (nbytes * 2) // self.page_bytes + 64)),
                           self.nb_full, self.page_bytes, **self.kw)
            passes = self.run_job(t)
            assert passes == 1
            pages = t.stats()["pages_used_max"]
            t.close()
            Job._footprint_cache[key] = (pages, 4 * self.nb_full + pages * self.page_bytes)
        return Job._footprint_cache[key]

    def table_params(self):
        pages_F, F = self.footprint()
        if self.ratio <= 1.0:
            # in-budget tables: four times as many buckets as keys (load ~0.25: shorter chains for the
            # misses that go to HBM — head insertion leaves a Zipf key's old entry behind the later ones;
            # C2 0.5x pass 1: load 1 28.5, 0.5 25.8 -> 22.7, 0.25 21.9, 0.125 21.6 ms,
            # profiles/r02/ab_directory_ib.jsonl, ab_nb_r3.jsonl). SEPO_BENCH_NB_IB overrides the multiple.
            nb = self.nb_full * int(os.environ.get("SEPO_BENCH_NB_IB", "4"))
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
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ins_ms, launches, recs_ins, kb_ins, vb_ins, p1_ms = 0.0, 0, 0, 0, 0, 0.0
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(steps):
        if route_fn is not None:  # sharded: route this rank's slice by key owner every step
            route_fn()
            launches += 2
        t.reset()
        job.run_job(t)
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


def cpu_info():
    """host CPU model, nproc and the affinity mask size (SURVEY §8(d) timing protocol)"""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except Exception:
        pass
    try:
        aff = len(os.sched_getaffinity(0))
    except Exception:
        aff = None
    return {"cpu_model": model, "nproc": os.cpu_count(), "affinity": aff}


def time_text_jobs(t, text, steps, stream):
    """`steps` raw-text jobs (sepo_run_text) back to back, CUDA events on the table's stream"""
    import torch
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    p1, launches = 0.0, 0
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(steps):
        t.reset()
        t.run_text(text)
        st = t.stats()
        p1 += st["t_insert_ms_per_pass"][0]
        launches += st["kernel_launches"]
    e1.record(stream)
    torch.cuda.synchronize()
    return e0.elapsed_time(e1), dict(p1_ms=p1, launches=launches, last=st)


def roofline_of(alg_bytes, p1_ms_total, steps, pk, kernel, extra=None):
    achieved = alg_bytes * steps / (p1_ms_total / 1e3) / 1e9
    r = {"bound": "hbm", "achieved": achieved, "peak": pk["hbm_gbs"], "unit": "GB/s", "frac": achieved / pk["hbm_gbs"],
         "kernel": kernel, "alg_bytes_per_launch": alg_bytes, "launch_ms": p1_ms_total / steps,
         "peak_source": "MEASURED_PEAKS.json hbm_gbs (copy, burst)" if not pk.get("_fallback") else "fallback 6.65 TB/s"}
    if extra:
        r.update(extra)
    return r


def traffic_of(name):
    """dram read+write bytes and warp instructions per launch from a committed ncu --set full capture"""
    tj = os.path.join(ROOT, "profiles", name)
    if not os.path.exists(tj):
        return None
    return json.load(open(tj))


def issue_of(tr, n_records, launch_ms, clocks):
    """instruction-issue roofline of a kernel (148 SMs x 4 schedulers x 1 warp instruction / cycle)"""
    if not tr or "warp_instructions" not in tr:
        return None
    peak_wi = 148 * 4 * (clocks.get("sm_mhz") or 1965.0) * 1e6
    wi_per_s = tr["warp_instructions"] / (launch_ms / 1e3)
    return {"warp_instructions_per_launch": tr["warp_instructions"], "warp_instructions_per_record": tr["warp_instructions"] / n_records,
            "achieved_warp_instr_per_s": wi_per_s, "peak_warp_instr_per_s": peak_wi, "frac": wi_per_s / peak_wi,
            "ncu_issue_active": tr.get("issue_active_pct", 0) / 100.0, "source": tr.get("launch")}


def e2e_text(t, text_dev, n_words, steps, world=1):
    """the headline job end to end: pinned HOST text -> sepo_run_text (H2D pipelined with pass 1,
    all passes, page D2H) -> sepo_export (host result assembly); wall clock, synchronized"""
    import torch
    tb = text_dev.numel()
    ht = torch.empty(tb, dtype=torch.uint8, pin_memory=True)
    ht.copy_(text_dev)
    t.reset(); t.run_text(ht); t.export(copy=False)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    d2h = 0
    for _ in range(steps):
        t.reset()
        t.run_text(ht)
        t.export(copy=False)
        d2h += t.stats()["bytes_evicted"]
    el = (time.perf_counter() - t0) / steps
    del ht
    return {"value": world * tb / el / 1e9, "unit": "GB/s of raw text", "kv_inserts_per_s": world * n_words / el,
            "h2d_bytes_per_step": tb, "d2h_bytes_per_step": d2h // steps,
            "note": "sepo_run_text on pinned host text + sepo_export: H2D (pipelined with pass 1), all passes, page D2H, "
                    "host result assembly"}


def e2e_csr(t, k, o, v, csr, n, steps, world=1):
    import torch
    hk = torch.empty(k.numel(), dtype=torch.uint8, pin_memory=True); hk.copy_(k)
    ho = torch.empty(o.numel(), dtype=torch.int64, pin_memory=True).copy_(o) if o is not None else None
    hv = torch.empty(v.numel(), dtype=torch.uint8, pin_memory=True).copy_(v) if v is not None else None
    t.reset(); t.run(hk, ho, hv); t.export(copy=False)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    d2h = 0
    for _ in range(steps):
        t.reset()
        t.run(hk, ho, hv)
        t.export(copy=False)
        d2h += t.stats()["bytes_evicted"]
    el = (time.perf_counter() - t0) / steps
    return {"value": world * csr / el / 1e9, "unit": "GB/s", "h2d_bytes_per_step": csr, "d2h_bytes_per_step": d2h // steps,
            "kv_inserts_per_s": world * n / el,
            "note": "sepo_run on pinned host CSR + sepo_export: H2D (pipelined), all passes, page D2H, host result assembly"}


def run_ours(args):
    import torch
    import torch.distributed as dist
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    routed = world > 1 or args.route
    if routed:
        return run_routed(args, world, rank, local)
    job = Job(args.config, args.ratio, scale=args.scale)
    stream = torch.cuda.current_stream()
    pk = peaks()
    text_ok = args.text and job.stream.family == 0 and job.stream.val == "one"
    nb, pages, F = job.table_params()
    t = job.table()
    k, o, v = job.inputs()
    n = job.stream.n
    csr = job.csr_bytes()
    sampler = ClockSampler(local)

    # ---- headline: the whole SEPO job on the RAW text, tokenizer inside (sepo_run_text)
    text = job.stream.text_device() if text_ok else None
    if text_ok:
        tb = text.numel()
        for _ in range(max(args.warmup, 3)):
            t.reset(); t.run_text(text)
        sampler.start()
        ms, info = time_text_jobs(t, text, args.steps, stream)
        value = tb * args.steps / (ms / 1e3) / 1e9
        recs_per_s = n * args.steps / (ms / 1e3)
        st = info["last"]
        head = {"metric_input": "raw text bytes (each word + one separator), tokenized inside the insert kernel",
                "text_bytes": tb}
    # ---- the same job on pre-tokenised CSR input (sepo_run; sub-line, or the headline for C3/C4/C5)
    for _ in range(max(args.warmup, 3)):
        t.reset(); t.run(k, o, v)
    if not text_ok:
        sampler.start()
    ms_c, info_c = timed_steps(job, t, args.steps, stream)
    st_c = info_c["last"]
    csr_line = {"value": csr * args.steps / (ms_c / 1e3) / 1e9, "unit": "GB/s of CSR (key bytes + 8 B offsets [+ values])",
                "ms_per_step": ms_c / args.steps, "kv_inserts_per_s": n * args.steps / (ms_c / 1e3),
                "passes": st_c["passes"], "postponed_per_pass": st_c["postponed_per_pass"],
                "pass1_ms": info_c["p1_ms"] / args.steps}
    if not text_ok:
        ms, info, st = ms_c, info_c, st_c
        value = csr_line["value"]
        recs_per_s = csr_line["kv_inserts_per_s"]
        head = {"metric_input": "CSR bytes: key bytes + 8 B offsets [+ values]", "csr_bytes": csr}

    # ---- M1: in-budget sepo_insert_batch, pass-1 insert kernel; C2 at 0.5x (+ C3 at P = 1)
    m1 = None
    if args.m1 and args.config == "C2" and args.scale == 1.0:
        jib = Job("C2", 0.5)
        jib._inputs = job._inputs
        tib = jib.table()
        for _ in range(2):
            tib.reset(); tib.run(k, o, v)
        msi, ii = timed_steps(jib, tib, args.steps, stream)
        tr = traffic_of("r02_traffic_m1.json")
        m1 = roofline_of(csr, ii["p1_ms"], args.steps, pk, "sepo::insert_lean_kernel<false,IN_CSR,32> (C2, 0.5x: in budget, 1 pass)",
                         {"traffic": (tr["dram_read_bytes"] + tr["dram_write_bytes"]) if tr else None,
                          "traffic_note": tr.get("launch") if tr else None, "share_of_step": ii["p1_ms"] / msi,
                          "job_ms": msi / args.steps, "passes": ii["last"]["passes"]})
        m1["issue"] = issue_of(tr, n, m1["launch_ms"], {"sm_mhz": None})
        tib.close()
    m1_c3 = None
    if args.m1_c3 and args.config == "C2" and args.scale == 1.0:
        j3 = Job("C3", 1.0)
        t3 = j3.table()
        k3, o3, v3 = j3.inputs()
        for _ in range(2):
            t3.reset(); t3.run(k3, o3, v3)
        ms3, i3 = timed_steps(j3, t3, 3, stream)
        tr3 = traffic_of("r02_traffic_c3.json")
        m1_c3 = roofline_of(j3.csr_bytes(), i3["p1_ms"], 3, pk, "sepo::insert_stream_kernel<false,1024,IN_CSR> (C3 URLs, P = 1, in budget)",
                            {"traffic": (tr3["dram_read_bytes"] + tr3["dram_write_bytes"]) if tr3 else None,
                             "job_ms": ms3 / 3, "records": j3.stream.n, "passes": i3["last"]["passes"]})
        t3.close()
        del j3, k3, o3, v3
        torch.cuda.empty_cache()
    clocks = sampler.stop()
    if m1 and m1.get("issue") is not None:
        m1["issue"] = issue_of(traffic_of("r02_traffic_m1.json"), n, m1["launch_ms"], clocks)

    # the headline step's own dominant kernel (pass 1 of the raw-text job: insert_text_kernel)
    if text_ok:
        trt = traffic_of("r02_traffic_text.json")
        roof_head = roofline_of(tb, info["p1_ms"], args.steps, pk, "sepo::insert_text_kernel (pass 1 of the headline job)",
                                {"share_of_step": info["p1_ms"] / ms,
                                 "traffic": (trt["dram_read_bytes"] + trt["dram_write_bytes"]) if trt else None})
    else:
        roof_head = roofline_of(csr, info["p1_ms"], args.steps, pk, "pass-1 insert kernel of the headline job",
                                {"share_of_step": info["p1_ms"] / ms})

    # host link: page bytes evicted over the eviction phase, vs measured pinned D2H
    host_link = None
    try:
        d2h_peak = json.load(open(os.path.join(ROOT, "PEAKS_EXTRA.json"))).get("d2h_GBps")
    except Exception:
        d2h_peak = None
    if st["t_evict_ms"] > 0:
        gbs = st["bytes_evicted"] / (st["t_evict_ms"] / 1e3) / 1e9
        host_link = {"bytes_evicted_per_step": st["bytes_evicted"], "evict_ms_per_step": st["t_evict_ms"],
                     "achieved": gbs, "unit": "GB/s", "peak": d2h_peak, "frac": (gbs / d2h_peak) if d2h_peak else None,
                     "note": "evict phase includes seal/classify kernels and the directory reset; peak = measured "
                             "pinned D2H (PEAKS_EXTRA.json)"}

    # slowdown curves (M3): job time at table/budget 0.5 .. 4 relative to 0.5 (headline job; CSR job too)
    curve = curve_csr = None
    if args.curve:
        curve, curve_csr = {}, {}
        base = base_c = None
        for r in (0.5, 1.0, 2.0, 3.0, 4.0):
            j2 = Job(args.config, r, scale=args.scale)
            j2._inputs = job._inputs
            t2 = j2.table()
            if text_ok:
                for _ in range(2):
                    t2.reset(); t2.run_text(text)
                m2, i2 = time_text_jobs(t2, text, 2, stream)
                base = base or m2 / 2
                curve[str(r)] = {"ms": m2 / 2, "slowdown": m2 / 2 / base, "passes": i2["last"]["passes"]}
            for _ in range(2):
                t2.reset(); t2.run(k, o, v)
            m2, i2 = timed_steps(j2, t2, 2, stream)
            base_c = base_c or m2 / 2
            curve_csr[str(r)] = {"ms": m2 / 2, "slowdown": m2 / 2 / base_c, "passes": i2["last"]["passes"]}
            t2.close()
        if not text_ok:
            curve = curve_csr

    # end to end through the public API from pinned HOST buffers (H2D + job + export in the timed region)
    e2e = e2e_c = None
    if args.e2e_steps > 0:
        e2e_c = e2e_csr(t, k, o, v, csr, n, args.e2e_steps)
        e2e = e2e_text(t, text, n, args.e2e_steps) if text_ok else e2e_c
    csr_line["e2e"] = e2e_c
    csr_line["slowdown_curve"] = curve_csr
    if text is not None:
        del text
        torch.cuda.empty_cache()

    cpu = None
    if rank == 0 and args.cpu_baseline:
        gbs, rps, nrec, tsec = oracle_sample(job, args.ref_records, budget_s=args.ref_seconds)
        cpu = {"value": gbs, "unit": "GB/s", "cores": 1, "kind": "oracle",
               "sample": f"first {nrec} records of {args.config} as CSR ({tsec:.1f} s; oracle/oracle.cpp std::unordered_map, "
                         f"one thread; generation excluded)", "kv_inserts_per_s": rps,
               "metric_input": "CSR bytes (the oracle takes tokenised records)", **cpu_info()}

    line = {"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": max(args.warmup, 3), "ms_per_step": ms / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
            "kv_inserts_per_s": recs_per_s,
            "config": {"workload": CONFIG_TEXT[args.config] + (" [raw text job, tokenizer fused]" if text_ok else ""),
                       **head, "records": n, "input_csr_bytes": csr,
                       "distinct_keys": job.distinct, "ratio_table_over_budget": args.ratio,
                       "table_footprint_bytes": F, "device_budget_bytes": job.sepo.budget_for(nb, job.page_bytes, pages),
                       "n_buckets": nb, "page_bytes": job.page_bytes, "pool_pages": pages,
                       "passes": st["passes"], "postponed_per_pass": st["postponed_per_pass"],
                       "bytes_evicted": st["bytes_evicted"], "l2": "inputs (8-16 GB) far larger than L2 (126 MB): no flush needed",
                       "parallelism": "1 GPU",
                       "phase_ms": {kk: st[kk] for kk in ("t_insert_ms", "t_reprobe_ms", "t_compact_ms", "t_evict_ms")}},
            "roofline": m1 if m1 is not None else roof_head, "roofline_headline_kernel": roof_head, "roofline_m1_c3": m1_c3,
            "host_link": host_link, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
            "gpu_launches": info["launches"], "slowdown_curve": curve, "csr_job": csr_line}
    if rank == 0:
        print(json.dumps(line), flush=True)
    t.close()
    if dist.is_initialized():
        dist.destroy_process_group()


def run_routed(args, world, rank, local):
    """N GPUs (torchrun) or --route at N=1: key-hash sharding of ONE global CSR stream (strong scaling):
    rank r holds records [r n/N, (r+1) n/N) and every step routes them by key owner (sepo_partition +
    NCCL all-to-all), then runs the SEPO job on the records it owns."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_mokhtaris17_b200 import shard
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29511")
        dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", local))
    job = Job(args.config, args.ratio, scale=args.scale)
    stream = torch.cuda.current_stream()
    fixed = job.stream.family == 2
    n_all = job.stream.n
    j0, j1 = rank * n_all // world, (rank + 1) * n_all // world
    sk, so, sv = job.stream.device(j0, j1 - j0)
    if fixed:
        so = None
    lib_plane = args.plane == "lib"
    router = shard.Router(route_seed=0x5eed, fixed_key_width=8 if fixed else 0,
                          fixed_val_width=job.stream.val_width if sv is not None else 0,
                          # hot-key pre-combine + 32-byte wire records for keys <= 16 B (SURVEY §8(e) makes
                          # it mandatory for Zipf load balance); longer keys (URLs) go as a CSR partition
                          combine=not args.no_combine)
    routed = {}

    def attach(t):  # the library's own NCCL communicator (rank 0 makes the id, torch.distributed carries it)
        if not getattr(t, "_attached", False):
            uid = [job.sepo.nccl_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            t.attach_nccl(uid[0], world, rank)
            t._attached = True

    if lib_plane:
        # sepo_run_sharded: route + NCCL exchange of chunk c+1 on a second stream beside chunk c's insert
        route_fn = None

        def run_lib(t, k=sk, o=so, v=sv):
            attach(t)
            return t.run_sharded(k, o, v)
        job.run_fn = run_lib
    else:
        def route_fn():
            routed["r"] = router.route(sk, so, sv)
            return routed["r"]
        job.run_fn = lambda t: shard.Router.run(t, routed["r"])
        route_fn()
    job.distinct = max(1, job.distinct // world)  # keys per rank (sizes the directory)
    slice_bytes = sk.numel() + (8 * (so.numel() - 1) if so is not None else 0) + (sv.numel() if sv is not None else 0)
    job.bytes_hint = slice_bytes
    nb, pages, F = job.table_params()
    t = job.table()
    for _ in range(max(args.warmup, 3)):
        if route_fn is not None:
            route_fn()
        t.reset()
        job.run_fn(t)
    sampler = ClockSampler(local)
    dist.barrier()
    torch.cuda.synchronize()
    sampler.start()
    ms, info = timed_steps(job, t, args.steps, stream, route_fn)
    clocks = sampler.stop()
    tt = torch.tensor([ms], device="cuda")
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    ms = float(tt.item())
    tb = torch.tensor([slice_bytes], device="cuda", dtype=torch.float64)
    dist.all_reduce(tb)
    csr = float(tb.item())
    value = csr * args.steps / (ms / 1e3) / 1e9
    st = info["last"]
    # e2e: each rank's slice from pinned host memory -> H2D -> route -> job -> export, max over ranks
    e2e = None
    if args.e2e_steps > 0:
        hk = torch.empty(sk.numel(), dtype=torch.uint8, pin_memory=True); hk.copy_(sk)
        ho = torch.empty(so.numel(), dtype=torch.int64, pin_memory=True).copy_(so) if so is not None else None
        hv = torch.empty(sv.numel(), dtype=torch.uint8, pin_memory=True).copy_(sv) if sv is not None else None
        torch.cuda.synchronize()
        dist.barrier()
        t0 = time.perf_counter()
        d2h = 0
        for _ in range(args.e2e_steps):
            dk = hk.to("cuda", non_blocking=True)
            do = ho.to("cuda", non_blocking=True) if ho is not None else None
            dv = hv.to("cuda", non_blocking=True) if hv is not None else None
            torch.cuda.current_stream().synchronize()  # (the table works on its own stream)
            t.reset()
            if lib_plane:
                job.run_fn(t, dk, do, dv)
            else:
                shard.Router.run(t, router.route(dk, do, dv))
            t.export(copy=False)
            d2h += t.stats()["bytes_evicted"]
        torch.cuda.synchronize()
        el = torch.tensor([time.perf_counter() - t0], device="cuda")
        dist.all_reduce(el, op=dist.ReduceOp.MAX)
        el = float(el.item()) / args.e2e_steps
        e2e = {"value": csr / el / 1e9, "unit": "GB/s", "h2d_bytes_per_step": slice_bytes,
               "d2h_bytes_per_step": d2h // args.e2e_steps, "kv_inserts_per_s": n_all / el,
               "note": "per rank: pinned host slice -> H2D -> " + (
                   "sepo_run_sharded (route + NCCL exchange pipelined with pass 1, re-issue passes)" if lib_plane else
                   "route (partition + all-to-all) -> sepo_run") + " -> sepo_export; max over ranks"}
    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": "GB/s", "n_gpus": world, "steps": args.steps,
                "warmup": max(args.warmup, 3), "ms_per_step": ms / args.steps, "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "u64", "data": "synthetic",
                "kv_inserts_per_s": n_all * args.steps / (ms / 1e3),
                "config": {"workload": CONFIG_TEXT[args.config] + " [CSR job, key-hash sharded]", "records": n_all,
                           "input_csr_bytes": csr, "ratio_table_over_budget": args.ratio, "n_buckets": nb,
                           "page_bytes": job.page_bytes, "pool_pages": pages, "passes": st["passes"],
                           "parallelism": f"key-hash sharded x{world} " + (
                               "(sepo_run_sharded: in-library NCCL send/recv, exchange pipelined with pass 1)" if lib_plane
                               else "(sepo_partition / pre-combine + torch.distributed all-to-all)"),
                           "l2": "inputs far larger than L2 (126 MB): no flush needed"},
                "roofline": roofline_of(slice_bytes, info["p1_ms"], args.steps, peaks(),
                                        "pass-1 insert kernel of this rank's job", {"share_of_step": info["p1_ms"] / ms}),
                "route": {"plane": "libsepo NCCL (sepo_run_sharded)"} if lib_plane else router.last_stats(), "e2e": e2e, "clocks": clocks, "gpu_launches": info["launches"],
                "cpu_baseline": None}
        print(json.dumps(line), flush=True)
    t.close()
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
    ap.add_argument("--no-text", dest="text", action="store_false", help="headline on the CSR job instead of raw text")
    ap.add_argument("--no-m1", dest="m1", action="store_false", help="skip the in-budget (0.5x) M1 roofline job")
    ap.add_argument("--no-m1-c3", dest="m1_c3", action="store_false", help="skip the C3 (P = 1) M1 sub-line")
    ap.add_argument("--ref-records", type=int, default=120_000_000)
    ap.add_argument("--ref-seconds", type=float, default=15.0)
    ap.add_argument("--route", action="store_true", help="run the sharded (router) path even at N=1")
    ap.add_argument("--no-combine", action="store_true", help="routed path: CSR partition without the pre-combine")
    ap.add_argument("--plane", choices=["lib", "torch"], default="lib",
                    help="routed path: the library's pipelined NCCL job (sepo_run_sharded) or torch.distributed all-to-all")
    ap.add_argument("--traffic", type=float, default=None, help="dram bytes/launch from an ncu --set full capture")
    args = ap.parse_args()
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
