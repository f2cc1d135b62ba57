"""Time the raw-text word-count job (sepo_run_text, fused tokenizer) on C2 next to the CSR job:
python tools/time_text.py [RATIO ...]  -> JSON lines (CUDA events on the table's stream; input in HBM)"""
import json, sys
sys.path.insert(0, '.')
import torch, bench
ratios = [float(x) for x in sys.argv[1:]] or [4.0, 0.5]
for r in ratios:
    job = bench.Job("C2", r)
    t = job.table()
    text = job.stream.text_device()
    tb = text.numel()
    s = torch.cuda.current_stream()
    for _ in range(2):
        t.reset(); t.run_text(text)
    ms = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record(s)
        t.reset(); p = t.run_text(text)
        e1.record(s); torch.cuda.synchronize()
        ms.append(e0.elapsed_time(e1))
    st = t.stats()
    print(json.dumps({"cfg": "C2-text", "ratio": r, "text_bytes": tb, "ms_per_job": min(ms), "text_gbs": tb / min(ms) / 1e6,
                      "words_per_s": job.stream.n / min(ms) * 1e3, "passes": p, "insert_ms_per_pass": [round(x, 3) for x in st["t_insert_ms_per_pass"][:p]],
                      "evict_ms": st["t_evict_ms"], "post": st["postponed_per_pass"][:p]}), flush=True)
    t.close(); del text
