"""Time SEPO lookups (sepo_lookup, NEXT-4) on the C2 table at table/budget 4 and 1: every
generation is restored into the pool and probed. Queries: the 1.1e9 words of the stream itself
(all present) and the 4.19 M distinct words. CUDA events on the table's stream; JSON lines."""
import json, sys
sys.path.insert(0, '.')
import torch, bench
ratios = [float(x) for x in sys.argv[1:]] or [4.0, 1.0]
for r in ratios:
    job = bench.Job("C2", r)
    t = job.table()
    k, o, v = job.inputs()
    s = torch.cuda.current_stream()
    for name, qk, qo in (("stream", k, o),):
        res = []
        for rep in range(3):
            t.reset(); passes = t.run(k, o, v); torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            found, vals, bm = t.lookup(qk, qo)
            e1.record(s); torch.cuda.synchronize()
            res.append(e0.elapsed_time(e1))
        n = qo.numel() - 1
        st = t.stats()
        print(json.dumps({"cfg": "C2", "ratio": r, "queries": name, "n": n, "found": found, "passes": passes,
                          "generations": passes, "ms": min(res), "lookups_per_s": n / min(res) * 1e3,
                          "table_bytes_restored": st["bytes_evicted"]}), flush=True)
    t.close()
