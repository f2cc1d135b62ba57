import sys, time, json
sys.path.insert(0, '.')
import torch, gen, numpy as np
import paper_conf_ipps_mokhtaris17_b200 as sepo
s = gen.config("C2", scale=1 / 64)
k, o, _ = s.device()
n = o.numel() - 1
ones = torch.ones(n, dtype=torch.int64, device="cuda").view(torch.uint8)
def rep(name, fn, pages):
    t = sepo.Table(sepo.budget_for(1 << 18, 16384, pages), 1 << 18, 16384)
    torch.cuda.synchronize(); t0 = time.perf_counter()
    p = fn(t)
    torch.cuda.synchronize(); t1 = time.perf_counter()
    st = t.stats()
    print(json.dumps({"case": name, "ms": (t1 - t0) * 1e3, "passes": p, "ins": [round(x, 2) for x in st["t_insert_ms_per_pass"][:p]],
                      "post": st["postponed_per_pass"][:p]}), flush=True)
    t.close()
for pages in (4096, 300):
    rep("implicit", lambda t: t.run(k, o), pages)
    rep("vals8", lambda t: t.run(k, o, ones), pages)
