"""Time the router kernels alone (CUDA events): CSR partition and pre-combine at P parts.
python tools/time_route.py CFG SCALE P... -> JSON lines"""
import json, sys
sys.path.insert(0, '.')
import torch, gen
from paper_conf_ipps_mokhtaris17_b200 import shard
cfg, scale = sys.argv[1], float(sys.argv[2])
Ps = [int(x) for x in sys.argv[3:]] or [1, 8]
s = gen.config(cfg, scale=scale)
k, o, v = s.device()
fixed = s.family == gen.GEN_PAIRS
ko = None if fixed else o
kw = 8 if fixed else 0
vw = 8 if v is not None else 0
nbytes = k.numel() + (0 if fixed else 8 * s.n) + (v.numel() if v is not None else 0)
st = torch.cuda.current_stream()
for P in Ps:
    first = shard.route_combine(k, ko, v, P, 7, kw, vw)
    buf = first[0] if first is not None else None
    for name, fn in (("partition", lambda: shard.partition(k, ko, v, P, 7, kw, vw)),
                     ("combine", lambda: shard.route_combine(k, ko, v, P, 7, kw, vw, out=buf))):
        if name == "combine" and buf is None:
            continue
        r = fn()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize(); e0.record(st)
        for _ in range(3):
            fn()
        e1.record(st); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(json.dumps({"cfg": cfg, "P": P, "kernel": name, "ms": ms, "input_gbs": nbytes / ms / 1e6, "records": s.n}), flush=True)
