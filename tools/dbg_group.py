import sys; sys.path.insert(0, '.')
import torch, gen, json
import paper_conf_ipps_mokhtaris17_b200 as sepo
for sc in (1/64,):
    s = gen.config("C4", scale=sc)
    k, o, v = s.device()
    t = sepo.Table(sepo.budget_for(1 << 18, 16384, (8 << 30) // 16384), 1 << 18, 16384, mode=sepo.GROUP, fixed_val_width=4)
    t.run(k, o, v)
    r = t.export(copy=False)
    st = t.stats()
    print(json.dumps({"scale": sc, "n": s.n, "keys": r["n_keys"], "vals": r["n_vals"], "pages": st["pages_used_max"],
                      "MB": st["pages_used_max"] * 16384 / 2**20, "chunks": st["value_chunks"], "slots": st["value_slots"],
                      "dead": st["dead_bytes"], "ins_ms": st["t_insert_ms"]}))
