"""Shared test helpers: run the CUDA path on a generated stream and canonicalise results."""
import numpy as np

import gen
import oracle


def oracle_expected(stream, j0=0, cnt=None):
    keys, offs, vals = stream.host(j0, cnt)
    if stream.val == "doc":
        return oracle.group(keys, offs, vals, val_width=4).as_dict()
    if stream.val == "u64":
        return oracle.combine(keys, offs, vals, 8).as_dict()
    return oracle.combine(keys, offs).as_dict()


def device_inputs(stream, j0=0, cnt=None):
    """(keys, key_offsets or None, vals or None) on cuda; PAIRS use fixed-width 8 B keys"""
    k, o, v = stream.device(j0, cnt)
    if stream.family == gen.GEN_PAIRS:
        return k, None, v
    return k, o, v


def table_kwargs(stream):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    if stream.val == "doc":
        return dict(mode=sepo.GROUP, fixed_val_width=4)
    if stream.val == "u64":
        return dict(mode=sepo.COMBINE, fixed_key_width=8, fixed_val_width=8)
    return dict(mode=sepo.COMBINE)


def run_job(stream, budget, n_buckets, page_bytes, inputs=None, **kw):
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    args = table_kwargs(stream)
    args.update(kw)
    t = sepo.Table(budget, n_buckets, page_bytes, **args)
    k, o, v = inputs if inputs is not None else device_inputs(stream)
    passes = t.run(k, o, v)
    res = t.export()
    st = t.stats()
    got = sepo.result_dict(res, t.mode)
    t.close()
    return got, passes, st


def footprint_pages(stream, n_buckets, page_bytes, inputs=None, **kw):
    """pages an unconstrained run of this stream touches (F of SURVEY §8c reading 23)"""
    import paper_conf_ipps_mokhtaris17_b200 as sepo
    big = sepo.budget_for(n_buckets, page_bytes, 1 << 14)
    _, passes, st = run_job(stream, big, n_buckets, page_bytes, inputs=inputs, **kw)
    assert passes == 1
    return st["pages_used_max"]
