"""Helpers for GPU parity tests: run a trace through libarbalest via the binding."""
from __future__ import annotations

import numpy as np


def to_device(rec):
    import torch
    return torch.from_numpy(np.ascontiguousarray(rec, dtype=np.uint64).view(np.int64)).cuda()


def run_gpu(rec, base, size, *, flags=0, bucket_bits=0, report_capacity=0, flush_points=None,
            host=False, global_index=None, ctx=None):
    """Returns (rc, triples, shadow, stats).  flush_points: record indices where
    the trace is cut into separate flushes."""
    import torch
    from paper_conf_ipps_yuphs21_b200 import Context, reports_to_triples
    own = ctx is None
    if own:
        ctx = Context(base, size, flags=flags, bucket_bits=bucket_bits, report_capacity=report_capacity)
    cuts = [0] + list(flush_points or []) + [rec.shape[0]]
    triples = []
    rc = 0
    for a, b in zip(cuts[:-1], cuts[1:]):
        part = np.ascontiguousarray(rec[a:b])
        gi = None if global_index is None else np.ascontiguousarray(global_index[a:b], dtype=np.uint64)
        if b > a:
            if host:
                ctx.submit_events(part, global_index=gi)
            else:
                keep = (to_device(part), None if gi is None else to_device(gi))  # alive until flush
                ctx.submit_events(keep[0], global_index=keep[1])
        rc, n, _ = ctx.flush(check=False)
        if rc < 0:
            break
        triples += reports_to_triples(ctx.get_reports(n))
    shadow = ctx.get_shadow(base // 8, size // 8) if rc >= 0 else None
    st = ctx.stats()
    torch.cuda.synchronize()
    if own:
        ctx.close()
    return rc, triples, shadow, st
