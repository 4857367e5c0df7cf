"""Planner decisions and count/step times per config (create-time sample, row classes, deferral).
Usage: python scripts/exp_plan.py C1 C2 ...  (env EXTRA='dict(...)' handle options)"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

extra = eval(os.environ.get("EXTRA", "dict()"), {"lu": lu, "dict": dict})
dev = torch.device("cuda", 0)
for cfg in (int(x) for x in sys.argv[1:]):
    name, rp, ci = gen.config(cfg)
    n = len(rp) - 1
    trp, tci = torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev)
    h = lu.Symbolic(trp, tci, **extra)
    st = h.stats()
    ts = []
    for _ in range(2 if cfg in (4,) else 3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fc = h.count()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    st = h.stats()
    print(f"{name} {extra}: create ms {st['ms_create']:.1f} sample_sv {st['sample_mean_sv']:.0f} "
          f"classes {st['row_classes']} smem {st['visited_in_smem']} tpr {st['threads_per_row']} "
          f"rif {st['rows_in_flight']} | count ms {min(ts):.1f} tail {st['ms_tail']:.1f} "
          f"deferred {st['rows_deferred']} nnz {int(fc.sum())} sv {st['vertices_scanned_count']} "
          f"spills {st['spills']}", flush=True)
    h.close()
