"""cfg3 count-pass time and tail statistics with deferred rows (reading G8), several window
thresholds.  Usage: python scripts/exp_defer.py CONFIG W1 W2 ...  (W < 0: no deferral)"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg = int(sys.argv[1])
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
dev = torch.device("cuda", 0)
trp, tci = torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev)
ref = None
extra = eval(os.environ.get("EXTRA", "dict()"))
for w in (int(x) for x in sys.argv[2:]):
    h = lu.Symbolic(trp, tci, defer_windows=w, **extra)
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fc = h.count()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    st = h.stats()
    got = fc.cpu().numpy()
    if ref is None:
        ref = got
    print(f"{name} defer_windows={w} {extra}: count ms {min(ts):.1f} (median {np.median(ts):.1f}) "
          f"tail ms {st['ms_tail']:.2f} deferred {st['rows_deferred']} failed "
          f"{st['rows_merge_failed']} merge_read {st['merge_entries_read']} rounds "
          f"{st['merge_rounds']} waits {st['merge_waits']} "
          f"same={np.array_equal(got, ref)} nnz={int(got.sum())}", flush=True)
    h.close()
