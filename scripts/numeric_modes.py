"""Numeric phase in GLU3.0's dense column mode against the sparse (Alg. 6) mode:
device time of lu_numeric_factor_ex per mode on a few patterns (CUDA events, median of 3).
Usage: python scripts/numeric_modes.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

d = torch.device("cuda", 0)
for name, (rp, ci) in (("cfg1 lap2d64", gen.lap2d(64)), ("lap3d16", gen.lap3d(16)),
                       ("lap2d128", gen.lap2d(128)), ("circuit128", gen.circuit(128, 1))):
    val = gen.dominant_values(rp, ci, 1, dtype=np.float32)
    A = [torch.from_numpy(x).to(d) for x in (rp, ci, val)]
    h = lu.Symbolic(A[0], A[1])
    _, rp_lu, ci_lu = h.run()
    lv, nl = h.levelize(rp_lu, ci_lu, "glu3")
    h.close()
    lptr, lcols = lu.level_schedule(lv, nl)
    res = {}
    ref = None
    for mode in ("sparse", "dense", "auto"):
        ts = []
        for r in range(4):
            v = lu.numeric_scatter(A[0], A[1], A[2], rp_lu, ci_lu)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            lu.numeric_factor(rp_lu, ci_lu, lptr, lcols, v, mode=mode)
            e1.record()
            torch.cuda.synchronize()
            if r:
                ts.append(e0.elapsed_time(e1))
        out = v.cpu().numpy().astype(np.float64)
        if ref is None:
            ref = out
        rel = float(np.max(np.abs(out - ref)) / max(np.max(np.abs(ref)), 1e-30))
        res[mode] = (float(np.median(ts)), rel)
    print(name, f"levels {nl}", " ".join(f"{m}: {t:.2f} ms (max rel diff vs sparse {r:.1e})"
                                         for m, (t, r) in res.items()), flush=True)
