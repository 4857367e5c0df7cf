"""Timing of the fill2 count pass on row ranges (which rows bound the step).
Usage: python scripts/exp_ranges.py CONFIG lo1:hi1 lo2:hi2 ...  (negative = n + value)"""
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
h = lu.Symbolic(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev))
fc = torch.zeros(n, dtype=torch.int32, device=dev)
h.count(0, n, fc)
torch.cuda.synchronize()
for spec in sys.argv[2:]:
    a, b = (int(x) for x in spec.split(":"))
    a = a + n if a < 0 else a
    b = b + n if b <= 0 and spec.split(":")[1].startswith("-") else b
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h.count(a, b, fc)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    print(f"{name} rows [{a},{b}) ({b - a} rows): count ms {np.median(ts):.2f} (min {min(ts):.2f})",
          flush=True)
if os.environ.get("ROWPROF"):
    a, b = (int(x) for x in os.environ["ROWPROF"].split(":"))
    a = a + n if a < 0 else a
    b = b + n if b <= 0 else b
    prof = torch.zeros(4 * n, dtype=torch.int64, device=dev)
    h.set_row_profile(prof)
    h.count(a, b, fc)
    torch.cuda.synchronize()
    P = prof.view(n, 4).cpu().numpy()
    cyc = P[:, 0]
    order = np.argsort(-cyc)
    f = fc.cpu().numpy()
    print("rowprof [%d,%d): total %.3e max %.3e" % (a, b, cyc.sum(), cyc.max()))
    for r in order[:40]:
        print("row", r, "cycles %.3e (%.1f ms) sv %d bfs %d windows %d count %d" % (
            P[r, 0], P[r, 0] / 1.9e6, P[r, 1], P[r, 2], P[r, 3], f[r]))
    np.savez_compressed(f"gpurun_out/rowprof_cfg{cfg}_{a}_{b}.npz", prof=P, counts=f)
