"""Per-row profile of the fill2 count pass (the paper's Fig. 3 analog: per-row work grows with
the row id, L249/L272).  Usage: python scripts/row_profile.py CONFIG [out.npz]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 3
out = sys.argv[2] if len(sys.argv) > 2 else f"gpurun_out/rowprof_cfg{cfg}.npz"
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
dev = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev))
prof = torch.zeros(4 * n, dtype=torch.int64, device=dev)
h.count()                       # warm-up
h.set_row_profile(prof)
s0, e0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s0.record()
fc = h.count()
e0.record()
torch.cuda.synchronize()
P = prof.view(n, 4).cpu().numpy()
np.savez_compressed(out, prof=P, counts=fc.cpu().numpy(), ms=s0.elapsed_time(e0))
cyc = P[:, 0]
order = np.argsort(-cyc)
print(name, "count ms", s0.elapsed_time(e0), "stats", h.stats()["rows_in_flight"])
print("total row-cycles %.3e, max %.3e (row %d), p50 %.0f" % (cyc.sum(), cyc.max(), order[0],
      np.median(cyc)))
for q in (10, 100, 1000):
    print(f"top {q} rows: {cyc[order[:q]].sum() / cyc.sum() * 100:.1f}% of cycles")
for r in order[:10]:
    print("row", r, "cycles %.3e sv %d bfs %d windows %d count %d" % (P[r, 0], P[r, 1], P[r, 2], P[r, 3], fc[r]))
print("sum(row cycles)/SMs = %.3e cycles (%.0f ms at 1.9 GHz); max row %.3e cycles (%.0f ms)" % (
    cyc.sum() / 148, cyc.sum() / 148 / 1.9e6, cyc.max(), cyc.max() / 1.9e6))
