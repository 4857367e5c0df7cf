"""Count pass over the top R rows of a config (the heaviest ones), for ncu captures of the
latency-bound classes: python scripts/profile_rows.py CONFIG ROWS [threads_per_row]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg, rows = int(sys.argv[1]), int(sys.argv[2])
tpr = int(sys.argv[3]) if len(sys.argv) > 3 else 0
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
dev = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev), threads_per_row=tpr)
prof = torch.zeros(4 * n, dtype=torch.int64, device=dev)
h.set_row_profile(prof)
s0, e0 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
s0.record()
fc = h.count(n - rows, n)
e0.record()
torch.cuda.synchronize()
P = prof.view(n, 4).cpu().numpy()[n - rows:]
st = h.stats()
print(name, f"rows [{n - rows},{n}) count ms {s0.elapsed_time(e0):.2f}", "rows_in_flight",
      st["rows_in_flight"])
print("per row: cycles %.3e  sv %.3e  bfs %.1f  windows %.1f  cycles/sv %.2f" % (
    P[:, 0].mean(), P[:, 1].mean(), P[:, 2].mean(), P[:, 3].mean(), P[:, 0].sum() / P[:, 1].sum()))
