"""cfg3 per-step count times in the bench's step pattern (L2 flush, count, scan, emit, levelize),
to look at run-to-run variation.  python scripts/cfg3_steps.py [steps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

name, rp, ci = gen.config(3)
n = len(rp) - 1
d = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
flush = torch.empty((256 << 20) // 4, dtype=torch.int32, device=d)
out = []
for k in range(int(sys.argv[1]) if len(sys.argv) > 1 else 8):
    flush.fill_(k)
    fc = torch.zeros(n, dtype=torch.int32, device=d)
    h.count(0, n, fc)
    rp_lu, nnz = h.scan(fc)
    ci_lu = torch.empty(nnz, dtype=torch.int32, device=d)
    h.emit(rp_lu, ci_lu, 0, n)
    lv, nl = h.levelize(rp_lu, ci_lu, "u")
    st = h.stats()
    out.append((round(st["ms_count"], 1), round(st["ms_tail"], 1), st["rows_deferred"]))
print(out, flush=True)
