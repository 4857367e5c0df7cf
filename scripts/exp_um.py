"""SURVEY 8(f2) / PAPER.md Figs. 5-6, Table 3 analog: out-of-core scratch (the planner sizes rows
in flight to the HBM that is free) against unified-memory scratch (cudaMallocManaged, with and
without prefetch) when that scratch is oversubscribed.  A ballast allocation leaves FREE_GB of
HBM; the UM handle is given a scratch budget of UM_X times that, so its pages must migrate
during the traversal.  nsys is not in this image, so the share of time spent servicing faults
is estimated as the slowdown against the out-of-core run: (t_UM - t_OOC) / t_UM.
Usage: python scripts/exp_um.py CONFIG [FREE_GB] [UM_X]"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg = int(sys.argv[1]) if len(sys.argv) > 1 else 2
free_gb = float(sys.argv[2]) if len(sys.argv) > 2 else 3.0
um_x = float(sys.argv[3]) if len(sys.argv) > 3 else 4.0
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
d = torch.device("cuda", 0)
trp, tci = torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d)
ref_h = lu.Symbolic(trp, tci)
ref = ref_h.count()
torch.cuda.synchronize()
ref_h.close()
del ref_h
torch.cuda.empty_cache()
free, total = torch.cuda.mem_get_info()
ballast_bytes = max(0, int(free - free_gb * 2**30))
ballast = torch.empty(ballast_bytes // 4, dtype=torch.int32, device=d)
ballast.fill_(1)
torch.cuda.synchronize()
free2, _ = torch.cuda.mem_get_info()
budget = int(free2 * 0.8)
out = {"config": name, "free_gb_after_ballast": free2 / 2**30}


def run(tag, **kw):
    h = lu.Symbolic(trp, tci, **kw)
    ts = []
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fc = h.count()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    st = h.stats()
    ok = bool(torch.equal(fc, ref))
    out[tag] = {"ms": ts, "scratch_gb": st["scratch_bytes"] / 2**30,
                "rows_in_flight": st["rows_in_flight"], "exact": ok}
    print(tag, json.dumps(out[tag]), flush=True)
    h.close()
    torch.cuda.empty_cache()


run("ooc", scratch_budget_bytes=budget)
run("um", scratch_budget_bytes=int(budget * um_x), flags=lu.F_MANAGED)
run("um_prefetch", scratch_budget_bytes=int(budget * um_x), flags=lu.F_MANAGED_PREFETCH)
t_ooc = min(out["ooc"]["ms"])
for k in ("um", "um_prefetch"):
    t = min(out[k]["ms"])
    out[k]["fault_share_est"] = max(0.0, (t - t_ooc) / t)
print(json.dumps(out))
