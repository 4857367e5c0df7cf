"""e2e of cfg2 through lu_sym_run_host with outputs from the capacity bound, for several chunk
counts (GPU events around: create, bound, pinned allocation, run_host, levelize, level D2H).
    python scripts/e2e_chunks.py [--config 2] [--chunks 0,8,16,32,64] [--reps 4]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from inputs import gen  # noqa: E402
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", type=int, default=2)
ap.add_argument("--chunks", default="0,8,16,32,64")
ap.add_argument("--reps", type=int, default=4)
a = ap.parse_args()
name, rp_np, ci_np = gen.config(a.config)
n = len(rp_np) - 1
dev = torch.device("cuda", 0)
rp_h = torch.from_numpy(rp_np).pin_memory()
ci_h = torch.from_numpy(ci_np).pin_memory()
for nc in [int(x) for x in a.chunks.split(",")]:
    ts = []
    for r in range(a.reps + 1):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        he = lu.Symbolic(rp_h.to(dev, non_blocking=True), ci_h.to(dev, non_blocking=True))
        cap = he.nnz_bound()
        out_rp = torch.empty(n + 1, dtype=torch.int64, pin_memory=True)
        out_ci = torch.empty(cap, dtype=torch.int32, pin_memory=True)
        out_lv = torch.empty(n, dtype=torch.int32, pin_memory=True)
        fc, rp_lu, ci_lu = he.run_host(cap, out_rp, out_ci, nchunks=nc)
        lv, nl = he.levelize(rp_lu, ci_lu)
        out_lv.copy_(lv, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        he.close()
        if r:
            ts.append(e0.elapsed_time(e1))
        del out_rp, out_ci, out_lv, fc, rp_lu, ci_lu, lv
    print(f"{name} nchunks={nc}: e2e ms median {np.median(ts):.2f} min {min(ts):.2f}", flush=True)
