"""Levelize time (S8+S9) of a config: median of REPS calls on one handle (CUDA events).
Usage: python scripts/lev_time.py CONFIG [rule]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg = int(sys.argv[1])
rule = sys.argv[2] if len(sys.argv) > 2 else "u"
name, rp, ci = gen.config(cfg)
d = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
fc, rp_lu, ci_lu = h.run()
lv0, nl0 = h.levelize(rp_lu, ci_lu, rule)
ts = []
for _ in range(int(os.environ.get("REPS", "7"))):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    lv, nl = h.levelize(rp_lu, ci_lu, rule)
    e1.record()
    torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
    assert nl == nl0 and torch.equal(lv, lv0)
print(f"{name} rule {rule}: levelize ms median {np.median(ts):.3f} min {min(ts):.3f} levels {nl0} "
      f"checksum {int(lv0.double().sum().item())}", flush=True)
