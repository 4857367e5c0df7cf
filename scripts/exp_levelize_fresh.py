"""Levelize time on a fresh handle against a reused one (e2e phases), cfg2."""
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

name, rp, ci = gen.config(int(sys.argv[1]) if len(sys.argv) > 1 else 2)
d = torch.device("cuda", 0)
A = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
h0 = lu.Symbolic(*A)
fc, rp_lu, ci_lu = h0.run()
torch.cuda.synchronize()
for k in range(4):
    for tag, h in (("reused", h0), ("fresh", None), ("no-handle", "none")):
        hh = lu.Symbolic(*A) if h is None else (None if h == "none" else h)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        lv, nl = lu.levelize(rp_lu, ci_lu, "u", handle=hh)
        e1.record()
        torch.cuda.synchronize()
        print(k, tag, f"events {e0.elapsed_time(e1):.2f} ms wall {1e3 * (time.perf_counter() - t0):.2f} ms",
              flush=True)
        if h is None:
            hh.close()
