"""Where the e2e time goes: host wall time of each public-API call of one end-to-end step
(fresh handle every step, as bench.py's e2e does), each call followed by a device sync.

    python scripts/e2e_probe.py [--config 2] [--steps 4]
"""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from inputs import gen  # noqa: E402
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=2)
    ap.add_argument("--steps", type=int, default=4)
    a = ap.parse_args()
    name, rp_np, ci_np = gen.config(a.config)
    n = len(rp_np) - 1
    dev = torch.device("cuda", 0)
    rp_h = torch.from_numpy(rp_np).pin_memory()
    ci_h = torch.from_numpy(ci_np).pin_memory()
    for k in range(a.steps):
        t = {}
        torch.cuda.synchronize()

        def tick(tag, t0=[time.perf_counter()]):
            torch.cuda.synchronize()
            now = time.perf_counter()
            t[tag] = round((now - t0[0]) * 1e3, 3)
            t0[0] = now

        rpd = rp_h.to(dev, non_blocking=True)
        cid = ci_h.to(dev, non_blocking=True)
        tick("h2d")
        he = lu.Symbolic(rpd, cid)
        tick("create")
        fc = torch.zeros(n, dtype=torch.int32, device=dev)
        he.count(0, n, fc)
        tick("count")
        rp_lu, nz = he.scan(fc)
        tick("scan")
        ci_lu = torch.empty(nz, dtype=torch.int32, device=dev)
        out_ci = torch.empty(nz, dtype=torch.int32, pin_memory=True)
        tick("alloc")
        he.emit(rp_lu, ci_lu, 0, n)
        tick("emit")
        level, nl = he.levelize(rp_lu, ci_lu, "u")
        tick("levelize")
        level2, nl = he.levelize(rp_lu, ci_lu, "u")
        tick("levelize_again")
        out_ci.copy_(ci_lu, non_blocking=True)
        tick("d2h")
        st = he.stats()
        he.close()
        tick("close")
        print(f"step {k}: {t}  ms_create(lib)={st['ms_create']:.3f} ms_lev(lib)={st['ms_levelize']:.3f}",
              flush=True)


if __name__ == "__main__":
    main()
