"""Time the numeric phase (lu_numeric_factor, Alg. 2) on BASELINE-shaped patterns (under gpurun).

Prints one JSON line per workload: ms per factorization (CUDA events on the launching stream,
after warm-up), Alg. 2 updates (sum over columns j of |L(:,j)| * |U(j,:)|, 2 flops each), the
number of GLU3 levels (one launch each)."""
import json
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402


def run(name, rp, ci, reps=3):
    d = torch.device("cuda", 0)
    val = gen.dominant_values(rp, ci, 1, dtype=np.float32)
    trp, tci, tv = (torch.from_numpy(x).to(d) for x in (rp, ci, val))
    h = lu.Symbolic(trp, tci)
    _, rp_lu, ci_lu = h.run()
    level, nl = lu.levelize(rp_lu, ci_lu, rule="glu3")
    torch.cuda.synchronize()
    lv_ms = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        lu.levelize(rp_lu, ci_lu, rule="glu3", level=level, handle=h)
        b.record()
        torch.cuda.synchronize()
        lv_ms.append(a.elapsed_time(b))
    h.close()
    lptr, lcols = lu.level_schedule(level, nl)
    rph, cih = rp_lu.cpu().numpy(), ci_lu.cpu().numpy()
    n = len(rph) - 1
    row = np.repeat(np.arange(n), np.diff(rph))
    nl_col = np.bincount(cih[cih < row], minlength=n)
    nu_row = np.bincount(row[cih > row], minlength=n)
    updates = int((nl_col.astype(np.int64) * nu_row).sum())
    s = torch.cuda.current_stream()
    ts = []
    for r in range(reps + 1):
        v = lu.numeric_scatter(trp, tci, tv, rp_lu, ci_lu)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        lu.numeric_factor(rp_lu, ci_lu, lptr, lcols, v)
        e1.record(s)
        torch.cuda.synchronize()
        if r:
            ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts))
    import os
    mode = "per-level" if os.environ.get("LUSYM_NUMERIC_LAUNCH_PER_LEVEL") == "1" else "coop"
    if mode == "coop" and os.environ.get("LUSYM_NUMERIC_TABLE") == "0":
        mode = "coop-no-table"
    print(json.dumps({"workload": name, "mode": mode, "n": n, "nnz_lu": int(len(cih)), "levels_glu3": nl,
                      "updates": updates, "levelize_glu3_ms": float(np.median(lv_ms)), "ms": ms, "gflops": 2 * updates / ms / 1e6,
                      "us_per_level": 1e3 * ms / max(nl, 1)}), flush=True)


if __name__ == "__main__":
    cases = {"cfg1 lap2d_k64": lambda: gen.lap2d(64), "lap3d_k16": lambda: gen.lap3d(16),
             "lap2d_k128": lambda: gen.lap2d(128), "circuit_s128": lambda: gen.circuit(128, 1),
             "lap3d_k24": lambda: gen.lap3d(24)}
    for name in (sys.argv[1:] or cases):
        run(name, *cases[name]())
