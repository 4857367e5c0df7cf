"""Count-pass time of one config on a row range under several handle options (A/B of planner
knobs).  Usage: python scripts/exp_knobs.py CONFIG LO HI 'dict(...)' 'dict(...)' ..."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg, lo, hi = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
hi = n if hi <= 0 else hi
dev = torch.device("cuda", 0)
trp, tci = torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev)
ref = None
for spec in sys.argv[4:]:
    kw = eval(spec, {"lu": lu, "dict": dict})
    h = lu.Symbolic(trp, tci, **kw)
    fc = torch.zeros(n, dtype=torch.int32, device=dev)
    ts = []
    for _ in range(int(os.environ.get('REPS', '2'))):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        h.count(lo, hi, fc)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    got = fc[lo:hi].cpu().numpy()
    if ref is None:
        ref = got
    st = h.stats()
    print(f"{name} [{lo},{hi}) {spec}: count ms {min(ts):.3f} same={np.array_equal(got, ref)} "
          f"rif={st['rows_in_flight']} tpr={st['threads_per_row']} smem={st['smem_bytes_per_row']} "
          f"classes={st['row_classes']} q={st['queue_capacity']} spills={st['spills']}", flush=True)
    h.close()
