"""One count pass over rows [LO, HI) of a config, for ncu captures of the traversal kernel on a
restricted row range (cfg4/cfg5 profiled on their heaviest rows).
Usage: python scripts/prof_count.py CONFIG [LO [HI]]   (HI <= 0: n + HI)"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

cfg = int(sys.argv[1])
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
lo = int(sys.argv[2]) if len(sys.argv) > 2 else 0
hi = int(sys.argv[3]) if len(sys.argv) > 3 else n
hi = n + hi if hi <= 0 else hi
dev = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(dev), torch.from_numpy(ci).to(dev))
fc = torch.zeros(n, dtype=torch.int32, device=dev)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
h.count(lo, hi, fc)
e1.record()
torch.cuda.synchronize()
st = h.stats()
print(f"{name} rows [{lo},{hi}): count {e0.elapsed_time(e1):.2f} ms, SV {st['vertices_scanned_count']}, "
      f"classes {st['row_classes']}, deferred {st['rows_deferred']}")
h.close()
