import os, sys
sys.path.insert(0, "/root/repo") if os.path.exists("/root/repo") else None
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
import numpy as np, torch
import oracle, paper_conf_ppopp_xia0ar23_b200 as lu
from inputs import gen
from tests.test_gpu_multirank import _hubs
d = torch.device("cuda", 0)
for world in (2, 3):
  for name, (rp, ci) in (("lap3d9", gen.lap3d(9)), ("circuit48", gen.circuit(48, 3)), ("hubs", _hubs()), ("random", gen.random_pattern(800, 2.2, seed=4))):
    ref = oracle.fill2(rp, ci); n = len(rp) - 1
    A = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    b = lu.partition_rows(lu.row_cost_upper_bound(rp), world)
    hs = [lu.Symbolic(*A, flags=lu.F_DEFER_GLOBAL, defer_windows=2) for _ in range(world)]
    fc = torch.zeros(n, dtype=torch.int32, device=d); flags = torch.zeros(n, dtype=torch.int32, device=d)
    for r in range(world):
        part = torch.zeros(n, dtype=torch.int32, device=d)
        hs[r].count(int(b[r]), int(b[r+1]), part); fc += part; flags |= hs[r].deferred_flags()
    torch.cuda.synchronize(); print(name, world, "counted", int(flags.sum()), flush=True)
    rp_lu, nnz = hs[0].scan(fc)
    for r in range(1, world): hs[r].scan(fc)
    ci_lu = torch.zeros(nnz, dtype=torch.int32, device=d)
    for r in range(world): hs[r].emit(rp_lu, ci_lu, int(b[r]), int(b[r+1]))
    torch.cuda.synchronize(); print(name, "emitted", flush=True)
    for r in range(world):
        fcr, rpr = fc.clone(), rp_lu.clone()
        nnz2 = hs[r].merge_deferred(flags, fcr, rpr, ci_lu)
        out = hs[r].emit(rpr, torch.empty(nnz2, dtype=torch.int32, device=d))
        torch.cuda.synchronize()
        print(name, world, r, np.array_equal(out.cpu().numpy(), ref["col_idx"]), flush=True)
    for h in hs: h.close()
