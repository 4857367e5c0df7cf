"""Small end-to-end runs of every kernel family for compute-sanitizer (memcheck, racecheck,
synccheck): validate + plan + fill2 count/stage (shared, split, HBM and sparse classes) + row-merge
tail (single CTA and cluster) + scan + place / emit + levelize (both rules) + schedule + level
types + numeric scatter/factor + the pipelined host run.  Each result is checked against the
oracle.  Usage: compute-sanitizer --tool T python scripts/sanitize.py"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import paper_conf_ppopp_xia0ar23_b200 as lu  # noqa: E402
from inputs import gen  # noqa: E402

d = torch.device("cuda", 0)


def hubs(n=600, k=4, deg=200):
    rp0, ci0 = gen.random_pattern(n, 1.5, seed=7)
    R = [np.repeat(np.arange(n), np.diff(rp0))]
    C = [ci0.astype(np.int64)]
    for hub in range(n - k, n):
        nb = np.random.default_rng(hub).choice(n, deg, replace=False)
        R += [np.full(nb.size, hub), nb]
        C += [nb, np.full(nb.size, hub)]
    return gen.csr_from_edges(n, np.concatenate(R), np.concatenate(C))


cases = [("lap2d16", gen.lap2d(16)), ("lap3d7", gen.lap3d(7)), ("circuit24", gen.circuit(24, 1)),
         ("hubs", hubs())]
knobs = [dict(), dict(defer_windows=1), dict(flags=lu.F_FORCE_CLASSES, queue_capacity=32),
         dict(flags=lu.F_GLOBAL_BITMAP), dict(flags=lu.F_TWO_PASS),
         dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS, queue_capacity=2048),
         dict(threads_per_row=1025, flags=lu.F_ASYNC_BFS | lu.F_GLOBAL_BITMAP)]
ok = True
for name, (rp, ci) in cases:
    ref = oracle.fill2(rp, ci)
    A = (torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
    for kn in knobs:
        h = lu.Symbolic(*A, **kn)
        fc, rp_lu, ci_lu = h.run()
        good = np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
        for rule in ("u", "glu3"):
            lv, nl = h.levelize(rp_lu, ci_lu, rule)
            good &= np.array_equal(lv.cpu().numpy(), oracle.levels(ref["row_ptr"], ref["col_idx"], rule)[0])
        if not kn:
            nnz = int(ref["row_ptr"][-1])
            hc = torch.empty(nnz, dtype=torch.int32).pin_memory()
            h.run_host(nnz, None, hc, nchunks=3)
            torch.cuda.synchronize()
            good &= np.array_equal(hc.numpy(), ref["col_idx"])
        h.close()
        print(name, kn, "OK" if good else "MISMATCH", flush=True)
        ok &= bool(good)
    # sparse class + cluster tail with many deferred rows
    os.environ["LUSYM_FORCE_SPARSE"] = "1"
    h = lu.Symbolic(*A, defer_windows=1)
    fc, rp_lu, ci_lu = h.run()
    good = np.array_equal(ci_lu.cpu().numpy(), ref["col_idx"])
    del os.environ["LUSYM_FORCE_SPARSE"]
    h.close()
    # deferred rows across shards (two handles)
    n = len(rp) - 1
    hs = [lu.Symbolic(*A, flags=lu.F_DEFER_GLOBAL, defer_windows=1) for _ in range(2)]
    b = [0, n // 2, n]
    fcs = torch.zeros(n, dtype=torch.int32, device=d)
    flags = torch.zeros(n, dtype=torch.int32, device=d)
    for r in range(2):
        part = torch.zeros(n, dtype=torch.int32, device=d)
        hs[r].count(b[r], b[r + 1], part)
        fcs += part
        flags |= hs[r].deferred_flags()
    rp_lu, nnz = hs[0].scan(fcs)
    hs[1].scan(fcs)
    ci0 = torch.zeros(nnz, dtype=torch.int32, device=d)
    for r in range(2):
        hs[r].emit(rp_lu, ci0, b[r], b[r + 1])
    nnz2 = hs[1].merge_deferred(flags, fcs, rp_lu, ci0)
    out = hs[1].emit(rp_lu, torch.empty(nnz2, dtype=torch.int32, device=d))
    good &= np.array_equal(out.cpu().numpy(), ref["col_idx"])
    for hh in hs:
        hh.close()
    print(name, "sparse+tail+shards", "OK" if good else "MISMATCH", flush=True)
    ok &= bool(good)
# numeric phase
rp, ci = gen.lap2d(10)
val = gen.dominant_values(rp, ci, 3, dtype=np.float32)
lu.factorize(*(torch.from_numpy(x).to(d) for x in (rp, ci, val)))
torch.cuda.synchronize()
print("numeric OK")
print("ALL OK" if ok else "FAILED")
sys.exit(0 if ok else 1)
