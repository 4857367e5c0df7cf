"""Exact method work of one traversal per config, from the ORACLE only:
TE = adjacency entries read (seed row + each scanned vertex's row, reading R24), SV = scanned
vertices, nnz(L+U).  Grids (cfg1, 2, 4, 5) use the pinned closed forms TE = sum row_ptr[i+1],
SV = n(n-1)/2 (tests/test_oracle_pins.py: test_closed_form_*); cfg3 runs the oracle (about a
minute on 16 cores).  Writes tests/golden/work_units.json, read by bench.py's roofline.
Usage: python scripts/work_units.py [configs...]"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle  # noqa: E402
from inputs import gen  # noqa: E402

GRID = {1: True, 2: True, 3: False, 4: True, 5: True}
NNZ_GRID = {1: 520_318, 2: 199_868_878, 4: 2_146_437_118, 5: 2_114_707_582}
path = os.path.join(ROOT, "tests", "golden", "work_units.json")
out = json.load(open(path)) if os.path.exists(path) else {}
cfgs = [int(c) for c in sys.argv[1:]] or [1, 2, 3, 4, 5]
for c in cfgs:
    name, rp, ci = gen.config(c)
    n = len(rp) - 1
    if GRID[c]:
        te, sv, nnz, how = int(rp[1:].sum()), n * (n - 1) // 2, NNZ_GRID[c], "closed form"
    else:
        r = oracle.fill2(rp, ci, emit=False, threads=os.cpu_count() or 1)
        te, sv, nnz, how = int(r["te"].sum()), int(r["sv"].sum()), int(r["counts"].sum()), \
            "oracle"
    out[f"cfg{c}"] = {"name": name, "n": n, "nnz_a": int(rp[-1]), "te": te, "sv": sv,
                      "nnz_lu": nnz, "source": how}
    print(c, out[f"cfg{c}"])
json.dump(out, open(path, "w"), indent=1, sort_keys=True)
