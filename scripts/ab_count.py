"""A/B of kernel variants: count-pass time per config/row range for each library build.
Usage: python scripts/ab_count.py LIB1 LIB2 ... (env AB_CASES='2:0:0,5:250000:0,...', REPS)
Each (lib, case) runs in its own process (LUSYM_LIB selects the build); libraries alternate
per repetition so clock drift hits all of them alike."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
cases = [tuple(int(x) for x in c.split(":")) for c in
         os.environ.get("AB_CASES", "2:0:0,5:250000:0,3:0:0,4:1040000:0").split(",")]
reps = int(os.environ.get("REPS", "2"))
libs = sys.argv[1:]
CHILD = r'''
import os, sys, json, torch, numpy as np
sys.path.insert(0, %r)
import paper_conf_ppopp_xia0ar23_b200 as lu
from inputs import gen
cfg, lo, hi = %d, %d, %d
name, rp, ci = gen.config(cfg)
n = len(rp) - 1
hi = n + hi if hi <= 0 else hi
d = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
fc = torch.zeros(n, dtype=torch.int32, device=d)
h.count(lo, hi, fc); torch.cuda.synchronize()
ts = []
for _ in range(3):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(); h.count(lo, hi, fc); e1.record(); torch.cuda.synchronize()
    ts.append(e0.elapsed_time(e1))
print(json.dumps({"ms": min(ts), "sum": int(fc[lo:hi].sum())}))
'''
res = {}
for r in range(reps):
    for lib in libs:
        for c in cases:
            env = dict(os.environ, LUSYM_LIB=os.path.abspath(lib))
            out = subprocess.run([sys.executable, "-c", CHILD % ((ROOT,) + c)], env=env,
                                 capture_output=True, text=True)
            try:
                j = json.loads(out.stdout.strip().splitlines()[-1])
            except Exception:
                print("FAILED", lib, c, out.stderr[-2000:], flush=True)
                continue
            res.setdefault((lib, c), []).append(j)
            print(os.path.basename(lib), c, f"{j['ms']:.2f} ms", j["sum"], flush=True)
print("\nsummary (min over reps):")
for c in cases:
    base = None
    for lib in libs:
        v = res.get((lib, c))
        if not v:
            continue
        ms = min(x["ms"] for x in v)
        sums = {x["sum"] for x in v}
        base = base or ms
        print(f"  cfg{c[0]} [{c[1]},{c[2]}) {os.path.basename(lib):28s} {ms:9.2f} ms  "
              f"{(ms / base - 1) * 100:+6.1f}%  sums {sums}")
