import os, sys, torch
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import paper_conf_ppopp_xia0ar23_b200 as lu
from inputs import gen
name, rp, ci = gen.config(3)
d = torch.device("cuda", 0)
h = lu.Symbolic(torch.from_numpy(rp).to(d), torch.from_numpy(ci).to(d))
fc = h.count()
torch.cuda.synchronize()
st = h.stats()
print({k: st[k] for k in ("rows_deferred", "rows_merge_failed", "merge_entries_read", "merge_rounds", "merge_waits", "ms_tail")})
