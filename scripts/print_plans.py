import sys, torch
sys.path.insert(0, '.')
from inputs import gen
import paper_conf_ppopp_xia0ar23_b200 as lu
for c in (2, 3, 4, 5):
    name, rp, ci = gen.config(c)
    print("cfg", c, name, flush=True)
    h = lu.Symbolic(torch.from_numpy(rp).cuda(), torch.from_numpy(ci).cuda())
    h.close()
