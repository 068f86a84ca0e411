"""Run one config's solve a few times (for ncu / sanitizer captures).
usage: python tools/run_one.py CONFIG [reps] [key=value ...]   (handle options, e.g. protocol=1)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

name = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[3:])}
s = synth.make(name)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(reps):
    h.solve(b, x)
h.check()
print(name, opts, "ok")
