"""Run a named synthetic system's solve a few times (ncu target). usage: run_sys.py diag|lev10 reps [opt=v ...]"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_icpp_suz0hw0w20_b200 as cap
name, reps = sys.argv[1], int(sys.argv[2])
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[3:])}
s = synth.gen_diag(1_000_000) if name == "diag" else synth.gen_leveled(1_000_000, int(name[3:]), 1, 1, 2, name)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(reps):
    h.solve(b, x)
h.check()
