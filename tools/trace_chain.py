"""Publish-time trace of a pure chain (bidiagonal) solve: in-warp step and warp-boundary hop.
usage: python tools/trace_chain.py N [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

n = int(sys.argv[1])
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
s = synth.gen_chain(n)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
h.check()
x, tr = h.trace(b, x)
t = tr.cpu().numpy().astype(np.int64)[: s.n]
t = (t - t.min()) / 1e3
inf = h.info()
R = 32 * inf["rows_per_lane"]
dt = np.diff(t)
bnd = (np.arange(1, n) % R) == 0
q = lambda a: [round(float(np.percentile(a, p)), 4) for p in (10, 50, 90)]
print(json.dumps({"n": n, "opts": opts, "engine": inf["engine"], "R": R, "total_us": round(float(t.max()), 1),
                  "step_us_p10_50_90": q(dt[~bnd]), "step_us_mean": round(float(dt[~bnd].mean()), 4),
                  "boundary_us_p10_50_90": q(dt[bnd]), "boundary_us_mean": round(float(dt[bnd].mean()), 4)}))
