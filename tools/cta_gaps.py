"""LEAN trace: per-CTA entry / loaded / done, and the slot-free -> next-CTA-entry gap.
usage: python tools/cta_gaps.py CONFIG [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

name = sys.argv[1]
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
s = synth.make(name)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
x, tr = h.trace(b, x)
tt = tr.cpu().numpy().astype(np.int64)
n = s.n
pub, start, ent = tt[:n], tt[2 * n:3 * n], tt[3 * n + 3:4 * n + 3]
t0 = ent.min()
C = 256
nc = (n + C - 1) // C
pad = nc * C - n
def per(a, f):
    a = np.concatenate([a, np.full(pad, a[-1])]).reshape(nc, C)
    return f(a, axis=1)
e = per(ent - t0, np.min) / 1e3
ld = per(start - t0, np.max) / 1e3
dn = per(pub - t0, np.max) / 1e3
res = int(sys.argv[-1].split("=")[1]) if sys.argv[-1].startswith("res=") else 740
# slot-free -> entry: CTA c (c >= res) takes the slot freed by the (c - res)-th earliest-finishing CTA
order = np.sort(dn)
gap = e[res:] - order[: nc - res]
out = {"cfg": name, "ctas": nc, "total_us": round(float(dn.max()), 2),
       "entry_to_loaded_us_p10_50_90": [round(float(np.percentile(ld - e, q)), 2) for q in (10, 50, 90)],
       "loaded_to_done_us_p10_50_90": [round(float(np.percentile(dn - ld, q)), 2) for q in (10, 50, 90)],
       "lifetime_us_p10_50_90": [round(float(np.percentile(dn - e, q)), 2) for q in (10, 50, 90)],
       "slotfree_to_entry_us_p10_50_90": [round(float(np.percentile(gap, q)), 2) for q in (10, 50, 90)],
       "entry_us_every_370": [round(float(a), 2) for a in e[::370]],
       "done_us_every_370": [round(float(a), 2) for a in dn[::370]]}
print(json.dumps(out))
