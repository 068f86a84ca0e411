"""Per-level decomposition of a leveled solve (c4-shaped, synth.gen_leveled): for every row of
level >= 1 with its nearest dependency c = the last off-diagonal,
  detect  = when the row consumed c  - when c was published   (publish -> seen)
  compute = when the row published   - when it consumed c       (mul/add, division, publish)
  late    = the row's loads landed after c was published (ingest behind the wavefront)
and the level-completion increments.  usage: python tools/trace_levels.py N LEVELS KANY [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

n, L, k = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
opts = {kk: int(v) for kk, v in (a.split("=") for a in sys.argv[4:])}
s = synth.gen_leveled(n, L, 1, k, 4, "lev")
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
h.check()
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=d)
if not os.environ.get("NOFLUSH"):
    flush.zero_()
x, tr = h.trace(b, x)
h.check()
t = tr.cpu().numpy().astype(np.int64)
W = n // L
pub, cons, load = t[:n], t[n:2 * n], t[2 * n:3 * n]
t0 = pub[:W].min()
rows = np.arange(W, n)
c = s.colidx[s.rowptr[rows + 1] - 2]
ok = (cons[rows] > 0)
q = lambda a: [round(float(np.percentile(a, p)) / 1e3, 3) for p in (10, 50, 90, 99)] if len(a) else []
det = (cons[rows] - pub[c])[ok]
comp = (pub[rows] - cons[rows])[ok]
late = (load[rows] > pub[c]) & (load[rows] > 0)
lev_done = np.array([pub[l * W:(l + 1) * W].max() for l in range(L)])
inc = np.diff(lev_done)
# the critical row of each level (its last publisher) and its own decomposition
crit = np.array([l * W + int(np.argmax(pub[l * W:(l + 1) * W])) for l in range(1, L)])
cc = s.colidx[s.rowptr[crit + 1] - 2]
out = {"n": n, "levels": L, "k": k, "opts": opts, "engine": h.info()["engine"],
       "total_us": round((lev_done[-1] - t0) / 1e3, 1), "per_level_us_p10_50_90_99": q(inc),
       "detect_us_p10_50_90_99": q(det), "compute_us_p10_50_90_99": q(comp),
       "late_rows_frac": round(float(late.mean()), 4),
       "crit_detect_us_p50": q((cons[crit] - pub[cc]))[1] if (cons[crit] > 0).all() else None,
       "crit_compute_us_p50": q(pub[crit] - cons[crit])[1] if (cons[crit] > 0).all() else None,
       "crit_dep_is_prev_crit_frac": round(float(np.mean(cc == crit - W + 0 * cc) if False else np.mean(np.isin(cc, crit))), 3),
       "crit_late_frac": round(float(np.mean(load[crit] > pub[cc])), 3)}
print(json.dumps(out))
