"""Per-CTA life of a LEAN solve (lower, all thread-level): entry -> rows loaded -> last dependency
published -> last row published; what the CTA's critical (last-publishing) row waited for.
usage: python tools/trace_cta.py CONFIG [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

name = sys.argv[1]
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
opts.setdefault("engine", 3)
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
pub, seen, loaded = tt[:n], tt[n:2 * n], tt[2 * n:3 * n]
entry = tt[3 * n + 3:4 * n + 3]
t0 = entry.min()
pub, loaded, entry = (pub - t0) / 1e3, (loaded - t0) / 1e3, (entry - t0) / 1e3
rps, cis = s.rowptr.astype(np.int64), s.colidx.astype(np.int64)
rows = np.repeat(np.arange(n), np.diff(rps))
off = cis != rows
dep = np.full(n, -1e9)
np.maximum.at(dep, rows[off], pub[cis[off]])
CT = h.info()["cta_threads"]
nc = (n + CT - 1) // CT
q = lambda a: [round(float(np.percentile(a, p)), 2) for p in (10, 50, 90)]
ent = entry[::CT][:nc]
end = np.array([pub[c * CT:(c + 1) * CT].max() for c in range(nc)])
crit = np.array([c * CT + int(np.argmax(pub[c * CT:(c + 1) * CT])) for c in range(nc)])
ld_c, dep_c, pub_c = loaded[crit], dep[crit], pub[crit]
waited_dep = dep_c > ld_c
out = {"cfg": name, "opts": opts, "ctas": nc, "total_us": round(float(pub.max()), 2),
       "cta_life_us_p10_50_90": q(end - ent),
       "cta_entry_to_rows_loaded_us_p10_50_90": q(np.array([loaded[c * CT:(c + 1) * CT].max() for c in range(nc)]) - ent),
       "crit_row_waited_for_dep_frac": round(float(waited_dep.mean()), 3),
       "crit_row_publish_minus_dep_publish_us_p10_50_90 (waited)": q((pub_c - dep_c)[waited_dep]) if waited_dep.any() else None,
       "crit_row_publish_minus_loaded_us_p10_50_90 (not waited)": q((pub_c - ld_c)[~waited_dep]) if (~waited_dep).any() else None,
       "crit_row_loaded_minus_entry_us_p10_50_90": q(ld_c - ent),
       "all_rows_react_us_p10_50_90 (dep after load)": q((pub - dep)[(dep > loaded)]),
       "all_rows_publish_minus_loaded_us_p10_50_90 (dep before load)": q((pub - loaded)[(dep <= loaded) & (dep > -1e8)])}
print(json.dumps(out))
