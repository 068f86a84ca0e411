"""LEAN row timeline (c2-shaped): per row, CTA entry -> loads landed -> last dependency consumed -> published,
and the waiting rows' dependency distance.  usage: python tools/trace_lean.py SYS [key=value ...] (SYS as probe.py)"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_suz0hw0w20_b200 as cap
from probe import build

s = build(sys.argv[1])
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=d)
flush.zero_()
x, tr = h.trace(b, x)
h.check()
n = s.n
t = tr.cpu().numpy().astype(np.int64)
pub, cons, load, ent = t[:n], t[n:2 * n], t[2 * n:3 * n], t[3 * n + 3:4 * n + 3]
t0, t1 = t[3 * n], t[3 * n + 1]
q = lambda a: [round(float(np.percentile(a, p)) / 1e3, 3) for p in (10, 50, 90, 99)] if len(a) else []
has = cons > 0  # rows that consumed at least one dependency
offd = np.diff(s.rowptr) > 1
last = np.where(offd, s.colidx[np.maximum(s.rowptr[1:] - 2, 0)], -1)
waited = has & (cons - load > 200)  # consumed their last dependency > 0.2 us after the loads landed
out = {"sys": sys.argv[1], "opts": opts, "engine": h.info()["engine"], "kernel_us": round((t1 - t0) / 1e3, 2),
       "entry_to_loaded_us": q(load - ent), "loaded_to_consumed_us": q((cons - load)[has]),
       "consumed_to_pub_us": q((pub - cons)[has]), "entry_to_pub_us": q(pub - ent),
       "frac_rows_waited": round(float(waited.mean()), 4),
       "waited_dep_pub_minus_loaded_us": q((pub[last] - load)[waited & (last >= 0)]),
       "waited_dep_distance_rows_p50": float(np.median((np.arange(n) - last)[waited & (last >= 0)])) if waited.any() else None,
       "cta_entry_spread_us": q(ent - t0), "pub_spread_us": q(pub - t0)}
print(json.dumps(out))
