"""Timeline of a small one-CTA solve (c1-shaped): when rows load, when each level publishes.
usage: python tools/trace_small.py SYS [key=value ...]   (SYS as in probe.py)"""
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
n = s.n
t = tr.cpu().numpy().astype(np.int64)
t0 = t[3 * n]
pub = (t[:n] - t0) / 1e3
last = np.where(t[n:2 * n] > 0, (t[n:2 * n] - t0) / 1e3, np.nan)
start = np.where(t[2 * n:3 * n] > 0, (t[2 * n:3 * n] - t0) / 1e3, np.nan)
lv = np.zeros(n, dtype=np.int64)
for i in range(n):
    c = s.colidx[s.rowptr[i]:s.rowptr[i + 1] - 1]
    lv[i] = 1 + (lv[c].max() if len(c) else 0)
L = lv.max()
out = {"sys": sys.argv[1], "opts": opts, "engine": h.info()["engine"], "levels": int(L),
       "kernel_us": round(float((t[3 * n + 1] - t0) / 1e3), 3),
       "rows_loaded_p50_max": [round(float(np.nanpercentile(start, 50)), 3), round(float(np.nanmax(start)), 3)]}
per = []
for l in range(1, L + 1):
    m = lv == l
    per.append((round(float(pub[m].min()), 3), round(float(pub[m].max()), 3)))
out["level_pub_min_max_us"] = per
print(json.dumps(out))
