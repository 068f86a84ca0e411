"""Per-hop publish gaps of a chain solve (row i depends on i-S): in-warp vs warp-boundary hops.
usage: python tools/trace_hops.py N S [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_icpp_suz0hw0w20_b200 as cap
from probe import build

n, S = int(sys.argv[1]), int(sys.argv[2])
s = build(f"stride:{n}:{S}")
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[3:])}
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
x, tr = h.trace(b, x)
t = tr.cpu().numpy().astype(np.int64)[:n]
g = np.diff(t[::S]) if S == 1 else np.diff(t)
idx = np.arange(1, len(g) + 1)
wb = (idx % 32) == 0
q = lambda a: [round(float(np.percentile(a, p)), 1) for p in (10, 50, 90, 99)] if len(a) else []
print(json.dumps({"n": n, "S": S, "opts": opts, "engine": h.info()["engine"], "total_us": round((t.max() - t.min()) / 1e3, 2),
                  "inwarp_ns_p10_50_90_99": q(g[~wb]), "warpboundary_ns_p10_50_90_99": q(g[wb]),
                  "first_gaps_ns": [int(a) for a in g[:40]]}))
