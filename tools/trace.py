"""Publish-time trace of one solve: where does the critical path spend its time?
usage: python tools/trace.py CONFIG [key=value ...]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, oracle
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
h.check()
x, tr = h.trace(b, x)
t = tr.cpu().numpy().astype(np.int64)
t = t - t.min()
lv = oracle.levels_dp(s.rowptr, s.colidx)
nl = int(lv.max()) + 1
# completion time of each level = max publish time of its rows
lvl_done = np.full(nl, 0, np.int64)
np.maximum.at(lvl_done, lv, t)
lvl_first = np.full(nl, np.iinfo(np.int64).max, np.int64)
np.minimum.at(lvl_first, lv, t)
out = {"cfg": name, "opts": opts, "total_us": float(t.max()) / 1e3, "levels": nl,
       "per_level_us_mean": float(np.diff(lvl_done).mean()) / 1e3 if nl > 1 else None}
q = np.percentile(np.diff(lvl_done), [10, 50, 90]) / 1e3 if nl > 1 else []
out["per_level_us_p10_50_90"] = [round(float(a), 3) for a in q]
if nl <= 40:
    out["level_done_us"] = [round(float(a) / 1e3, 2) for a in lvl_done]
    out["level_first_us"] = [round(float(a) / 1e3, 2) for a in lvl_first]
if name == "chain":
    dt = np.diff(t)
    idx = np.arange(1, s.n)
    inwarp = (idx % 32) != 0
    cta_b = (idx % 256) == 0
    warp_b = ((idx % 32) == 0) & ~cta_b
    out["hop_ns_inwarp_median"] = float(np.median(dt[inwarp]))
    out["hop_ns_warp_boundary_median"] = float(np.median(dt[warp_b]))
    out["hop_ns_cta_boundary_median"] = float(np.median(dt[cta_b]))
    out["sum_us"] = {"inwarp": float(dt[inwarp].sum()) / 1e3, "warp_b": float(dt[warp_b].sum()) / 1e3,
                     "cta_b": float(dt[cta_b].sum()) / 1e3}
print(json.dumps(out))
if name == "c3":
    g = 2048
    T = t.reshape(g, g)
    row_start = T.min(axis=1); row_end = T.max(axis=1)
    print(json.dumps({"c3_row_start_us": [round(float(row_start[r]) / 1e3, 1) for r in range(0, g, 128)],
                      "c3_row_end_us": [round(float(row_end[r]) / 1e3, 1) for r in range(0, g, 128)],
                      "row0_cells_us": [round(float(T[0, c]) / 1e3, 2) for c in range(0, 2048, 128)]}))
