"""Publish-time trace of one solve: where does the critical path spend its time?
usage: python tools/trace.py CONFIG [key=value ...]"""
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
h.check()
x, tr = h.trace(b, x)
tt = tr.cpu().numpy().astype(np.int64)
t0 = tt[: s.n].min()
if tt.size >= 3 * s.n + 3 and tt[3 * s.n + 1] > 0:
    print(json.dumps({"kernel_entry_to_first_publish_us": round((t0 - tt[3 * s.n]) / 1e3, 2),
                      "last_publish_to_last_exit_us": round((tt[3 * s.n + 1] - tt[: s.n].max()) / 1e3, 2),
                      "ctas": int(tt[3 * s.n + 2])}))
t = tt[: s.n] - t0
seen = np.where(tt[s.n:2 * s.n] > 0, tt[s.n:2 * s.n] - t0, -1)
start = np.where(tt[2 * s.n:3 * s.n] > 0, tt[2 * s.n:3 * s.n] - t0, -1)
lv = h.levels()[0].cpu().numpy()  # the GPU level diagnostic (tools/ never run the oracle)
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
    stv = tt[2 * s.n:3 * s.n]
    if (stv > 0).all():
        st0 = stv - t0
        out["level_start_p0_50_100_us"] = [[round(float(np.percentile(st0[lv == l], q)) / 1e3, 2) for q in (0, 50, 100)]
                                           for l in range(nl)]
        out["level_publish_p50_us"] = [round(float(np.percentile(t[lv == l], 50)) / 1e3, 2) for l in range(nl)]
    ent = tt[3 * s.n + 3:4 * s.n + 3] if tt.size >= 4 * s.n + 3 else np.zeros(0)
    if ent.size and (ent > 0).all():
        e0 = ent - t0
        out["level_entry_p0_50_100_us"] = [[round(float(np.percentile(e0[lv == l], q)) / 1e3, 2) for q in (0, 50, 100)]
                                           for l in range(nl)]
        if (stv > 0).all():
            ld = (stv - ent)
            out["load_latency_ns_p10_50_90"] = [int(np.percentile(ld, q)) for q in (10, 50, 90)]
if name.startswith("chain"):
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
# ---- reaction time: publish(i) - max publish(dependencies of i), per row (the hop under load)
rp, ci = s.rowptr.astype(np.int64), s.colidx.astype(np.int64)
rows = np.repeat(np.arange(s.n), np.diff(rp))
off = ci != rows
dep_t = np.zeros(s.n, np.int64)
np.maximum.at(dep_t, rows[off], t[ci[off]])
has = np.bincount(rows[off], minlength=s.n) > 0
react = (t - dep_t)[has]
sv = seen[has]
okm = sv >= 0
vis = (sv - dep_t[has])[okm]       # dependency published -> seen ready by the consumer
proc = (t[has] - sv)[okm]          # seen ready -> consumer published
st_h = start[has]
wait_before_start = (st_h - dep_t[has])[st_h >= 0]  # > 0: the consumer started after its dep was published
print(json.dumps({"consumer_started_after_dep_frac": round(float((wait_before_start > 0).mean()), 3) if wait_before_start.size else None,
                  "start_minus_dep_ns_p10_50_90": [int(np.percentile(wait_before_start, q)) for q in (10, 50, 90)] if wait_before_start.size else None,
                  "row_start_us_by_decile": [round(float(np.percentile(start[start >= 0], q)) / 1e3, 2) for q in range(0, 101, 10)] if (start >= 0).any() else None}))
print(json.dumps({"visibility_ns_p10_50_90": [int(np.percentile(vis, q)) for q in (10, 50, 90)] if okm.any() else None,
                  "seen_to_publish_ns_p10_50_90": [int(np.percentile(proc, q)) for q in (10, 50, 90)] if okm.any() else None}))
print(json.dumps({"react_ns_p10_50_90_99": [int(np.percentile(react, q)) for q in (10, 50, 90, 99)],
                  "nodep_publish_us_p10_50_90_max": [round(float(np.percentile(t[~has], q)) / 1e3, 2) for q in (10, 50, 90, 100)] if (~has).any() else None,
                  "frac_react_gt_2us": round(float((react > 2000).mean()), 4)}))
