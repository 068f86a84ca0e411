"""Publish-time trace of the 2D grid (c3-shaped) solve: north / west hop costs and the wavefront.
usage: python tools/trace_grid.py G [key=value ...]   (G x G 5-point lower factor)"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

g = int(sys.argv[1])
opts = {k: int(v) for k, v in (a.split("=") for a in sys.argv[2:])}
s = synth.gen_grid(g)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v, **opts)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
h.check()
x, tr = h.trace(b, x)
t = tr.cpu().numpy().astype(np.int64)[: s.n]
t = (t - t.min()).reshape(g, g) / 1e3  # us
inf = h.info()
K = inf["rows_per_lane"]
R = 32 * K
north = t[1:, :] - t[:-1, :]          # T(r,c) - T(r-1,c)
west = t[:, 1:] - t[:, :-1]           # T(r,c) - T(r,c-1)
wb = (np.arange(1, g) % R) == 0       # west step crossing a warp boundary
q = lambda a: [round(float(np.percentile(a, p)), 3) for p in (10, 50, 90)]
rows_done = t.max(axis=1)
rows_first = t.min(axis=1)
out = {"g": g, "opts": opts, "engine": inf["engine"], "K": K, "total_us": round(float(t.max()), 1),
       "north_us_p10_50_90": q(north), "west_inwarp_us_p10_50_90": q(west[:, ~wb]),
       "west_warp_boundary_us_p10_50_90": q(west[:, wb]),
       "row_span_us_p10_50_90": q(rows_done - rows_first),
       "row_first_gap_us_p10_50_90": q(np.diff(rows_first)),
       "row_done_gap_us_p10_50_90": q(np.diff(rows_done)),
       "col0_per_row_us": round(float(t[-1, 0] / (g - 1)), 3),
       "lastcol_per_row_us": round(float((t[-1, -1] - t[0, -1]) / (g - 1)), 3)}
pos = np.arange(g) % R
for name, m in (("pos0", pos == 0), ("pos1", pos == 1), ("pos2_7", (pos >= 2) & (pos < 8)),
                ("pos8_31", (pos >= 8) & (pos < 32)), ("pos32_63", pos >= 32)):
    if m.any():
        out["north_us_p50_" + name] = round(float(np.percentile(north[:, m], 50)), 3)
out["north_us_p50_col0"] = round(float(np.percentile(north[:, 0], 50)), 3)
# how far the row below trails inside one warp: publish time of the warp's first cell relative to
# the north warp's last cell
first = t[1:, ::R]
north_last = t[:-1, R - 1::R][:, : first.shape[1]]
out["warp_first_minus_north_warp_last_us_p10_50_90"] = q(first[:, : north_last.shape[1]] - north_last)
# north split: [n+i] = when cell (r,c) consumed its north (external) dependency (CHAIN / LEAN)
tc = tr.cpu().numpy().astype(np.int64)[s.n: 2 * s.n]
if (tc[g:] > 0).mean() > 0.5:
    t0 = tr.cpu().numpy().astype(np.int64)[: s.n].min()
    tcu = ((tc - t0) / 1e3).reshape(g, g)
    seen = tcu[1:, :] - t[:-1, :]      # north published -> consumed by the cell below
    pub = t[1:, :] - tcu[1:, :]        # north consumed -> the cell's own publish
    ok = tc.reshape(g, g)[1:, :] > 0
    out["north_seen_us_p10_50_90"] = q(seen[ok])
    out["north_consumed_to_publish_us_p10_50_90"] = q(pub[ok])
    # CHAINP: [2n+i] = when the chain warp started a run at row i (0 = not a run start)
    rs = tr.cpu().numpy().astype(np.int64)[2 * s.n: 3 * s.n]
    if (rs > 0).any():
        rsu = ((rs - t0) / 1e3).reshape(g, g)
        okr = (rs.reshape(g, g) > 0) & (tc.reshape(g, g) > 0)
        okr[0, :] = False
        out["run_starts_per_row"] = round(float(okr.sum() / (g - 1)), 2)
        out["handover_us_p10_50_90"] = q((rsu - tcu)[okr])
        out["runstart_to_publish_us_p10_50_90"] = q((t - rsu)[okr])
        ho = tr.cpu().numpy().astype(np.int64)[3 * s.n + 3: 4 * s.n + 3]
        if (ho > 0).any():
            hou = ((ho - t0) / 1e3).reshape(g, g)
            okh = okr & (ho.reshape(g, g) > 0)
            out["consumed_to_handed_us_p10_50_90"] = q((hou - tcu)[okh])
            out["handed_to_runstart_us_p10_50_90"] = q((rsu - hou)[okh])
            # pair boundaries (c % R == 0, c > 0): west published -> west consumed -> handed -> run -> publish
            bc = np.arange(R, g, R)
            if bc.size:
                wp = t[:, bc - 1]
                out["bnd_west_pub_to_consumed_us_p10_50_90"] = q((tcu[:, bc] - wp).ravel())
                out["bnd_consumed_to_handed_us_p10_50_90"] = q((hou[:, bc] - tcu[:, bc]).ravel())
                out["bnd_handed_to_runstart_us_p10_50_90"] = q((rsu[:, bc] - hou[:, bc]).ravel())
                out["bnd_runstart_to_pub_us_p10_50_90"] = q((t[:, bc] - rsu[:, bc]).ravel())
                out["bnd_north_pub_minus_west_pub_us_p10_50_90"] = q((np.vstack([t[:1, bc] * 0, t[:-1, bc]]) - wp)[1:].ravel())
        c0 = okr[:, 0]
        out["col0_seen_handover_publish_us"] = [round(float(np.median(seen[:, 0])), 3),
                                                 round(float(np.median((rsu - tcu)[c0, 0])), 3),
                                                 round(float(np.median((t - rsu)[c0, 0])), 3)]
print(json.dumps(out))
