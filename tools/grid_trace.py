"""GRID timeline on c3 (measurement build -DSPTRSV_GRID_TRACE): per-row publish times -> per band the step time,
the start lag behind the previous band, and the hand-over delay (band k-1 lane 31 publishes line y -> band k
lane 0 publishes line y).  usage: python paper_conf_icpp_suz0hw0w20_b200/build.py --force -DSPTRSV_GRID_TRACE;
python tools/grid_trace.py"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

s = synth.gen_c3()
m = 2048
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
h = cap.analyse(rp, ci, v)
x = torch.empty_like(b)
for _ in range(3):
    h.solve(b, x)
x, tr = h.trace(b, x)
t = tr[: s.n].cpu().numpy().astype(np.int64).reshape(m, m)  # [line][col]
t = t - t[t > 0].min()
nb = m // 32
print("total span us", t.max() / 1e3)
first = t[:, 0::32]   # lane 0 of each band, per line
last = t[:, 31::32]   # lane 31
step = np.diff(first, axis=0)  # per line step time of lane 0
print("lane-0 step ns: p50 %.0f p90 %.0f" % (np.median(step), np.percentile(step, 90)))
start = first[0]
print("band start lag (us) p50 %.2f p90 %.2f" % (np.median(np.diff(start)) / 1e3, np.percentile(np.diff(start), 90) / 1e3))
hand = first[:, 1:] - last[:, :-1]  # band k lane 0 line y - band k-1 lane 31 line y
print("hand-over ns (pub k-1 lane 31 -> pub k lane 0, same line): p10 %.0f p50 %.0f p90 %.0f" % tuple(np.percentile(hand, [10, 50, 90])))
skew = last - first  # within a band: lane 31 line y - lane 0 line y
print("in-band skew (lane 31 - lane 0, same line) us p50 %.2f" % (np.median(skew) / 1e3))

# the ring warp: when band k stored line y's west value (trace[n + y * nb + k]) vs band k-1's lane 31 publish
ring = tr[s.n: s.n + m * nb].cpu().numpy().astype(np.int64).reshape(m, nb)
t0 = tr[: s.n].cpu().numpy().astype(np.int64)
base = t0[t0 > 0].min()
ring = ring - base
pub31 = (tr[: s.n].cpu().numpy().astype(np.int64).reshape(m, m)[:, 31::32] - base)  # band k lane 31, line y
det = ring[:, 1:] - pub31[:, :-1]
print("ring detection ns (band k-1 lane 31 publish -> band k ring stored): p10 %.0f p50 %.0f p90 %.0f" % tuple(np.percentile(det, [10, 50, 90])))
use = first[:, 1:] - ring[:, 1:] - base * 0  # band k lane 0 publish - ring store (same line)
use = (t[:, 0::32][:, 1:]) - ring[:, 1:]
print("ring store -> band k lane 0 publish ns: p10 %.0f p50 %.0f p90 %.0f" % tuple(np.percentile(use, [10, 50, 90])))
