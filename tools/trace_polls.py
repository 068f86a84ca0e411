"""Last-dependency poll timing of warp / sub-warp rows (c4-shaped), from a SPTRSV_MEASURE_POLLS build:
wait_start = lane 0 starts polling its last dependency, last_issue = the successful poll's issue,
polls = how many.  Splits detection into 'already published when the wait began' (one poll round
trip) and 'published during the wait' (visibility + poll cadence).
usage: python tools/trace_polls.py N LEVELS KANY [key=value ...]"""
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
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device=d)
flush.zero_()
x, tr = h.trace(b, x)
h.check()
t = tr.cpu().numpy().astype(np.int64)
W = n // L
pub, cons, ws = t[:n], t[n:2 * n], t[2 * n:3 * n]
enc = t[3 * n + 3:4 * n + 3]
npolls = enc >> 40
tl = enc & ((1 << 40) - 1)
rows = np.arange(W, n)
c = s.colidx[s.rowptr[rows + 1] - 2]
gt_hi = pub[rows] & ~((1 << 40) - 1)
last_issue = gt_hi | tl[rows]
q = lambda a: [round(float(np.percentile(a, p)) / 1e3, 3) for p in (10, 50, 90, 99)] if len(a) else []
pre = ws[rows] >= pub[c]          # the dependency was published before the wait began
rtt = (cons[rows] - last_issue)    # successful poll: issue -> consumed (one round trip + mul/add)
inf = h.info()
print(json.dumps({"opts": opts, "n": n, "k": k, "sub_tasks": inf["n_sub_tasks"], "warp_rows": inf["n_warp_rows"], "frac_published_before_wait": round(float(pre.mean()), 3),
                  "polls_p50_p90_p99": [int(np.percentile(npolls[rows], p)) for p in (50, 90, 99)],
                  "rtt_us_if_prepublished": q(rtt[pre]), "rtt_us_all": q(rtt),
                  "detect_us_prepublished": q((cons[rows] - pub[c])[pre]),
                  "detect_us_during_wait": q((cons[rows] - pub[c])[~pre]),
                  "visible_after_pub_us_during_wait": q((last_issue - pub[c])[~pre]),
                  # with a SPTRSV_MEASURE_ROWSTART build, ws = the row's task start instead:
                  "start_before_dep_pub_us": q((pub[c] - ws[rows])),
                  "start_to_wait_us": q((last_issue - ws[rows]))}))
