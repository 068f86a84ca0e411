"""Thread- vs warp-level rows on random (non-leveled) lower matrices, against the nearest-dependency
distance statistic (scratch probe for the f2 dispatch rule).  usage: python tools/dispatch_probe.py"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")


def t_us(h, b, x, reps=10):
    h.solve(b, x)
    h.check()
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    return float(np.median(ts))


for n, k in ((200_000, 2), (200_000, 4), (200_000, 8), (200_000, 12), (200_000, 16), (200_000, 24), (20_000, 4), (20_000, 12)):
    s = synth.gen_random_lower(n, k, seed=k + n % 7)
    rows = np.repeat(np.arange(s.n), np.diff(s.rowptr)); off = s.colidx != rows
    d = rows[off] - s.colidx[off]; dmin = np.full(s.n, 10**9); np.minimum.at(dmin, rows[off], d)
    med = float(np.median(dmin[dmin < 10**9]))
    dev = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(dev) for a in (s.rowptr, s.colidx, s.val, s.b))
    rec = {"n": n, "k": k, "nnz_row": round(s.nnz / s.n, 2), "median_dmin": med}
    for name, opts in (("thread", dict(mode=1)), ("warp", dict(mode=2)), ("auto", {})):
        with cap.analyse(rp, ci, v, **opts) as h:
            x = torch.empty_like(b)
            rec[name] = round(t_us(h, b, x), 1)
            rec[name + "_engine"] = h.info()["engine"]
    print(json.dumps(rec), flush=True)
