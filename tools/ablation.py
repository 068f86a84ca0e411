"""SURVEY rows f2 + f3: the paper's kernels vs ours across parallel granularity delta, on B200.

For synthetic leveled matrices spanning the paper's (n_level, nnz_row) plane (Fig.3/4/6,
PAPER.md:216-220, :363, :393-397) it times
  alg3  the paper's SyncFree, warp per row        (Alg.3)
  alg4  the paper's Two-Phase CapelliniSpTRSV     (Alg.4)
  alg5  the paper's Writing-First, literal         (Alg.5)
  thread / warp / auto  this repo's product path with MODE_THREAD / MODE_WARP / AUTO
and reports GFLOPS, delta (Eq.1, Table-6 reading), the paper's headline ratios
(alg5/alg4 -- 28.9x on GTX 1080; alg5/alg3 -- 4.97x avg, Table 5) and the
thread-vs-warp crossover that sets SPTRSV_OPT_WARP_THRESHOLD (f2, sec.4.4).

usage: python tools/ablation.py [n] [out.jsonl]
"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import math
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

n = int(sys.argv[1]) if len(sys.argv) > 1 else 200_000
out = open(sys.argv[2], "w") if len(sys.argv) > 2 else None
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")

def delta_table6(n_level, nnz_row):
    """Eq. 1's parallel granularity in DESIGN.md reading G1 (reporting only)."""
    return math.log10(math.log10(n_level) / (math.log10(nnz_row) + 0.01) + 0.01)

VARIANTS = {"alg3": dict(variant=3), "alg4": dict(variant=4), "alg5": dict(variant=5),
            "thread": dict(mode=1, engine=0), "warp": dict(mode=2, engine=0), "auto": dict()}
if os.environ.get("ABLATION_SET") == "f2":  # thread / sub-warp widths / warp, and AUTO variants
    VARIANTS = {"thread": dict(mode=1), "lean": dict(mode=1, engine=3), "leanp": dict(mode=1, engine=9),
                "warp": dict(mode=2),
                "sub_e1": dict(mode=3, subwarp=1), "sub_e2": dict(mode=3, subwarp=2), "sub_e4": dict(mode=3, subwarp=4),
                "sub_e8": dict(mode=3, subwarp=8), "auto": dict(), "auto_e2": dict(subwarp=2),
                "auto_e4": dict(subwarp=4), "auto_e8": dict(subwarp=8)}


def timeit(h, b, x, reps=5, limit_s=20.0):
    h.solve(b, x)
    h.check()
    ts, t_start = [], time.time()
    for _ in range(reps):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        h.solve(b, x)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e-3)
        if time.time() - t_start > limit_s:
            break
    h.check()
    return float(np.median(ts))


rows = []
LEVELS = [int(v) for v in os.environ.get("ABLATION_LEVELS", "10,100,1000,10000").split(",")]
for levels in LEVELS:
    W = n // levels
    for deps in (2, 4, 8, 16, 32, 64):
        if deps - 1 >= W:
            continue
        s = synth.gen_leveled(n, levels, 1, deps - 1, 40 + levels + deps, f"lev{levels}_d{deps}")
        d = torch.device("cuda")
        rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
        ref = s.x_true  # results are checked against the generator's x_true (tools/ never run the oracle)
        nnz_row = s.nnz / s.n
        rec = {"n": s.n, "levels": levels, "n_level": W, "nnz_row": round(nnz_row, 3),
               "delta": round(delta_table6(W, nnz_row), 4), "gflops": {}}
        for name, opts in VARIANTS.items():
            with cap.analyse(rp, ci, v, **opts) as h:
                x = torch.empty_like(b)
                t = timeit(h, b, x)
                err = float(np.max(np.abs(x.cpu().numpy() - ref) / np.abs(ref)))
                assert err <= 1e-12, (name, err)
                rec["gflops"][name] = round(2 * s.nnz / t / 1e9, 3)
        g = rec["gflops"]
        if "alg5" in g:
            rec["alg5_over_alg4"] = round(g["alg5"] / g["alg4"], 2)
            rec["alg5_over_alg3"] = round(g["alg5"] / g["alg3"], 2)
            rec["ours_over_alg5"] = round(g["auto"] / g["alg5"], 2)
        rec["thread_over_warp"] = round(g["thread"] / g["warp"], 2)
        ours = [v for k, v in g.items() if not k.startswith("alg")]
        rec["auto_over_best"] = round(g["auto"] / max(ours), 3)
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")
        rows.append(rec)
        del rp, ci, v, b
if out:
    out.close()
