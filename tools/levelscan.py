"""Solve time vs number of levels at fixed n (c2 construction): T(L) = T0 + L * t_level."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap
opts = json.loads(sys.argv[1]) if len(sys.argv) > 1 else {}
flush = torch.empty(64 * 1024 * 1024, dtype=torch.float32, device="cuda")
for L in (1, 2, 5, 10, 20, 50, 100):
    if L == 1:
        s = synth.gen_diag(1_000_000)
    else:
        s = synth.gen_leveled(1_000_000, L, 1, 1, 2, f"lev{L}")
    d = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    h = cap.analyse(rp, ci, v, **opts)
    x = torch.empty_like(b)
    for _ in range(3):
        h.solve(b, x)
    ts = []
    for _ in range(7):
        flush.zero_()
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) * 1e3)
    h.check()
    print(json.dumps({"levels": L, "nnz": s.nnz, "t_us": round(float(np.median(ts)), 2), "opts": opts}), flush=True)
    h.close()
