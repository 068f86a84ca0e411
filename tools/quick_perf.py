"""Scratch perf probe: per-config solve time (CUDA events, L2 flushed), GFLOPS, %HBM roof."""
import json, sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

PEAK = 6539.9e9
cfgs = sys.argv[1].split(",") if len(sys.argv) > 1 else ["c1", "c2", "c3", "c4", "chain"]
opts = json.loads(sys.argv[2]) if len(sys.argv) > 2 else {}
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
for p in (0, 1, 2, 3, 4, 5, 6, 7):
    print("flag_latency proto", p, "%.1f ns @ %.0f MHz" % cap.flag_latency(20000, p, True), flush=True)
for name in cfgs:
    s = synth.make(name)
    d = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    for mode, proto in [(m, pr) for m in ([0, 1, 2] if name in ("c4",) else [0]) for pr in (0, 1)]:
        h = cap.analyse(rp, ci, v, mode=mode, protocol=proto, **opts)
        x = torch.empty_like(b)
        for _ in range(3):
            h.solve(b, x)
        h.check()
        ts = []
        for _ in range(20):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        h.check()
        t = float(np.median(ts))
        err = float(np.max(np.abs(x.cpu().numpy() - s.x_true) / np.abs(s.x_true))) if s.x_true is not None else -1
        print(json.dumps({"cfg": name, "mode": mode, "proto": proto, "n": s.n, "nnz": s.nnz, "t_us": round(t * 1e6, 2),
                          "gflops": round(2 * s.nnz / t / 1e9, 2), "roof": round(s.alg_bytes() / t / PEAK, 4),
                          "err_vs_xtrue": err, "plan": [h.info()[k] for k in ("n_thread_groups","n_warp_rows")], "opts": opts}), flush=True)
        h.close()
