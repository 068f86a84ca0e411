"""Option sweep: median solve time (CUDA events, L2 flushed) per config x option set.
usage: python tools/sweep.py c2,c4 '[{"protocol":1},{"protocol":1,"backoff_max_ns":128}]' [reps]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

cfgs = sys.argv[1].split(",")
optsets = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [{}]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 15
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
for name in cfgs:
    s = synth.make(name)
    d = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    for opts in optsets:
        h = cap.analyse(rp, ci, v, **opts)
        x = torch.empty_like(b)
        for _ in range(3):
            h.solve(b, x)
        h.check()
        ts = []
        for _ in range(reps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        h.check()
        t = float(np.median(ts))
        ok = bool(np.allclose(x.cpu().numpy(), s.x_true, rtol=1e-12, atol=0)) if s.x_true is not None else None
        print(json.dumps({"cfg": name, "opts": opts, "t_us": round(t * 1e6, 2), "p10_p90": [round(float(np.percentile(ts, q)) * 1e6, 1) for q in (10, 90)],
                          "gflops": round(2 * s.nnz / t / 1e9, 2), "ok": ok}), flush=True)
        h.close()
