"""Scratch e2e probe: sptrsv_solve_host per-step time (CUDA events, L2 flushed) for host_io modes.
usage: python tools/e2e_probe.py CONFIG '[{"host_io":0}, ...]'"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

s = synth.make(sys.argv[1])
sets = json.loads(sys.argv[2])
d = torch.device("cuda")
rp, ci, v = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val))
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=d)
bh = torch.from_numpy(s.b).pin_memory()
xh = torch.empty(s.n, dtype=torch.float64).pin_memory()
st = torch.cuda.current_stream()
for rnd in range(2):
    for opts in sets:
        with cap.analyse(rp, ci, v, **opts) as h:
            for _ in range(3):
                h.solve_host(bh, xh)
            ts, wall = [], []
            import time
            for _ in range(20):
                flush.zero_()
                a, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(st)
                w0 = time.perf_counter()
                h.solve_host(bh, xh)
                wall.append((time.perf_counter() - w0) * 1e6)
                b_.record(st)
                b_.synchronize()
                ts.append(a.elapsed_time(b_) * 1e3)
            t = float(np.median(ts))
            print(json.dumps({"cfg": sys.argv[1], "pass": rnd, "opts": opts, "us": round(t, 1), "wall_us": round(float(np.median(wall)), 1),
                              "gflops": round(2 * s.nnz / t / 1e3, 2)}), flush=True)
