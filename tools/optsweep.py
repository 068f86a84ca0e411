"""Scratch perf probe: one config, several handle-option sets, median solve time (CUDA events, L2 flushed).
usage: python tools/optsweep.py CONFIG '[{"prefetch": 0}, {"prefetch": 740}]' [reps]"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

PEAK = 6539.9e9
name = sys.argv[1]
sets = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [{}]
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 30
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
FLUSH = os.environ.get("FLUSH", "dirty")  # dirty (bench.py's 256 MiB write), clean (write + read), none
sink = torch.empty(1, dtype=torch.float32, device="cuda")


def do_flush():
    if FLUSH == "none":
        return
    flush.zero_()
    if FLUSH == "clean":
        sink.add_(flush.sum())
s = synth.make(name)
d = torch.device("cuda")
rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
for rnd in range(2):  # two passes: the spread between them is the noise floor
    for opts in sets:
        h = cap.analyse(rp, ci, v, **opts)
        x = torch.empty_like(b)
        for _ in range(3):
            h.solve(b, x)
        h.check()
        ts = []
        for _ in range(reps):
            do_flush()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        h.check()
        t = float(np.median(ts))
        err = float(np.max(np.abs(x.cpu().numpy() - s.x_true) / np.abs(s.x_true))) if s.x_true is not None else -1
        inf = h.info()
        print(json.dumps({"cfg": name, "pass": rnd, "flush": FLUSH, "opts": opts, "t_us": round(t * 1e6, 2),
                          "p10": round(float(np.percentile(ts, 10)) * 1e6, 2),
                          "p90": round(float(np.percentile(ts, 90)) * 1e6, 2),
                          "gflops": round(2 * s.nnz / t / 1e9, 2), "roof": round(s.alg_bytes() / t / PEAK, 4),
                          "err": err, "engine": inf.get("engine"), "cta": inf.get("cta_threads")}), flush=True)
        h.close()
