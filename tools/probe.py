"""Scratch perf probe over systems x option sets (CUDA events, L2 flushed between solves).

usage: python tools/probe.py SYS[,SYS...] [OPTS_JSON_LIST]
  SYS: c1..c5 | chain | grid:G | stride:N:S (row i depends on i-S only) | lev:N:L:KANY | diag:N | rand:N:K
  OPTS_JSON_LIST: JSON list of option dicts (default [{}]), e.g. '[{}, {"backoff_max": 64}]'
Prints one JSON line per (system, options): median / mean solve time, GFLOPS, engine, parity vs x_true."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap


def build(spec):
    p = spec.split(":")
    if p[0] == "grid":
        return synth.gen_grid(int(p[1]))
    if p[0] == "stride":
        n, S = int(p[1]), int(p[2])
        rng = np.random.default_rng(5)
        rows = np.arange(S, n, dtype=np.int64)
        rp, ci = synth._assemble(n, (rows, rows - S))
        return synth.from_pattern(spec, rp, ci, rng, {"levels": (n + S - 1) // S})
    if p[0] == "lev":
        return synth.gen_leveled(int(p[1]), int(p[2]), 1, int(p[3]), 9, spec)
    if p[0] == "rand":  # rand:N:K -- row i: min(K, i) distinct columns uniform in [0, i) (c1's recipe)
        return synth.gen_random_lower(int(p[1]), int(p[2]), 11, spec)
    if p[0] == "diag":
        return synth.gen_diag(int(p[1]))
    return synth.make(spec)


def main():
    specs = sys.argv[1].split(",")
    optsets = json.loads(sys.argv[2]) if len(sys.argv) > 2 else [{}]
    reps = int(os.environ.get("PROBE_REPS", "20"))
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    d = torch.device("cuda")
    for spec in specs:
        s = build(spec)
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
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record()
                h.solve(b, x)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1) * 1e-3)
            h.check()
            xt = s.x_true
            err = float(np.max(np.abs(x.cpu().numpy() - xt) / np.abs(xt))) if xt is not None else -1.0
            t = float(np.median(ts))
            inf = h.info()
            print(json.dumps({"sys": spec, "opts": opts, "n": s.n, "nnz": s.nnz, "t_us": round(t * 1e6, 2),
                              "mean_us": round(float(np.mean(ts)) * 1e6, 2), "p90_us": round(float(np.percentile(ts, 90)) * 1e6, 2), "gflops": round(2 * s.nnz / t / 1e9, 2),
                              "engine": inf["engine"], "cta": inf["cta_threads"], "K": inf["rows_per_lane"],
                              "err": err}), flush=True)
            h.close()
        del rp, ci, v, b
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
