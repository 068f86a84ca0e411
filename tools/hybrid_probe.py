"""HYBRID (engine 6) vs staged one-shot (engine 0) on plans with warp-level rows.
usage: python tools/hybrid_probe.py [protocol 0|1]"""
import json, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, synth
import paper_conf_icpp_suz0hw0w20_b200 as cap
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
def t_of(h, b, x, reps=15):
    for _ in range(3): h.solve(b, x)
    h.check(); ts=[]
    for _ in range(reps):
        flush.zero_(); e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
        e0.record(); h.solve(b,x); e1.record(); torch.cuda.synchronize(); ts.append(e0.elapsed_time(e1)*1e3)
    h.check(); return float(np.median(ts))
cases = [("c4", lambda: synth.gen_c4()), ("c4_500lv", lambda: synth.gen_c4(nlevels=500)),
         ("lev100_d32", lambda: synth.gen_leveled(1_000_000, 100, 1, 31, 9, "l")),
         ("lev1000_d20", lambda: synth.gen_leveled(1_000_000, 1000, 1, 19, 9, "l")),
         ("lev10_d64", lambda: synth.gen_leveled(1_000_000, 10, 1, 63, 9, "l")),
         ("dense2k", lambda: synth.gen_dense_lower(2000)),
         ("rand_k30", lambda: synth.gen_random_lower(300_000, 30, 5))]
for name, g in cases:
    s = g(); d = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    x = torch.empty_like(b); r = {"cfg": name, "n": s.n, "nnz": s.nnz}
    P = int(sys.argv[1]) if len(sys.argv) > 1 else 1
    for lab, o in [("auto", {}), ("hyb", {"engine": 6}), ("oneshot_c128", {"engine": 0, "cta_threads": 128}), ("oneshot_c256", {"engine": 0, "cta_threads": 256})]:
        with cap.analyse(rp, ci, v, protocol=P, **o) as h:
            r[lab] = round(t_of(h, b, x), 1)
            if lab == "auto": r["plan"] = [h.info()[k] for k in ("n_thread_groups", "n_warp_rows", "engine")]
    print(json.dumps(r), flush=True)
