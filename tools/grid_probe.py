"""GRID engine probe: per system and engine, solve time (CUDA events, L2 flushed), GFLOPS, bit-exactness
vs the CHAIN engine.  usage: grid_probe.py [systems] [engines]   systems: c3,g1000,s3d ...; engines: 10,7,5"""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

SYS = {"c3": lambda: synth.gen_c3(), "g1024": lambda: synth.gen_grid(1024), "g1000": lambda: synth.gen_grid(1000),
       "g500": lambda: synth.gen_grid(500), "g4096": lambda: synth.gen_grid(4096),
       "r8192x512": lambda: synth.gen_stencil(8192, 512), "r512x8192": lambda: synth.gen_stencil(512, 8192),
       "s3d": lambda: synth.gen_stencil(128, 128, 128), "s3d64": lambda: synth.gen_stencil(64, 64, 256),
       "b1": lambda: synth.gen_stencil(32, 65536), "b2": lambda: synth.gen_stencil(64, 32768),
       "b8": lambda: synth.gen_stencil(256, 8192), "w16k": lambda: synth.gen_stencil(16384, 64),
       "w4k": lambda: synth.gen_stencil(4096, 256), "g100": lambda: synth.gen_grid(100),
       "g300": lambda: synth.gen_grid(300), "g64x48x20": lambda: synth.gen_stencil(64, 48, 20), "b1f": lambda: synth.gen_stencil(32, 64, 1024)}
names = sys.argv[1].split(",") if len(sys.argv) > 1 else ["c3", "g1000", "s3d"]
engines = [int(e) for e in sys.argv[2].split(",")] if len(sys.argv) > 2 else [10, 7, 5]
opts = json.loads(sys.argv[3]) if len(sys.argv) > 3 else {}
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
for name in names:
    s = SYS[name]()
    d = torch.device("cuda")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    # reference: the CHAIN engine's result (thread-level rows, Alg.1 arithmetic: bit-identical across
    # engines; the oracle parity itself is tests/test_gpu_grid.py)
    with cap.analyse(rp, ci, v, engine=7) as hr:
        xr = torch.empty_like(b)
        hr.solve(b, xr)
        hr.check()
        ref = xr.cpu().numpy()
    for eng in engines:
        try:
            h = cap.analyse(rp, ci, v, engine=eng, **opts)
        except cap.SptrsvError as e:
            print(json.dumps({"sys": name, "engine": eng, "error": str(e)}), flush=True)
            continue
        x = torch.empty_like(b)
        for _ in range(3):
            h.solve(b, x)
        h.check()
        ts = []
        for _ in range(10):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
            e0.record(); h.solve(b, x); e1.record(); torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) * 1e-3)
        h.check()
        t = float(np.mean(ts))
        info = h.info()
        print(json.dumps({"sys": name, "engine": eng, "ran": info["engine"], "n": s.n, "nnz": s.nnz,
                          "t_us_mean": round(t * 1e6, 1), "t_us_min": round(min(ts) * 1e6, 1),
                          "gflops": round(2 * s.nnz / t / 1e9, 3), "same_as_chain": bool(np.array_equal(x.cpu().numpy(), ref)),
                          "opts": opts}), flush=True)
        h.close()
