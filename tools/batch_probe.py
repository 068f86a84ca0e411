"""One launch over the block-diagonal concatenation of the 8 C5 systems vs 8 back-to-back launches
(CUDA events, L2 flushed before each step).  usage: python tools/batch_probe.py [NSYS]"""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth
import paper_conf_icpp_suz0hw0w20_b200 as cap

ns = int(sys.argv[1]) if len(sys.argv) > 1 else 8
sy = [synth.gen_c5(k) for k in range(ns)]
d = torch.device("cuda")
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=d)


def timeit(fn, reps=20):
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) * 1e3)
    return float(np.median(ts)), float(np.mean(ts))


hs, bufs = [], []
for s in sy:
    t = [torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b)]
    hs.append(cap.analyse(t[0], t[1], t[2])); bufs.append((t[3], torch.empty_like(t[3])))
sep = timeit(lambda: [h.solve(b, x) for h, (b, x) in zip(hs, bufs)])
# block-diagonal concatenation
off_r = np.cumsum([0] + [s.n for s in sy])
off_z = np.cumsum([0] + [int(s.rowptr[-1]) for s in sy])
rp = np.concatenate([s.rowptr[:-1].astype(np.int64) + off_z[k] for k, s in enumerate(sy)] + [[off_z[-1]]]).astype(np.int32)
ci = np.concatenate([s.colidx.astype(np.int64) + off_r[k] for k, s in enumerate(sy)]).astype(np.int32)
va = np.concatenate([s.val for s in sy]); bb = np.concatenate([s.b for s in sy])
t = [torch.from_numpy(a).to(d) for a in (rp, ci, va, bb)]
H = cap.analyse(t[0], t[1], t[2]); X = torch.empty_like(t[3])
one = timeit(lambda: H.solve(t[3], X))
H.check()
ok = all(torch.equal(X[off_r[k]:off_r[k + 1]], bufs[k][1]) for k in range(ns))
nnz = int(off_z[-1])
print(json.dumps({"systems": ns, "separate_us": sep, "one_launch_us": one, "bit_identical": ok,
                  "gflops_separate": round(2 * nnz / sep[0] / 1e3, 1), "gflops_one": round(2 * nnz / one[0] / 1e3, 1),
                  "engine_one": H.info()["engine"]}))
