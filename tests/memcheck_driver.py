"""Small solves through every engine / form for compute-sanitizer (memcheck / racecheck-free kernels):
usage: compute-sanitizer --tool memcheck python tests/memcheck_driver.py (a test harness: it runs the oracle)"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import synth, oracle
import paper_conf_icpp_suz0hw0w20_b200 as cap

d = torch.device("cuda")
def run(s, flags=0, **opt):
    rp, ci, v, b = (torch.from_numpy(np.ascontiguousarray(a)).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, upper=bool(flags & 1), unit_diag=bool(flags & 2), **opt) as h:
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags) if flags else oracle.solve(s.rowptr, s.colidx, s.val, s.b)
        assert np.array_equal(x.cpu().numpy(), ref), (s.name, flags, opt)

bases = [synth.gen_random_lower(1025, 4, seed=3), synth.gen_grid(40), synth.gen_chain(700), synth.gen_c2i(n=2000)]
for s in bases:
    for eng in (0, 3, 6, 7, 8, 9):
        for proto in (0, 1):
            run(s, engine=eng, protocol=proto)
    for flags in (1, 2, 3):
        s2 = synth.to_upper(s) if flags & 1 else s
        s2 = synth.to_unit(s2, upper=bool(flags & 1)) if flags & 2 else s2
        for eng in (3, 7, 8, 9):
            run(s2, flags, engine=eng)
    run(s, engine=8, chain_div=2)  # SMALL's verified re-run
print("memcheck_small ok")
