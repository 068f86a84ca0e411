"""Full-size BASELINE.json configs on the GPU, in the launch configuration bench.py times
(default options, auto dispatch), compared with the oracle on every component."""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-12


def _run(s, **opt):
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, **opt) as h:
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        x1 = x.cpu().numpy()
        x.fill_(float("nan"))
        h.solve(b, x)  # second solve: epoch path
        h.check()
        return x1, x.cpu().numpy(), h.info()


@pytest.mark.parametrize("proto,engine", [(0, 0), (1, 0), (0, 3), (1, 3), (0, 9), (1, 9), (1, 5)])
def test_c2_full(proto, engine):
    s = synth.gen_c2()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, x2, info = _run(s, protocol=proto, engine=engine)
    assert info["n_warp_rows"] == 0  # 2.8 nnz/row -> thread level everywhere
    assert np.array_equal(x1, ref) and np.array_equal(x2, ref)


@pytest.mark.parametrize("proto,K", [(0, 1), (1, 1), (1, 2)])
def test_c3_full_ones_and_random(proto, K):
    s = synth.gen_c3(ones=True)
    x1, x2, _ = _run(s, protocol=proto, rows_per_lane=K)
    assert np.array_equal(x1, np.ones(s.n)) and np.array_equal(x2, np.ones(s.n))
    s = synth.gen_c3()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, _, _ = _run(s, protocol=proto, rows_per_lane=K)
    assert np.array_equal(x1, ref)


@pytest.mark.parametrize("proto", [0, 1])
def test_c4_full_auto_picks_warp(proto):
    s = synth.gen_c4()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, x2, info = _run(s, protocol=proto)
    assert info["n_thread_groups"] <= 32  # only the diagonal-only level-0 groups stay thread level
    err = np.max(np.abs(x1 - ref) / np.abs(ref))
    assert err <= TOL, err
    assert np.array_equal(x1, x2)  # deterministic summation order


def test_c5_system_full():
    s = synth.gen_c5(3)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, _, _ = _run(s)
    assert np.array_equal(x1, ref)


@pytest.mark.parametrize("proto", [0, 1])
def test_chain_full_closed_form(proto):
    s = synth.gen_chain()
    x1, _, _ = _run(s, protocol=proto)
    want = np.array([1.0 - 2.0 ** -(i + 1) if i <= 52 else 1.0 for i in range(s.n)])
    assert np.array_equal(x1, want)


@pytest.mark.parametrize("proto", [0, 1])
def test_c2_full_default_launch(proto):
    """c2 in exactly the bench.py configuration: default options, AUTO -> LEANP."""
    s = synth.gen_c2()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, x2, info = _run(s, protocol=proto)
    assert info["engine"] == 9
    assert np.array_equal(x1, ref) and np.array_equal(x2, ref)


def test_c3_full_default_launch():
    """c3 in the bench.py configuration: AUTO -> GRID (wavefront bands; 192-thread CTAs: consumer,
    four producers, ring warp)."""
    s = synth.gen_c3(ones=True)
    x1, x2, info = _run(s)
    assert (info["engine"], info["cta_threads"]) == (10, 192), info
    assert np.array_equal(x1, np.ones(s.n)) and np.array_equal(x2, np.ones(s.n))
    s = synth.gen_c3()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, x2, _ = _run(s)
    assert np.array_equal(x1, ref) and np.array_equal(x2, ref)


@pytest.mark.parametrize("cfg,flags", [("c2", 1), ("c2", 2), ("c2", 3), ("c3", 1), ("c3", 2), ("c3", 3),
                                       ("c4", 1), ("c4", 3)])
def test_f4_forms_full(cfg, flags):
    """SURVEY f4 at full BASELINE sizes, the bench's triangular_forms_leg configuration (AUTO):
    upper (flags 1), unit lower (2), unit upper (3) -- LEANP (c2), GRID (c3), HYBRID (c4)."""
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    s = {"c2": synth.gen_c2, "c3": synth.gen_c3, "c4": synth.gen_c4}[cfg]()
    if flags & 1:
        s = synth.to_upper(s)
    if flags & 2:
        s = synth.to_unit(s)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(np.ascontiguousarray(a)).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, upper=bool(flags & 1), unit_diag=bool(flags & 2)) as h:
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        info = h.info()
        got = x.cpu().numpy()
    assert info["engine"] == {"c2": 9, "c3": 10, "c4": 6}[cfg], info
    if cfg == "c4":
        assert np.max(np.abs(got - ref) / np.abs(ref)) <= TOL
    else:
        assert np.array_equal(got, ref)


@pytest.mark.parametrize("cfg", ["c2", "c3", "c4"])
def test_levels_full_size_bit_exact(cfg):
    """a10 at full BASELINE size: the GPU level diagnostic (sptrsv_levels) against the oracle's Kahn
    BFS -- every component's level, the level count and every per-level count, bit for bit (beta =
    n / levels of Table 6) -- and the generator's closed form (10 x 1e5; 4095 with
    min(k+1, 4095-k) per anti-diagonal; 1000 x 1000)."""
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    s = {"c2": synth.gen_c2, "c3": synth.gen_c3, "c4": synth.gen_c4}[cfg]()
    d = torch.device("cuda:0")
    rp, ci, v = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val))
    with cap.analyse(rp, ci, v) as h:
        lv, nl, counts = h.levels()
        deg = h.indegree().cpu().numpy()
    olv = oracle.levels_bfs(s.rowptr, s.colidx)
    onl, ocounts = oracle.level_counts(olv)
    assert nl == onl
    assert np.array_equal(lv.cpu().numpy(), olv)
    assert np.array_equal(counts.cpu().numpy(), ocounts)
    assert np.array_equal(deg, oracle.indegree(s.rowptr, s.colidx))
    want = {"c2": [100_000] * 10, "c4": [1000] * 1000,
            "c3": [min(k + 1, 4095 - k) for k in range(4095)]}[cfg]
    assert ocounts.tolist() == want
