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


@pytest.mark.parametrize("proto,K,engine", [(0, 1, 0), (1, 1, 0), (1, 2, 0), (1, 4, 0), (1, 1, 2), (1, 2, 2),
                                             (0, 2, 2)])
def test_c2_full(proto, K, engine):
    s = synth.gen_c2()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x1, x2, info = _run(s, protocol=proto, rows_per_lane=K, engine=engine)
    assert info["n_warp_rows"] == 0  # 2.8 nnz/row -> thread level everywhere
    assert np.array_equal(x1, ref) and np.array_equal(x2, ref)


@pytest.mark.parametrize("proto,K", [(0, 1), (1, 1), (1, 4)])
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
