"""GPU parity for ENGINE_SMALL (8): the whole system in one CTA's shared memory (solve_small.cuh).

Bar: BIT-EXACT against the oracle (oracle.solve / oracle.solve_tri) for every form -- every row is
thread-level (separately rounded multiply and add in row order, Alg.1 l.3-4) and
the division is the Markstein candidate whose remainder proof runs after the sweep; a failed proof
re-runs the sweep with the verified division, so the result is IEEE a / d whichever path ran.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

U, UNIT = oracle.UPPER, oracle.UNIT_DIAG
FORMS = [0, U, UNIT, U | UNIT]
SMALL = 8


@pytest.fixture(scope="module")
def cap():
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    return cap


def form(s, flags):
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:
        s = synth.to_unit(s, upper=bool(flags & U))
    return s


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda:0")


def ref_of(s, flags):
    return oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags) if flags else oracle.solve(s.rowptr, s.colidx,
                                                                                              s.val, s.b)


def small_solve(cap, s, flags=0, **opt):
    rp, ci, v, b = (dev(a) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, upper=bool(flags & U), unit_diag=bool(flags & UNIT), **opt) as h:
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        return x.cpu().numpy(), h.info()


@pytest.mark.parametrize("n", [1, 2, 31, 33, 257, 1000, 2500])
@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("cta", [32, 256, 1024])
def test_small_random_bit_exact(cap, n, flags, cta):
    """Ragged sizes (several threads' worth of rows per thread at 32 threads, idle threads at 1024),
    every triangular form: bit-identical to the oracle."""
    s = form(synth.gen_random_lower(n, 4, seed=n + 31), flags)
    x, info = small_solve(cap, s, flags, engine=SMALL, cta_threads=cta)
    assert (info["engine"], info["cta_threads"]) == (SMALL, min(cta, (n + 31) // 32 * 32))
    assert np.array_equal(x, ref_of(s, flags), equal_nan=True), (n, flags, cta)


@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("which", ["c1", "grid", "chain", "dense", "diag", "leveled", "wide"])
def test_small_structures_bit_exact(cap, flags, which):
    s = {"c1": synth.gen_c1, "grid": lambda: synth.gen_grid(40), "chain": lambda: synth.gen_chain(3000),
         "dense": lambda: synth.gen_dense_lower(120), "diag": lambda: synth.gen_diag(4000),
         "leveled": lambda: synth.gen_leveled(2000, 20, 1, 3, 5, "l"),
         "wide": lambda: synth.gen_random_lower(600, 20, seed=3)}[which]()
    s = form(s, flags)
    x, info = small_solve(cap, s, flags, engine=SMALL)
    assert info["engine"] == SMALL
    assert np.array_equal(x, ref_of(s, flags), equal_nan=True), (which, flags)


def test_small_unit_diagonal_only_has_no_entries(cap):
    """A unit-diagonal handle of a diagonal matrix stores nnz = 0 entries: x = b."""
    s = synth.to_unit(synth.gen_diag(500))
    assert s.rowptr[-1] == 0
    x, info = small_solve(cap, s, UNIT, engine=SMALL)
    assert info["engine"] == SMALL
    assert np.array_equal(x, s.b)


def _midpoint_system(rng, n, wild=0.0):
    """Bidiagonal rows with zero off-diagonals, so x_i = b_i / d_i goes through the row's division;
    (b_i, d_i) within a few ulps of rounding midpoints (test_gpu_parity._near_midpoint_quotients);
    `wild`: that fraction of operands pushed outside the guarded range [2^-400, 2^401)."""
    d = rng.uniform(1.0, 2.0, size=n)
    q = rng.uniform(0.5, 1.0, size=n)
    a = (q + np.spacing(q) / 2) * d
    steps = rng.integers(-3, 4, size=n)
    for k in range(3):
        up, dn = steps > k, steps < -k
        a[up] = np.nextafter(a[up], np.inf)
        a[dn] = np.nextafter(a[dn], -np.inf)
    if wild:
        w = rng.random(n) < wild
        d[w] = np.ldexp(d[w], rng.integers(-600, 600, w.sum()))
        w = rng.random(n) < wild
        a[w] = np.ldexp(a[w], rng.integers(-600, 600, w.sum()))
    rp = np.r_[0, np.arange(1, 2 * n, 2)].astype(np.int32)
    ci = np.empty(2 * n - 1, np.int32)
    v = np.empty(2 * n - 1)
    ci[0], ci[1::2], ci[2::2] = 0, np.arange(0, n - 1), np.arange(1, n)
    v[0], v[2::2] = d[0], d[1:]
    v[1::2] = 0.0
    return synth.CSRSystem("mid", n, rp, ci, v, a, None, {}), a / d


@pytest.mark.parametrize("wild", [0.0, 0.01])
@pytest.mark.parametrize("chain_div", [0, 2])
def test_small_division_proof_and_rerun(cap, wild, chain_div):
    """The deferred proof: quotients next to rounding midpoints (some candidates are rejected) and
    operands outside the guarded range force the verified re-run; CHAIN_DIV = 2 forces it always.
    Every path ends bit-identical to IEEE a / d."""
    rng = np.random.default_rng(77 + int(wild * 100) + chain_div)
    s, want = _midpoint_system(rng, 3000, wild)
    x, info = small_solve(cap, s, 0, engine=SMALL, chain_div=chain_div)
    assert info["engine"] == SMALL
    assert np.array_equal(x.view(np.int64), want.view(np.int64))


def test_small_special_values(cap):
    """NaN / inf in b, zero right-hand sides and a subnormal diagonal (outside the guarded range: the
    verified re-run) propagate exactly as in the oracle (IEEE).  (A zero diagonal is refused by
    analyse, SPTRSV_ERR_ZERO_DIAG.)"""
    s = synth.gen_random_lower(700, 3, seed=9)
    b = s.b.copy()
    b[[3, 100, 400]] = [np.nan, np.inf, -np.inf]
    b[[5, 6]] = 0.0
    val = s.val.copy()
    val[s.rowptr[11] - 1] = 1e-310  # L_10,10 subnormal
    s = synth.CSRSystem("special", s.n, s.rowptr, s.colidx, val, b, None, {})
    with np.errstate(all="ignore"):
        ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    x, _ = small_solve(cap, s, 0, engine=SMALL)
    assert np.array_equal(x, ref, equal_nan=True)


def test_small_auto_choice(cap):
    """AUTO takes SMALL for small near-dependency systems that fit one CTA and are not pure chains;
    pure chains stay on CHAIN, far / no dependencies on LEAN, systems too large for shared memory or
    above 4096 rows on the multi-CTA engines.  Forcing SMALL on a system that does not fit fails."""
    for gen, want in ((synth.gen_c1, SMALL), (lambda: synth.gen_grid(32), SMALL),
                      (lambda: synth.gen_random_lower(600, 20, seed=3), SMALL),
                      (lambda: synth.gen_chain(3000), 7), (lambda: synth.gen_diag(4000), 9),
                      (lambda: synth.gen_random_lower(5000, 3, seed=4), None),
                      (lambda: synth.gen_random_lower(4000, 6, seed=4), None)):
        s = gen()
        x, info = small_solve(cap, s)
        if want is None:
            assert info["engine"] != SMALL, (s.name, info)
        else:
            assert info["engine"] == want, (s.name, info)
        assert np.array_equal(x, oracle.solve(s.rowptr, s.colidx, s.val, s.b)) or info["engine"] == 6
    s = synth.gen_random_lower(4000, 6, seed=4)  # 24 B x 4000 + 12 B x ~24k > 226 KB
    rp, ci, v, _ = (dev(a) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v) as h:
        with pytest.raises(cap.SptrsvError):
            h.set_option(cap._lib.OPT_ENGINE, SMALL)


@pytest.mark.parametrize("flags", [0, U | UNIT])
@pytest.mark.parametrize("pinned", [True, False])
def test_small_solve_host(cap, flags, pinned):
    """sptrsv_solve_host on SMALL: pinned buffers are read / written by the kernel through the UVA
    mapping (no copy launches), pageable ones staged; repeated solves on one handle."""
    s = form(synth.gen_c1(), flags)
    ref = ref_of(s, flags)
    rp, ci, v = (dev(a) for a in (s.rowptr, s.colidx, s.val))
    with cap.analyse(rp, ci, v, upper=bool(flags & U), unit_diag=bool(flags & UNIT)) as h:
        assert h.info()["engine"] == SMALL
        if pinned:
            bh = torch.from_numpy(s.b).pin_memory()
            xh = torch.full((s.n,), float("nan"), dtype=torch.float64).pin_memory()
        else:
            bh, xh = s.b.copy(), np.full(s.n, np.nan)
        for _ in range(3):
            (xh.fill_ if pinned else xh.fill)(float("nan"))
            h.solve_host(bh, xh)
            assert np.array_equal(xh.numpy() if pinned else xh, ref)


def test_small_graph_replay_and_stale_refusal(cap):
    """A captured SMALL solve replays exactly; after a re-configuration (new generation) a replay of
    the old graph is refused with SPTRSV_ERR_STALE_LAUNCH like every other engine, and a new capture
    solves exactly."""
    s = synth.gen_c1()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    rp, ci, v, b = (dev(a) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v) as h:
        assert h.info()["engine"] == SMALL
        st = torch.cuda.Stream()
        x = torch.empty_like(b)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.stream(st):
            h.solve(b, x, stream=st)
            st.synchronize()
            with torch.cuda.graph(g, stream=st):
                h.solve(b, x, stream=st)
        for _ in range(3):
            x.fill_(float("nan"))
            g.replay()
            torch.cuda.synchronize()
            h.check(st)
            assert np.array_equal(x.cpu().numpy(), ref)
        h.set_option(cap.OPT_CTA_THREADS, 128)
        with torch.cuda.stream(st):
            h.solve(b, x, stream=st)  # the new configuration's first launch bumps the generation
        st.synchronize()
        h.check(st)
        g.replay()
        torch.cuda.synchronize()
        with pytest.raises(cap.SptrsvError) as e:
            h.check(st)
        assert e.value.status == cap._lib.ERR_STALE_LAUNCH
        g2 = torch.cuda.CUDAGraph()
        with torch.cuda.stream(st):
            with torch.cuda.graph(g2, stream=st):
                h.solve(b, x, stream=st)
        x.fill_(float("nan"))
        g2.replay()
        torch.cuda.synchronize()
        h.check(st)
        assert np.array_equal(x.cpu().numpy(), ref)


@pytest.mark.parametrize("flags", [0, U])
def test_small_multi_rhs(cap, flags):
    """sptrsv_solve_multi on a SMALL handle (lower: the multi-RHS kernel; upper: column by column
    through SMALL): bit-exact per column."""
    s = form(synth.gen_c1(), flags)
    rng = np.random.default_rng(5)
    B = rng.uniform(-1, 1, (s.n, 4))
    rp, ci, v = (dev(a) for a in (s.rowptr, s.colidx, s.val))
    with cap.analyse(rp, ci, v, upper=bool(flags & U)) as h:
        assert h.info()["engine"] == SMALL
        X = h.solve_multi(dev(B))
        h.check()
        X = X.cpu().numpy()
    for c in range(4):
        want = (oracle.solve_tri(s.rowptr, s.colidx, s.val, B[:, c].copy(), flags) if flags else
                oracle.solve(s.rowptr, s.colidx, s.val, B[:, c].copy()))
        assert np.array_equal(X[:, c], want), c
