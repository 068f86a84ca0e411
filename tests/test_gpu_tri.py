"""GPU parity for SURVEY row f4: upper-triangular and unit-diagonal solves through
``sptrsv_analyse_csr_ex`` (include/sptrsv.h), against oracle.solve_tri (G25).

Bar: BIT-EXACT -- the LEAN engine sums each row's off-diagonals in stored order with
separately rounded multiply and add and an IEEE-exact division, as the oracle does.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

U, UNIT = oracle.UPPER, oracle.UNIT_DIAG
FORMS = [U, UNIT, U | UNIT]
TOL = 1e-12  # warp-level rows (lane-strided sums), as tests/test_gpu_parity.py


def relerr(a, ref):
    return float(np.max(np.abs(a - ref) / np.maximum(np.abs(ref), 1e-300)))


@pytest.fixture(scope="module")
def cap():
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    return cap


def form(s, flags):
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:
        s = synth.to_unit(s)
    return s


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda:0")


def analyse(cap, s, flags, **opt):
    return cap.analyse(dev(s.rowptr), dev(s.colidx), dev(s.val), upper=bool(flags & U),
                       unit_diag=bool(flags & UNIT), **opt)


def gpu_solve(cap, s, flags, **opt):
    with analyse(cap, s, flags, **opt) as h:
        b = dev(s.b)
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        return x.cpu().numpy(), h.info()


GENS = {
    "rand4": lambda n: synth.gen_random_lower(n, 4, seed=n),
    "rand12": lambda n: synth.gen_random_lower(n, 12, seed=n + 1),
}


@pytest.mark.parametrize("n", [1, 2, 31, 33, 255, 257, 1000, 4099, 20_001])
@pytest.mark.parametrize("gen", list(GENS))
@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("proto", [0, 1])
def test_tri_random_sizes_bit_exact(cap, n, gen, flags, proto):
    s = form(GENS[gen](n), flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, info = gpu_solve(cap, s, flags, protocol=proto, mode=1)  # thread level: bit-exact
    # LEANP, CHAIN for long aligned previous-row runs, SMALL for small near-dependency systems
    assert info["engine"] in (7, 8, 9)
    assert np.array_equal(x, ref)
    for engine in (3, 7, 8, 9):  # the thread-level engines, forced (SMALL where the system fits one CTA)
        if engine == 8 and (s.n > 4096 or 24 * s.n + 12 * int(s.rowptr[-1]) > 220 * 1024):
            continue
        x, info = gpu_solve(cap, s, flags, protocol=proto, engine=engine, mode=1)
        assert info["engine"] == engine
        assert np.array_equal(x, ref)


@pytest.mark.parametrize("which", ["c2", "c2i", "grid", "c4", "dense", "chain"])
@pytest.mark.parametrize("flags", FORMS)
def test_tri_structured_bit_exact(cap, which, flags):
    base = {"c2": lambda: synth.gen_c2(n=300_000), "c2i": lambda: synth.gen_c2i(n=100_000),
            "grid": lambda: synth.gen_grid(300), "c4": lambda: synth.gen_c4(n=100_000, nlevels=200),
            "dense": lambda: synth.gen_dense_lower(400), "chain": lambda: synth.gen_chain(30_000)}[which]()
    s = form(base, flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, _ = gpu_solve(cap, s, flags, mode=1)  # thread level everywhere: bit-exact
    assert np.array_equal(x, ref)
    x, _ = gpu_solve(cap, s, flags)  # AUTO (warp rows where long): warp-mode bound
    assert relerr(x, ref) <= TOL


@pytest.mark.parametrize("flags", [0, U, UNIT, U | UNIT])
def test_tri_exact_integer_systems(cap, flags):
    s = synth.integerize(synth.gen_random_lower(50_000, 6, 21))
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:  # integer unit form: drop the diagonal, b = x + N x exactly
        rows = np.repeat(np.arange(s.n), np.diff(s.rowptr))
        keep = s.colidx != rows
        rp = np.zeros(s.n + 1, np.int64)
        np.cumsum(np.bincount(rows[keep], minlength=s.n), out=rp[1:])
        ci, v = s.colidx[keep], s.val[keep]
        b = s.x_true + np.bincount(rows[keep], weights=v * s.x_true[ci], minlength=s.n)
        s = synth.CSRSystem("u", s.n, rp.astype(np.int32), ci, v, b, s.x_true, {})
    x, _ = gpu_solve(cap, s, flags)
    assert np.array_equal(x, s.x_true)


def test_upper_bidiagonal_closed_form(cap):
    """U_ii = 2, U_{i,i+1} = -1, b = 1: x_i = 1 - 2^-(n-i) (exact for n - i <= 53), and the
    rest of a long chain converges to 1 -- a 100k-long dependency chain in reverse order."""
    n = 100_000
    rp = np.r_[np.arange(0, 2 * n, 2), 2 * n - 1].astype(np.int32)
    ci = np.empty(2 * n - 1, np.int32)
    v = np.empty(2 * n - 1)
    ci[0::2], v[0::2] = np.arange(n), 2.0
    ci[1::2], v[1::2] = np.arange(1, n), -1.0
    s = synth.CSRSystem("ub", n, rp, ci, v, np.ones(n), None, {})
    x, _ = gpu_solve(cap, s, U)
    k = np.arange(n - 53, n)
    assert np.array_equal(x[k], 1.0 - 2.0 ** -(n - k).astype(float))
    assert np.array_equal(x, oracle.solve_tri(rp, ci, v, np.ones(n), U))


def test_unit_identity_and_empty_rows(cap):
    """Unit lower with NO stored entries (nnz = 0, colidx/val empty): x = b."""
    n = 10_000
    s = synth.CSRSystem("id", n, np.zeros(n + 1, np.int32), np.zeros(0, np.int32), np.zeros(0),
                        np.random.default_rng(0).uniform(-1, 1, n), None, {})
    for flags in (UNIT, U | UNIT):
        x, _ = gpu_solve(cap, s, flags)
        assert np.array_equal(x, s.b)


def test_unit_lower_chain_closed_form(cap):
    """Unit lower, L_{i,i-1} = -1, b = 1: x_i = i + 1 (row 0 empty)."""
    n = 50_000
    rp = np.r_[0, np.arange(0, n)].astype(np.int32)
    ci = np.arange(0, n - 1, dtype=np.int32)
    s = synth.CSRSystem("uc", n, rp, ci, -np.ones(n - 1), np.ones(n), None, {})
    x, _ = gpu_solve(cap, s, UNIT)
    assert np.array_equal(x, np.arange(1, n + 1, dtype=float))


@pytest.mark.parametrize("n", [1, 2, 33, 1000, 4099])
@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("proto", [0, 1])
def test_tri_warp_mode(cap, n, flags, proto):
    """MODE = 2: one warp per row (k_solve_tri_warp); lane-strided sums -> warp-mode bound."""
    s = form(synth.gen_random_lower(n, 40, seed=n + 3), flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, info = gpu_solve(cap, s, flags, mode=2, protocol=proto)
    assert info["engine"] == 6 and info["n_warp_rows"] == n
    assert relerr(x, ref) <= TOL


@pytest.mark.parametrize("flags", FORMS)
def test_tri_c4_auto_picks_warp(cap, flags):
    """c4-like rows (~64 entries) in each form: AUTO plans every row warp-level."""
    s = form(synth.gen_c4(n=100_000, nlevels=100), flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, info = gpu_solve(cap, s, flags)
    assert info["engine"] == 6
    assert relerr(x, ref) <= TOL
    assert relerr(x, s.x_true) <= TOL


@pytest.mark.parametrize("flags", FORMS)
def test_tri_integer_warp_mode_bit_exact(cap, flags):
    """Exact-integer values: any summation order is exact, so warp rows are bit-exact too."""
    s = synth.integerize(synth.gen_random_lower(20_000, 30, 31))
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:
        rows = np.repeat(np.arange(s.n), np.diff(s.rowptr))
        keep = s.colidx != rows
        rp = np.zeros(s.n + 1, np.int64)
        np.cumsum(np.bincount(rows[keep], minlength=s.n), out=rp[1:])
        ci, v = s.colidx[keep], s.val[keep]
        b = s.x_true + np.bincount(rows[keep], weights=v * s.x_true[ci], minlength=s.n)
        s = synth.CSRSystem("u", s.n, rp.astype(np.int32), ci, v, b, s.x_true, {})
    x, _ = gpu_solve(cap, s, flags, mode=2)
    assert np.array_equal(x, s.x_true)


@pytest.mark.parametrize("flags", FORMS)
def test_tri_full_size_c2(cap, flags):
    """BASELINE c2 shape (n = 1e6) in each f4 form, the bench launch configuration."""
    s = form(synth.gen_c2(), flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, _ = gpu_solve(cap, s, flags)
    assert np.array_equal(x, ref)
    assert np.max(np.abs(x - s.x_true) / np.abs(s.x_true)) <= 1e-12


@pytest.mark.parametrize("proto", [0, 1])
def test_tri_interleaved_handles_graph_and_epochs(cap, proto):
    """Upper, unit and lower handles interleaved on one stream, many solves each with new b,
    then a CUDA graph replay of an upper solve (device-side epoch)."""
    base = synth.gen_c2(n=200_000)
    systems = {f: form(base, f) for f in (0, U, UNIT, U | UNIT)}
    hs = {f: analyse(cap, s, f, protocol=proto) for f, s in systems.items()}
    rng = np.random.default_rng(5)
    try:
        for it in range(6):
            for f, s in systems.items():
                bb = rng.uniform(-1, 1, s.n)
                x = torch.full((s.n,), float("nan"), dtype=torch.float64, device="cuda:0")
                hs[f].solve(dev(bb), x)
                hs[f].check()
                assert np.array_equal(x.cpu().numpy(), oracle.solve_tri(s.rowptr, s.colidx, s.val, bb, f)), (it, f)
        s = systems[U]
        b = dev(s.b)
        x = torch.empty_like(b)
        st = torch.cuda.Stream()
        with torch.cuda.stream(st):
            hs[U].solve(b, x)  # warm-up on the capture stream
        st.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            hs[U].solve(b, x, stream=st)
        ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, U)
        for _ in range(5):
            x.fill_(float("nan"))
            g.replay()
            torch.cuda.synchronize()
            assert np.array_equal(x.cpu().numpy(), ref)
        hs[U].check()
    finally:
        for h in hs.values():
            h.close()


def test_tri_solve_host(cap):
    s = form(synth.gen_c2(n=100_000), U)
    with analyse(cap, s, U) as h:
        x = np.empty(s.n)
        h.solve_host(np.ascontiguousarray(s.b), x)
        assert np.array_equal(x, oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, U))


@pytest.mark.parametrize("flags", FORMS)
def test_tri_indegree(cap, flags):
    s = form(synth.gen_c4(n=20_000, nlevels=100), flags)
    with analyse(cap, s, flags) as h:
        deg = np.diff(s.rowptr) - (0 if flags & UNIT else 1)
        assert np.array_equal(h.indegree().cpu().numpy(), deg)


TRI_CASES = [  # (rowptr, colidx, val, flags) -- oracle.validate_tri decides the code
    ([0, 1, 3], [0, 0, 1], [1, 1, 1], U),          # entry below the diagonal
    ([0, 1, 2], [1, 1], [1, 1], U),                # diagonal not first
    ([0, 2, 3], [0, 1, 1], [0, 1, 1], U),          # zero diagonal
    ([0, 2, 3], [1, 0, 1], [1, 1, 1], U),          # unsorted
    ([0, 1, 1], [0], [1], U),                      # empty row (non-unit)
    ([0, 1, 1], [0], [1], UNIT),                   # stored diagonal under UNIT
    ([0, 0, 2], [0, 0], [1, 1], UNIT),             # duplicate
    ([0, 1, 1], [0], [1], U | UNIT),               # stored diagonal
    ([0, 0, 1], [0], [1], U | UNIT),               # below the diagonal
    ([0, 1, 1], [2], [1], U | UNIT),               # column out of range
]


@pytest.mark.parametrize("case", range(len(TRI_CASES)))
def test_tri_validation_codes_match_oracle(cap, case):
    rp, ci, v, flags = TRI_CASES[case]
    code, _ = oracle.validate_tri(np.array(rp, np.int32), np.array(ci, np.int32), np.array(v, float), flags)
    assert code != 0
    with pytest.raises(cap.SptrsvError) as e:
        cap.analyse(torch.tensor(rp, dtype=torch.int32, device="cuda:0"),
                    torch.tensor(ci, dtype=torch.int32, device="cuda:0"),
                    torch.tensor(v, dtype=torch.float64, device="cuda:0"),
                    upper=bool(flags & U), unit_diag=bool(flags & UNIT))
    assert e.value.status == code


def test_tri_unsupported_calls_fail_loudly(cap):
    s = form(synth.gen_c2(n=10_000), U)
    with analyse(cap, s, U) as h:
        with pytest.raises(cap.SptrsvError):
            h.levels()
        with pytest.raises(cap.SptrsvError):
            h.set_option(cap._lib.OPT_VARIANT, 5)
        # still solves correctly after the refused calls
        b = dev(s.b)
        x = h.solve(b)
        h.check()
        assert np.array_equal(x.cpu().numpy(), oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, U))


@pytest.mark.parametrize("which", ["grid", "chain", "c2i", "rand4"])
@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("proto", [0, 1])
@pytest.mark.parametrize("K,cta", [(1, 128), (2, 128), (2, 64), (2, 256)])
def test_tri_chain_engine_bit_exact(cap, which, flags, proto, K, cta):
    """CHAIN (in-warp chains in registers) on f4 handles: logical rows reversed for upper, the
    diagonal first / implicit, entries walked earliest-solved first -- bit-exact vs solve_tri."""
    base = {"grid": lambda: synth.gen_grid(150), "chain": lambda: synth.gen_chain(20_000),
            "c2i": lambda: synth.gen_c2i(n=60_000), "rand4": lambda: synth.gen_random_lower(4099, 4, seed=5)}[which]()
    s = form(base, flags)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    x, info = gpu_solve(cap, s, flags, protocol=proto, engine=7, rows_per_lane=K, cta_threads=cta, mode=1)
    assert (info["engine"], info["rows_per_lane"], info["cta_threads"]) == (7, K, cta), info
    assert np.array_equal(x, ref)


@pytest.mark.parametrize("flags", FORMS)
def test_tri_chain_auto_choice_and_closed_forms(cap, flags):
    """AUTO sends f4 grids to GRID (a 200^2 grid factor in every form) and f4 chains to CHAIN; the f4
    bidiagonal closed forms stay exact."""
    s = form(synth.gen_grid(200), flags)
    x, info = gpu_solve(cap, s, flags)
    assert info["engine"] == 10, info
    assert np.array_equal(x, oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags))
    s = form(synth.gen_c2(n=100_000), flags)
    _, info = gpu_solve(cap, s, flags)
    assert info["engine"] == 9, info  # far dependencies: LEANP
    n = 100_000  # upper bidiagonal U_ii = 2, U_{i,i+1} = -1, b = 1 (as test_upper_bidiagonal_closed_form)
    rp = np.r_[np.arange(0, 2 * n, 2), 2 * n - 1].astype(np.int32)
    ci = np.empty(2 * n - 1, np.int32)
    v = np.empty(2 * n - 1)
    ci[0::2], v[0::2] = np.arange(n), 2.0
    ci[1::2], v[1::2] = np.arange(1, n), -1.0
    sb = synth.CSRSystem("ub", n, rp, ci, v, np.ones(n), None, {})
    x, info = gpu_solve(cap, sb, U)
    assert info["engine"] == 7
    k = np.arange(n - 53, n)
    assert np.array_equal(x[k], 1.0 - 2.0 ** -(n - k).astype(float))


@pytest.mark.parametrize("nrhs", [1, 3, 8])
@pytest.mark.parametrize("flags", FORMS)
@pytest.mark.parametrize("which", ["c2", "grid", "c4"])
def test_tri_multi_rhs_columns(cap, nrhs, flags, which):
    """sptrsv_solve_multi on f4 handles: column by column through the handle's engine (LEAN,
    CHAIN or HYBRID), padded leading dimensions -- every column vs oracle.solve_tri."""
    base = {"c2": lambda: synth.gen_c2(n=100_000), "grid": lambda: synth.gen_grid(200),
            "c4": lambda: synth.gen_c4(n=20_000, nlevels=100)}[which]()
    s = form(base, flags)
    # columns (1 + r/8) b: solutions (1 + r/8) x_true with |x| >= 1, where the warp-row tolerance
    # is derived
    B = np.stack([s.b * (1.0 + r / 8.0) for r in range(nrhs)], axis=1)
    ref = np.stack([oracle.solve_tri(s.rowptr, s.colidx, s.val, B[:, r].copy(), flags) for r in range(nrhs)], axis=1)
    with analyse(cap, s, flags) as h:
        eng = h.info()["engine"]
        Bp = torch.zeros((s.n, nrhs + 2), dtype=torch.float64, device="cuda:0")
        Bp[:, :nrhs] = dev(B)
        Xp = torch.full((s.n, nrhs + 3), float("nan"), dtype=torch.float64, device="cuda:0")
        h.solve_multi(Bp[:, :nrhs], Xp[:, :nrhs])
        h.check()
        got = Xp[:, :nrhs].cpu().numpy()
        if eng == 6:
            assert relerr(got, ref) <= TOL
        else:
            assert np.array_equal(got, ref)
        assert torch.isnan(Xp[:, nrhs:]).all()
