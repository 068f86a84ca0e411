"""ENGINE_GRID (solve_grid.cuh): wavefront bands for stencil-shaped lower factors, against the oracle.

Every GRID row is Alg.1's row (far, north, west entries in column order, separately rounded mul and
add, proven division), so the bar is BIT-EXACT vs oracle.solve.  Coverage: 5-point
grids with line lengths that are / are not multiples of 32 (ragged last band), ragged last lines,
7-point grids (far entries through the protocol), both protocols, both division modes, zero
numerators (the division guard), NaN-poisoned x, repeated solves (epochs), graph replay, the
watchdog, the division-proof failure path, analyse's eligibility (AUTO picks GRID on grids only,
forcing it on other shapes is refused) and the full-size c3 config.
"""
import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

GRID = 10


@pytest.fixture(scope="module")
def cap():
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    return cap


def dev(s, b=None):
    d = torch.device("cuda:0")
    return (torch.from_numpy(s.rowptr).to(d), torch.from_numpy(s.colidx).to(d),
            torch.from_numpy(s.val).to(d), torch.from_numpy(s.b if b is None else b).to(d))


def solve(cap, s, b=None, solves=1, **opt):
    rp, ci, v, bd = dev(s, b)
    with cap.analyse(rp, ci, v, **opt) as h:
        info = h.info()
        out = []
        for _ in range(solves):
            x = torch.full_like(bd, float("nan"))
            h.solve(bd, x)
            h.check()
            out.append(x.cpu().numpy())
        return out, info


SHAPES = [  # (nx, ny, nz, rows)
    (64, 64, 1, None), (100, 37, 1, None), (33, 70, 1, None), (2, 300, 1, None), (31, 40, 1, None),
    (96, 50, 1, 96 * 50 - 17), (257, 9, 1, None), (40, 6, 5, None), (70, 5, 3, 900), (32, 4, 9, None),
]


@pytest.mark.parametrize("shape", SHAPES, ids=lambda t: "x".join(str(v) for v in t))
@pytest.mark.parametrize("proto", [0, 1])
@pytest.mark.parametrize("div", [0, 1])
def test_grid_forced_bit_exact(cap, shape, proto, div):
    nx, ny, nz, rows = shape
    s = synth.gen_stencil(nx, ny, nz, seed=nx * 7 + ny, rows=rows)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    xs, info = solve(cap, s, solves=2, engine=GRID, protocol=proto, chain_div=div)
    assert info["engine"] == GRID
    for x in xs:
        assert np.array_equal(x, ref)


@pytest.mark.parametrize("g", [100, 300, 1024])
def test_grid_auto_picks_grid(cap, g):
    s = synth.gen_grid(g)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    xs, info = solve(cap, s)
    assert info["engine"] == GRID
    assert np.array_equal(xs[0], ref)


def test_grid_3d_forced(cap):
    """A 7-point grid (far entries: the plane below, polled by the producers): forced GRID, bit-exact
    over repeated solves.  (AUTO keeps 3D grids on the level-parallel engines: their wavefront is much
    shorter than their line count.)"""
    s = synth.gen_stencil(64, 48, 20, seed=5)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    xs, info = solve(cap, s, solves=3, engine=GRID)
    assert info["engine"] == GRID
    for x in xs:
        assert np.array_equal(x, ref)


@pytest.mark.parametrize("gen", ["c2", "chain", "random", "diag"])
def test_grid_refused_on_other_shapes(cap, gen):
    s = {"c2": lambda: synth.gen_c2(n=50_000), "chain": lambda: synth.gen_chain(5000),
         "random": lambda: synth.gen_random_lower(3000, 4, seed=3), "diag": lambda: synth.gen_diag(4000)}[gen]()
    rp, ci, v, b = dev(s)
    with cap.analyse(rp, ci, v) as h:
        assert h.info()["engine"] != GRID
        with pytest.raises(cap.SptrsvError):
            h.set_option(cap._lib.OPT_ENGINE, GRID)


def test_grid_zero_numerators_and_specials(cap):
    """b = 0 on whole lines (zero numerators fall outside the division guard: the in-loop full
    division), tiny and huge magnitudes, NaN / Inf in b: IEEE propagation identical to Alg.1."""
    s = synth.gen_stencil(96, 80, seed=9)
    b = s.b.copy()
    b[: 96 * 3] = 0.0
    b[96 * 10 + 5] = 1e-300
    b[96 * 20 + 40] = 1e300
    b[96 * 30 + 64] = np.nan
    b[96 * 40 + 33] = np.inf
    b[96 * 50 + 31] = -0.0
    ref = oracle.solve(s.rowptr, s.colidx, s.val, b)
    for div in (0, 1):
        xs, _ = solve(cap, s, b=b, engine=GRID, chain_div=div)
        bad = np.nonzero(~((xs[0] == ref) | (np.isnan(xs[0]) & np.isnan(ref))))[0]
        assert bad.size == 0, (div, bad.size, bad[:8], xs[0][bad[:4]], ref[bad[:4]])
        assert np.array_equal(np.signbit(xs[0]), np.signbit(ref))


def test_grid_graph_replay(cap):
    s = synth.gen_stencil(128, 60, seed=4)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    rp, ci, v, b = dev(s)
    with cap.analyse(rp, ci, v, engine=GRID) as h:
        st = torch.cuda.Stream()
        x = torch.empty_like(b)
        with torch.cuda.stream(st):
            h.solve(b, x, stream=st)  # warm: configuration reset outside the capture
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=st):
                h.solve(b, x, stream=st)
        for _ in range(5):
            x.fill_(float("nan"))
            g.replay()
            torch.cuda.synchronize()
            h.check()
            assert np.array_equal(x.cpu().numpy(), ref)


def test_grid_watchdog_then_exact(cap):
    s = synth.gen_stencil(256, 200, seed=6)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    rp, ci, v, b = dev(s)
    with cap.analyse(rp, ci, v, engine=GRID) as h:
        default = h.get_option(cap.OPT_SPIN_LIMIT)
        h.set_option(cap.OPT_SPIN_LIMIT, 1)
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        with pytest.raises(cap.SptrsvError) as e:
            h.check()
        assert e.value.status == cap._lib.ERR_TIMEOUT
        h.check()
        h.set_option(cap.OPT_SPIN_LIMIT, default)
        x.fill_(float("nan"))
        h.solve(b, x)
        h.check()
        assert np.array_equal(x.cpu().numpy(), ref)


def test_grid_division_proof_failure_path(cap):
    """chain_div = 2 (test hook): the off-chain proof reports a failure -> SPTRSV_ERR_INEXACT, the
    handle switches to the in-loop proof (chain_div = 1) and the next solve is exact."""
    s = synth.gen_stencil(96, 64, seed=8)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    rp, ci, v, b = dev(s)
    with cap.analyse(rp, ci, v, engine=GRID, chain_div=2) as h:
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        with pytest.raises(cap.SptrsvError) as e:
            h.check()
        assert e.value.status == cap._lib.ERR_INEXACT
        assert h.get_option(cap._lib.OPT_CHAIN_DIV) == 1
        x.fill_(float("nan"))
        h.solve(b, x)
        h.check()
        assert np.array_equal(x.cpu().numpy(), ref)


@pytest.mark.parametrize("proto", [0, 1])
def test_c3_full_grid(cap, proto):
    s = synth.gen_c3()
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    xs, info = solve(cap, s, solves=2, engine=GRID, protocol=proto)
    assert info["engine"] == GRID
    for x in xs:
        assert np.array_equal(x, ref)


def test_grid_solve_host_and_multi_rhs(cap):
    """A GRID handle through sptrsv_solve_host (pinned host b / x) and sptrsv_solve_multi (the multi-RHS
    kernel, engine-independent): bit-exact per column."""
    s = synth.gen_stencil(200, 90, seed=13)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    rp, ci, v, b = dev(s)
    with cap.analyse(rp, ci, v) as h:
        assert h.info()["engine"] == GRID
        bh = torch.from_numpy(s.b).pin_memory()
        xh = torch.full((s.n,), float("nan"), dtype=torch.float64).pin_memory()
        h.solve_host(bh, xh)
        assert np.array_equal(xh.numpy(), ref)
        rng = np.random.default_rng(7)
        B = rng.uniform(-1, 1, (s.n, 5))
        X = h.solve_multi(torch.from_numpy(B).cuda())
        h.check()
        assert np.array_equal(X.cpu().numpy(), oracle.solve_multi(s.rowptr, s.colidx, s.val, B))
        x = torch.full_like(b, float("nan"))  # and a device solve after the host / multi paths
        h.solve(b, x)
        h.check()
        assert np.array_equal(x.cpu().numpy(), ref)


def test_grid_batch_of_grids(cap):
    """Independent grids of one line length as one block-diagonal batch handle: still grid-shaped (each
    system starts on a line boundary), solved by GRID in one launch, every block bit-exact."""
    systems = [synth.gen_stencil(96, 40, seed=21), synth.gen_stencil(96, 70, seed=22), synth.gen_stencil(96, 33, seed=23)]
    d = torch.device("cuda:0")
    devs = [tuple(torch.from_numpy(a).to(d) for a in (t.rowptr, t.colidx, t.val)) for t in systems]
    refs = [oracle.solve(t.rowptr, t.colidx, t.val, t.b) for t in systems]
    b = torch.from_numpy(np.concatenate([t.b for t in systems])).to(d)
    with cap.analyse_batch(devs, engine=GRID) as h:
        assert h.info()["engine"] == GRID
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        got = x.cpu().numpy()
        off = h.offsets
        for k, ref in enumerate(refs):
            assert np.array_equal(got[off[k]:off[k + 1]], ref), k


F4_SHAPES = [(64, 64, 1), (100, 37, 1), (33, 70, 1), (257, 9, 1), (40, 6, 5), (32, 4, 9)]


@pytest.mark.parametrize("shape", F4_SHAPES, ids=lambda t: "x".join(str(v) for v in t))
@pytest.mark.parametrize("flags", [1, 2, 3])
@pytest.mark.parametrize("proto", [0, 1])
def test_grid_triangular_forms(cap, shape, flags, proto):
    """SURVEY f4 on GRID: upper (backward substitution in logical rows), unit lower, unit upper --
    bit-exact vs oracle.solve_tri (the same order of operations: Alg.1 under the reversal, DESIGN G25)."""
    nx, ny, nz = shape
    s = synth.gen_stencil(nx, ny, nz, seed=nx + 3 * ny + flags)
    if flags & 1:
        s = synth.to_upper(s)
    if flags & 2:
        s = synth.to_unit(s, upper=bool(flags & 1))
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(np.ascontiguousarray(a)).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, upper=bool(flags & 1), unit_diag=bool(flags & 2), engine=GRID, protocol=proto) as h:
        assert h.info()["engine"] == GRID
        for _ in range(2):
            x = torch.full_like(b, float("nan"))
            h.solve(b, x)
            h.check()
            assert np.array_equal(x.cpu().numpy(), ref)


def test_grid_upper_needs_whole_lines(cap):
    """An upper handle whose last grid line is ragged is not grid-shaped (GRID needs n % m == 0 there):
    forcing GRID is refused, AUTO runs another engine, the result is exact."""
    s = synth.to_upper(synth.gen_stencil(96, 50, rows=96 * 50 - 17, seed=4))
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, 1)
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(np.ascontiguousarray(a)).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    with cap.analyse(rp, ci, v, upper=True) as h:
        assert h.info()["engine"] != GRID
        with pytest.raises(cap.SptrsvError):
            h.set_option(cap._lib.OPT_ENGINE, GRID)
        x = torch.full_like(b, float("nan"))
        h.solve(b, x)
        h.check()
        assert np.array_equal(x.cpu().numpy(), ref)
