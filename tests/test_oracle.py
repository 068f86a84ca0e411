"""Pins for the CPU oracle (-m "not gpu").

Each test checks oracle/ against something other than itself: LAPACK / SciPy
triangular solves, closed forms, exact-integer systems, generator-guaranteed
level histograms, brute force on tiny inputs, and the numbers the paper prints
(tests/golden/).  A plausible slip in oracle.c -- a dropped term, a sign error,
an off-by-one in the row loop, dividing by the wrong entry, a transposed
pattern in the BFS -- fails at least one of these.
"""
import itertools
import math
import os

import numpy as np
import pytest
import scipy.linalg
import scipy.sparse
import scipy.sparse.linalg

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _dense(s):
    A = np.zeros((s.n, s.n))
    rows = np.repeat(np.arange(s.n), np.diff(s.rowptr))
    A[rows, s.colidx] = s.val
    return A


def _sp(s):
    return scipy.sparse.csr_matrix((s.val, s.colidx, s.rowptr), shape=(s.n, s.n))


# ---------------------------------------------------------------- solve (Alg. 1)

@pytest.mark.parametrize("n", [1, 2, 3, 7, 33, 64, 300])
def test_solve_matches_lapack_dense(n):
    """Brute force: dense LAPACK dtrtrs (scipy.linalg.solve_triangular) on a full lower triangle."""
    s = synth.gen_dense_lower(n, seed=100 + n)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    ref = scipy.linalg.solve_triangular(_dense(s), s.b, lower=True)
    err = np.linalg.norm(x - ref, np.inf) / np.linalg.norm(ref, np.inf)
    assert err <= 1e-13, err


@pytest.mark.parametrize("n,k,seed", [(50, 5, 1), (1000, 3, 1), (3000, 9, 5)])
def test_solve_matches_lapack_sparse_pattern(n, k, seed):
    s = synth.gen_random_lower(n, k, seed)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    if n <= 1000:
        ref = scipy.linalg.solve_triangular(_dense(s), s.b, lower=True)
    else:
        ref = scipy.sparse.linalg.spsolve_triangular(_sp(s), s.b, lower=True)
    assert np.max(np.abs(x - ref) / np.abs(ref)) <= 1e-13


@pytest.mark.parametrize("gen", [lambda: synth.gen_c2(n=50_000),
                                 lambda: synth.gen_c2i(n=20_000),
                                 lambda: synth.gen_c4(n=20_000, nlevels=40),
                                 lambda: synth.gen_grid(96)])
def test_solve_matches_scipy_spsolve_triangular(gen):
    s = gen()
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    ref = scipy.sparse.linalg.spsolve_triangular(_sp(s), s.b, lower=True)
    assert np.max(np.abs(x - ref) / np.abs(ref)) <= 1e-13
    # and b = L x_true with known x_true (strictly dominant L, well conditioned)
    assert np.max(np.abs(x - s.x_true) / np.abs(s.x_true)) <= 1e-13


def test_solve_diagonal_closed_form_bit_exact():
    s = synth.gen_diag(10_000)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    assert np.array_equal(x, s.b / s.val)  # one correctly rounded division per row


def test_solve_bidiagonal_closed_form_bit_exact():
    """L_ii = 2, L_i,i-1 = -1, b = 1  ->  x_i = 1 - 2^-(i+1) exactly; 1.0 from i = 52 on
    (x_52 = (1 + x_51)/2 = (2 - 2^-52)/2 is exact; x_53: 2 - 2^-53 rounds to 2 -> 1.0)."""
    s = synth.gen_chain(200)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    want = np.array([1.0 - 2.0 ** -(i + 1) if i <= 52 else 1.0 for i in range(200)])
    assert np.array_equal(x, want)


def test_solve_integer_chain_closed_form():
    """L_ii = 1, L_i,i-1 = -1, b = 1  ->  x_i = i + 1 exactly."""
    s = synth.gen_chain(5000)
    v = s.val.copy()
    v[s.rowptr[1:] - 1] = 1.0
    x = oracle.solve(s.rowptr, s.colidx, v, s.b)
    assert np.array_equal(x, np.arange(1, 5001, dtype=np.float64))


@pytest.mark.parametrize("gen", [lambda: synth.gen_c1(),
                                 lambda: synth.gen_c2(n=20_000),
                                 lambda: synth.gen_c2i(n=20_000),
                                 lambda: synth.gen_c4(n=5_000, nlevels=50),
                                 lambda: synth.gen_dense_lower(40)])
def test_solve_exact_integer_systems(gen):
    """Exact-integer values: x must equal x_true bit-for-bit (all partials exact)."""
    s = synth.integerize(gen())
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    assert np.array_equal(x, s.x_true)


def test_solve_grid_ones_bit_exact():
    s = synth.gen_grid(64, ones=True)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    assert np.array_equal(x, np.ones(s.n))


def test_solve_uses_diagonal_not_another_entry():
    """Hand system where dividing by the first entry, or summing the diagonal, is detectable."""
    rp = np.array([0, 1, 3, 6], dtype=np.int32)
    ci = np.array([0, 0, 1, 0, 1, 2], dtype=np.int32)
    v = np.array([2.0, 3.0, 5.0, 7.0, 11.0, 13.0])
    b = np.array([4.0, 6.0 + 5.0 * 1.0, 7.0 * 2.0 + 11.0 * 1.0 + 13.0 * 3.0])
    # x0 = 4/2 = 2 ; x1 = (11 - 3*2)/5 = 1 ; x2 = (64 - 14 - 11)/13 = 3
    x = oracle.solve(rp, ci, v, b)
    assert np.array_equal(x, [2.0, 1.0, 3.0])


def test_solve_componentwise_backward_error():
    s = synth.gen_c4(n=10_000, nlevels=100)
    x = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    A = _sp(s)
    r = np.abs(s.b - A @ x)
    denom = abs(A) @ np.abs(x) + np.abs(s.b)
    k = int(np.max(np.diff(s.rowptr)))
    u = 2.0 ** -53
    assert np.max(r / denom) <= 2 * k * u / (1 - k * u)


@pytest.mark.parametrize("n,nrhs", [(1, 1), (40, 3), (200, 8)])
def test_solve_multi_matches_lapack(n, nrhs):
    """Multi-RHS oracle vs LAPACK dtrtrs with a matrix right-hand side (one call, all columns)."""
    s = synth.gen_dense_lower(n, seed=300 + n)
    B = np.random.default_rng(n).uniform(-1, 1, (n, nrhs))
    X = oracle.solve_multi(s.rowptr, s.colidx, s.val, B)
    ref = scipy.linalg.solve_triangular(_dense(s), B, lower=True)
    assert np.max(np.abs(X - ref)) / np.max(np.abs(ref)) <= 1e-13


def test_solve_multi_integer_columns_bit_exact():
    s = synth.integerize(synth.gen_c2(n=5000))
    rng = np.random.default_rng(3)
    XT = rng.integers(-8, 9, size=(s.n, 5)).astype(float)
    A = scipy.sparse.csr_matrix((s.val, s.colidx, s.rowptr), shape=(s.n, s.n))
    B = A @ XT
    assert np.array_equal(oracle.solve_multi(s.rowptr, s.colidx, s.val, B), XT)


def test_solve_empty():
    x = oracle.solve(np.zeros(1, np.int32), np.zeros(0, np.int32), np.zeros(0), np.zeros(0))
    assert x.shape == (0,)


# ---------------------------------------------------------------- indegree

def test_indegree_closed_form_and_hand():
    s = synth.gen_c2(n=10_000)
    assert np.array_equal(oracle.indegree(s.rowptr, s.colidx), np.diff(s.rowptr) - 1)
    g = synth.gen_grid(16)
    r, c = np.divmod(np.arange(256), 16)
    assert np.array_equal(oracle.indegree(g.rowptr, g.colidx), (r > 0).astype(int) + (c > 0))
    rp, ci = synth.gen_fig2_pattern()
    assert oracle.indegree(rp, ci).tolist() == [0, 1, 1, 2, 2, 1]


# ---------------------------------------------------------------- levels

def _brute_levels(rp, ci):
    """Longest path into each node by exhaustive recursion over explicit dependency sets."""
    n = len(rp) - 1
    deps = [[int(c) for c in ci[rp[i]:rp[i + 1]] if c < i] for i in range(n)]
    memo = {}

    def lv(i):
        if i not in memo:
            memo[i] = 0 if not deps[i] else 1 + max(lv(j) for j in deps[i])
        return memo[i]
    return [lv(i) for i in range(n)]


@pytest.mark.parametrize("seed", range(6))
def test_levels_dp_bfs_brute_agree_tiny(seed):
    s = synth.gen_random_lower(40, 1 + seed % 3, seed)
    want = _brute_levels(s.rowptr, s.colidx)
    assert oracle.levels_dp(s.rowptr, s.colidx).tolist() == want
    assert oracle.levels_bfs(s.rowptr, s.colidx).tolist() == want


def test_levels_fig2_golden():
    rows = [ln.split() for ln in open(os.path.join(GOLDEN, "fig2_levels.txt"))
            if ln.strip() and not ln.startswith("#")]
    want = [int(r[2]) for r in rows]
    rp, ci = [0], []
    for r in rows:  # build the pattern from the fixture's dependency column
        ci += ([] if r[1] == "-" else [int(c) for c in r[1].split(",")]) + [int(r[0])]
        rp.append(len(ci))
    rp, ci = np.array(rp, np.int32), np.array(ci, np.int32)
    g_rp, g_ci = synth.gen_fig2_pattern()
    assert np.array_equal(rp, g_rp) and np.array_equal(ci, g_ci)
    assert oracle.levels_bfs(rp, ci).tolist() == want
    assert oracle.levels_dp(rp, ci).tolist() == want


@pytest.mark.parametrize("n,L", [(20_000, 10), (50_000, 10)])
def test_levels_generator_histogram_c2(n, L):
    s = synth.gen_c2(n=n, nlevels=L)
    lv = oracle.levels_bfs(s.rowptr, s.colidx)
    assert np.array_equal(lv, oracle.levels_dp(s.rowptr, s.colidx))
    assert np.array_equal(lv, np.arange(n) // (n // L))  # contiguous level blocks
    nl, counts = oracle.level_counts(lv)
    assert nl == L and np.all(counts == n // L)


def test_levels_generator_histogram_c2i():
    s = synth.gen_c2i(n=20_000)
    lv = oracle.levels_bfs(s.rowptr, s.colidx)
    assert np.array_equal(lv, np.arange(20_000) % 10)


def test_levels_generator_histogram_c4():
    s = synth.gen_c4(n=30_000, nlevels=30)
    lv = oracle.levels_dp(s.rowptr, s.colidx)
    assert np.array_equal(lv, oracle.levels_bfs(s.rowptr, s.colidx))
    nl, counts = oracle.level_counts(lv)
    assert nl == 30 and np.all(counts == 1000)
    assert s.nnz == 1000 + 29_000 * 64


@pytest.mark.parametrize("g", [1, 2, 5, 64])
def test_levels_grid_closed_form(g):
    s = synth.gen_grid(g)
    lv = oracle.levels_bfs(s.rowptr, s.colidx)
    r, c = np.divmod(np.arange(g * g), g)
    assert np.array_equal(lv, r + c)  # anti-diagonal wavefronts
    nl, counts = oracle.level_counts(lv)
    assert nl == 2 * g - 1
    assert counts.tolist() == [min(k + 1, 2 * g - 1 - k) for k in range(2 * g - 1)]
    assert s.nnz == 3 * g * g - 2 * g


def test_levels_chain_diag_dense():
    s = synth.gen_chain(1000)
    assert oracle.level_counts(oracle.levels_bfs(s.rowptr, s.colidx))[0] == 1000
    d = synth.gen_diag(777)
    nl, counts = oracle.level_counts(oracle.levels_bfs(d.rowptr, d.colidx))
    assert nl == 1 and counts.tolist() == [777]
    t = synth.gen_dense_lower(30)
    assert oracle.levels_dp(t.rowptr, t.colidx).tolist() == list(range(30))


# ---------------------------------------------------------------- validation

def _case(rp, ci, v):
    return oracle.validate(np.array(rp, np.int32), np.array(ci, np.int32), np.array(v, float))


def test_validate_codes():
    assert _case([0, 1, 3], [0, 0, 1], [1, 1, 1]) == (oracle.OK, -1)
    assert _case([0, 1, 3], [0, 1, 1], [1, 1, 1]) == (oracle.UNSORTED, 1)      # duplicate
    assert _case([0, 2, 3], [0, 1, 1], [1, 1, 1]) == (oracle.NOT_LOWER, 0)     # upper entry
    assert _case([0, 1, 3], [0, 1, 0], [1, 1, 1]) == (oracle.UNSORTED, 1)      # diag not last
    assert _case([0, 1, 2], [0, 0], [1, 1]) == (oracle.MISSING_DIAG, 1)
    assert _case([0, 1, 1], [0], [1]) == (oracle.MISSING_DIAG, 1)              # empty row
    assert _case([0, 1, 3], [0, 0, 1], [1, 1, 0]) == (oracle.ZERO_DIAG, 1)
    assert _case([1, 1, 3], [0, 0, 1], [1, 1, 1])[0] == oracle.BAD_ROWPTR
    assert _case([0, 1, 0, 3], [0, 0, 1], [1, 1, 1]) == (oracle.BAD_ROWPTR, 1)
    assert _case([0, 1, 3], [0, -1, 1], [1, 1, 1]) == (oracle.BAD_COL, 1)
    assert _case([0], [], []) == (oracle.OK, -1)


# ---------------------------------------------------------------- Eq. 1 vs Table 6

def _table6():
    out = []
    for ln in open(os.path.join(GOLDEN, "table6.txt")):
        if ln.strip() and not ln.startswith("#"):
            name, d, a, b = ln.split()
            out.append((name, float(d), float(a), float(b)))
    return out


def test_delta_table6_reading_reproduces_paper():
    rows = _table6()
    assert len(rows) == 3
    for name, d, alpha, beta in rows:
        got = oracle.parallel_granularity(beta, alpha, "table6")
        assert round(got, 2) == d, (name, got, d)


def test_delta_printed_form_does_not_reproduce_all_rows():
    """Documents DESIGN.md reading G1: b1 inside log(nnz_row + b1) misses Table 6."""
    rows = _table6()
    got = [round(oracle.parallel_granularity(b, a, "printed"), 2) for _, _, a, b in rows]
    assert got != [d for _, d, _, _ in rows]


def test_delta_closed_forms():
    # log10(log10(100)/(log10(10)+0.01)+0.01)
    assert math.isclose(oracle.parallel_granularity(100, 10), math.log10(2 / 1.01 + 0.01))
    assert math.isnan(oracle.parallel_granularity(1, 3))


def test_gflops_convention():
    assert oracle.gflops(500_000_000, 1.0) == 1.0


def test_analyse_summary():
    s = synth.gen_c2(n=100_000)
    a = oracle.analyse(s.rowptr, s.colidx)
    assert a["nlevels"] == 10 and a["n_level"] == 10_000 and a["nnz"] == 280_000
    assert math.isclose(a["nnz_row"], 2.8)
