"""Pins for the f4 oracle (oracle.solve_tri / oracle.validate_tri; G25):
upper-triangular (backward substitution) and unit-diagonal solves, checked against LAPACK /
SciPy, closed forms and exact-integer systems -- never against the oracle itself."""
import numpy as np
import pytest
import scipy.linalg
import scipy.sparse
import scipy.sparse.linalg

import oracle
import synth

U, UNIT = oracle.UPPER, oracle.UNIT_DIAG


def _dense(s):
    A = np.zeros((s.n, s.n))
    rows = np.repeat(np.arange(s.n), np.diff(s.rowptr))
    A[rows, s.colidx] = s.val
    return A


def _csr_of_dense(A, keep_diag=True):
    """CSR (ascending columns) of the nonzeros of A; the diagonal dropped if not keep_diag."""
    n = A.shape[0]
    M = A.copy()
    if not keep_diag:
        np.fill_diagonal(M, 0.0)
    rp, ci, v = [0], [], []
    for i in range(n):
        nz = np.nonzero(M[i])[0]
        ci += nz.tolist()
        v += M[i, nz].tolist()
        rp.append(len(ci))
    return np.array(rp, np.int32), np.array(ci, np.int32), np.array(v, float)


@pytest.mark.parametrize("n", [1, 2, 5, 33, 200])
@pytest.mark.parametrize("flags", [U, UNIT, U | UNIT])
def test_solve_tri_matches_lapack_dense(n, flags):
    """Dense triangle drawn HERE (not by synth), LAPACK dtrtrs with lower/unit_diagonal flags."""
    rng = np.random.default_rng(1000 + n + 7 * flags)
    A = rng.uniform(-0.5, 0.5, size=(n, n))
    A = np.triu(A) if flags & U else np.tril(A)
    np.fill_diagonal(A, 1.0 + np.abs(A).sum(axis=1))
    if flags & UNIT:  # row-scaled so that the implicit unit diagonal keeps it well conditioned
        A = A / np.diag(A)[:, None]
    b = rng.uniform(-1, 1, size=n)
    rp, ci, v = _csr_of_dense(A, keep_diag=not (flags & UNIT))
    assert oracle.validate_tri(rp, ci, v, flags) == (oracle.OK, -1)
    x = oracle.solve_tri(rp, ci, v, b, flags)
    ref = scipy.linalg.solve_triangular(A, b, lower=not (flags & U), unit_diagonal=bool(flags & UNIT))
    assert np.max(np.abs(x - ref)) <= 1e-13 * max(1.0, np.max(np.abs(ref)))


@pytest.mark.parametrize("gen", [lambda: synth.gen_random_lower(3000, 6, 4),
                                 lambda: synth.gen_c2(n=30_000),
                                 lambda: synth.gen_grid(64)])
@pytest.mark.parametrize("flags", [U, UNIT, U | UNIT])
def test_solve_tri_matches_scipy_sparse(gen, flags):
    s = gen()
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:
        s = synth.to_unit(s)
    assert oracle.validate_tri(s.rowptr, s.colidx, s.val, flags) == (oracle.OK, -1)
    x = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    A = scipy.sparse.csr_matrix((s.val, s.colidx, s.rowptr), shape=(s.n, s.n))
    ref = scipy.sparse.linalg.spsolve_triangular(A, s.b, lower=not (flags & U),
                                                 unit_diagonal=bool(flags & UNIT))
    assert np.max(np.abs(x - ref) / np.abs(ref)) <= 1e-12
    assert np.max(np.abs(x - s.x_true) / np.abs(s.x_true)) <= 1e-12


def test_upper_bidiagonal_closed_form_bit_exact():
    """U_ii = 2, U_{i,i+1} = -1, b = 1: x_i = 1 - 2^-(n-i), exact in fp64 for n - i <= 53."""
    n = 40
    rp = np.arange(0, 2 * n, 2, dtype=np.int32)
    rp = np.append(rp, 2 * n - 1).astype(np.int32)
    ci, v = [], []
    for i in range(n):
        ci += [i] + ([i + 1] if i + 1 < n else [])
        v += [2.0] + ([-1.0] if i + 1 < n else [])
    x = oracle.solve_tri(rp, np.array(ci, np.int32), np.array(v), np.ones(n), U)
    assert np.array_equal(x, 1.0 - 2.0 ** -(n - np.arange(n, dtype=float)))


def test_unit_lower_bidiagonal_closed_form_bit_exact():
    """Unit lower, L_{i,i-1} = -1, b = 1: x_i = i + 1.  Row 0 is EMPTY (allowed for UNIT)."""
    n = 1000
    rp = np.concatenate([[0], np.arange(0, n, dtype=np.int32)]).astype(np.int32)
    ci = np.arange(0, n - 1, dtype=np.int32)
    x = oracle.solve_tri(rp, ci, -np.ones(n - 1), np.ones(n), UNIT)
    assert np.array_equal(x, np.arange(1, n + 1, dtype=float))


def test_unit_upper_all_ones_closed_form():
    """Unit upper with every U_ij = 1 (j > i), b = 1: x_{n-1} = 1, x_i = 1 - sum_{j>i} x_j = 0."""
    n = 50
    A = np.triu(np.ones((n, n)), 1)
    rp, ci, v = _csr_of_dense(A)
    x = oracle.solve_tri(rp, ci, v, np.ones(n), U | UNIT)
    assert np.array_equal(x, np.r_[np.zeros(n - 1), 1.0])


@pytest.mark.parametrize("flags", [0, U, UNIT, U | UNIT])
def test_solve_tri_exact_integer_systems(flags):
    """Integer entries / x_true: every partial sum is an exact small integer, so x == x_true
    bit-exactly whatever the order (catches a transposed operand or a wrong diagonal)."""
    s = synth.integerize(synth.gen_random_lower(2000, 5, 9))
    if flags & U:
        s = synth.to_upper(s)
    if flags & UNIT:  # keep integer values: drop the diagonal, b = x + N x
        rows = np.repeat(np.arange(s.n), np.diff(s.rowptr))
        keep = s.colidx != rows
        rp = np.zeros(s.n + 1, np.int64)
        np.cumsum(np.bincount(rows[keep], minlength=s.n), out=rp[1:])
        ci, v = s.colidx[keep], s.val[keep]
        b = s.x_true + np.bincount(rows[keep], weights=v * s.x_true[ci], minlength=s.n)
        s = synth.CSRSystem("u", s.n, rp.astype(np.int32), ci, v, b, s.x_true, {})
    x = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    assert np.array_equal(x, s.x_true)


def test_solve_tri_lower_is_algorithm1_bit_exact():
    s = synth.gen_c2(n=20_000)
    assert np.array_equal(oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, 0),
                          oracle.solve(s.rowptr, s.colidx, s.val, s.b))


@pytest.mark.parametrize("gen", [lambda: synth.gen_random_lower(5000, 7, 12), lambda: synth.gen_c2(n=40_000),
                                 lambda: synth.gen_grid(80)])
def test_upper_is_mirror_of_algorithm1_bit_exact(gen):
    """U = P L P (P the reversal): backward substitution on U IS Alg. 1 on L with b reversed,
    operation for operation (G25's descending-column order), so the results agree bit-exactly
    -- a pin through oracle.solve, which test_oracle.py ties to LAPACK / closed forms."""
    s = gen()
    u = synth.to_upper(s)
    xl = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    xu = oracle.solve_tri(u.rowptr, u.colidx, u.val, u.b, U)
    assert np.array_equal(xu, xl[::-1])


def test_upper_sum_order_descending_column():
    """Row 0 = [1 | 1, e, e] over columns (0 | 1, 2, 3), e = 1e-16, x1 = x2 = x3 = 1.  Descending
    column: (e + e) + 1 = 1 + 2^-52; ascending: (1 + e) + e = 1.  Fixes G25's order, not just
    the value."""
    e = 1e-16
    rp = np.array([0, 4, 5, 6, 7], np.int32)
    ci = np.array([0, 1, 2, 3, 1, 2, 3], np.int32)
    v = np.array([1.0, 1.0, e, e, 1.0, 1.0, 1.0])
    x = oracle.solve_tri(rp, ci, v, np.array([0.0, 1.0, 1.0, 1.0]), U)
    assert np.array_equal(x[1:], [1.0, 1.0, 1.0])
    assert x[0] == -(1.0 + 2.0 ** -52)


def test_upper_uses_first_entry_as_diagonal():
    """Row 0 = [U00=4, U01=2]; the diagonal is the FIRST entry: x1 = 3/5, x0 = (1 - 2*3/5)/4."""
    rp = np.array([0, 2, 3], np.int32)
    x = oracle.solve_tri(rp, np.array([0, 1, 1], np.int32), np.array([4.0, 2.0, 5.0]), np.array([1.0, 3.0]), U)
    assert x[1] == 3.0 / 5.0 and x[0] == (1.0 - 2.0 * (3.0 / 5.0)) / 4.0


def _case(rp, ci, v, f):
    return oracle.validate_tri(np.array(rp, np.int32), np.array(ci, np.int32), np.array(v, float), f)


def test_validate_tri_codes():
    # upper: diagonal first
    assert _case([0, 2, 3], [0, 1, 1], [1, 1, 1], U) == (oracle.OK, -1)
    assert _case([0, 1, 3], [0, 0, 1], [1, 1, 1], U) == (oracle.NOT_LOWER, 1)     # below the diagonal
    assert _case([0, 1, 2], [1, 1], [1, 1], U) == (oracle.MISSING_DIAG, 0)
    assert _case([0, 2, 3], [0, 1, 1], [0, 1, 1], U) == (oracle.ZERO_DIAG, 0)
    assert _case([0, 2, 3], [1, 0, 1], [1, 1, 1], U) == (oracle.UNSORTED, 0)     # col 1 then col 0
    assert _case([0, 1, 1], [0], [1], U) == (oracle.MISSING_DIAG, 1)              # empty row
    # unit lower: diagonal must be absent; rows may be empty
    assert _case([0, 0, 1], [0], [1], UNIT) == (oracle.OK, -1)
    assert _case([0, 1, 1], [0], [1], UNIT) == (oracle.NOT_LOWER, 0)              # stored diagonal
    assert _case([0, 0, 2], [0, 0], [1, 1], UNIT) == (oracle.UNSORTED, 1)
    # unit upper
    assert _case([0, 1, 1], [1], [1], U | UNIT) == (oracle.OK, -1)
    assert _case([0, 1, 1], [0], [1], U | UNIT) == (oracle.NOT_LOWER, 0)
    assert _case([0, 0, 1], [0], [1], U | UNIT) == (oracle.NOT_LOWER, 1)
    # shared rules
    assert _case([0, 1, 1], [2], [1], U | UNIT) == (oracle.BAD_COL, 0)
    assert _case([1, 1, 1], [0], [1], UNIT)[0] == oracle.BAD_ROWPTR
    assert _case([0, 0], [], [], 4)[0] == oracle.INVALID_ARG
    # flags 0 agrees with the lower validator
    for rp, ci, v in (([0, 1, 3], [0, 0, 1], [1, 1, 1]), ([0, 2, 3], [0, 1, 1], [1, 1, 1]),
                      ([0, 1, 3], [0, 0, 1], [1, 1, 0]), ([0, 1, 3], [0, 0, 9], [1, 1, 1]),
                      ([0, 1, 3], [0, -1, 1], [1, 1, 1])):
        assert _case(rp, ci, v, 0) == oracle.validate(np.array(rp, np.int32), np.array(ci, np.int32),
                                                      np.array(v, float))
