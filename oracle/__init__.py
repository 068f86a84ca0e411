"""CPU oracle for the CapelliniSpTRSV hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_icpp_suz0hw0w20_b200``) never imports it and shares
no code with it; ``liboracle.so`` is compiled from ``oracle/oracle.c`` alone.

Paper: /root/reference/PAPER.md (Su et al., ICPP '20), cited ``PAPER.md:<line>``.

What is here (each function cites the passage it follows):

* :func:`validate`      -- the CSR shape Alg. 1 assumes
* :func:`solve`         -- Algorithm 1, sequential forward substitution
* :func:`solve_multi`   -- Algorithm 1 per column of B (multiple right-hand sides)
* :func:`validate_tri` / :func:`solve_tri` -- upper / unit-diagonal forms (G25)
* :func:`indegree`      -- dependencies per component
* :func:`levels_dp`     -- level of each component, row-order recurrence
* :func:`levels_bfs`    -- the same levels by Kahn's BFS (independent algorithm)
* :func:`level_counts`  -- components per level-set; nlevels (Table 6 beta :421)
* :func:`parallel_granularity` -- Eq. 1, both readings (G1)
* :func:`gflops`        -- the 2*nnz/t convention (G9)

Every function is pinned by ``tests/test_oracle.py`` against something other
than itself (LAPACK/SciPy, closed forms, exact-integer systems, the paper's
Table 6 numbers in ``tests/golden/``).  None is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

# Error codes, restated from oracle.c (same meaning as include/sptrsv.h; no shared header).
OK, INVALID_ARG, NOT_LOWER, MISSING_DIAG, ZERO_DIAG, UNSORTED, BAD_ROWPTR, BAD_COL = 0, -1, -2, -3, -4, -5, -6, -7

_i32p = np.ctypeslib.ndpointer(dtype=np.int32, flags="C_CONTIGUOUS")
_f64p = np.ctypeslib.ndpointer(dtype=np.float64, flags="C_CONTIGUOUS")
_i64p = ctypes.POINTER(ctypes.c_int64)


def build(force: bool = False) -> str:
    """Compile liboracle.so from oracle.c (single thread, -O2 -ffp-contract=off)."""
    with _lock:
        if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
            tmp = _LIB + ".tmp.%d" % os.getpid()
            subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c11",
                                   "-shared", "-fPIC", "-o", tmp, _SRC])
            os.replace(tmp, _LIB)
    return _LIB


def _get():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        lib.oracle_validate.argtypes = [ctypes.c_int32, _i32p, _i32p, _f64p, ctypes.c_int64, _i64p]
        lib.oracle_validate.restype = ctypes.c_int
        lib.oracle_solve.argtypes = [ctypes.c_int32, _i32p, _i32p, _f64p, _f64p, _f64p]
        lib.oracle_solve.restype = None
        lib.oracle_indegree.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p]
        lib.oracle_indegree.restype = None
        lib.oracle_levels_dp.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p]
        lib.oracle_levels_dp.restype = None
        lib.oracle_levels_bfs.argtypes = [ctypes.c_int32, _i32p, _i32p, _i32p]
        lib.oracle_levels_bfs.restype = ctypes.c_int32
        lib.oracle_level_counts.argtypes = [ctypes.c_int32, _i32p, _i32p]
        lib.oracle_level_counts.restype = ctypes.c_int32
        lib.oracle_validate_tri.argtypes = [ctypes.c_int32, _i32p, _i32p, _f64p, ctypes.c_int64,
                                            ctypes.c_int32, _i64p]
        lib.oracle_validate_tri.restype = ctypes.c_int
        lib.oracle_solve_tri.argtypes = [ctypes.c_int32, _i32p, _i32p, _f64p, ctypes.c_int32, _f64p, _f64p]
        lib.oracle_solve_tri.restype = None
        _lib = lib
    return _lib


def _csr(rowptr, colidx, val=None):
    rp = np.ascontiguousarray(rowptr, dtype=np.int32)
    ci = np.ascontiguousarray(colidx, dtype=np.int32)
    if val is None:
        return rp, ci
    return rp, ci, np.ascontiguousarray(val, dtype=np.float64)


def validate(rowptr, colidx, val):
    """CSR rules of Alg. 1 (diagonal is the last entry of each row).

    Returns ``(code, bad_row)``; code 0 == OK.  Row-ordered: the first bad row wins.
    """
    rp, ci, v = _csr(rowptr, colidx, val)
    n = rp.shape[0] - 1
    bad = ctypes.c_int64(-1)
    if v.shape[0] == 0:  # keep ndpointer happy on empty arrays
        v = np.zeros(1)
    if ci.shape[0] == 0:
        ci = np.zeros(1, dtype=np.int32)
    code = _get().oracle_validate(n, rp, ci, v, int(rp[-1]) if n >= 0 else 0, ctypes.byref(bad))
    return int(code), int(bad.value)


def solve(rowptr, colidx, val, b):
    """Algorithm 1: sequential CSR forward substitution, fp64, mul+add unfused."""
    rp, ci, v = _csr(rowptr, colidx, val)
    n = rp.shape[0] - 1
    bb = np.ascontiguousarray(b, dtype=np.float64)
    x = np.zeros(max(n, 1), dtype=np.float64)
    if n > 0:
        _get().oracle_solve(n, rp, ci, v, bb, x)
    return x[:n]


def solve_multi(rowptr, colidx, val, B):
    """Multiple right-hand sides: Algorithm 1 applied to each
    column of B (n x nrhs) independently -- the definition of X = L^{-1} B column by column."""
    B = np.asarray(B, dtype=np.float64)
    X = np.empty_like(B)
    for r in range(B.shape[1]):
        X[:, r] = solve(rowptr, colidx, val, np.ascontiguousarray(B[:, r]))
    return X


UPPER, UNIT_DIAG = 1, 2  # f4 flags (restated from oracle.c)


def validate_tri(rowptr, colidx, val, flags):
    """CSR rules for the four triangular forms (G25): lower / upper
    (diagonal last / first), unit diagonal (diagonal not stored, rows may be empty)."""
    rp, ci, v = _csr(rowptr, colidx, val)
    n = rp.shape[0] - 1
    bad = ctypes.c_int64(-1)
    if v.shape[0] == 0:
        v = np.zeros(1)
    if ci.shape[0] == 0:
        ci = np.zeros(1, dtype=np.int32)
    code = _get().oracle_validate_tri(n, rp, ci, v, int(rp[-1]) if n >= 0 else 0, int(flags),
                                      ctypes.byref(bad))
    return int(code), int(bad.value)


def solve_tri(rowptr, colidx, val, b, flags):
    """Substitution for the four triangular forms (G25): Alg. 1
     for lower, backward substitution (row order reversed, diagonal the first
    stored entry, off-diagonals summed in DESCENDING column order = earliest-solved first, the
    mirror of Alg. 1) for UPPER; UNIT_DIAG drops the division.  flags=0 equals :func:`solve`."""
    rp, ci, v = _csr(rowptr, colidx, val)
    n = rp.shape[0] - 1
    bb = np.ascontiguousarray(b, dtype=np.float64)
    x = np.zeros(max(n, 1), dtype=np.float64)
    if v.shape[0] == 0:
        v = np.zeros(1)
    if ci.shape[0] == 0:
        ci = np.zeros(1, dtype=np.int32)
    if n > 0:
        _get().oracle_solve_tri(n, rp, ci, v, int(flags), bb, x)
    return x[:n]


def indegree(rowptr, colidx):
    """In-degree of each component: stored entries with column < row."""
    rp, ci = _csr(rowptr, colidx)
    n = rp.shape[0] - 1
    out = np.zeros(max(n, 1), dtype=np.int32)
    if n > 0:
        _get().oracle_indegree(n, rp, ci, out)
    return out[:n]


def levels_dp(rowptr, colidx):
    """level[i] = 0 if no dependency else 1 + max level[j] (row order is topological)."""
    rp, ci = _csr(rowptr, colidx)
    n = rp.shape[0] - 1
    out = np.zeros(max(n, 1), dtype=np.int32)
    if n > 0:
        _get().oracle_levels_dp(n, rp, ci, out)
    return out[:n]


def levels_bfs(rowptr, colidx):
    """Levels by Kahn's BFS over the dependency DAG (independent of :func:`levels_dp`)."""
    rp, ci = _csr(rowptr, colidx)
    n = rp.shape[0] - 1
    out = np.zeros(max(n, 1), dtype=np.int32)
    popped = 0
    if n > 0:
        popped = _get().oracle_levels_bfs(n, rp, ci, out)
    if popped != n:
        raise ValueError("dependency graph is not a DAG (popped %d of %d)" % (popped, n))
    return out[:n]


def level_counts(level):
    """Components per level-set (PAPER.md:70; Table 6 beta, :421). Returns (nlevels, counts[:nlevels])."""
    lv = np.ascontiguousarray(level, dtype=np.int32)
    n = lv.shape[0]
    if n == 0:
        return 0, np.zeros(0, dtype=np.int32)
    counts = np.zeros(n, dtype=np.int32)
    nlev = _get().oracle_level_counts(n, lv, counts)
    return int(nlev), counts[:nlev].copy()


def parallel_granularity(n_level, nnz_row, form="table6", b1=0.01, b2=0.01):
    """Eq. 1, default bases 10 and b1 = b2 = 0.01.

    ``form="printed"``: log10( log10(n_level) / log10(nnz_row + b1) + b2 ), as typeset.
    ``form="table6"`` : log10( log10(n_level) / (log10(nnz_row) + b1) + b2 ) -- the only
    placement of b1 that reproduces all three delta values of Table 6;
    DESIGN.md reading G1.  n_level = average components per level, nnz_row = nnz / n.
    """
    if n_level <= 1.0:
        return float("nan")  # log10(1) = 0 numerator; delta undefined (pure chains)
    if form == "printed":
        inner = math.log10(n_level) / math.log10(nnz_row + b1) + b2
    elif form == "table6":
        inner = math.log10(n_level) / (math.log10(nnz_row) + b1) + b2
    else:
        raise ValueError(form)
    return math.log10(inner)


def gflops(nnz: int, seconds: float) -> float:
    """GFLOPS = 2*nnz / t (G9): per row (nnz_i - 1) mul+add, 1 sub, 1 div = 2*nnz_i."""
    return 2.0 * nnz / seconds / 1e9


def analyse(rowptr, colidx):
    """Summary used by tests and the bench: nlevels, counts, n_level (beta), nnz_row (alpha), delta."""
    rp = np.asarray(rowptr)
    n = rp.shape[0] - 1
    nnz = int(rp[-1])
    lv = levels_bfs(rowptr, colidx)
    nlev, counts = level_counts(lv)
    n_level = n / nlev if nlev else 0.0
    nnz_row = nnz / n if n else 0.0
    return {
        "n": n, "nnz": nnz, "nlevels": nlev, "counts": counts,
        "n_level": n_level, "nnz_row": nnz_row,
        "delta_table6": parallel_granularity(n_level, nnz_row, "table6") if n else float("nan"),
        "delta_printed": parallel_granularity(n_level, nnz_row, "printed") if n else float("nan"),
    }
