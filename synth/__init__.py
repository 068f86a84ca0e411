"""Seeded synthetic lower-triangular CSR systems -- shared input generators.

This module holds NO arithmetic of the method (no triangular solve, no level
analysis, no flag protocol).  It only draws sparsity patterns and values with
numpy's PCG64 (``numpy.random.default_rng(seed)``) and forms ``b = L @ x_true``
(a sparse matrix-vector product, not the solve).  It is the one module both the
oracle tests and the CUDA path's tests/bench use, as the task rules allow.

Every system satisfies the CSR contract of Algorithm 1: int32
``rowptr``/``colidx``, fp64 ``val``, columns strictly increasing per row, the
diagonal stored LAST.  Off-diagonals are U[-0.5, 0.5]; ``L_ii = 1 + sum_j |L_ij|``
(strict row diagonal dominance); ``x_true ~ U[1, 2]``.

Configs follow BASELINE.json ``configs`` and SURVEY.md section 8(d):

=====  =====================================================  ==========
name   construction                                            seed
=====  =====================================================  ==========
c1     n=1000, row i: min(3,i) distinct cols uniform in [0,i)   1
c2     n=1e6, 10 contiguous levels x 1e5; 2 deps per row        2
c2i    c2 histogram, level(i)=i mod 10 (intra-warp chains)      2
c3     2048x2048 5-point grid lower factor, diag 4, off -1      3
c4     n=1e6, 1000 levels x 1000; 63 deps per row               4
c5     8 systems, c2 construction at n=2e6 (10 x 2e5)           500..507
chain  bidiagonal n=1e5, L_ii=2, L_i,i-1=-1, b=1                6
=====  =====================================================  ==========
"""
from __future__ import annotations

import dataclasses
import hashlib

import numpy as np

__all__ = [
    "CSRSystem", "gen_c1", "gen_c2", "gen_c2i", "gen_c3", "gen_grid", "gen_c4", "gen_c5",
    "gen_chain", "gen_diag", "gen_dense_lower", "gen_random_lower", "gen_leveled",
    "gen_fig2_pattern", "integerize", "from_pattern", "to_upper", "to_unit", "CONFIGS", "make",
]


@dataclasses.dataclass
class CSRSystem:
    name: str
    n: int
    rowptr: np.ndarray      # int32 [n+1]
    colidx: np.ndarray      # int32 [nnz]
    val: np.ndarray         # float64 [nnz]
    b: np.ndarray           # float64 [n]
    x_true: np.ndarray | None
    meta: dict

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def sha256(self) -> dict:
        return {k: hashlib.sha256(np.ascontiguousarray(getattr(self, k)).tobytes()).hexdigest()[:16]
                for k in ("rowptr", "colidx", "val", "b")}

    def alg_bytes(self) -> int:
        """Algorithmic HBM bytes of one solve: rowptr 4(n+1) + colidx/val 12*nnz + b 8n + x 8n + flags 4n."""
        return 4 * (self.n + 1) + 12 * self.nnz + 20 * self.n


# ----------------------------------------------------------------------------- helpers

def _rows_of(rowptr: np.ndarray) -> np.ndarray:
    n = rowptr.shape[0] - 1
    return np.repeat(np.arange(n, dtype=np.int64), np.diff(rowptr.astype(np.int64)))


def from_pattern(name, rowptr, colidx, rng, meta=None, x_true=None, offdiag=None, diag=None):
    """Assign the standard values to a pattern (diag last in each row) and form b = L @ x_true."""
    rowptr = np.ascontiguousarray(rowptr, dtype=np.int32)
    colidx = np.ascontiguousarray(colidx, dtype=np.int32)
    n = rowptr.shape[0] - 1
    nnz = int(rowptr[-1])
    rows = _rows_of(rowptr)
    is_diag = colidx.astype(np.int64) == rows
    if offdiag is None:
        val = rng.uniform(-0.5, 0.5, size=nnz)
    else:
        val = np.asarray(offdiag, dtype=np.float64).copy()
    if diag is None:
        s = np.bincount(rows[~is_diag], weights=np.abs(val[~is_diag]), minlength=n)
        dvals = 1.0 + s
    else:
        dvals = np.broadcast_to(np.asarray(diag, dtype=np.float64), (n,))
    val[is_diag] = dvals[rows[is_diag]]
    if x_true is None:
        x_true = rng.uniform(1.0, 2.0, size=n)
    x_true = np.asarray(x_true, dtype=np.float64)
    b = np.bincount(rows, weights=val * x_true[colidx], minlength=n).astype(np.float64)
    m = dict(meta or {})
    return CSRSystem(name, n, rowptr, colidx, np.ascontiguousarray(val), np.ascontiguousarray(b),
                     x_true, m)


def _assemble(n, offcols_per_row):
    """offcols_per_row: (row_ids int64 sorted-by-row, cols int64) of off-diagonals, sorted within row."""
    rows, cols = offcols_per_row
    cnt = np.bincount(rows, minlength=n).astype(np.int64) + 1
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(cnt, out=rowptr[1:])
    colidx = np.empty(int(rowptr[-1]), dtype=np.int64)
    # position of each off-diagonal: rowptr[row] + rank within row
    if rows.size:
        first = np.searchsorted(rows, rows, side="left")
        rank = np.arange(rows.size) - first
        colidx[rowptr[rows] + rank] = cols
    colidx[rowptr[1:] - 1] = np.arange(n)
    return rowptr.astype(np.int32), colidx.astype(np.int32)


# ----------------------------------------------------------------------------- configs

def gen_random_lower(n: int, k: int, seed: int, name: str | None = None) -> CSRSystem:
    """Row i has min(k, i) distinct off-diagonal columns drawn uniformly from [0, i)."""
    rng = np.random.default_rng(seed)
    rows_l, cols_l = [], []
    for i in range(1, n):
        m = min(k, i)
        c = np.sort(rng.choice(i, size=m, replace=False))
        rows_l.append(np.full(m, i, dtype=np.int64))
        cols_l.append(c.astype(np.int64))
    rows = np.concatenate(rows_l) if rows_l else np.zeros(0, np.int64)
    cols = np.concatenate(cols_l) if cols_l else np.zeros(0, np.int64)
    rp, ci = _assemble(n, (rows, cols))
    return from_pattern(name or f"random_n{n}_k{k}", rp, ci, rng, {"seed": seed, "k": k})


def gen_c1(seed: int = 1) -> CSRSystem:
    """C1: n=1000, ~4 nnz/row (min(3,i) off-diagonals) -> nnz = 3994."""
    return gen_random_lower(1000, 3, seed, name="c1")


def _distinct_draws(rng, lo, hi, k, must):
    """Per row r: k distinct ints uniform in [lo_r, hi_r), all different from must[r].
    Duplicates (the later of an equal pair after sorting, or any equal to must) are redrawn
    until none remain.  Returns (M, k) int64 sorted per row."""
    out = rng.integers(lo[:, None], hi[:, None], size=(lo.shape[0], k))
    todo = np.arange(lo.shape[0])
    while todo.size:
        sub = np.sort(out[todo], axis=1)
        dup = np.zeros(sub.shape, dtype=bool)
        dup[:, 1:] = sub[:, 1:] == sub[:, :-1]
        dup |= sub == must[todo, None]
        out[todo] = sub
        bad = np.nonzero(dup.any(axis=1))[0]
        if bad.size == 0:
            break
        rr, cc = np.nonzero(dup[bad])
        glob = todo[bad[rr]]
        out[glob, cc] = rng.integers(lo[glob], hi[glob])
        todo = todo[bad]
    return out


def gen_leveled(n: int, nlevels: int, k_prev: int, k_any: int, seed: int, name: str) -> CSRSystem:
    """Contiguous level blocks of W = n/nlevels rows: rows [l*W, (l+1)*W) form level l.

    Level-0 rows are diagonal only.  A row in level l >= 1 has one column uniform in
    level l-1 (k_prev must be 1) and k_any further distinct columns uniform in
    [0, l*W); so its level is exactly l and the histogram is nlevels x W.
    """
    assert k_prev == 1 and n % nlevels == 0
    rng = np.random.default_rng(seed)
    W = n // nlevels
    r = np.arange(W, n, dtype=np.int64)
    lev = r // W
    a = rng.integers((lev - 1) * W, lev * W)
    if k_any:
        others = _distinct_draws(rng, np.zeros_like(lev), lev * W, k_any, a)
        cols = np.concatenate([a[:, None], others], axis=1)
    else:
        cols = a[:, None]
    cols.sort(axis=1)
    k = cols.shape[1]
    rows = np.repeat(r, k)
    rp, ci = _assemble(n, (rows, cols.reshape(-1)))
    return from_pattern(name, rp, ci, rng, {"seed": seed, "levels": nlevels, "width": W,
                                             "deps_per_row": k})


def gen_c2(seed: int = 2, n: int = 1_000_000, nlevels: int = 10, name: str = "c2") -> CSRSystem:
    """C2: n=1e6, 10 levels x 1e5, 2 deps per row (one in level l-1) -> nnz = 2.8e6."""
    return gen_leveled(n, nlevels, 1, 1, seed, name)


def gen_c2i(seed: int = 2, n: int = 1_000_000, nlevels: int = 10) -> CSRSystem:
    """C2i (deadlock stress): level(i) = i mod L. Row i with l = i mod L >= 1 depends on i-1
    and on one uniform earlier row of level < l other than i-1 (omitted when none exists).
    Rows with i mod L == 0 are diagonal only.  ~half the dependencies stay inside a warp."""
    rng = np.random.default_rng(seed)
    L = nlevels
    i = np.arange(n, dtype=np.int64)
    lv = i % L
    q = i // L
    has = lv >= 1
    ii, ll, qq = i[has], lv[has], q[has]
    cnt = qq * ll + ll - 1
    u = (rng.random(ii.size) * np.maximum(cnt, 1)).astype(np.int64)
    u = np.minimum(u, np.maximum(cnt - 1, 0))
    in_prev = u < qq * ll
    rq = np.where(in_prev, u // np.maximum(ll, 1), qq)
    ro = np.where(in_prev, u % np.maximum(ll, 1), u - qq * ll)
    other = rq * L + ro
    ok = cnt > 0
    rows = np.concatenate([ii[ok], ii])
    cols = np.concatenate([other[ok], ii - 1])
    order = np.lexsort((cols, rows))
    rp, ci = _assemble(n, (rows[order], cols[order]))
    return from_pattern("c2i", rp, ci, rng, {"seed": seed, "levels": L})


def gen_grid(g: int = 2048, seed: int = 3, ones: bool = False, name: str | None = None) -> CSRSystem:
    """Lower factor pattern of a g x g 5-point grid (row-major i = r*g + c): diag 4,
    -1 at (i, i-1) if c > 0 and at (i, i-g) if r > 0.  nnz = 3n - 2g; levels 2g-1.
    ``ones``: b = L @ 1 (x = 1 exactly); else x_true ~ U[1,2]."""
    rng = np.random.default_rng(seed)
    n = g * g
    i = np.arange(n, dtype=np.int64)
    r, c = i // g, i % g
    s_rows = i[r > 0]
    w_rows = i[c > 0]
    rows = np.concatenate([s_rows, w_rows])
    cols = np.concatenate([s_rows - g, w_rows - 1])
    order = np.lexsort((cols, rows))
    rp, ci = _assemble(n, (rows[order], cols[order]))
    nnz = int(rp[-1])
    off = np.full(nnz, -1.0)
    x_true = np.ones(n) if ones else None
    return from_pattern(name or ("c3" if g == 2048 else f"grid{g}"), rp, ci, rng,
                        {"seed": seed, "grid": g, "ones": ones}, x_true=x_true, offdiag=off,
                        diag=4.0)


def gen_stencil(nx: int, ny: int, nz: int = 1, seed: int = 12, rows: int | None = None,
                name: str | None = None) -> CSRSystem:
    """Lower factor pattern of an nx x ny (x nz) 5-point (7-point) grid, row-major
    i = (z*ny + y)*nx + x: off-diagonals at i-1 (x > 0), i-nx (y > 0), i-nx*ny (z > 0); the
    standard values (off-diagonals U[-0.5, 0.5], diag 1 + sum |L_ij|, x_true ~ U[1, 2]).
    ``rows``: keep only the leading rows (a ragged last grid line)."""
    rng = np.random.default_rng(seed)
    n = nx * ny * nz
    i = np.arange(n, dtype=np.int64)
    x, y, z = i % nx, (i // nx) % ny, i // (nx * ny)
    parts_r, parts_c = [i[x > 0]], [i[x > 0] - 1]
    parts_r.append(i[y > 0]), parts_c.append(i[y > 0] - nx)
    if nz > 1:
        parts_r.append(i[z > 0]), parts_c.append(i[z > 0] - nx * ny)
    r_all, c_all = np.concatenate(parts_r), np.concatenate(parts_c)
    if rows is not None:
        keep = r_all < rows
        r_all, c_all, n = r_all[keep], c_all[keep], rows
    order = np.lexsort((c_all, r_all))
    rp, ci = _assemble(n, (r_all[order], c_all[order]))
    return from_pattern(name or f"stencil{nx}x{ny}x{nz}", rp, ci, rng,
                        {"seed": seed, "nx": nx, "ny": ny, "nz": nz})


def gen_c3(seed: int = 3, ones: bool = False) -> CSRSystem:
    return gen_grid(2048, seed, ones, name="c3")


def gen_c4(seed: int = 4, n: int = 1_000_000, nlevels: int = 1000, k_any: int = 62,
           name: str = "c4") -> CSRSystem:
    """C4: n=1e6, 1000 levels x 1000 rows, 63 deps per row -> nnz = 63,937,000."""
    return gen_leveled(n, nlevels, 1, k_any, seed, name)


def gen_c5(system: int, n: int = 2_000_000) -> CSRSystem:
    """C5 system s (0..7): the C2 construction at n=2e6 (10 levels x 2e5), seed 500+s."""
    return gen_leveled(n, 10, 1, 1, 500 + system, f"c5_{system}")


def gen_chain(n: int = 100_000, closed_form: bool = True, seed: int = 6) -> CSRSystem:
    """Bidiagonal chain.  closed_form: L_ii = 2, L_i,i-1 = -1, b = 1, whose solution is
    x_i = 1 - 2^-(i+1) exactly (i <= 52) and 1.0 after; else standard U values."""
    rng = np.random.default_rng(seed)
    rows = np.arange(1, n, dtype=np.int64)
    rp, ci = _assemble(n, (rows, rows - 1))
    if closed_form:
        nnz = int(rp[-1])
        val = np.full(nnz, -1.0)
        val[rp[1:] - 1] = 2.0
        b = np.ones(n)
        return CSRSystem("chain", n, rp, ci, val, b, None, {"seed": seed, "closed_form": True})
    return from_pattern("chain_u", rp, ci, rng, {"seed": seed})


def gen_diag(n: int, seed: int = 7) -> CSRSystem:
    """Diagonal only: d ~ U[1,2], b ~ U[-1,1] -> x_i = b_i / d_i (one IEEE division)."""
    rng = np.random.default_rng(seed)
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    d = rng.uniform(1.0, 2.0, size=n)
    b = rng.uniform(-1.0, 1.0, size=n)
    return CSRSystem("diag", n, rp, ci, d, b, None, {"seed": seed})


def gen_dense_lower(n: int, seed: int = 8) -> CSRSystem:
    """Fully dense lower triangle (n levels of one component)."""
    rng = np.random.default_rng(seed)
    rows = np.repeat(np.arange(n, dtype=np.int64), np.arange(n))
    cols = np.concatenate([np.arange(i, dtype=np.int64) for i in range(n)]) if n else np.zeros(0, np.int64)
    rp, ci = _assemble(n, (rows, cols))
    return from_pattern(f"dense{n}", rp, ci, rng, {"seed": seed})


def gen_fig2_pattern() -> tuple[np.ndarray, np.ndarray]:
    """The part of the paper's 8x8 example recoverable from prose (PAPER.md:196, :226, :230,
    :240, :242, :244, :297): row 0 diagonal only; L(1,0); L(2,1); L(3,1), L(3,2);
    L(4,0), L(4,1); L(5,2).  Rows 6-7 are unknown (Fig. 1 is missing) and omitted."""
    deps = {0: [], 1: [0], 2: [1], 3: [1, 2], 4: [0, 1], 5: [2]}
    rows = np.concatenate([np.full(len(v), k, dtype=np.int64) for k, v in deps.items()])
    cols = np.concatenate([np.array(v, dtype=np.int64) for v in deps.values()])
    return _assemble(6, (rows, cols))


def integerize(sys: CSRSystem, seed: int = 11, lim: int = 8) -> CSRSystem:
    """Same pattern, exact-integer values: off-diagonals in {-2..2}, diag in {-1, 1, 2, -2, 4},
    x_true integers in [-lim, lim], b = L @ x_true exactly (all partial sums are small
    integers < 2^53), so x == x_true bit-exactly in ANY summation order, fused or not."""
    rng = np.random.default_rng(seed)
    n = sys.n
    rows = _rows_of(sys.rowptr)
    is_diag = sys.colidx.astype(np.int64) == rows
    val = rng.integers(-2, 3, size=sys.nnz).astype(np.float64)
    dch = np.array([-1.0, 1.0, 2.0, -2.0, 4.0])
    x_true = rng.integers(-lim, lim + 1, size=n).astype(np.float64)
    d = dch[rng.integers(0, dch.size, size=n)]
    val[is_diag] = d[rows[is_diag]]
    b = np.bincount(rows, weights=val * x_true[sys.colidx], minlength=n).astype(np.float64)
    return CSRSystem(sys.name + "_int", n, sys.rowptr, sys.colidx, val, b, x_true,
                     dict(sys.meta, integer=True))


def to_upper(sys: CSRSystem) -> CSRSystem:
    """the upper-triangular system U = P L P with P the reversal permutation
    (U_ij = L_{n-1-i, n-1-j}); b and x_true reversed.  Row i of U is row n-1-i of L with
    columns mapped c -> n-1-c and re-sorted ascending, so the diagonal comes FIRST.  Same
    dependency DAG (reversed), same values, same nnz per row."""
    n = sys.n
    rp = sys.rowptr.astype(np.int64)
    lens = np.diff(rp)[::-1]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(lens, out=rowptr[1:])
    # the flattened entries of L reversed are exactly: row n-1 reversed, row n-2 reversed, ...
    src = np.arange(sys.nnz - 1, -1, -1, dtype=np.int64)
    colidx = (n - 1 - sys.colidx[src].astype(np.int64)).astype(np.int32)
    val = sys.val[src].copy()
    xt = None if sys.x_true is None else sys.x_true[::-1].copy()
    return CSRSystem(sys.name + "_upper", n, rowptr.astype(np.int32), colidx, val, sys.b[::-1].copy(),
                     xt, dict(sys.meta, upper=True))


def to_unit(sys: CSRSystem, upper: bool = False) -> CSRSystem:
    """the unit-diagonal system D^{-1} T (T = sys, D its diagonal) with the
    diagonal NOT stored: every off-diagonal divided by its row's diagonal (the form an
    incomplete factorisation produces), b = (I + N) @ x_true with N the stored entries.
    ``upper`` says which side of each row holds the diagonal (first / last entry)."""
    n = sys.n
    rows = _rows_of(sys.rowptr)
    is_diag = sys.colidx.astype(np.int64) == rows
    d = np.ones(n)
    d[rows[is_diag]] = sys.val[is_diag]
    keep = ~is_diag
    colidx = sys.colidx[keep].copy()
    val = sys.val[keep] / d[rows[keep]]
    rowptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows[keep], minlength=n), out=rowptr[1:])
    xt = sys.x_true if sys.x_true is not None else np.ones(n)
    b = xt + np.bincount(rows[keep], weights=val * xt[colidx], minlength=n)
    return CSRSystem(sys.name + "_unit", n, rowptr.astype(np.int32), colidx, val, b.astype(np.float64),
                     xt.copy(), dict(sys.meta, unit=True))


CONFIGS = {
    "c1": gen_c1,
    "c2": gen_c2,
    "c2i": gen_c2i,
    "c3": gen_c3,
    "c4": gen_c4,
    "c5": lambda: gen_c5(0),
    "chain": gen_chain,
}


def make(name: str, **kw) -> CSRSystem:
    if name.startswith("c5_"):
        return gen_c5(int(name[3:]), **kw)
    if name.startswith("diag:"):  # scratch shapes for the perf tools: diag:N, lev:N:L
        return gen_diag(int(name.split(":")[1]))
    if name.startswith("chain:"):
        return gen_chain(int(name.split(":")[1]))
    if name.startswith("lev:"):
        _, n, nl = name.split(":")
        return gen_leveled(int(n), int(nl), 1, 1, 2, name)
    return CONFIGS[name](**kw)
