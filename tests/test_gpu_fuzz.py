"""Randomised parity sweep (GPU): seeded random structures x engines x protocols x geometries
against the oracle.  The synchronisation-free solve's failure modes are schedule-dependent
(a missed dependency, a stale value, a deadlock on an unusual row mix), so besides the
structured cases of test_gpu_parity.py every engine also sees many irregular ones:
variable row lengths (1..300 entries, mixing thread- and warp-level rows), banded,
near-diagonal and far dependencies, empty-ish rows, ragged sizes.

Bar: bit-exact where every row is thread level, else max componentwise
relative error <= 1e-12 (the solutions are x_true ~ U[1, 2], |x| >= 1).
"""
import os

import numpy as np
import pytest

import oracle
import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-12


def random_structure(rng):
    """A random lower-triangular CSR pattern: per-row off-diagonal counts from a mixed
    distribution, columns drawn from a mixture of bands (near), uniform (far) and the
    previous row (chains)."""
    n = int(rng.choice([1, 2, 31, 33, 257, 1000, 4099, 20_000, 60_000]))
    kind = rng.integers(0, 4)
    rows, cols = [], []
    for i in range(1, n):
        if kind == 0:    # short rows, far dependencies
            m = min(i, int(rng.integers(0, 4)))
        elif kind == 1:  # mixed lengths incl. long (warp-level) rows
            m = min(i, int(rng.choice([0, 1, 2, 3, 8, 40, 120, 300], p=[.1, .2, .2, .2, .1, .1, .05, .05])))
        elif kind == 2:  # banded
            m = min(i, int(rng.integers(1, 6)))
        else:            # chains with occasional far entries
            m = min(i, 1 + int(rng.random() < 0.3))
        if m == 0:
            continue
        if kind == 2:
            lo = max(0, i - int(rng.integers(m, 200)))
            c = rng.choice(np.arange(lo, i), size=min(m, i - lo), replace=False)
        elif kind == 3:
            c = np.unique(np.r_[i - 1, rng.integers(0, i, size=m - 1)])
        else:
            c = rng.choice(i, size=m, replace=False)
        c = np.sort(np.asarray(c, dtype=np.int64))
        rows.append(np.full(c.size, i, dtype=np.int64))
        cols.append(c)
    rows = np.concatenate(rows) if rows else np.zeros(0, np.int64)
    cols = np.concatenate(cols) if cols else np.zeros(0, np.int64)
    allr = np.r_[rows, np.arange(n)]
    allc = np.r_[cols, np.arange(n)]
    o = np.lexsort((allc, allr))
    allr, allc = allr[o], allc[o]
    rowptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(allr, minlength=n), out=rowptr[1:])
    return synth.from_pattern(f"fuzz{kind}", rowptr, allc, rng)


ENGINES = [(5, {}), (0, {}), (3, {}), (6, {}), (7, {}),
           (0, {"cta_threads": 1024}), (7, {"rows_per_lane": 1, "cta_threads": 64}), (3, {"cta_threads": 128}),
           (7, {"cta_threads": 512}), (3, {"cta_threads": 1024}), (8, {}), (8, {"cta_threads": 64}), (9, {})]


def small_fits(s):
    """ENGINE_SMALL accepts systems whose CSR, b and x fit one CTA's shared memory (sptrsv.cu)."""
    n, nnz = s.n, int(s.rowptr[-1])
    up = lambda v: (v + 15) // 16 * 16
    z = max(nnz, 1)
    return n <= (1 << 20) and 3 * up(8 * n) + up(8 * z) + up(4 * (n + 1)) + up(4 * z) + 64 <= 226 * 1024


@pytest.mark.parametrize("seed", range(int(os.environ.get("SPTRSV_FUZZ_SEEDS", "100"))))
def test_fuzz_engines_vs_oracle(seed):
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    rng = np.random.default_rng(1000 + seed)
    s = random_structure(rng)
    ref = oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(a).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    picks = rng.choice(len(ENGINES), size=3, replace=False)
    for k in picks:
        engine, extra = ENGINES[k]
        proto = int(rng.integers(0, 2))
        if engine == 8 and (s.n == 0 or not small_fits(s)):
            continue
        with cap.analyse(rp, ci, v, engine=engine, protocol=proto, **extra) as h:
            for _ in range(2):  # two solves: the epoch path
                x = torch.full_like(b, float("nan"))
                h.solve(b, x)
                h.check()
                got = x.cpu().numpy()
                info = h.info()
                if info["n_warp_rows"] == 0 and info["n_sub_tasks"] == 0:
                    assert np.array_equal(got, ref), (s.name, s.n, engine, proto, extra, info)
                else:
                    err = float(np.max(np.abs(got - ref) / np.abs(ref))) if s.n else 0.0
                    assert err <= TOL, (s.name, s.n, engine, proto, extra, info, err)


@pytest.mark.parametrize("seed", range(int(os.environ.get("SPTRSV_FUZZ_SEEDS", "100")) // 2))
def test_fuzz_triangular_forms_vs_oracle(seed):
    """The same random structures as upper / unit-lower / unit-upper systems through
    AUTO and the forced thread-level engines (LEAN, CHAIN), two solves each, vs oracle.solve_tri."""
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    rng = np.random.default_rng(5000 + seed)
    s = random_structure(rng)
    flags = int(rng.integers(1, 4))  # 1 upper, 2 unit lower, 3 unit upper
    if flags & 1:
        s = synth.to_upper(s)
    if flags & 2:
        s = synth.to_unit(s)
    ref = oracle.solve_tri(s.rowptr, s.colidx, s.val, s.b, flags)
    d = torch.device("cuda:0")
    rp, ci, v, b = (torch.from_numpy(np.ascontiguousarray(a)).to(d) for a in (s.rowptr, s.colidx, s.val, s.b))
    for opts in ({}, {"engine": 3, "mode": 1}, {"engine": 7, "mode": 1}, {"engine": 8}, {"engine": 9, "mode": 1}):
        proto = int(rng.integers(0, 2))
        if opts.get("engine") == 8 and (s.n == 0 or not small_fits(s)):
            continue
        with cap.analyse(rp, ci, v, upper=bool(flags & 1), unit_diag=bool(flags & 2), protocol=proto, **opts) as h:
            for _ in range(2):
                x = torch.full_like(b, float("nan"))
                h.solve(b, x)
                h.check()
                got = x.cpu().numpy()
                inf = h.info()
                if inf["n_warp_rows"] == 0 and inf["n_sub_tasks"] == 0:
                    assert np.array_equal(got, ref), (s.name, s.n, flags, opts, proto)
                else:
                    err = float(np.max(np.abs(got - ref) / np.abs(ref))) if s.n else 0.0
                    assert err <= TOL, (s.name, s.n, flags, opts, proto, err)
