"""Event model of synchronization-free SpTRSV scheduling (c2-like leveled matrices).

Rows are dispensed in order in UNITS (CTA = units of `unit` rows) to at most `slots_units`
resident units.  A row starts after its unit starts + load; it completes at
max(start, dep_done + hop) + proc.  A unit frees its slot when ALL its rows completed
(coupled) or row-by-row (decoupled: each freed row slot immediately takes the next row).
"""
import heapq
import sys
import numpy as np

sys.path.insert(0, __file__.rsplit("/tools/", 1)[0])
import synth


def deps_of(s):
    rp, ci = s.rowptr.astype(np.int64), s.colidx.astype(np.int64)
    rows = np.repeat(np.arange(s.n), np.diff(rp))
    off = ci != rows
    # latest dependency index per row (all deps are earlier rows; the latest-completing one matters)
    return rows[off], ci[off]


def simulate_coupled(n, dep_rows, dep_cols, unit=256, resident=592, load=1.5, hop=0.6, proc=0.2, launch=0.3):
    done = np.full(n, np.inf)
    # per-row dependency lists
    order = np.argsort(dep_rows, kind="stable")
    dr, dc = dep_rows[order], dep_cols[order]
    ptr = np.searchsorted(dr, np.arange(n + 1))
    nunits = (n + unit - 1) // unit
    free_at = [0.0] * resident
    heapq.heapify(free_at)
    for u in range(nunits):
        t_start = heapq.heappop(free_at) + launch
        r0, r1 = u * unit, min(n, (u + 1) * unit)
        t_ready = t_start + load
        fin = t_ready
        for i in range(r0, r1):
            d = dc[ptr[i]:ptr[i + 1]]
            t = t_ready if d.size == 0 else max(t_ready, done[d].max() + hop)
            done[i] = t + proc
        fin = done[r0:r1].max()
        heapq.heappush(free_at, fin)
    return done.max()


def simulate_decoupled(n, dep_rows, dep_cols, slots=151552, load=1.5, hop=0.6, proc=0.2):
    order = np.argsort(dep_rows, kind="stable")
    dr, dc = dep_rows[order], dep_cols[order]
    ptr = np.searchsorted(dr, np.arange(n + 1))
    done = np.full(n, np.inf)
    free_at = [0.0] * slots
    heapq.heapify(free_at)
    for i in range(n):
        t0 = heapq.heappop(free_at) + load
        d = dc[ptr[i]:ptr[i + 1]]
        t = t0 if d.size == 0 else max(t0, done[d].max() + hop)
        done[i] = t + proc
        heapq.heappush(free_at, done[i])
    return done.max()


if __name__ == "__main__":
    s = synth.gen_c2()
    dr, dc = deps_of(s)
    for resident in (592, 1184, 2368):
        print("coupled   unit=256 resident=%5d  T=%.1f us" % (resident, simulate_coupled(s.n, dr, dc, resident=resident)))
    for unit, res in ((32, 4736), (1024, 148)):
        print("coupled   unit=%d resident=%d  T=%.1f us" % (unit, res, simulate_coupled(s.n, dr, dc, unit=unit, resident=res)))
    for slots in (151552, 303104, 606208):
        print("decoupled slots=%6d  T=%.1f us" % (slots, simulate_decoupled(s.n, dr, dc, slots=slots)))
