#!/usr/bin/env python
"""Benchmark: SpTRSV GFLOPS (2*nnz / solve time, fp64) and % of HBM roofline on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2] [--impl cuda|reference]

One step = one pass of the whole hot path (one ``sptrsv_solve`` launch per system) over the
config's synthetic system(s), inputs resident in HBM, L2 flushed (256 MiB write) between steps
outside the timed events.  ``value`` = 2*nnz*K / (sum of the K step times), ``ms_per_step`` the
mean step -- ``roofline.frac`` is computed from that same mean.

N = 1: the headline workload is BASELINE.json configs[1] ("c2": n=1e6, ~3 nnz/row, 10 levels x
1e5).  The same line carries a ``configs`` leg that times every other BASELINE config (c1, c3,
c4, one C5 system; plus the aux pure chain) under the same rules, each with its roofline
fraction (measured and nominal HBM peak), critical-path latency bound, t / max(T_bw, T_lat) and
the ncu-measured DRAM bytes of one cold launch (``--no-ncu`` to skip).

N > 1: ``value`` is WEAK scaling of the headline: every GPU solves its own c2-shaped system (seed + GPU),
so the driver's per-N values compare like for like; ``c5_batch_leg`` is BASELINE.json configs[4]: the 8
fixed C5 systems, system s on GPU s mod N (strong scaling; ``--config c5`` makes it the value).  The
N = 1 line carries the same 8-system batch on one GPU (``configs.c5batch``).  No data is exchanged, so
no NCCL (``paper_conf_icpp_suz0hw0w20_b200.batch``):
  * without torchrun, this one process drives N devices, one stream each;
  * under torchrun (WORLD_SIZE > 1), each rank drives its own GPU and the barrier / max over
    ranks go through a CPU (gloo) process group -- control plane only.
Either way the timed region's length is the max over devices of their CUDA-event spans, and
``value`` = all systems' flops / that time.  Fewer visible GPUs than N is an error.

The oracle (oracle/, the plain CPU implementation) is used here only for the cpu_baseline leg
and for --impl reference, as the task rules allow; the reference arm never imports the product
package (it loads no libsptrsv.so).
"""
from __future__ import annotations

import argparse
import json
import os
import shutil
import subprocess
import sys
import tempfile
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "SpTRSV GFLOPS (2*nnz/solve time, fp64)"
UNIT = "GFLOPS"
NOMINAL_HBM_GBS = 8000.0  # B200 HBM3e nominal (north_star's "~8 TB/s")
WORKLOADS = {
    "c1": "random lower-triangular CSR n=1000, ~4 nnz/row, diagonally dominant, fp64, single RHS",
    "c2": "n=1,000,000, ~3 nnz/row (2.8 nnz/row), 10 levels x 100,000 components (warp-underutilisation regime)",
    "c3": "lower factor of a 2D 5-point grid 2048x2048 (n=4,194,304, 4095 anti-diagonal levels)",
    "c4": "n=1,000,000, ~64 nnz/row, 1000 levels x 1000 (warp-per-row regime)",
    "c5": "batch of 8 independent n=2,000,000 low-nnz systems (10 levels x 200,000), system s on GPU s mod N",
    "c5sys": "one C5 system: n=2,000,000, 2.8 nnz/row, 10 levels x 200,000",
    "chain": "bidiagonal chain n=100,000 (pure dependency chain, aux)",
}
ENGINES = {0: "one-shot (staged, in-CTA x copy)", 3: "lean", 6: "hybrid (warp tasks + 32-row thread groups)",
           7: "chain (in-warp chains)", 8: "small (one CTA, shared memory)", 9: "leanp (persistent, pipelined)",
           10: "grid (wavefront bands of 32 columns)", 33: "paper Alg.3", 34: "paper Alg.4", 35: "paper Alg.5"}
KERNELS = {0: "k_solve", 3: "k_solve_lean", 6: "k_solve_tri_warp", 7: "k_solve_chain", 8: "k_solve_small",
           9: "k_solve_leanp", 10: "k_solve_grid",
           33: "k_paper_alg3", 34: "k_paper_alg4", 35: "k_paper_alg5"}
EXTRA_CONFIGS = ["c1", "c3", "c4", "c5sys", "chain"]


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default=None, choices=sorted(WORKLOADS),
                    help="workload (default c2; N > 1: c2 on every GPU, plus the C5 batch leg)")
    ap.add_argument("--impl", default="cuda", choices=["cuda", "reference"])
    ap.add_argument("--mode", type=int, default=0, help="0 auto, 1 thread, 2 warp")
    ap.add_argument("--cpu-seconds", type=float, default=10.0, help="cpu_baseline sample budget")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the per-config leg (N=1)")
    ap.add_argument("--no-ncu", action="store_true", help="skip the ncu DRAM-traffic pass")
    ap.add_argument("--profile", action="store_true", help="headline only (for ncu): no extra legs")
    ap.add_argument("--opt", action="append", default=[], help="extra handle option key=value")
    ap.add_argument("--no-flags-leg", action="store_true", help="skip the FLAGS-protocol / no-window legs")
    ap.add_argument("--no-tri-leg", action="store_true", help="skip the upper / unit-diagonal (f4) leg")
    ap.add_argument("--nrhs", type=int, default=8, help="right-hand sides of the multi-RHS leg (0 = skip)")
    ap.add_argument("--no-c5-leg", action="store_true", help="N > 1: skip the C5 strong-scaling leg")
    ap.add_argument("--ncu-child", default=None, help=argparse.SUPPRESS)
    a = ap.parse_args(argv)
    if a.config is None:
        a.config = "c2"
    return a


# ------------------------------------------------------------------ workloads (host only: no product import)

def make_system(name: str, rank: int = 0):
    import synth
    if name == "c2":
        return synth.gen_c2(seed=2 + rank)
    if name == "c3":
        return synth.gen_c3(seed=3 + rank)
    if name == "c4":
        return synth.gen_c4(seed=4 + rank)
    if name == "c1":
        return synth.gen_c1(seed=1 + rank)
    if name == "c5sys":
        return synth.gen_c5(0)
    if name == "chain":
        return synth.gen_chain()
    raise ValueError(name)


def c5_systems(owned):
    import synth
    return [synth.gen_c5(s) for s in owned]


def generator_levels(s):
    """Level count the generator guarantees by construction (synth), or None."""
    m = s.meta or {}
    if "levels" in m:
        return int(m["levels"])
    if s.name.startswith("grid") or s.name == "c3":
        g = int(round(np.sqrt(s.n)))
        return 2 * g - 1
    if s.name == "chain":
        return s.n
    return None


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy bandwidth)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks (nvidia-smi during the timed region)

class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap,clocks_event_reasons.hw_power_brake_slowdown")

    def __init__(self, indices):
        self.indices = ",".join(str(i) for i in indices)
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", self.indices, f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            time.sleep(0.3)
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) >= 7:
                self.rows.append(parts)

    def __exit__(self, *exc):
        if self.proc:
            time.sleep(0.15)
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap", "hw_power_brake"]
        reasons = sorted({names[k] for r in self.rows for k in range(5) if r[2 + k].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# ------------------------------------------------------------------ reference arm (the CPU oracle)

def run_reference(args, rank, world):
    """The oracle as it stands (single thread, plain C Alg.1), on the same workload; rank 0 only."""
    import oracle
    if rank != 0:
        return
    if args.config == "c5":
        systems = c5_systems(range(8))
    else:
        systems = [make_system(args.config)]
    for _ in range(args.warmup):
        for s in systems:
            oracle.solve(s.rowptr, s.colidx, s.val, s.b)
    times = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        for s in systems:
            oracle.solve(s.rowptr, s.colidx, s.val, s.b)
        times.append(time.perf_counter() - t0)
    nnz = sum(s.nnz for s in systems)
    tot = float(np.sum(times))
    value = 2.0 * nnz * args.steps / tot / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": tot / args.steps * 1e3,
        "higher_is_better": True, "scaling": "weak" if args.config != "c5" else "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {WORKLOADS[args.config]}", "n": int(sum(s.n for s in systems)),
                   "nnz": int(nnz)},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                         "sample": f"{len(systems)} full system(s) per step, {args.steps} steps, single-thread C "
                                   f"oracle (Alg. 1), host {os.cpu_count()} cores"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def cpu_baseline(s, budget_s):
    import oracle
    reps = 0
    oracle.solve(s.rowptr, s.colidx, s.val, s.b)  # warm
    t0 = time.perf_counter()
    while True:
        oracle.solve(s.rowptr, s.colidx, s.val, s.b)
        reps += 1
        el = time.perf_counter() - t0
        if el >= budget_s or reps >= 2000:
            break
    return {"value": 2.0 * s.nnz * reps / el / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"{reps} repeated full solves of the headline system ({s.name}, n={s.n}, nnz={s.nnz}) in "
                      f"{el:.1f}s, single-thread C oracle (Alg. 1, gcc -O2); host has {os.cpu_count()} cores"}


# ------------------------------------------------------------------ timing helpers (CUDA arm)

def time_steps(torch, solve, stream, flush, steps, warmup):
    """Per-step ms: CUDA events on `stream` around `solve()`; L2 flushed before every step,
    outside the events; synchronised on both sides of the timed region."""
    for _ in range(warmup):
        flush.zero_()
        solve()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    for i in range(steps):
        flush.zero_()
        ev[i][0].record(stream)
        solve()
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    return np.array([a.elapsed_time(b) for a, b in ev])


def roofline(s, mean_s, peak, peak_src, kernel, traffic=None):
    alg = s.alg_bytes()
    ach = alg / mean_s / 1e9
    return {"bound": "hbm", "kernel": kernel, "achieved": round(ach, 2), "peak": peak, "unit": "GB/s",
            "frac": round(ach / peak, 4), "peak_source": peak_src,
            "frac_of_nominal_8tbs": round(ach / NOMINAL_HBM_GBS, 4),
            "traffic": (traffic or {}).get("total"), "traffic_read": (traffic or {}).get("read"),
            "traffic_write": (traffic or {}).get("write"),
            "traffic_source": (traffic or {}).get("source", "not measured"),
            "alg_bytes_per_launch": alg, "alg_bytes_formula": "4(n+1) + 12*nnz + 8n (b) + 8n (x) + 4n (flags)"}


def latency_bound(levels, hops, mean_s, alg_bytes, peak, engine=None):
    """T_lat = (levels - 1) * t_hop per die placement; t / max(T_bw, T_lat)."""
    t_bw = alg_bytes / (peak * 1e9)
    out = {"levels": int(levels), "t_bw_us": round(t_bw * 1e6, 3),
           "model": "(levels - 1) * t_hop with the cross-SM record hop: a bound when every level boundary crosses "
                    "SMs; CHAIN resolves in-warp levels in registers (~0.1 us per step), so for chains and grids it "
                    "is a model, not a bound"}
    if engine == 10:
        out["model"] = ("GRID crosses SMs only at band boundaries (ceil(m/32) - 1 record hops, lane 0 of a band "
                        "waiting on lane 31 of the previous one); the other level boundaries are register / "
                        "shuffle steps inside a warp (~0.23 us each under load), so (levels - 1) * t_hop is a "
                        "reference scale here, not a bound")
    if engine == 8:
        out["model"] = ("SMALL solves the whole system in ONE SM's shared memory: no level boundary crosses SMs, so "
                        "the cross-SM hop figures below are a reference scale only, not a bound")
    for place, hop in hops.items():
        if hop is None:
            continue
        t_lat = (levels - 1) * hop * 1e-9
        out[place] = {"t_hop_ns": round(hop, 1), "bound_us": round(t_lat * 1e6, 2),
                      "frac": round(t_lat / mean_s, 4), "t_over_max_bound": round(mean_s / max(t_bw, t_lat), 3)}
    return out


def hop_placements(cap):
    """One-way hop of the solve's FUSED record protocol between two SMs, placement-controlled:
    every SM pair (0, b) is measured (one CTA per SM, sptrsv_hop_scan) and split into the two
    latency modes (same die / cross die; the B200 has two dies of 74 SMs)."""
    try:
        sms, ns = cap.hop_scan(1500, 1)
    except Exception as e:  # pragma: no cover - diagnostics only
        return {"error": str(e)}
    ns = np.asarray(ns)
    lo, hi = np.percentile(ns, 5), np.percentile(ns, 95)
    thr = 0.5 * (lo + hi)
    near, far = ns[ns <= thr], ns[ns > thr]
    same = float(np.median(near)) if near.size else None
    cross = float(np.median(far)) if far.size and (hi - lo) > 0.08 * lo else None
    return {"same_die": same, "cross_die": cross, "pairs": int(ns.size),
            "split": {"near": int(near.size), "far": int(far.size), "threshold_ns": round(float(thr), 1)},
            "spread_near_p10_p90": [round(float(np.percentile(near, q)), 1) for q in (10, 90)] if near.size else None,
            "spread_far_p10_p90": [round(float(np.percentile(far, q)), 1) for q in (10, 90)] if far.size else None}


# ------------------------------------------------------------------ ncu DRAM traffic (one cold launch per config)

def ncu_child(spec_dir):
    """Child process run under ncu: one solve per saved system, in the order of manifest.json."""
    import torch
    import paper_conf_icpp_suz0hw0w20_b200 as cap
    man = json.load(open(os.path.join(spec_dir, "manifest.json")))
    dev = torch.device("cuda", 0)
    for ent in man:
        arrs = np.load(os.path.join(spec_dir, ent["file"]))
        t = [torch.from_numpy(arrs[k]).to(dev) for k in ("rowptr", "colidx", "val", "b")]
        h = cap.analyse(t[0], t[1], t[2], **ent["opts"])
        x = torch.empty_like(t[3])
        h.solve(t[3], x)
        h.check()
        h.close()


def ncu_traffic(entries, opts, timeout_s=420):
    """dram__bytes_{read,write}.sum of each system's solve launch (cold: ncu --cache-control all),
    measured by re-running this script under ncu.  entries: [(name, CSRSystem)]."""
    ncu = shutil.which("ncu") or ("/usr/local/cuda/bin/ncu" if os.path.exists("/usr/local/cuda/bin/ncu") else None)
    if ncu is None:
        return {}, "ncu not found"
    tmp = tempfile.mkdtemp(prefix="sptrsv_ncu_")
    try:
        man = []
        for k, (name, s) in enumerate(entries):
            f = f"sys{k}.npz"
            np.savez(os.path.join(tmp, f), rowptr=s.rowptr, colidx=s.colidx, val=s.val, b=s.b)
            man.append({"name": name, "file": f, "opts": opts})
        json.dump(man, open(os.path.join(tmp, "manifest.json"), "w"))
        csv = os.path.join(tmp, "ncu.csv")
        cmd = [ncu, "--metrics", "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum",
               "--cache-control", "all", "--clock-control", "none", "-k", "regex:^k_(solve|paper)",
               "--csv", "--log-file", csv, sys.executable, os.path.abspath(__file__), "--ncu-child", tmp]
        r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout_s)
        if r.returncode != 0 or not os.path.exists(csv):
            return {}, f"ncu rc={r.returncode}: {(r.stderr or r.stdout)[-300:]}"
        import csv as _csv
        rows = [row for row in _csv.reader(open(csv)) if len(row) > 5]
        hdr = rows[0]
        iid, iname, imet, ival = (hdr.index("ID"), hdr.index("Kernel Name"), hdr.index("Metric Name"),
                                  hdr.index("Metric Value"))
        per = {}
        for row in rows[1:]:
            if row[iid] == "ID":
                continue
            d = per.setdefault(int(row[iid]), {"kernel": row[iname]})
            d[row[imet]] = float(row[ival].replace(",", ""))
        launches = [per[k] for k in sorted(per)]
        out = {}
        for (name, _), L in zip(entries, launches):
            rd, wr = L.get("dram__bytes_read.sum", 0.0), L.get("dram__bytes_write.sum", 0.0)
            # ncu reports bytes in the unit row; the csv values above are in the unit of the header
            out[name] = {"read": int(rd), "write": int(wr), "total": int(rd + wr), "kernel": L["kernel"],
                         "source": "ncu --cache-control all (cold L2), one launch, measured by bench.py"}
        return out, None
    except Exception as e:  # pragma: no cover - diagnostics only
        return {}, f"ncu failed: {e}"
    finally:
        shutil.rmtree(tmp, ignore_errors=True)


# ------------------------------------------------------------------ N = 1: headline + legs

def run_single(args):
    import torch
    import paper_conf_icpp_suz0hw0w20_b200 as cap

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    opts = {"mode": args.mode, "protocol": 1}
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = int(v)
    if args.config == "c5":
        systems = c5_systems(range(8))
    else:
        systems = [make_system(args.config)]
    handles, bufs = [], []
    for s in systems:
        t = [torch.from_numpy(a).to(dev) for a in (s.rowptr, s.colidx, s.val, s.b)]
        handles.append(cap.analyse(t[0], t[1], t[2], **opts))
        bufs.append((*t, torch.empty_like(t[3])))
    # warm analyse: a second handle on the same (already resident) arrays -- the setup a user
    # pays per matrix once the process and the CUDA context are up (Table 1 analogue)
    warm = []
    for _ in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        h2 = cap.analyse(bufs[0][0], bufs[0][1], bufs[0][2], **opts)
        warm.append((time.perf_counter() - t0) * 1e3)
        h2.close()
    stream = torch.cuda.current_stream(dev)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)  # > 126 MB L2
    peak, peak_src = peaks()

    def step():
        for h, (_, _, _, b, x) in zip(handles, bufs):
            h.solve(b, x, stream=stream)

    sampler = ClockSampler([0]) if not args.profile else None
    if sampler:
        sampler.__enter__()
    step_ms = time_steps(torch, step, stream, flush, args.steps, args.warmup)
    if sampler:
        sampler.__exit__(None, None, None)
    for h in handles:
        h.check(stream)
    tot_s = float(step_ms.sum()) * 1e-3
    mean_s = tot_s / args.steps
    nnz_all = sum(s.nnz for s in systems)
    value = 2.0 * nnz_all * args.steps / tot_s / 1e9
    per_solve_s = mean_s / len(systems)

    def leg(set_opt, key, on, off):
        for h in handles:
            h.set_option(key, off)
        ms = time_steps(torch, step, stream, flush, args.steps, args.warmup)
        for h in handles:
            h.check(stream)
            h.set_option(key, on)
        t = float(ms.sum()) * 1e-3
        return {"value": round(2.0 * nnz_all * args.steps / t / 1e9, 3), "unit": UNIT,
                "ms_per_step": round(t / args.steps * 1e3, 5)}

    legs = {}
    if not args.no_flags_leg and not args.profile:
        if opts.get("protocol", 1) != 0:
            legs["flags_protocol_leg"] = {"protocol": "flags (st.release.gpu / ld.acquire.gpu epoch flags)",
                                          **leg(None, cap.OPT_PROTOCOL, opts.get("protocol", 1), 0)}
        if opts.get("l2_window", 1) != 0:
            legs["no_l2_window_leg"] = {"what": "same solve, no persisting L2 window over the ready words "
                                                "(SPTRSV_OPT_L2_WINDOW=0)",
                                        **leg(None, cap.OPT_L2_WINDOW, 1, 0)}

    # ---- multi-RHS leg
    if args.nrhs > 0 and not args.profile:
        Bs = [torch.from_numpy(np.ascontiguousarray(np.repeat(s.b[:, None], args.nrhs, axis=1)
                                                    * (1.0 + np.arange(args.nrhs)[None, :]))).to(dev)
              for s in systems]
        Xs = [torch.empty_like(B) for B in Bs]

        def mstep():
            for h, B, X in zip(handles, Bs, Xs):
                h.solve_multi(B, X, stream=stream)
        ms = time_steps(torch, mstep, stream, flush, args.steps, args.warmup)
        for h in handles:
            h.check(stream)
        mt = float(ms.sum()) * 1e-3
        legs["multi_rhs_leg"] = {
            "nrhs": args.nrhs, "value": round(2.0 * nnz_all * args.nrhs * args.steps / mt / 1e9, 3), "unit": UNIT,
            "ms_per_step": round(mt / args.steps * 1e3, 5),
            "column0_matches_single_rhs": bool(torch.equal(Xs[0][:, 0], bufs[0][4])),
            "layout": "row-major B[i*nrhs + r], r-th column = (r+1) * b"}
        del Bs, Xs

    # ---- triangular-forms leg: U = P L P (upper), unit lower, unit upper
    if not args.no_tri_leg and not args.profile:
        import synth
        tri = {}
        for name, up, un in (("upper", True, False), ("unit_lower", False, True), ("unit_upper", True, True)):
            ts = [synth.to_unit(synth.to_upper(s) if up else s) if un else (synth.to_upper(s) if up else s)
                  for s in systems]
            th, tb = [], []
            for t in ts:
                a = [torch.from_numpy(np.ascontiguousarray(z)).to(dev) for z in (t.rowptr, t.colidx, t.val, t.b)]
                th.append(cap.analyse(a[0], a[1], a[2], upper=up, unit_diag=un, protocol=opts.get("protocol", 1)))
                tb.append((*a, torch.empty_like(a[3])))

            def tstep():
                for h, (_, _, _, b, x) in zip(th, tb):
                    h.solve(b, x, stream=stream)
            ms = time_steps(torch, tstep, stream, flush, args.steps, args.warmup)
            for h in th:
                h.check(stream)
            tt = float(ms.sum()) * 1e-3
            nnz_t = sum(t.nnz for t in ts)
            err = max(float(np.max(np.abs(x.cpu().numpy() - t.x_true) / np.abs(t.x_true)))
                      for t, (_, _, _, _, x) in zip(ts, tb))
            tri[name] = {"value": round(2.0 * nnz_t * args.steps / tt / 1e9, 3), "unit": UNIT,
                         "ms_per_step": round(tt / args.steps * 1e3, 5), "nnz": int(nnz_t),
                         "engine": ENGINES.get(th[0].info()["engine"]), "max_rel_err_vs_x_true": err}
            for h in th:
                h.close()
            del tb
        legs["triangular_forms_leg"] = tri

    # ---- e2e: through the C-ABI host-buffer call, H2D + solve + D2H inside the timed region
    e2e = None
    if not args.no_e2e and not args.profile:
        hb = [torch.from_numpy(s.b).pin_memory() for s in systems]
        hx = [torch.empty(s.n, dtype=torch.float64).pin_memory() for s in systems]
        for h, b_, x_ in zip(handles, hb, hx):
            h.solve_host(b_, x_, stream=stream)
        torch.cuda.synchronize()
        e_ms = []
        for i in range(args.steps):
            flush.zero_()
            a, bb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            for h, b_, x_ in zip(handles, hb, hx):
                h.solve_host(b_, x_, stream=stream)
            bb.record(stream)
            bb.synchronize()
            e_ms.append(a.elapsed_time(bb))
        torch.cuda.synchronize()
        et = float(np.sum(e_ms)) * 1e-3
        ok = all(np.array_equal(x_.numpy(), x.cpu().numpy()) for x_, (_, _, _, _, x) in zip(hx, bufs))
        e2e = {"value": 2.0 * nnz_all * args.steps / et / 1e9, "unit": UNIT,
               "ms_per_step": round(et / args.steps * 1e3, 5),
               "h2d_bytes_per_step": int(sum(8 * s.n for s in systems)),
               "d2h_bytes_per_step": int(sum(8 * s.n for s in systems)),
               "matches_device_path": bool(ok),
               "note": "pinned host b / x; sptrsv_solve_host overlaps both copies with the solve (DESIGN.md 8)"}

    # ---- every other BASELINE config, same timing rules (N=1 only)
    hops = {"same_die": None, "cross_die": None}
    placement = None
    if not args.profile:
        placement = hop_placements(cap)
        hops = {k: placement.get(k) for k in ("same_die", "cross_die")}
    configs = {}
    ncu_entries = [(args.config if args.config != "c5" else "c5sys", systems[0])]
    if not args.no_configs and not args.profile:
        for name in EXTRA_CONFIGS:
            if name == args.config:
                continue
            s = make_system(name)
            t = [torch.from_numpy(a).to(dev) for a in (s.rowptr, s.colidx, s.val, s.b)]
            h = cap.analyse(t[0], t[1], t[2], **opts)
            x = torch.empty_like(t[3])
            steps = args.steps if name not in ("chain",) else max(3, args.steps // 4)
            ms = time_steps(torch, lambda: h.solve(t[3], x, stream=stream), stream, flush, steps, args.warmup)
            h.check(stream)
            m = float(ms.mean()) * 1e-3
            xt = x.cpu().numpy()
            ref = s.x_true if s.x_true is not None else None
            _, nlev, _ = h.levels(stream)
            inf = h.info()
            configs[name] = {
                "workload": WORKLOADS[name], "n": s.n, "nnz": s.nnz, "steps": steps,
                "value": round(2.0 * s.nnz / m / 1e9, 3), "unit": UNIT, "ms_per_step": round(m * 1e3, 5),
                "engine": ENGINES.get(inf["engine"], str(inf["engine"])), "cta_threads": inf["cta_threads"],
                "rows_per_lane": inf["rows_per_lane"], "analyse_ms": round(inf["analyse_ms"], 3),
                "roofline": roofline(s, m, peak, peak_src, KERNELS.get(inf["engine"], "?")),
                "latency_bound": latency_bound(nlev, hops, m, s.alg_bytes(), peak, inf["engine"]),
                "levels_gpu": int(nlev), "levels_generator": generator_levels(s),
                "max_rel_err_vs_x_true": (float(np.max(np.abs(xt - ref) / np.abs(ref))) if ref is not None
                                          else None)}
            ncu_entries.append((name, s))
            h.close()
            del t, x
            torch.cuda.empty_cache()

    # ---- BASELINE configs[4] at N = 1: the 8 C5 systems back to back on this GPU (the N = 1 point of
    # the C5 strong-scaling leg of the N > 1 lines)
    if not args.no_configs and not args.profile:
        from paper_conf_icpp_suz0hw0w20_b200.batch import MultiDeviceBatch
        c5 = c5_systems(range(8))
        batch = MultiDeviceBatch([(t.rowptr, t.colidx, t.val, t.b) for t in c5], [0], **opts)
        fl = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
        for _ in range(args.warmup):
            batch.timed_solve(lambda g: fl.zero_())
        per = np.array([batch.timed_solve(lambda g: fl.zero_())[0] for _ in range(args.steps)])
        batch.check()
        m = float(per.mean()) * 1e-3
        configs["c5batch"] = {"workload": WORKLOADS["c5"], "systems": 8, "n_per_system": c5[0].n,
                              "value": round(2.0 * sum(t.nnz for t in c5) / m / 1e9, 3), "unit": UNIT,
                              "ms_per_step": round(m * 1e3, 5), "steps": args.steps,
                              "engine": ENGINES.get(batch.handles[0].info()["engine"]),
                              "timing": "one step = the 8 solves back to back on one stream (CUDA events)"}
        batch.close()
        # the same 8 systems as block-diagonal BATCH handles (sptrsv_analyse_csr_batch): one launch per
        # group of g systems -- 8 x 1 (= the leg above, through one handle each), 4 x 2, 1 x 8
        stream = torch.cuda.current_stream()
        grouped = {}
        dsys = [tuple(torch.from_numpy(a).to(dev) for a in (t.rowptr, t.colidx, t.val)) for t in c5]
        for g in (2, 8):
            hs = [cap.analyse_batch(dsys[k:k + g], **opts) for k in range(0, 8, g)]
            bs = [torch.from_numpy(np.concatenate([t.b for t in c5[k:k + g]])).to(dev) for k in range(0, 8, g)]
            xs = [torch.empty_like(b) for b in bs]
            ms = time_steps(torch, lambda: [h.solve(b, x, stream=stream) for h, b, x in zip(hs, bs, xs)], stream,
                            fl, args.steps, args.warmup)
            for h in hs:
                h.check(stream)
            mg = float(ms.mean()) * 1e-3
            grouped[f"{g}_per_launch"] = {"launches": len(hs), "value": round(2.0 * sum(t.nnz for t in c5) / mg / 1e9, 3),
                                          "ms_per_step": round(mg * 1e3, 5),
                                          "engine": ENGINES.get(hs[0].info()["engine"])}
            for h in hs:
                h.close()
            del hs, bs, xs
        configs["c5batch"]["one_launch_groups"] = grouped
        del c5, fl, dsys
        torch.cuda.empty_cache()

    # ---- roofline of the headline kernel (mean step), latency bound, ncu-measured DRAM traffic
    traffic, ncu_err = ({}, "skipped")
    if not args.no_ncu and not args.profile:
        del flush
        torch.cuda.empty_cache()
        traffic, ncu_err = ncu_traffic(ncu_entries, opts)
    head = args.config if args.config != "c5" else "c5sys"
    info = handles[0].info()
    roof = roofline(systems[0], per_solve_s, peak, peak_src, KERNELS.get(info["engine"], "?"), traffic.get(head))
    for name, c in configs.items():
        tr = traffic.get(name)
        if tr:
            c["roofline"].update({"traffic": tr["total"], "traffic_read": tr["read"], "traffic_write": tr["write"],
                                  "traffic_source": tr["source"]})
    lat = None
    if not args.profile:
        _, nlev, _ = handles[0].levels(stream)
        lat = latency_bound(nlev, hops, per_solve_s, systems[0].alg_bytes(), peak)
        lat["levels_generator"] = generator_levels(systems[0])

    cpu = None
    if not args.no_cpu_baseline and not args.profile:
        cpu = cpu_baseline(systems[0], args.cpu_seconds)

    line = {
        "metric": METRIC, "value": round(value, 3), "unit": UNIT, "n_gpus": 1,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(mean_s * 1e3, 5),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{args.config}: {WORKLOADS[args.config]}",
                   "n": systems[0].n, "nnz": systems[0].nnz, "systems": len(systems),
                   "mode": {0: "auto", 1: "thread", 2: "warp"}[args.mode],
                   "plan": {"thread_groups": info["n_thread_groups"], "warp_rows": info["n_warp_rows"]},
                   "engine": ENGINES.get(info["engine"], str(info["engine"])),
                   "cta_threads": info["cta_threads"], "rows_per_lane": info["rows_per_lane"],
                   "analyse_ms_cold": round(info["analyse_ms"], 3),
                   "analyse_ms_warm": round(float(np.median(warm)), 3),
                   "l2": "flushed between timed steps (256 MiB write, outside the per-step events): CSR, b and x "
                         "are read / written cold; the solver's ready words (16-B records per row) sit in a "
                         "persisting L2 access-policy window (north_star) -- see no_l2_window_leg",
                   "parallelism": "1 GPU", "options": opts},
        "protocol": {1: "fused (epoch-tagged 16-byte value records, no fences)",
                     0: "flags (st.release.gpu / ld.acquire.gpu)"}[opts.get("protocol", 1)],
        **legs,
        "roofline": roof,
        "latency_bound": lat,
        "hop_placement": placement,
        "configs": configs or None,
        "ncu": ncu_err,
        "e2e": e2e,
        "gpu_launches": args.steps * len(systems),
        "cpu_baseline": cpu,
        "clocks": sampler.summary() if sampler else None,
    }
    print(json.dumps(line), flush=True)
    for h in handles:
        h.close()


# ------------------------------------------------------------------ N > 1: batches over devices / ranks

class CudaEnv:
    """What run_batch needs from the machine: devices, the batch runner, L2 flushes, pinned host
    buffers, clock sampling.  (tests/test_multiproc.py swaps in a CPU stand-in to run the same
    rank / shard / max-over-ranks path under gloo without a GPU.)"""

    def __init__(self):
        import torch
        self.torch = torch

    def devices(self, args, rank, world):
        ndev = self.torch.cuda.device_count()
        if world > 1:
            local = int(os.environ.get("LOCAL_RANK", "0"))
            if local >= ndev:
                raise SystemExit(f"bench.py: rank {rank} needs GPU {local} but only {ndev} visible")
            return [local]
        if args.gpus > ndev:
            raise SystemExit(f"bench.py --gpus {args.gpus}: only {ndev} CUDA device(s) visible")
        return list(range(args.gpus))

    def make_batch(self, systems, devices, opts):
        from paper_conf_icpp_suz0hw0w20_b200.batch import MultiDeviceBatch
        return MultiDeviceBatch([(s.rowptr, s.colidx, s.val, s.b) for s in systems], devices, **opts)

    def make_flush(self, batch):
        torch = self.torch
        bufs = []
        for d in batch.devices:
            with torch.cuda.device(d):
                bufs.append(torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=d))
        return lambda g: bufs[g].zero_()

    def host_buffers(self, systems):
        torch = self.torch
        return ([torch.from_numpy(s.b).pin_memory() for s in systems],
                [torch.empty(s.n, dtype=torch.float64).pin_memory() for s in systems])

    @staticmethod
    def numpy(t):
        return t.cpu().numpy()

    def clocks(self, devices):
        return ClockSampler(devices)


def _measure_batch(args, env, systems, devices, opts, dist, e2e=True):
    """One workload through MultiDeviceBatch: warm-up, K timed steps (per-device CUDA events, step =
    max over devices, L2 flushed before each step outside the events), max / sum over ranks, and the
    end-to-end leg.  Every collective runs on every rank."""
    from paper_conf_icpp_suz0hw0w20_b200.batch import max_over_ranks, sum_over_ranks

    batch = env.make_batch(systems, devices, opts)
    flush = env.make_flush(batch)
    for _ in range(args.warmup):
        batch.timed_solve(flush)
    batch.check()
    if dist is not None:
        dist.barrier()
    batch.synchronize()
    per_dev = np.array([batch.timed_solve(flush) for _ in range(args.steps)])  # [steps, devices] ms
    batch.synchronize()
    if dist is not None:
        dist.barrier()
    batch.check()
    step_ms = per_dev.max(axis=1)  # a step ends when the last device is done
    tot_s = max_over_ranks(float(step_ms.sum()) * 1e-3, dist)
    nnz_all = sum_over_ranks(float(sum(s.nnz for s in systems)), dist)
    out = {"value": 2.0 * nnz_all * args.steps / tot_s / 1e9, "tot_s": tot_s, "per_dev": per_dev,
           "launches": int(sum_over_ranks(float(args.steps * len(systems)), dist)),
           "systems_total": int(sum_over_ranks(float(len(systems)), dist)),
           "info": batch.handles[0].info()}
    if e2e:  # pinned host b -> device -> solve -> host x, every step, through the public API
        hb, hx = env.host_buffers(systems)
        batch.solve_host(hb, hx)
        if dist is not None:
            dist.barrier()
        e_t = []
        for _ in range(args.steps):
            t0 = time.perf_counter()
            batch.solve_host(hb, hx)
            e_t.append(time.perf_counter() - t0)
        et = max_over_ranks(float(np.sum(e_t)), dist)
        ok = all(np.array_equal(env.numpy(hx[k]), env.numpy(batch.x(k))) for k in range(len(systems)))
        ok = sum_over_ranks(0.0 if ok else 1.0, dist) == 0.0
        h2d = int(sum_over_ranks(float(sum(8 * s.n for s in systems)), dist))
        out["e2e"] = {"value": 2.0 * nnz_all * args.steps / et / 1e9, "unit": UNIT,
                      "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": h2d, "matches_device_path": bool(ok),
                      "timing": "host wall clock per step around sptrsv_solve_host of every owned system (one host "
                                "thread per device), max over ranks"}
    batch.close()
    return out


def run_batch(args, rank, world, dist=None, env=None):
    """N > 1 (or --config c5): independent systems over N GPUs.  world > 1: this process is one rank of
    torchrun and drives GPU LOCAL_RANK; world == 1: this process drives args.gpus devices.
    The line's `value` is WEAK scaling of the headline config (every GPU solves its own c2-shaped
    system, seed + GPU), comparable with the N = 1 line; `c5_batch_leg` is BASELINE configs[4]: the 8
    fixed C5 systems, s -> GPU s mod N (strong scaling).  `--config c5` makes C5 the value."""
    from paper_conf_icpp_suz0hw0w20_b200.batch import shard

    env = env or CudaEnv()
    devices = env.devices(args, rank, world)
    n_gpus = args.gpus if world == 1 else world
    opts = {"mode": args.mode, "protocol": 1}
    for kv in args.opt:
        k, v = kv.split("=")
        opts[k] = int(v)
    c5 = c5_systems(shard(8, rank, world))  # ranks own systems s = rank (mod world); devices split them further
    if args.config == "c5":
        main_sys, scaling = c5, "strong"
    else:
        main_sys = [make_system(args.config, rank * len(devices) + k) for k in range(len(devices))]
        scaling = "weak"
    sampler = env.clocks(devices)
    sampler.__enter__()
    m = _measure_batch(args, env, main_sys, devices, opts, dist)
    sampler.__exit__(None, None, None)
    leg = None
    if args.config != "c5" and not args.no_c5_leg:
        c = _measure_batch(args, env, c5, devices, opts, dist, e2e=False)
        leg = {"workload": f"c5: {WORKLOADS['c5']}", "value": round(c["value"], 3), "unit": UNIT,
               "ms_per_step": round(c["tot_s"] / args.steps * 1e3, 5), "scaling": "strong",
               "systems_total": c["systems_total"], "gpu_launches": c["launches"],
               "per_device_ms_mean": [round(float(v), 5) for v in c["per_dev"].mean(axis=0)]}
    info = m["info"]
    if rank == 0:
        line = {
            "metric": METRIC, "value": round(m["value"], 3), "unit": UNIT, "n_gpus": n_gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(m["tot_s"] / args.steps * 1e3, 5),
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": f"{args.config}: {WORKLOADS[args.config]}"
                       + ("" if args.config == "c5" else f" -- one per GPU (seed + GPU), weak scaling"),
                       "systems_total": m["systems_total"],
                       "n_per_system": main_sys[0].n, "nnz_per_system": main_sys[0].nnz,
                       "engine": ENGINES.get(info["engine"], str(info["engine"])),
                       "parallelism": (f"{n_gpus} GPUs, system s on GPU s mod {n_gpus}, one stream per device, "
                                       "no inter-GPU exchange (no NCCL)") + (
                           "; torchrun ranks, gloo control plane" if world > 1 else "; one host process"),
                       "timing": "per-device CUDA events around each device's solves on its stream; step = max over "
                                 "devices; L2 flushed before every step outside the events",
                       "options": opts},
            "per_device_ms_mean": [round(float(v), 5) for v in m["per_dev"].mean(axis=0)],
            "c5_batch_leg": leg,
            "e2e": m["e2e"],
            "gpu_launches": m["launches"],
            "cpu_baseline": None,
            "clocks": sampler.summary(),
        }
        print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.ncu_child:
        ncu_child(args.ncu_child)
        return
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo")  # control plane only (barrier, max / sum over ranks)
        try:
            run_batch(args, rank, world, dist)
        finally:
            dist.destroy_process_group()
        return
    if args.gpus > 1 or args.config == "c5":
        run_batch(args, 0, 1)
        return
    run_single(args)


if __name__ == "__main__":
    main()
