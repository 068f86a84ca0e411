"""B200-native CapelliniSpTRSV: synchronization-free fp64 sparse lower-triangular solve.

Thin Python layer over the C ABI in ``include/sptrsv.h`` (``libsptrsv.so``).
PyTorch supplies device memory and streams only; every step of the solve is a
hand-written sm_100a kernel.  Paper: Su et al., ICPP '20.

    import torch, paper_conf_icpp_suz0hw0w20_b200 as cap
    L = cap.analyse(rowptr, colidx, val)      # torch CUDA tensors, int32/int32/float64
    L.solve(b, x)                             # async on the current stream
"""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import (MODE_AUTO, MODE_THREAD, MODE_WARP, OPT_BACKOFF_MAX_NS, OPT_BACKOFF_MIN_NS,
                   OPT_CTA_THREADS, OPT_L2_WINDOW, OPT_LOCAL, OPT_MODE, OPT_PROTOCOL, OPT_SPIN_LIMIT,
                   OPT_STAGE_SMEM, OPT_WARP_THRESHOLD, PROTO_FLAGS, PROTO_FUSED, SptrsvError, check)

__all__ = ["analyse", "analyse_batch", "Handle", "SptrsvError", "flag_latency", "hop_scan", "MODE_AUTO", "MODE_THREAD",
           "MODE_WARP", "PROTO_FLAGS", "PROTO_FUSED", "lib"]

lib = _lib.lib


def _stream_ptr(stream, device=None) -> int | None:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream(device)
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _need(t, dtype, n, name, device=None):
    import torch
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor")
    if device is not None and t.device != device:
        raise ValueError(f"{name} is on {t.device}, the handle on {device}")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if n is not None and t.numel() != n:
        raise ValueError(f"{name} must have {n} elements, got {t.numel()}")


class Handle:
    """An analysed matrix (``sptrsv_analyse_csr`` / ``sptrsv_analyse_csr_ex``).  Keeps the CSR
    tensors alive.  ``upper`` / ``unit_diag`` select the f4 triangular forms (include/sptrsv.h)."""

    def __init__(self, rowptr, colidx, val, upper=False, unit_diag=False):
        import torch
        _need(rowptr, torch.int32, None, "rowptr")
        n = rowptr.numel() - 1
        if n < 0:
            raise ValueError("rowptr must have n+1 >= 1 entries")
        _need(colidx, torch.int32, None, "colidx")
        _need(val, torch.float64, colidx.numel(), "val")
        if not (rowptr.device == colidx.device == val.device):
            raise ValueError("CSR tensors must live on one device")
        self.device = rowptr.device
        self.n = n
        self._keep = (rowptr, colidx, val)
        self._h = ctypes.c_void_p()
        self.tri = (_lib.TRI_UPPER if upper else 0) | (_lib.TRI_UNIT_DIAG if unit_diag else 0)
        with torch.cuda.device(self.device):
            torch.cuda.current_stream().synchronize()  # analyse runs on the legacy default stream
            check(lib.sptrsv_analyse_csr_ex(n, rowptr.data_ptr(), colidx.data_ptr() if colidx.numel() else None,
                                            val.data_ptr() if val.numel() else None, self.tri,
                                            ctypes.byref(self._h)),
                  "sptrsv_analyse_csr_ex")

    @classmethod
    def batch(cls, systems, upper=False, unit_diag=False):
        """``sptrsv_analyse_csr_batch``: independent systems [(rowptr, colidx, val), ...] on one device as
        ONE block-diagonal handle (the library owns the concatenation); solve / solve_host then take
        the concatenated b / x (system s at rows offsets[s] .. offsets[s + 1])."""
        import numpy as np
        import torch
        if not systems:
            raise ValueError("no systems")
        dev = systems[0][0].device
        ns = []
        for rp, ci, v in systems:
            _need(rp, torch.int32, None, "rowptr", dev)
            _need(ci, torch.int32, None, "colidx", dev)
            _need(v, torch.float64, ci.numel(), "val", dev)
            ns.append(rp.numel() - 1)
        self = cls.__new__(cls)
        self.device = dev
        self.n = int(sum(ns))
        self.offsets = np.concatenate([[0], np.cumsum(ns)]).astype(np.int64)
        self._keep = tuple(systems)
        self._h = ctypes.c_void_p()
        self.tri = (_lib.TRI_UPPER if upper else 0) | (_lib.TRI_UNIT_DIAG if unit_diag else 0)
        k = len(systems)
        n_arr = (ctypes.c_int32 * k)(*ns)
        rp_arr = (ctypes.c_void_p * k)(*[rp.data_ptr() for rp, _, _ in systems])
        ci_arr = (ctypes.c_void_p * k)(*[ci.data_ptr() if ci.numel() else None for _, ci, _ in systems])
        v_arr = (ctypes.c_void_p * k)(*[v.data_ptr() if v.numel() else None for _, _, v in systems])
        with torch.cuda.device(dev):
            torch.cuda.current_stream().synchronize()
            check(lib.sptrsv_analyse_csr_batch(k, ctypes.addressof(n_arr), ctypes.addressof(rp_arr),
                                               ctypes.addressof(ci_arr), ctypes.addressof(v_arr), self.tri,
                                               ctypes.byref(self._h)), "sptrsv_analyse_csr_batch")
        return self

    # -- solve -------------------------------------------------------------------------
    def solve(self, b, x=None, stream=None):
        """x <- L^{-1} b (fp64, device tensors), enqueued on ``stream`` (default: current)."""
        import torch
        _need(b, torch.float64, self.n, "b", self.device)
        if x is None:
            x = torch.empty_like(b)
        _need(x, torch.float64, self.n, "x", self.device)
        if self.n:
            with torch.cuda.device(self.device):
                check(lib.sptrsv_solve(self._h, b.data_ptr(), x.data_ptr(), _stream_ptr(stream, self.device)), "sptrsv_solve")
        return x

    def solve_multi(self, B, X=None, stream=None):
        """X <- L^{-1} B for B of shape (n, nrhs) (row-major rows, nrhs <= 32), one launch."""
        import torch
        if not isinstance(B, torch.Tensor) or not B.is_cuda or B.dtype != torch.float64 or B.dim() != 2:
            raise TypeError("B must be a 2-D float64 CUDA tensor")
        if B.shape[0] != self.n or B.stride(1) != 1:
            raise ValueError("B must be (n, nrhs) with unit column stride")
        if B.device != self.device:
            raise ValueError(f"B is on {B.device}, the handle on {self.device}")
        nrhs = B.shape[1]
        if X is None:
            X = torch.empty_like(B)
        if X.shape != B.shape or X.stride(1) != 1 or X.dtype != torch.float64 or X.device != B.device:
            raise ValueError("X must match B")
        if self.n and nrhs:
            with torch.cuda.device(self.device):
                check(lib.sptrsv_solve_multi(self._h, B.data_ptr(), X.data_ptr(), nrhs, B.stride(0), X.stride(0),
                                             _stream_ptr(stream, self.device)), "sptrsv_solve_multi")
        return X

    def solve_host(self, b_host, x_host, stream=None):
        """End to end from host buffers (numpy float64 or pinned CPU tensors); synchronous."""
        import numpy as np
        import torch

        def ptr(a):
            if isinstance(a, np.ndarray):
                assert a.dtype == np.float64 and a.flags.c_contiguous and a.size == self.n
                return a.ctypes.data
            assert isinstance(a, torch.Tensor) and a.device.type == "cpu" and a.dtype == torch.float64
            assert a.is_contiguous() and a.numel() == self.n
            return a.data_ptr()
        with torch.cuda.device(self.device):
            check(lib.sptrsv_solve_host(self._h, ptr(b_host), ptr(x_host), _stream_ptr(stream, self.device)),
                  "sptrsv_solve_host")
        return x_host

    def check(self, stream=None):
        """Synchronise and raise SptrsvError(ERR_TIMEOUT) if the watchdog fired."""
        check(lib.sptrsv_check(self._h, _stream_ptr(stream, self.device)), "sptrsv_check")

    # -- diagnostics ---------------------------------------------------------------------
    def indegree(self, stream=None):
        import torch
        out = torch.empty(self.n, dtype=torch.int32, device=self.device)
        check(lib.sptrsv_get_indegree(self._h, out.data_ptr() if self.n else None, _stream_ptr(stream, self.device)),
              "sptrsv_get_indegree")
        return out

    def levels(self, stream=None):
        """(level[n] int32, nlevels, counts[nlevels] int32) computed on the GPU."""
        import torch
        lv = torch.empty(self.n, dtype=torch.int32, device=self.device)
        counts = torch.empty(self.n, dtype=torch.int32, device=self.device)
        nl = ctypes.c_int32(0)
        if self.n:
            check(lib.sptrsv_levels(self._h, lv.data_ptr(), counts.data_ptr(), ctypes.byref(nl),
                                    _stream_ptr(stream, self.device)), "sptrsv_levels")
        return lv, int(nl.value), counts[: nl.value]

    def trace(self, b, x=None, stream=None):
        """Diagnostic solve: (x, trace) with trace[:n] = publish time (ns, %globaltimer) of each
        x_i, trace[n:2n] = when (thread-level) row i consumed its last dependency (0 = none) and
        trace[2n:3n] = when its solve loop started (0 = not recorded), trace[3n:3n+3] = kernel
        first entry / last exit / CTAs started, trace[3n+3:4n+3] = when row i's CTA entered (LEAN)."""
        import torch
        tr = torch.zeros(4 * self.n + 3, dtype=torch.int64, device=self.device)
        tr[3 * self.n] = (1 << 63) - 1
        check(lib.sptrsv_set_trace(self._h, tr.data_ptr()), "sptrsv_set_trace")
        try:
            x = self.solve(b, x, stream)
            self.check(stream)
        finally:
            check(lib.sptrsv_set_trace(self._h, None), "sptrsv_set_trace")
        return x, tr

    def info(self) -> dict:
        inf = _lib.sptrsv_info()
        check(lib.sptrsv_get_info(self._h, ctypes.byref(inf)), "sptrsv_get_info")
        return {f: getattr(inf, f) for f, _ in inf._fields_}

    def set_option(self, key: int, value: int) -> None:
        check(lib.sptrsv_set_option(self._h, key, int(value)), "sptrsv_set_option")

    def get_option(self, key: int) -> int:
        v = ctypes.c_int64(0)
        check(lib.sptrsv_get_option(self._h, key, ctypes.byref(v)), "sptrsv_get_option")
        return int(v.value)

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib.sptrsv_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def analyse(rowptr, colidx, val, upper=False, unit_diag=False, **options) -> Handle:
    """``sptrsv_analyse_csr[_ex]`` + options (mode=, warp_threshold=, cta_threads=, ...)."""
    h = Handle(rowptr, colidx, val, upper=upper, unit_diag=unit_diag)
    for k, v in options.items():
        h.set_option(_OPTION_KEYS[k], v)
    return h


_OPTION_KEYS = {"mode": OPT_MODE, "warp_threshold": OPT_WARP_THRESHOLD, "cta_threads": OPT_CTA_THREADS,
            "backoff_min_ns": OPT_BACKOFF_MIN_NS, "backoff_max_ns": OPT_BACKOFF_MAX_NS,
            "spin_limit": OPT_SPIN_LIMIT, "l2_window": OPT_L2_WINDOW, "stage_smem": OPT_STAGE_SMEM,
            "protocol": OPT_PROTOCOL, "local": OPT_LOCAL, "engine": _lib.OPT_ENGINE,
            "rows_per_lane": _lib.OPT_ROWS_PER_LANE,
            "variant": _lib.OPT_VARIANT, "lean_occupancy": _lib.OPT_LEAN_OCCUPANCY,
            "poll_gap_ns": _lib.OPT_POLL_GAP_NS,
            "poll_one": _lib.OPT_POLL_ONE,
            "warp_split_last": _lib.OPT_WARP_SPLIT_LAST,
            "host_io": _lib.OPT_HOST_IO, "subwarp": _lib.OPT_SUBWARP, "chain_div": _lib.OPT_CHAIN_DIV}


def analyse_batch(systems, upper=False, unit_diag=False, **options) -> Handle:
    """``sptrsv_analyse_csr_batch`` + options: independent systems as one block-diagonal handle."""
    h = Handle.batch(systems, upper=upper, unit_diag=unit_diag)
    for k, v in options.items():
        h.set_option(_OPTION_KEYS[k], v)
    return h


def hop_scan(iters: int = 4000, protocol: int = 1, capacity: int = 512):
    """Placement-controlled one-way hop (ns) from the lowest-id SM to every other SM of the current
    device (``sptrsv_hop_scan``): returns (partner SM ids, ns per hop) as numpy arrays."""
    import numpy as np
    sm_b = np.zeros(capacity, dtype=np.int32)
    ns = np.zeros(capacity, dtype=np.float64)
    a, cnt = ctypes.c_int32(0), ctypes.c_int32(0)
    check(lib.sptrsv_hop_scan(iters, protocol, capacity, ctypes.byref(a), sm_b.ctypes.data, ns.ctypes.data,
                              ctypes.byref(cnt)), "sptrsv_hop_scan")
    return sm_b[: cnt.value], ns[: cnt.value]


def flag_latency(iters: int = 20000, protocol: int = 0, with_clock: bool = False):
    """Mean one-way flag hop (ns) between two CTAs on the current device (sptrsv_flag_latency).
    protocol 0 = the solve's release/acquire pair; see include/sptrsv.h for 1-4."""
    v, mhz = ctypes.c_double(0.0), ctypes.c_double(0.0)
    check(lib.sptrsv_flag_latency(iters, protocol, ctypes.byref(v), ctypes.byref(mhz)), "sptrsv_flag_latency")
    return (float(v.value), float(mhz.value)) if with_clock else float(v.value)
