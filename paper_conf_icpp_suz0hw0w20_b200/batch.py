"""Batches of independent systems over 1..G GPUs.

A single solve does not shard: its dependency DAG crosses every row partition, and a cross-GPU
ready flag would put an NVLink round trip (~1.8k cycles) on a latency-bound critical path.  What
does spread over GPUs is a BATCH of independent systems: system s -> device s mod G, each device
solving its systems back to back on its own stream.  No data is exchanged, so there is no
collective and no NCCL on the data path.

Two launch shapes use the same sharding:
  * one host process driving G devices (``MultiDeviceBatch``: one stream per device, per-device
    CUDA events, the timed region's length = max over devices);
  * one process per GPU under torchrun (``bench.py``), where each rank builds a
    ``MultiDeviceBatch`` over its own device and the max over ranks goes through a CPU (gloo)
    all-reduce -- control plane only.
"""
from __future__ import annotations

from concurrent.futures import ThreadPoolExecutor


def shard(n_systems: int, rank: int, world: int) -> list[int]:
    """Systems owned by `rank`: s with s % world == rank (round-robin, deterministic)."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank/world")
    return [s for s in range(n_systems) if s % world == rank]


def replica_seed(base_seed: int, rank: int) -> int:
    """Weak scaling: every rank solves its own system of the same shape, seed base + rank."""
    return base_seed + rank


def max_over_ranks(value: float, dist=None) -> float:
    """The timed region's length is the max over ranks (never a wall clock).  `dist` must have a
    CPU-capable (gloo) process group: the reduction is control plane, not data path."""
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def sum_over_ranks(value: float, dist=None) -> float:
    if dist is None or not dist.is_initialized() or dist.get_world_size() == 1:
        return float(value)
    import torch
    t = torch.tensor([float(value)], dtype=torch.float64)
    dist.all_reduce(t)
    return float(t.item())


class MultiDeviceBatch:
    """Independent systems L_s x_s = b_s spread over devices: system s -> devices[s % G].

    ``systems``: sequence of (rowptr, colidx, val, b) host arrays (int32 / int32 / float64 /
    float64, the C ABI's CSR).  Every system is uploaded to and analysed on its device
    (``sptrsv_analyse_csr``); ``solve()`` enqueues every system's solve on its device's stream
    (asynchronous: the host issues all devices before any finishes).  ``options`` are handle
    options for every system (see ``analyse``).
    """

    def __init__(self, systems, devices, **options):
        import torch

        from . import analyse
        if not devices:
            raise ValueError("no devices")
        ndev = torch.cuda.device_count()
        bad = [d for d in devices if not 0 <= int(d) < ndev]
        if bad:
            raise RuntimeError(f"MultiDeviceBatch: devices {bad} requested but only {ndev} CUDA device(s) visible")
        self.devices = [torch.device("cuda", int(d)) for d in devices]
        self.owner = [s % len(self.devices) for s in range(len(systems))]
        self.streams = [torch.cuda.Stream(device=d) for d in self.devices]
        self.nnz = [int(s[0][-1]) for s in systems]
        self.n = [int(len(s[0]) - 1) for s in systems]
        self.handles, self.bufs = [], []
        for (rp, ci, v, b), g in zip(systems, self.owner):
            dev = self.devices[g]
            with torch.cuda.device(dev):
                t = [torch.as_tensor(a).to(dev) for a in (rp, ci, v, b)]
                self.handles.append(analyse(t[0], t[1], t[2], **options))
                self.bufs.append((*t, torch.empty_like(t[3])))
            torch.cuda.synchronize(dev)

    def systems_on(self, g: int) -> list[int]:
        return [s for s, o in enumerate(self.owner) if o == g]

    def solve(self) -> None:
        """One batch: every device solves its systems back to back on its stream (async)."""
        for g in range(len(self.devices)):
            st = self.streams[g]
            for s in self.systems_on(g):
                _, _, _, b, x = self.bufs[s]
                self.handles[s].solve(b, x, stream=st)

    def timed_solve(self, before=None) -> list[float]:
        """One batch with CUDA events around each device's work on its own stream; returns the
        per-device milliseconds (after synchronising every device).  `before(g)` runs on device
        g's stream ahead of its start event (e.g. an L2 flush), outside the timed span."""
        import torch
        evs = []
        for g, dev in enumerate(self.devices):
            st = self.streams[g]
            with torch.cuda.device(dev), torch.cuda.stream(st):
                if before is not None:
                    before(g)
                a, b_ = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(st)
                for s in self.systems_on(g):
                    _, _, _, b, x = self.bufs[s]
                    self.handles[s].solve(b, x, stream=st)
                b_.record(st)
                evs.append((a, b_))
        for a, b_ in evs:
            b_.synchronize()
        return [a.elapsed_time(b_) for a, b_ in evs]

    def solve_host(self, b_host, x_host) -> None:
        """End to end from host buffers (``sptrsv_solve_host`` per system; pinned host tensors
        overlap the copies with the solve).  One host thread per device so that devices overlap."""
        def run(g):
            for s in self.systems_on(g):
                self.handles[s].solve_host(b_host[s], x_host[s], stream=self.streams[g])
        with ThreadPoolExecutor(max_workers=len(self.devices)) as ex:
            list(ex.map(run, range(len(self.devices))))

    def synchronize(self) -> None:
        import torch
        for d in self.devices:
            torch.cuda.synchronize(d)

    def check(self) -> None:
        for h, g in zip(self.handles, self.owner):
            h.check(self.streams[g])

    def x(self, s: int):
        return self.bufs[s][4]

    def close(self) -> None:
        for h in self.handles:
            h.close()
        self.handles = []
