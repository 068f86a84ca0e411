"""N>1 host logic on CPU: world_size-2 gloo processes (the GPU box has one GPU)."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _load_batch():
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "_batch", os.path.join(ROOT, "paper_conf_icpp_suz0hw0w20_b200", "batch.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def _worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    b = _load_batch()
    mine = b.shard(8, rank, world)
    # every rank reports its shard; times are rank-dependent so max/sum are checkable
    t = b.max_over_ranks(1.0 + rank, dist)
    tot = b.sum_over_ranks(len(mine), dist)
    dist.barrier()
    q.put((rank, mine, t, tot, b.replica_seed(2, rank)))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharding_and_max_over_ranks_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    out.sort()
    shards = [o[1] for o in out]
    assert sorted(s for sh in shards for s in sh) == list(range(8))  # each system exactly once
    assert all(o[2] == float(world) for o in out)                    # max over ranks
    assert all(o[3] == 8.0 for o in out)                             # all systems accounted
    assert len({o[4] for o in out}) == world                         # distinct replica seeds


def test_shard_single_rank_and_errors():
    b = _load_batch()
    assert b.shard(8, 0, 1) == list(range(8))
    assert b.shard(8, 7, 8) == [7]
    with pytest.raises(ValueError):
        b.shard(8, 2, 2)


# ------------------------------------------------------------------ the bench's own N>1 rank path

class _CpuBatch:
    """CPU stand-in for MultiDeviceBatch with the same interface: every 'device' solves its systems
    with the oracle (wall clock as its event span) -- so bench.run_batch's rank / shard / timing /
    max-over-ranks path runs under gloo without a GPU."""

    def __init__(self, systems, devices):
        import oracle
        self.oracle = oracle
        self.systems = systems
        self.devices = devices
        self.owner = [s % len(devices) for s in range(len(systems))]
        self.xs = [np.zeros(s.n) for s in systems]
        self.solved = 0

    class _H:
        @staticmethod
        def info():
            return {"engine": 3}

    @property
    def handles(self):
        return [self._H()]

    def timed_solve(self, before=None):
        ms = []
        for g in range(len(self.devices)):
            if before:
                before(g)
            t0 = time.perf_counter()
            for s, o in enumerate(self.owner):
                if o == g:
                    sy = self.systems[s]
                    self.xs[s] = self.oracle.solve(sy.rowptr, sy.colidx, sy.val, sy.b)
                    self.solved += 1
            ms.append((time.perf_counter() - t0) * 1e3)
        return ms

    def solve_host(self, hb, hx):
        for s, sy in enumerate(self.systems):
            hx[s][:] = self.oracle.solve(sy.rowptr, sy.colidx, sy.val, hb[s])

    def synchronize(self):
        pass

    def check(self):
        pass

    def x(self, s):
        return self.xs[s]

    def close(self):
        pass


class _CpuEnv:
    def devices(self, args, rank, world):
        return [0] if world > 1 else list(range(args.gpus))

    def make_batch(self, systems, devices, opts):
        return _CpuBatch(systems, devices)

    def make_flush(self, batch):
        return lambda g: None

    def host_buffers(self, systems):
        return [s.b.copy() for s in systems], [np.zeros(s.n) for s in systems]

    @staticmethod
    def numpy(t):
        return t

    def clocks(self, devices):
        class _S:
            def __enter__(self):
                return self

            def __exit__(self, *a):
                pass

            def summary(self):
                return {"sm_mhz": None, "reasons": ["cpu stand-in"]}
        return _S()


def _bench_worker(rank, world, port, q, config):
    import contextlib
    import io
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update({"RANK": str(rank), "WORLD_SIZE": str(world), "LOCAL_RANK": "0"})
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    import bench
    args = bench.parse(["--gpus", str(world), "--steps", "2", "--warmup", "1", "--config", config, "--no-c5-leg"])
    env = _CpuEnv()
    out = io.StringIO()
    with contextlib.redirect_stdout(out):
        bench.run_batch(args, rank, world, dist, env=env)
    dist.destroy_process_group()
    q.put((rank, out.getvalue()))


import time  # noqa: E402

import numpy as np  # noqa: E402


@pytest.mark.parametrize("world", [2, 3])
def test_bench_rank_path_gloo(world):
    """bench.py's N>1 path itself (run_batch, as torchrun launches it), with a CPU stand-in for the
    device batch: the C5 systems are sharded s -> rank s mod N (each exactly once), only rank 0
    prints, the line reports n_gpus = N, all 8 systems' launches, and a value equal to
    (8 systems' 2*nnz * steps) / (max over ranks of the summed step times)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_worker, args=(r, world, port, q, "c5")) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import json
    assert all(not out[r].strip() for r in range(1, world))  # only rank 0 prints
    line = json.loads(out[0].strip().splitlines()[-1])
    assert line["n_gpus"] == world and line["scaling"] == "strong"
    assert line["gpu_launches"] == 8 * 2 and line["config"]["systems_total"] == 8
    assert line["e2e"]["matches_device_path"] is True
    assert line["e2e"]["h2d_bytes_per_step"] == 8 * 8 * 2_000_000
    nnz = 8 * 5_600_000
    assert abs(line["value"] - 2.0 * nnz * 2 / (line["ms_per_step"] * 2 * 1e-3) / 1e9) <= 1e-3 * line["value"]


def _bench_worker_weak(rank, world, port, q):
    import contextlib
    import io
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update({"RANK": str(rank), "WORLD_SIZE": str(world), "LOCAL_RANK": "0"})
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    import bench
    args = bench.parse(["--gpus", str(world), "--steps", "2", "--warmup", "1"])
    out = io.StringIO()
    with contextlib.redirect_stdout(out):
        bench.run_batch(args, rank, world, dist, env=_CpuEnv())
    dist.destroy_process_group()
    q.put((rank, out.getvalue()))


def test_bench_default_n2_is_weak_scaling_with_c5_leg():
    """The default N > 1 line (as the driver launches it): value = weak scaling of the c2 headline
    (one c2-shaped system per rank, seed + rank), plus the C5 strong-scaling leg over the same ranks."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_bench_worker_weak, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=900) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    import json
    line = json.loads(out[0].strip().splitlines()[-1])
    assert line["scaling"] == "weak" and line["n_gpus"] == world
    assert line["config"]["systems_total"] == world and line["config"]["n_per_system"] == 1_000_000
    assert line["gpu_launches"] == world * 2
    leg = line["c5_batch_leg"]
    assert leg["scaling"] == "strong" and leg["systems_total"] == 8 and leg["gpu_launches"] == 16
