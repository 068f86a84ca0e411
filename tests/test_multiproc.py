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
