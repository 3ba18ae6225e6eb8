"""Multi-process (world_size 2, gloo, CPU) tests of the N > 1 host logic: contiguous
sharding, the u64 checksum all-reduce (wraps mod 2^64 through int64), max-over-ranks
timing, and sharding invariance of the XSBench/RSBench checksums computed per rank (by the
oracle here; the GPU path is checked for the same invariance in test_gpu_xsbench)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_doerfertphtdcg22_b200 import sharding


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import gen
    import oracle
    res = {}
    # strong-scaling shard of 60k lookups; per-rank checksum; u64 all-reduce
    t = gen.XSTables(n_isotopes=68, n_gridpoints=300)
    first, count = sharding.shard(60_000, rank, world)
    v = oracle.xs_lookup(t, first, count)
    ck = torch.tensor([int(v.sum())], dtype=torch.uint64)
    sharding.allreduce_u64_sum(ck)
    res["xs_checksum"] = int(ck.numpy()[0])
    # wrap-around: each rank contributes 2^63 + rank
    w = torch.tensor([(1 << 63) + rank], dtype=torch.uint64)
    sharding.allreduce_u64_sum(w)
    res["wrap"] = int(w.numpy()[0])
    # weak shard ranges tile [0, world*per)
    res["weak"] = sharding.weak_shard(1000, rank)
    res["max"] = sharding.allreduce_max(float(rank) + 0.5, "cpu")
    f = torch.tensor([0.25 * (rank + 1)], dtype=torch.float64)
    sharding.allreduce_f64_sum(f)
    res["fsum"] = float(f.item())
    q.put((rank, res))
    dist.barrier()
    dist.destroy_process_group()


def test_world2_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    import gen
    import oracle
    t = gen.XSTables(n_isotopes=68, n_gridpoints=300)
    full = int(oracle.xs_lookup(t, 0, 60_000).sum())
    for r in range(world):
        assert out[r]["xs_checksum"] == full
        assert out[r]["wrap"] == ((1 << 63) * 2 + 1) % 2**64
        assert out[r]["max"] == 1.5
        assert out[r]["fsum"] == 0.75
    assert out[0]["weak"] == (0, 1000) and out[1]["weak"] == (1000, 1000)


def test_device_and_backend_choice():
    assert sharding.pick_device_and_backend(3, 8, 8) == (3, "nccl", False)
    assert sharding.pick_device_and_backend(0, 1, 1) == (0, "nccl", False)
    assert sharding.pick_device_and_backend(1, 2, 1) == (0, "gloo", True)  # test mode only
    with pytest.raises(RuntimeError):
        sharding.pick_device_and_backend(0, 1, 0)  # no GPU: no CPU fallback


def test_shard_partition_properties():
    for total in (0, 1, 7, 17_000_000, 10_000_001):
        for world in (1, 2, 3, 4, 8):
            spans = [sharding.shard(total, r, world) for r in range(world)]
            pos = 0
            for first, count in spans:
                assert first == pos and count >= 0
                pos += count
            assert pos == total
            assert max(c for _, c in spans) - min(c for _, c in spans) <= 1
    with pytest.raises(ValueError):
        sharding.shard(10, 2, 2)
