"""SURVEY §4 T-multi on one B200: two ranks (processes) share cuda:0 over gloo -- the
shared-GPU test mode of sharding.pick_device_and_backend -- and run BASELINE configs [2]-[4]
sharded as bench.py's N > 1 path does (contiguous shards, per-rank GPU kernels, the one
checksum all-reduce).  The all-reduced checksums must equal the one-launch values: bit-exact
for the u64 verification sums (C3, C4), within the C6 tolerance for the fp64 SU(3) sum."""
import os
import socket

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _checksums(rank, world, omprt, gen, sharding, dev, backend="gloo"):
    """(xs u64, rs u64, su3 f64) over this rank's shards, all-reduced when world > 1."""
    res = {}
    # C3: XSBench-shaped, flattened kernel on the B200 layouts, 200k lookups (small table)
    t = gen.XSTables(n_isotopes=68, n_gridpoints=2000)
    d = omprt.XSDeviceTables(t, dev, accel=True)
    first, cnt = sharding.shard(200_000, rank, world)
    ver = torch.empty(max(cnt, 1), dtype=torch.uint64, device=dev)
    ck = torch.zeros(1, dtype=torch.uint64, device=dev)
    omprt.omprt_xs_lookup(d, gen.XS_LOOKUP_SEED, first, cnt, ver, None, 0, 256,
                          omprt.OMPRT_XS_FLAT)
    omprt.omprt_u64_sum(ver, cnt, ck)
    # C4: RSBench-shaped, the bench's queued dynamic lock-step kernel, 50k lookups
    rd = omprt.RSDeviceTables(gen.RSTables(), dev)
    f4, c4 = sharding.shard(50_000, rank, world)
    v4 = torch.empty(max(c4, 1), dtype=torch.uint64, device=dev)
    ck4 = torch.zeros(1, dtype=torch.uint64, device=dev)
    omprt.omprt_rs_lookup(rd, gen.RS_LOOKUP_SEED, f4, c4, v4, None, 0, 128,
                          omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC | omprt.OMPRT_RS_QUEUE)
    omprt.omprt_u64_sum(v4, c4, ck4)
    # C5: SU(3) on 8^4 sites
    ns = 8 ** 4
    s0, sc = sharding.shard(ns, rank, world)
    A, B = gen.su3_inputs(sc, first_site=s0)
    At, Bt = torch.from_numpy(A).to(dev), torch.from_numpy(B).to(dev)
    Ct = torch.empty_like(At)
    cs = torch.zeros(1, dtype=torch.float64, device=dev)
    omprt.omprt_su3_mult(At, Bt, Ct, sc, cs, 0, 128, omprt.OMPRT_ASSUME_OVERSUB)
    # ... and with the TMA tensor tiles bench.py's sharded C5 runs (same elementwise C)
    Ct2 = torch.empty_like(At)
    cs2 = torch.zeros(1, dtype=torch.float64, device=dev)
    omprt.omprt_su3_mult(At, Bt, Ct2, sc, cs2, 0, 128, omprt.OMPRT_TMA_TILED)
    torch.cuda.synchronize()
    assert torch.equal(Ct, Ct2)
    if backend == "gloo":  # gloo reduces host tensors, NCCL device ones
        ck, ck4, cs = ck.cpu(), ck4.cpu(), cs.cpu()
    if world > 1:
        sharding.allreduce_u64_sum(ck)
        sharding.allreduce_u64_sum(ck4)
        sharding.allreduce_f64_sum(cs)
    res["xs"] = int(ck.cpu().numpy()[0])
    res["rs"] = int(ck4.cpu().numpy()[0])
    res["su3"] = float(cs.item())
    return res


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt, sharding
    gpu, backend, shared = sharding.pick_device_and_backend(rank, world,
                                                           torch.cuda.device_count())
    dist.init_process_group(backend, rank=rank, world_size=world)
    torch.cuda.set_device(gpu)
    omprt.omprt_init(gpu)
    q.put((rank, dict(_checksums(rank, world, omprt, gen, sharding, f"cuda:{gpu}", backend),
                      backend=backend, shared=shared)))
    dist.barrier()
    dist.destroy_process_group()


def test_two_ranks_match_one_launch(rt):
    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import sharding
    one = _checksums(0, 1, rt, gen, sharding, "cuda:0")
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for r in range(world):
        assert out[r]["xs"] == one["xs"]
        assert out[r]["rs"] == one["rs"]
        # C6 tolerance: the fp64 checksum of a different summation order
        assert abs(out[r]["su3"] - one["su3"]) <= 1e-12 * 36 * 8 ** 4
        if torch.cuda.device_count() < world:
            assert out[r]["backend"] == "gloo" and out[r]["shared"]
