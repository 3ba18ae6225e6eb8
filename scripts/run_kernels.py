"""Launch one config's runtime kernel and twin a few times (for ncu captures).
  python scripts/run_kernels.py rs|rs1m|rs10m|su3|generic|axpy|xs [reps]"""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch, gen
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt

which = sys.argv[1]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
torch.cuda.set_device(0)
omprt.omprt_init(0)
dev = "cuda"
A = omprt.OMPRT_ASSUME_OVERSUB
if which == "rs":
    t = gen.RSTables(); d = omprt.RSDeviceTables(t, dev); n = 1_000_000
    v = torch.empty(n, dtype=torch.uint64, device=dev)
    for _ in range(reps):
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, A)
        omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, 0)
elif which == "rs1m":  # nested and flattened, 1M lookups
    t = gen.RSTables(); d = omprt.RSDeviceTables(t, dev); n = 1_000_000
    v = torch.empty(n, dtype=torch.uint64, device=dev)
    for _ in range(reps):
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, A)
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, omprt.OMPRT_FLAT)
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128,
                              omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC)
        omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128,
                                   omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC)
        Q = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC | omprt.OMPRT_RS_QUEUE
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, Q)
        omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, Q)
elif which == "rs10m":  # the bench's C4 launch (queued, dynamic, flattened), 10M lookups
    t = gen.RSTables(); d = omprt.RSDeviceTables(t, dev); n = 10_000_000
    v = torch.empty(n, dtype=torch.uint64, device=dev)
    Q = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC | omprt.OMPRT_RS_QUEUE
    for _ in range(reps):
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, Q)
        omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, Q)
elif which == "rsd10m":  # dynamic flattened without the queue, 10M lookups
    t = gen.RSTables(); d = omprt.RSDeviceTables(t, dev); n = 10_000_000
    v = torch.empty(n, dtype=torch.uint64, device=dev)
    D = omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC
    for _ in range(reps):
        omprt.omprt_rs_lookup(d, 1070, 0, n, v, None, 0, 128, D)
        omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, v, None, 0, 128, D)
elif which == "su3":
    ns = 32 ** 4; Ah, Bh = gen.su3_inputs(ns)
    At, Bt = torch.from_numpy(Ah).to(dev), torch.from_numpy(Bh).to(dev); Ct = torch.empty_like(At)
    ck = torch.zeros(1, dtype=torch.float64, device=dev)
    for _ in range(reps):
        omprt.omprt_su3_mult(At, Bt, Ct, ns, ck, 0, 128, A)
        omprt.omprt_cuda_su3_mult(At, Bt, Ct, ns, ck, 0, 128, 0)
        for fl in (omprt.OMPRT_WARP_STAGED, omprt.OMPRT_TMA_TILED):
            omprt.omprt_su3_mult(At, Bt, Ct, ns, ck, 0, 128, fl)
            omprt.omprt_cuda_su3_mult(At, Bt, Ct, ns, ck, 0, 128, fl)
elif which == "generic":
    T = 4096; inp = torch.from_numpy(gen.generic_inputs(T, 256)).to(dev)
    out = torch.empty(T * 256, dtype=torch.float64, device=dev)
    for _ in range(reps):
        omprt.omprt_generic_team(T, 256, 256, inp, out, None, None, A)
        omprt.omprt_cuda_generic_team(T, 256, 256, inp, out)
        omprt.omprt_generic_team(T, 256, 256, inp, out, None, None, omprt.OMPRT_GENERAL_SM)
elif which == "axpy":
    n = 1 << 20; x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(dev), torch.from_numpy(c).to(dev); at = torch.empty_like(bt)
    s = torch.zeros(1, dtype=torch.float64, device=dev)
    for _ in range(reps):
        omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, 128)
        omprt.omprt_cuda_axpy_sum(n, x, bt, ct, at, s, 8, 128)
        omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, 128, omprt.OMPRT_TMA_STREAM)
        omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, 256, omprt.OMPRT_TMA_STREAM)
torch.cuda.synchronize()
print("done", which)
