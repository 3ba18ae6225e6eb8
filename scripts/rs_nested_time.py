import sys, torch, statistics
sys.path.insert(0, '.')
import gen
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
torch.cuda.set_device(0); omprt.omprt_init(0)
d = omprt.RSDeviceTables(gen.RSTables(), "cuda")
n = 10_000_000
v = torch.empty(n, dtype=torch.uint64, device="cuda")
s = torch.cuda.current_stream()
for name, fn, fl in (("rt_assume", omprt.omprt_rs_lookup, omprt.OMPRT_ASSUME_OVERSUB), ("twin", omprt.omprt_cuda_rs_lookup, 0), ("rt_loop", omprt.omprt_rs_lookup, 0)):
    ts = []
    for r in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s); fn(d, 1070, 0, n, v, None, 0, 128, fl); b.record(s); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    print(name, min(ts), int(v.sum().item()))
