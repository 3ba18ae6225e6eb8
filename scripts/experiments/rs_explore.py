"""Time RSBench body variants (scripts/experiments/rs_explore.cu) on the GPU."""
import ctypes as C, os, subprocess, sys, statistics, json
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
HERE = os.path.dirname(os.path.abspath(__file__))
SO = os.path.join(HERE, "librs_explore.so")

def build():
    subprocess.check_call(["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
                           "-lineinfo", "--shared", "-Xcompiler", "-fPIC", os.path.join(HERE, "rs_explore.cu"), "-o", SO])

def main():
    import torch, gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    L = C.CDLL(SO)
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    t = gen.RSTables()
    d = omprt.RSDeviceTables(t, "cuda")
    L.rsx_run.argtypes = [C.c_int, omprt.RSTablesC, C.c_uint64, C.c_int64, C.c_int32, C.c_void_p, C.c_void_p]
    n = 1_000_000
    ref = torch.zeros(n, dtype=torch.uint64, device="cuda")
    omprt.omprt_cuda_rs_lookup(d, 1070, 0, n, ref, None, 0, 128, 0)
    ver = torch.zeros(n, dtype=torch.uint64, device="cuda")
    s = torch.cuda.current_stream()
    res = {}
    for v in range(L.rsx_count()):
        ts = []
        for r in range(4):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            assert L.rsx_run(v, d.c, 1070, 0, n, ver.data_ptr(), s.cuda_stream) == 0
            b.record(s)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        res[v] = {"ms": statistics.median(ts[1:]), "regs": L.rsx_regs(v),
                  "mismatch": int((ver != ref).sum().item())}
        print(v, res[v], flush=True)

if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "build":
        build()
    else:
        main()
