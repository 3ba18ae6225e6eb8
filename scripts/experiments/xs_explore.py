"""Time XSBench body/launch variants (scripts/experiments/xs_explore.cu) on the GPU."""
import ctypes as C, os, subprocess, sys, statistics, json
ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)
HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.environ.get("XSX_SRC", "xs_explore.cu")
SO = os.path.join(HERE, "lib" + SRC.replace(".cu", ".so"))

def build():
    subprocess.check_call(["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
                           "-lineinfo", "--shared", "-Xcompiler", "-fPIC", os.path.join(HERE, SRC), "-o", SO])

def main():
    import torch, gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    if not os.path.exists(SO):
        build()
    L = C.CDLL(SO)
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    t = gen.XSTables(**gen.XS_SMALL)
    d = omprt.XSDeviceTables(t, "cuda", accel=os.environ.get("XSX_ACCEL") == "1",
                             log2_bins=int(os.environ.get("XSX_LOG2BINS", "16")))
    L.xsx_prepare.argtypes = [omprt.XSTablesC]
    L.xsx_run.argtypes = [C.c_int, omprt.XSTablesC, C.c_uint64, C.c_int64, C.c_int32, C.c_void_p, C.c_void_p]
    assert L.xsx_prepare(d.c) == 0
    n = 17_000_000
    ref = torch.zeros(n, dtype=torch.uint64, device="cuda")
    omprt.omprt_xs_lookup(d, 1070, 0, n, ref, None, 0, 256, omprt.OMPRT_ASSUME_OVERSUB)
    ver = torch.zeros(n, dtype=torch.uint64, device="cuda")
    scrub = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    res = {}
    for v in range(L.xsx_count()):
        ts = []
        for r in range(6):
            scrub.fill_(1.0)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            assert L.xsx_run(v, d.c, 1070, 0, n, ver.data_ptr(), s.cuda_stream) == 0
            b.record(s)
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ok = bool(torch.equal(ver, ref))
        res[v] = {"ms": statistics.median(ts[1:]), "regs": L.xsx_regs(v), "exact": ok}
        if hasattr(L, "xsx_name"):
            L.xsx_name.restype = C.c_char_p
            res[v]["name"] = L.xsx_name(v).decode()
        print(v, res[v], flush=True)
    print(json.dumps(res))

if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "build":
        build()
    else:
        main()
