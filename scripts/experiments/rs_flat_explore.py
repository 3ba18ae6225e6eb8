"""Time the flattened RSBench variants (scripts/experiments/rs_flat_explore.cu) on the GPU:
verification flips vs the library's nested kernel, macro xs normwise error, time at 1M/10M.
  python scripts/experiments/rs_flat_explore.py build | run"""
import ctypes as C
import json
import os
import statistics
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(os.path.dirname(HERE))
sys.path.insert(0, ROOT)
SRC = os.environ.get("RSX_SRC", "rs_flat_explore.cu")
SO = os.path.join(HERE, "lib" + SRC.replace(".cu", ".so"))


def build():
    subprocess.check_call(["nvcc", "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a",
                           "-lineinfo", "--shared", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
                           os.path.join(HERE, SRC), "-o", SO])


def main():
    import torch

    import gen
    from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
    L = C.CDLL(SO)
    L.rsf_name.restype = C.c_char_p
    L.rsf_run.argtypes = [C.c_int, omprt.RSTablesC, C.c_uint64, C.c_int64, C.c_int32,
                          C.c_void_p, C.c_void_p, C.c_void_p]
    torch.cuda.set_device(0)
    omprt.omprt_init(0)
    t = gen.RSTables()
    d = omprt.RSDeviceTables(t, "cuda")
    s = torch.cuda.current_stream()
    for n in (1_000_000, 10_000_000):
        ref = torch.zeros(n, dtype=torch.uint64, device="cuda")
        mref = torch.zeros(4 * n, dtype=torch.float64, device="cuda")
        omprt.omprt_rs_lookup(d, 1070, 0, n, ref, mref, 0, 128,
                              omprt.OMPRT_FLAT | omprt.OMPRT_SCHED_DYNAMIC)
        mref = mref.view(n, 4)
        ver = torch.zeros(n, dtype=torch.uint64, device="cuda")
        mac = torch.zeros(4 * n, dtype=torch.float64, device="cuda")
        for v in range(L.rsf_count()):
            ts = []
            for r in range(3 if n <= 1_000_000 else 2):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                assert L.rsf_run(v, d.c, 1070, 0, n, ver.data_ptr(), mac.data_ptr(), s.cuda_stream) == 0
                b.record(s)
                torch.cuda.synchronize()
                ts.append(a.elapsed_time(b))
            m = mac.view(n, 4)
            err = ((m - mref).abs().max(dim=1).values / mref.abs().max(dim=1).values).max().item()
            print(json.dumps({"n": n, "variant": L.rsf_name(v).decode(), "ms": min(ts),
                              "regs_local": L.rsf_regs(v), "flips": int((ver != ref).sum().item()),
                              "max_norm_err": err}), flush=True)


if __name__ == "__main__":
    build() if sys.argv[1:] == ["build"] else main()
