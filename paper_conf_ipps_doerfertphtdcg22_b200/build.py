"""Build libomprt.so (sm_100a) in-tree with nvcc and write a per-kernel resource report.

The library is one translation unit (csrc/libomprt.cu).  `ptxas -v` output is parsed into
build/resource_report.txt: registers, stack, shared memory per kernel (the paper's Fig. 11
"# Regs" / "SMem" columns) so runtime-vs-twin resource usage is visible without a
GPU.
"""
from __future__ import annotations

import os
import re
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libomprt.so")
REPORT = os.path.join(ROOT, "build", "resource_report.txt")

NVCC_FLAGS = [
    "-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
    "-Xptxas", "-v", "--shared", "-Xcompiler", "-fPIC,-O2", "-I", os.path.join(ROOT, "include"),
]


def _sources():
    out = []
    for d, _, fs in os.walk(CSRC):
        out += [os.path.join(d, f) for f in fs if f.endswith((".cu", ".cuh", ".h"))]
    out.append(os.path.join(ROOT, "include", "omprt.h"))
    return out


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in _sources())


def parse_ptxas(log: str):
    rows, cur = [], None
    for line in log.splitlines():
        m = re.search(r"Compiling entry function '([^']+)'", line)
        if m:
            cur = {"mangled": m.group(1)}
            rows.append(cur)
            continue
        if cur is None:
            continue
        m = re.search(r"Used (\d+) registers", line)
        if m:
            cur["regs"] = int(m.group(1))
            s = re.search(r"(\d+) bytes smem", line)
            cur["smem"] = int(s.group(1)) if s else 0
            st = re.search(r"(\d+) bytes cumulative stack size", line)
            cur["stack"] = int(st.group(1)) if st else 0
        m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads",
                      line)
        if m and "frame" not in cur:
            cur["frame"], cur["spill_st"], cur["spill_ld"] = map(int, m.groups())
    return rows


def demangle(names):
    try:
        p = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True)
        return p.stdout.splitlines()
    except OSError:
        return names


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and not needs_build():
        return LIB
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = ["nvcc", *NVCC_FLAGS, os.path.join(CSRC, "libomprt.cu"), "-o", tmp]
    p = subprocess.run(cmd, capture_output=True, text=True)
    if p.returncode != 0:
        sys.stderr.write(p.stdout + p.stderr)
        raise RuntimeError("nvcc failed building libomprt.so")
    os.replace(tmp, LIB)
    rows = parse_ptxas(p.stdout + p.stderr)
    names = demangle([r["mangled"] for r in rows])
    os.makedirs(os.path.dirname(REPORT), exist_ok=True)
    with open(REPORT, "w") as f:
        f.write("# ptxas resource report for libomprt.so (sm_100a)\n")
        f.write("# regs  stack  spill_st spill_ld  smem  kernel\n")
        for r, n in sorted(zip(rows, names), key=lambda x: x[1]):
            f.write(f"{r.get('regs', -1):5d} {r.get('stack', 0):6d} {r.get('spill_st', 0):8d} "
                    f"{r.get('spill_ld', 0):8d} {r.get('smem', 0):5d}  {n}\n")
    if verbose:
        print(open(REPORT).read())
    return LIB


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
