"""B200-native (sm_100a) OpenMP device-runtime hot path (Doerfert et al., IPDPS'22).

csrc/omprt/device/  header-only device runtime (init/deinit, Fig. 5 schedules, generic-mode
                    state machine, alloc_shared stack, team/league reductions, ICVs, debug)
csrc/kernels/       the five BASELINE workloads, runtime-driven and bare-CUDA twins
csrc/host/          the C ABI (include/omprt.h) -> libomprt.so
omprt.py            thin ctypes binding with the C names
"""
from . import omprt  # noqa: F401

__all__ = ["omprt"]
