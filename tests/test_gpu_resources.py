"""Resource parity with the bare CUDA twins (the paper's Fig. 11 "# Regs" / "SMem" columns,
P:290-470; north_star target: registers within 5% of the twin, no local memory, and 0 B of
runtime shared memory on SPMD kernels)."""
import pytest

pytestmark = pytest.mark.gpu

PAIRS = [
    ("omprt_axpy_rt", "cuda_axpy_twin", True),
    ("omprt_axpy_rt_assume", "cuda_axpy_twin", True),
    ("omprt_xs_rt_assume", "cuda_xs_twin", True),
    ("omprt_xs_rt", "cuda_xs_twin", True),
    ("omprt_xs_rt_fused", "cuda_xs_twin_fused", True),
    ("omprt_xs_rt_assume_accel", "cuda_xs_twin_accel", True),
    ("omprt_xs_rt_accel", "cuda_xs_twin_accel", True),
    ("omprt_xs_rt_fused_accel", "cuda_xs_twin_fused_accel", True),
    ("omprt_rs_rt_assume", "cuda_rs_twin", True),
    ("omprt_rs_rt", "cuda_rs_twin", True),
    ("omprt_su3_rt", "cuda_su3_twin", True),
    ("omprt_generic_rt", "cuda_generic_twin", False),
    ("omprt_axpy_chunk_rt", "cuda_axpy_chunk_twin", True),
    ("omprt_generic_spmd_rt", "cuda_generic_twin", True),
    ("omprt_generic_deglob_rt", "cuda_generic_twin", False),
    ("omprt_xs_flat_rt", "cuda_xs_flat_twin", True),
    ("omprt_xs_flat_rt_fused", "cuda_xs_flat_twin_fused", True),
    ("omprt_su3_wstaged_rt", "cuda_su3_wstaged_twin", True),
    ("omprt_su3_tiled_rt", "cuda_su3_tiled_twin", True),
    ("omprt_axpy_tma_rt", "cuda_axpy_tma_twin", True),
    ("omprt_rs_flat_rt", "cuda_rs_flat_twin", True),
    ("omprt_rs_dflat_rt", "cuda_rs_dflat_twin", True),
    ("omprt_rs_qflat_rt", "cuda_rs_qflat_twin", True),
    ("omprt_axpy_dyn_rt", "cuda_axpy_dyn_twin", True),
    ("omprt_axpy_rt_wide", "cuda_axpy_twin_wide", True),
]


def test_deglobalized_has_no_stack(rt):
    """NEXT f2: the deglobalized kernel carries only the twin's arrays (+ the team state and
    the argument sharing space), not the 4 KiB stack of the stack-based kernel."""
    tab = rt.kernel_table()
    assert tab["omprt_generic_deglob_rt"]["static_smem"] < tab["omprt_generic_rt"]["static_smem"]
    assert tab["omprt_generic_deglob_rt"]["static_smem"] <= tab["cuda_generic_twin"]["static_smem"] + 64


# Pairs whose register counts may differ by more than 5 % because the count cannot change
# the occupancy at the geometries they run: both kernels of a pair carry the same
# __maxnreg__ budget and the resident teams per SM are asserted equal at every listed team
# size instead.  C1 at 32 iterations per trip (teams of <= 256, axpy.cuh): budget 255,
# runtime 206 / twin 218 registers -- the same teams per SM at every multiple of 32 up to
# 256.
OCCUPANCY_EQUIVALENT = {("omprt_axpy_rt_wide", "cuda_axpy_twin_wide"): (range(32, 257, 32), 255)}


@pytest.mark.parametrize("rtk,twin,spmd", PAIRS)
def test_registers_and_smem_vs_twin(rt, rtk, twin, spmd):
    tab = rt.kernel_table()
    a, b = tab[rtk], tab[twin]
    if (rtk, twin) in OCCUPANCY_EQUIVALENT:
        sizes, budget = OCCUPANCY_EQUIVALENT[(rtk, twin)]
        for th in sizes:
            assert rt.omprt_kernel_occupancy(rtk, th) == rt.omprt_kernel_occupancy(twin, th), th
        assert a["regs"] <= budget and b["regs"] <= budget, (a, b)
    else:
        assert a["regs"] <= int(1.05 * b["regs"]) or a["regs"] <= b["regs"] + 1, (a, b)
    assert a["local_bytes"] <= b["local_bytes"], (a, b)
    if spmd:
        assert a["static_smem"] == b["static_smem"], (a, b)  # 0 B of runtime state
