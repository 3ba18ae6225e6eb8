"""The measurement side of the library (not the hot path): the roof probes bench.py
reports against and the occupancy query -- they run, and their numbers are physically
plausible for a B200 (so a broken probe cannot inflate or deflate a roofline fraction
unnoticed)."""
import pytest
import torch

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def test_roof_probes_plausible(rt):
    import bench
    p = bench.measure_peaks(rt, torch, torch.device(DEV), torch.cuda.current_stream())
    # L2 -> SM: above the HBM copy peak (~6.5 TB/s), below 4 x it
    assert 7000 < p["l2_stream_gbs"] < 26000, p
    assert 2000 < p["l2_sector32_gbs"] <= p["l2_stream_gbs"] * 1.05, p
    assert 2000 < p["l2_record96_gbs"] <= p["l2_stream_gbs"] * 1.05, p
    # FP64 FMA: B200 nominal ~37-40 TFLOP/s
    assert 20000 < p["fp64_fma_gflops"] < 45000, p
    # HBM -> SM by bulk copies: all SMs near the HBM peak (~7.7 TB/s nominal), 8 SMs a
    # fraction of it
    assert 4000 < p["hbm_stream_gbs"] < 8500, p
    assert 100 < p["hbm_stream_8sm_gbs"] < p["hbm_stream_gbs"] * 0.5, p
    assert 100 < p["hbm_read2write1_8sm_gbs"] < p["hbm_stream_gbs"] * 0.5, p


def test_probe_arguments_rejected(rt):
    buf = torch.ones(1024, dtype=torch.float64, device=DEV)
    sink = torch.zeros(1, dtype=torch.float64, device=DEV)
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_l2_read(buf, 8192, 3, 1, 8, sink)      # no mode 3
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_l2_read(buf, 8192, 1, 1, 7, sink)      # per_thread % 8
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_fp64_fma(0, sink)
    big = torch.ones(1 << 16, dtype=torch.float64, device=DEV)
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_hbm_stream(big, big.numel() * 8, 0, sink)       # no teams
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_hbm_stream(big, big.numel() * 8, 1000, sink)    # more teams than SMs
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_hbm_stream(big, 16384, 1, sink)                 # slice < 32 KB
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_hbm_stream(big, big.numel() * 8, 1, sink, None, 1)  # mode 1, no dst
    with pytest.raises(rt.OmprtError):
        rt.omprt_probe_hbm_stream(big, big.numel() * 8, 1, sink, None, 2)  # no mode 2


def test_hbm_probe_copies_what_it_reads(rt):
    """Mode 1 writes every second 16 KB chunk of each team's slice to dst (team b's writes
    at b * slice / 2): the copy is exact, so the probe moves the bytes it claims."""
    n = 8 * (1 << 20)  # 8 MiB, 4 teams -> slice 2 MiB = 128 chunks of 16 KB
    src = torch.arange(n // 8, dtype=torch.int64, device=DEV)
    dst = torch.zeros(n // 2 // 8, dtype=torch.int64, device=DEV)
    sink = torch.zeros(1, dtype=torch.float64, device=DEV)
    rt.omprt_probe_hbm_stream(src, n, 4, sink, dst, 1)
    torch.cuda.synchronize()
    chunk = 16384 // 8
    s = src.view(4, -1, chunk)[:, 1::2, :].reshape(-1)
    assert torch.equal(dst, s)


def test_occupancy_query(rt):
    # the headline kernel: 64 registers x 256 threads -> 4 resident teams per SM
    assert rt.omprt_kernel_occupancy("omprt_xs_flat_rt", 256) == 4
    assert rt.omprt_kernel_occupancy("omprt_rs_qflat_rt", 128) == 4
    with pytest.raises(rt.OmprtError):
        rt.omprt_kernel_occupancy("omprt_xs_flat_rt", 0)
