"""GPU parity: SPMD `distribute parallel for` -- Fig. 5 assignment (owner bit-exact,
every iteration exactly once) and C1 axpy + fp64 sum."""
import os
import subprocess
import sys

import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _run(rt, fn, n, T, N, flags, x, b, c):
    bt = torch.from_numpy(b).to(DEV)
    ct = torch.from_numpy(c).to(DEV)
    at = torch.full((max(n, 1),), float("nan"), dtype=torch.float64, device=DEV)
    s = torch.zeros(1, dtype=torch.float64, device=DEV)
    owner = torch.full((max(n, 1),), -1, dtype=torch.int32, device=DEV)
    count = torch.zeros(max(n, 1), dtype=torch.int32, device=DEV)
    fn(n, x, bt, ct, at, s, T, N, flags | rt.OMPRT_RECORD_OWNER, owner, count)
    torch.cuda.synchronize()
    return at.cpu().numpy()[:n], float(s.item()), owner.cpu().numpy()[:n], count.cpu().numpy()[:n]


CASES = [(0, 1, 32), (1, 8, 128), (1023, 8, 128), (1024, 8, 128), (1025, 8, 128),
         (1 << 20, 8, 128), ((1 << 20) + 7, 3, 96), (100003, 37, 64)]


@pytest.mark.parametrize("n,T,N", CASES)
@pytest.mark.parametrize("which", ["rt", "twin"])
def test_owner_exactly_once_bit_exact(rt, n, T, N, which):
    x, b, c = gen.axpy_inputs(n)
    fn = rt.omprt_spmd_axpy_sum if which == "rt" else rt.omprt_cuda_axpy_sum
    a, s, owner, count = _run(rt, fn, n, T, N, 0, x, b, c)
    ref_owner, ref_count = oracle.fig5_simulate(n, T, N)
    assert (count == 1).all()
    assert (owner == ref_owner).all()
    assert (a == oracle.axpy(x, b, c)).all()


def test_owner_with_assumption_17M(rt):
    """The XSBench geometry: 17e6 iterations, 66407 teams x 256 with the assumption."""
    n, N = 17_000_000, 256
    T = (n + N - 1) // N
    x, b, c = 1.0, np.zeros(n), np.zeros(n)
    a, s, owner, count = _run(rt, rt.omprt_spmd_axpy_sum, n, T, N, rt.OMPRT_ASSUME_OVERSUB, x, b, c)
    assert (count == 1).all()
    assert (owner == np.arange(n, dtype=np.int32)).all()  # closed form when n <= T*N


def test_assumption_violation_rejected(rt):
    n, T, N = 2049, 8, 256
    x, b, c = gen.axpy_inputs(n)
    with pytest.raises(rt.OmprtError) as e:
        _run(rt, rt.omprt_spmd_axpy_sum, n, T, N, rt.OMPRT_ASSUME_OVERSUB, x, b, c)
    assert e.value.code == rt.OMPRT_E_INVAL


@pytest.mark.parametrize("which", ["rt", "twin", "rt_assume"])
def test_axpy_exact_sum(rt, which):
    """Integer-valued inputs: every partial sum is exact, so sum == 2^30 bit for bit."""
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n, exact=True)
    if which == "rt_assume":
        T, N, flags, fn = 1024, 1024, rt.OMPRT_ASSUME_OVERSUB, rt.omprt_spmd_axpy_sum
    else:
        T, N, flags = 8, 128, 0
        fn = rt.omprt_spmd_axpy_sum if which == "rt" else rt.omprt_cuda_axpy_sum
    a, s, _, _ = _run(rt, fn, n, T, N, flags, x, b, c)
    assert s == float(1 << 30)
    assert (a == oracle.axpy(x, b, c)).all()


@pytest.mark.parametrize("n,T,N", [(1 << 20, 8, 128), ((1 << 20) + 7, 8, 128),
                                   ((1 << 20) + 7, 592, 256)])
def test_axpy_random_sum_tolerance(rt, n, T, N):
    x, b, c = gen.axpy_inputs(n)
    a_ref = oracle.axpy(x, b, c)
    bound = 1e-12 * oracle.sum_abs_f64(a_ref)
    ref = oracle.sum_f64(a_ref)
    sums = []
    for fn in (rt.omprt_spmd_axpy_sum, rt.omprt_cuda_axpy_sum):
        bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
        at = torch.empty_like(bt)
        s = torch.full((1,), 0.25, dtype=torch.float64, device=DEV)  # OpenMP: orig (+) sum
        fn(n, x, bt, ct, at, s, T, N)
        torch.cuda.synchronize()
        assert (at.cpu().numpy() == a_ref).all()
        sums.append(float(s.item()))
        assert abs(sums[-1] - (ref + 0.25)) <= bound
    assert sums[0] == sums[1]  # same reduction algorithm, same geometry -> same bits
    # deterministic run to run
    bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
    at = torch.empty_like(bt)
    s = torch.full((1,), 0.25, dtype=torch.float64, device=DEV)
    rt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, T, N)
    assert float(s.item()) == sums[0]


def test_int64_index_path(rt):
    """the host picks the 64-bit induction variable when n + 9*T*N needs it."""
    T, N = 1 << 20, 1024  # T*N = 2^30 -> Idx = int64
    m = 4096
    x, b, c = gen.axpy_inputs(m)
    a, s, owner, count = _run(rt, rt.omprt_spmd_axpy_sum, m, T, N, 0, x, b, c)
    assert (count == 1).all() and (owner == np.arange(m)).all()
    assert abs(s - oracle.sum_f64(oracle.axpy(x, b, c))) <= 1e-12 * s


_CHILD = r'''
import sys, torch, gen
from paper_conf_ipps_doerfertphtdcg22_b200 import omprt
torch.cuda.set_device(0)
omprt.omprt_init(0)
n, threads = int(sys.argv[1]), int(sys.argv[2])
x, b, c = gen.axpy_inputs(n)
bt, ct = torch.from_numpy(b).cuda(), torch.from_numpy(c).cuda()
at = torch.empty_like(bt); s = torch.zeros(1, dtype=torch.float64, device="cuda")
flags = omprt.OMPRT_ASSUME_OVERSUB | omprt.OMPRT_DEBUG_BUILD | omprt.OMPRT_UNCHECKED
omprt.omprt_spmd_axpy_sum(n, x, bt, ct, at, s, 8, threads, flags)
try:
    torch.cuda.synchronize()
    print("SYNC ok")
except Exception as e:
    print("SYNC failed", type(e).__name__)
print("STATUS", omprt.omprt_device_status(0)[0])
'''


def _child(n, threads, debug_env):
    env = dict(os.environ, OMPRT_DEBUG=debug_env,
               PYTHONPATH=os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    return subprocess.run([sys.executable, "-c", _CHILD, str(n), str(threads)],
                          capture_output=True, text=True, env=env, timeout=300)


def test_debug_build_legal_launch_traces(rt):
    """Debug build, OMPRT_DEBUG=3 (assert + trace), assumption holds: no error, traced."""
    p = _child(4096, 512, "3")
    assert p.returncode == 0, p.stderr
    assert "STATUS 0" in p.stdout and "[omprt]" in p.stdout


def test_debug_assert_fires_on_violated_assumption(rt):
    """the runtime asserts the oversubscription condition in debug runs; the device
    records OMPRT_E_ASSERT in the mapped error word and traps."""
    p = _child(8 * 128 + 1, 128, "1")
    assert "STATUS -5" in p.stdout, (p.stdout, p.stderr)
    assert "assertion failed" in p.stdout


def test_debug_build_runtime_bits_off_is_silent(rt):
    """Compiled-in debug code does nothing unless enabled at run time."""
    p = _child(8 * 128 + 1, 128, "0")
    assert "STATUS 0" in p.stdout and "[omprt]" not in p.stdout


CHUNK_CASES = [(0, 4, 1, 32), (1, 4, 8, 128), (1 << 20, 4, 8, 128), ((1 << 20) + 7, 4, 8, 128),
               ((1 << 20) + 5, 3, 3, 96), (100003, 16, 37, 64), (4096, 1, 8, 128),
               (2049, 4, 2, 256)]


@pytest.mark.parametrize("n,C,T,N", CHUNK_CASES)
@pytest.mark.parametrize("which", ["rt", "twin"])
def test_chunked_schedule_owner_and_values(rt, n, C, T, N, which):
    """NEXT f3: chunk k -> global thread k mod (T*N) (oracle_chunk_simulate), every iteration
    once, a[] bit-exact, sum within 1e-12 of the Neumaier reference."""
    x, b, c = gen.axpy_inputs(n)
    fn = rt.omprt_spmd_axpy_sum_chunked if which == "rt" else rt.omprt_cuda_axpy_sum_chunked
    bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
    at = torch.full((max(n, 1),), float("nan"), dtype=torch.float64, device=DEV)
    s = torch.zeros(1, dtype=torch.float64, device=DEV)
    owner = torch.full((max(n, 1),), -1, dtype=torch.int32, device=DEV)
    count = torch.zeros(max(n, 1), dtype=torch.int32, device=DEV)
    fn(n, C, x, bt, ct, at, s, T, N, rt.OMPRT_RECORD_OWNER, owner, count)
    torch.cuda.synchronize()
    ref_owner, _ = oracle.chunk_simulate(n, C, T, N)
    assert (count.cpu().numpy()[:n] == 1).all()
    assert (owner.cpu().numpy()[:n] == ref_owner).all()
    a_ref = oracle.axpy(x, b, c)
    assert (at.cpu().numpy()[:n] == a_ref).all()
    assert abs(s.item() - oracle.sum_f64(a_ref)) <= 1e-12 * max(oracle.sum_abs_f64(a_ref), 1e-300)


def test_chunked_vectorized_matches_twin_and_assumption(rt):
    n, C = 1 << 20, 4
    x, b, c = gen.axpy_inputs(n, exact=True)
    bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
    sums = []
    for fn, T, N, flags in [(rt.omprt_spmd_axpy_sum_chunked, 8, 128, 0),
                            (rt.omprt_cuda_axpy_sum_chunked, 8, 128, 0),
                            (rt.omprt_spmd_axpy_sum_chunked, 256, 1024, rt.OMPRT_ASSUME_OVERSUB)]:
        at = torch.empty_like(bt)
        s = torch.zeros(1, dtype=torch.float64, device=DEV)
        fn(n, C, x, bt, ct, at, s, T, N, flags)
        torch.cuda.synchronize()
        assert (at.cpu().numpy() == oracle.axpy(x, b, c)).all()
        sums.append(s.item())
    assert sums == [float(1 << 30)] * 3  # integer-valued: exact in any order
    with pytest.raises(rt.OmprtError) as e:  # 2^20 / 4 chunks > 128*1024 threads
        rt.omprt_spmd_axpy_sum_chunked(n, C, x, bt, ct, torch.empty_like(bt),
                                       torch.zeros(1, dtype=torch.float64, device=DEV), 128,
                                       1024, rt.OMPRT_ASSUME_OVERSUB)
    assert e.value.code == rt.OMPRT_E_INVAL


DYN_CASES = [(0, 4, 1, 32), (1, 1, 8, 128), ((1 << 20) + 7, 4, 8, 128), (100003, 16, 37, 64),
             (4096, 1, 8, 128), (2049, 3, 2, 256), (5000, 7, 300, 32)]


@pytest.mark.parametrize("n,C,T,N", DYN_CASES)
@pytest.mark.parametrize("which", ["rt", "twin"])
def test_dynamic_schedule_owner_and_values(rt, n, C, T, N, which):
    """schedule(dynamic, C) (reading R-D1): which thread runs a chunk is up to the hardware,
    so the GPU's owner[] is checked against the schedule's invariants (the same checks that
    pin oracle_dynamic_simulate) and the oracle's closed-form team of every iteration;
    a[] bit-exact, the sum within 1e-12 (its order follows the chunk hand-out)."""
    from test_oracle_schedule import _check_dynamic
    x, b, c = gen.axpy_inputs(n)
    fn = rt.omprt_spmd_axpy_sum_chunked if which == "rt" else rt.omprt_cuda_axpy_sum_chunked
    bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
    at = torch.full((max(n, 1),), float("nan"), dtype=torch.float64, device=DEV)
    s = torch.zeros(1, dtype=torch.float64, device=DEV)
    owner = torch.full((max(n, 1),), -1, dtype=torch.int32, device=DEV)
    count = torch.zeros(max(n, 1), dtype=torch.int32, device=DEV)
    fn(n, C, x, bt, ct, at, s, T, N, rt.OMPRT_RECORD_OWNER | rt.OMPRT_SCHED_DYNAMIC, owner,
       count)
    torch.cuda.synchronize()
    own = owner.cpu().numpy()[:n]
    _check_dynamic(n, C, T, N, own, count.cpu().numpy()[:n])
    if n:
        teams = np.array([oracle.dynamic_team_closed(i, n, T) for i in range(0, n, 97)])
        assert (own[::97] // N == teams).all()
    a_ref = oracle.axpy(x, b, c)
    assert (at.cpu().numpy()[:n] == a_ref).all()
    assert abs(s.item() - oracle.sum_f64(a_ref)) <= 1e-12 * max(oracle.sum_abs_f64(a_ref), 1e-300)


def test_dynamic_schedule_rejects_assumption(rt):
    n = 1024
    x, b, c = gen.axpy_inputs(n)
    bt, ct = torch.from_numpy(b).to(DEV), torch.from_numpy(c).to(DEV)
    with pytest.raises(rt.OmprtError):
        rt.omprt_spmd_axpy_sum_chunked(n, 1, x, bt, ct, torch.empty_like(bt),
                                       torch.zeros(1, dtype=torch.float64, device=DEV), 8, 128,
                                       rt.OMPRT_SCHED_DYNAMIC | rt.OMPRT_ASSUME_OVERSUB)


TMA_CASES = [(0, 1, 32), (1, 8, 128), (1023, 8, 128), (1024, 8, 128), (1025, 8, 128),
             (1 << 20, 8, 128), ((1 << 20) + 7, 3, 96), (100003, 37, 64), (16 * 1024 * 5 + 3, 8, 128),
             (300_000, 2, 256)]


@pytest.mark.parametrize("n,T,N", TMA_CASES)
@pytest.mark.parametrize("which", ["rt", "twin"])
def test_tma_stream_owner_values_and_sum(rt, n, T, N, which):
    """OMPRT_TMA_STREAM: the operands move by 2-D TMA boxes, the iterations stay Fig. 5's --
    owners bit-exact against the literal Fig. 5 simulation, every iteration once, a[]
    bit-exact, and the sum bit-identical to the register-path runtime kernel (the same
    iterations per thread in the same order); partial last boxes, a partial last trip and
    fewer iterations than threads included."""
    x, b, c = gen.axpy_inputs(n)
    fn = rt.omprt_spmd_axpy_sum if which == "rt" else rt.omprt_cuda_axpy_sum
    a, s, owner, count = _run(rt, fn, n, T, N, rt.OMPRT_TMA_STREAM, x, b, c)
    ref_owner, _ = oracle.fig5_simulate(n, T, N)
    assert (count == 1).all() and (owner == ref_owner).all()
    assert (a == oracle.axpy(x, b, c)).all()
    _, s_reg, _, _ = _run(rt, rt.omprt_spmd_axpy_sum, n, T, N, 0, x, b, c)
    assert s == s_reg
    if n:
        assert abs(s - oracle.sum_f64(a)) <= 1e-12 * oracle.sum_abs_f64(a)


def test_tma_stream_exact_sum_and_rejects(rt):
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n, exact=True)
    for fn in (rt.omprt_spmd_axpy_sum, rt.omprt_cuda_axpy_sum):
        _, s, _, _ = _run(rt, fn, n, 8, 128, rt.OMPRT_TMA_STREAM, x, b, c)
        assert s == float(1 << 30)
    with pytest.raises(rt.OmprtError):  # box width: at most 256 threads
        _run(rt, rt.omprt_spmd_axpy_sum, n, 8, 512, rt.OMPRT_TMA_STREAM, x, b, c)
    with pytest.raises(rt.OmprtError):
        _run(rt, rt.omprt_spmd_axpy_sum, 1024, 8, 128,
             rt.OMPRT_TMA_STREAM | rt.OMPRT_ASSUME_OVERSUB, x[:1] if False else x, b[:1024],
             c[:1024])


@pytest.mark.parametrize("dynamic", [False, True])
@pytest.mark.parametrize("n,T,N", [(0, 2, 64), (1, 1, 32), (1000, 3, 64), (20_011, 7, 128),
                                   (50_000, 148, 256)])
def test_lockstep_warp_collective_hook(rt, n, T, N, dynamic):
    """The lock-step flattened loops call a body's warp_collective(done) after every trip on
    all 32 lanes, report done exactly on an iteration's last step, before its end(); every
    iteration runs all its steps exactly once; under Fig. 5 (static) each warp runs as many
    trips as its busiest lane has steps."""
    steps = torch.full((max(n, 1),), -1, dtype=torch.int32, device="cuda:0")
    hooks = torch.zeros(T * N, dtype=torch.int32, device="cuda:0")
    errors = torch.zeros(1, dtype=torch.int32, device="cuda:0")
    rt.omprt_lockstep_probe(n, T, N, dynamic, steps, hooks, errors)
    torch.cuda.synchronize()
    assert int(errors.item()) == 0
    i = np.arange(n)
    L = 1 + (7 * i) % 13
    assert (steps.cpu().numpy()[:n] == L).all()
    h = hooks.cpu().numpy().reshape(-1, 32)
    assert (h == h[:, :1]).all()  # every lane of a warp saw every hook call
    if not dynamic:
        per_thread = np.zeros(T * N, dtype=np.int64)
        np.add.at(per_thread, i % (T * N), L)  # Fig. 5: iteration i on thread i mod T*N
        assert (h[:, 0] == per_thread.reshape(-1, 32).max(axis=1)).all()
