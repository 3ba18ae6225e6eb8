"""Oracle pins: the Fig. 5 static schedule (§III-F).

Two independent oracle implementations (closed form, literal Fig. 5 transliteration) are
checked against each other by brute force over every tiny shape, against the exactly-once
invariant, and against a hand-derived worked example of Fig. 5 (tests/golden)."""
import os

import numpy as np
import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "fig5_n10_T2_N3.txt")


def test_closed_form_equals_literal_fig5_bruteforce():
    for n in range(0, 71):
        for T in range(1, 6):
            for N in range(1, 10):
                owner, count = oracle.fig5_simulate(n, T, N)
                assert (count == 1).all(), (n, T, N)  # every iteration exactly once
                for iv in range(n):
                    tm, th = oracle.static_owner_closed(iv, n, T, N)
                    assert owner[iv] == tm * N + th, (n, T, N, iv)


def test_worked_example_fig5():
    rows = np.loadtxt(GOLD, dtype=np.int64, comments="#")
    owner, count = oracle.fig5_simulate(10, 2, 3)
    assert (count == 1).all()
    assert (owner == rows[:, 3]).all()
    for iv, tm, th, g in rows:
        assert oracle.static_owner_closed(int(iv), 10, 2, 3) == (tm, th)
    # the assumption breaks after one iteration: IV >= T*N never runs
    owner_a, count_a = oracle.fig5_simulate(10, 2, 3, assume_oversub=True)
    assert (count_a[:6] == 1).all() and (count_a[6:] == 0).all()


@pytest.mark.parametrize("n,T,N", [(0, 1, 1), (1, 8, 128), (1023, 8, 128), (1024, 8, 128),
                                   (1025, 8, 128), (7, 3, 5), (15, 3, 5), (16, 3, 5)])
def test_special_cases(n, T, N):
    owner, count = oracle.fig5_simulate(n, T, N)
    assert (count == 1).all()
    # n < T*N: threads g >= n idle;   n = k*T*N + r: thread g runs ceil((n-g)/(T*N)) iters
    runs = np.bincount(owner, minlength=T * N) if n else np.zeros(T * N, np.int64)
    g = np.arange(T * N)
    expect = np.where(g < n, (n - g + T * N - 1) // (T * N), 0)
    assert (runs == expect).all()


def test_assumption_equivalent_when_it_holds():
    for n in range(0, 40):
        for T in range(1, 5):
            for N in range(1, 8):
                if n > T * N:
                    continue
                a = oracle.fig5_simulate(n, T, N, assume_oversub=True)
                b = oracle.fig5_simulate(n, T, N, assume_oversub=False)
                assert (a[0] == b[0]).all() and (a[1] == b[1]).all()


def test_team_for_and_distribute_readings():
    # Q2: `for` in a team = Fig. 5 with NumBlocks=1; `distribute` = Fig. 5 with NumThreads=1
    for n in range(0, 50):
        for N in range(1, 9):
            owner, count = oracle.team_for_simulate(n, N)
            assert (count == 1).all() and (owner == np.arange(n) % N).all()
        for T in range(1, 6):
            owner, count = oracle.distribute_simulate(n, T)
            assert (count == 1).all() and (owner == np.arange(n) % T).all()


def test_cyclic_not_blocked():
    """the combined scheme is CUDA-style cyclic (chunk 1), not OpenMP's blocked
    schedule(static): consecutive iterations go to consecutive threads."""
    owner, _ = oracle.fig5_simulate(64, 2, 4)
    assert list(owner[:9]) == [0, 1, 2, 3, 4, 5, 6, 7, 0]


def test_chunked_schedule_closed_form_and_literal():
    """NEXT f3 (reading R-F3): chunk k -> global thread k mod (T*N); brute force over tiny
    shapes, exactly-once, and C = 1 reduces to Fig. 5 (the independent pin)."""
    for n in range(0, 60):
        for C in range(1, 7):
            for T in range(1, 4):
                for N in range(1, 6):
                    owner, count = oracle.chunk_simulate(n, C, T, N)
                    assert (count == 1).all()
                    for iv in range(n):
                        tm, th = oracle.static_chunk_owner_closed(iv, n, C, T, N)
                        assert owner[iv] == tm * N + th
                    if C == 1:
                        f5, _ = oracle.fig5_simulate(n, T, N)
                        assert (owner == f5).all()


def test_chunked_schedule_special_cases():
    owner, count = oracle.chunk_simulate(100, 1000, 4, 8)   # one chunk: all on thread 0
    assert (owner == 0).all() and (count == 1).all()
    owner, count = oracle.chunk_simulate(64, 4, 2, 8)        # consecutive chunks, round robin
    assert list(owner[:12]) == [0, 0, 0, 0, 1, 1, 1, 1, 2, 2, 2, 2]
    # assumption n <= T*N*C: at most one chunk per thread, identical assignment
    a = oracle.chunk_simulate(63, 4, 2, 8, assume_oversub=True)
    b = oracle.chunk_simulate(63, 4, 2, 8)
    assert (a[0] == b[0]).all() and (a[1] == b[1]).all()


def _check_dynamic(n, C, T, N, owner, count):
    """Structural pins of schedule(dynamic, C) under a blocked distribute (reading R-D1),
    none of which restates the oracle's loop: exactly once; team t's iterations are one
    contiguous run, in team order, every full team holding ceil(n/T); a chunk of C
    iterations of the team's run stays on one thread; thread k's first chunk is chunk k."""
    assert (count == 1).all()
    B = -(-n // T) if n else 0
    team = owner // N
    assert (np.diff(team) >= 0).all()                      # contiguous, ascending teams
    sizes = np.bincount(team, minlength=T) if n else np.zeros(T, np.int64)
    full = sizes[sizes > 0]
    assert (full[:-1] == B).all() and (full[-1:] <= B).all()
    start = 0
    for t in range(T):
        run = owner[start:start + sizes[t]]
        for c0 in range(0, len(run), C):
            assert (run[c0:c0 + C] == run[c0]).all()       # a chunk on one thread
        for k in range(min(N, -(-len(run) // C))):
            assert run[k * C] == t * N + k                 # thread k starts with chunk k
        start += sizes[t]


def test_dynamic_schedule_invariants_bruteforce():
    for n in range(0, 50):
        for C in (1, 2, 3, 5):
            for T in (1, 2, 3):
                for N in (1, 2, 4):
                    for seed in (0, 1):
                        owner, count = oracle.dynamic_simulate(n, C, T, N, seed)
                        _check_dynamic(n, C, T, N, owner, count)
                        for iv in range(n):
                            assert oracle.dynamic_team_closed(iv, n, T) == owner[iv] // N


def test_dynamic_schedule_special_cases():
    # one thread per team: the blocked distribute itself
    owner, _ = oracle.dynamic_simulate(10, 1, 3, 1, 7)
    assert list(owner) == [0, 0, 0, 0, 1, 1, 1, 1, 2, 2]
    # a chunk covering the whole block: thread 0 of each team runs its block
    owner, _ = oracle.dynamic_simulate(40, 64, 4, 8, 3)
    assert list(owner) == [t * 8 for t in range(4) for _ in range(10)]
    # different request orders are different (legal) executions of the same schedule
    a, _ = oracle.dynamic_simulate(4000, 2, 2, 16, 1)
    b, _ = oracle.dynamic_simulate(4000, 2, 2, 16, 2)
    assert (a != b).any() and ((a // 16) == (b // 16)).all()
    _check_dynamic(4000, 2, 2, 16, a, np.ones(4000, np.int32))
    assert oracle.dynamic_team_closed(-1, 10, 2) is None
