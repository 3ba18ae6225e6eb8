"""Oracle pins: generic-mode semantics and ICV values.

Expected ICV values are the OpenMP 5.1 definitions: inside a parallel
region of N threads level=1, active-level=(N>1); nested regions are serialized."""
import numpy as np
import pytest

import gen
import oracle


@pytest.mark.parametrize("teams,N,inner", [(3, 256, 256), (4, 96, 256), (2, 33, 256), (3, 5, 7),
                                           (2, 1, 16), (1, 300, 256)])
def test_generic_owner_and_join(teams, N, inner):
    inp = gen.generic_inputs(teams, inner)
    out, owner, post = oracle.generic_team(teams, N, inner, inp)
    # team `for` = Fig. 5 within the team: j -> thread j mod N (exactly once by construction)
    assert (owner.reshape(teams, inner) == np.arange(inner) % N).all()
    # join visibility + permutation invariant: sum_j w[perm j]/s = 1, so post = 1 + s
    for t in range(teams):
        s = (t + 1) * np.sum(inp[t * inner:(t + 1) * inner])
        assert abs(post[t] - (1.0 + s)) <= 1e-12 * (1.0 + s)


def test_generic_constant_input_closed_form():
    teams, inner = 5, 256
    out, owner, post = oracle.generic_team(teams, 64, inner, np.ones(teams * inner))
    # w = t+1, s = 256 (t+1) exactly  ->  out = 1/256 + (t+1) exactly
    expect = np.repeat(np.arange(1, teams + 1) + 1.0 / 256, inner)
    assert (out == expect).all()


def test_generic_perm_is_bijection():
    teams, inner = 3, 256
    inp = np.tile(np.arange(1, inner + 1, dtype=np.float64), teams)
    out, _, _ = oracle.generic_team(teams, 256, inner, inp)
    for t in range(teams):
        w = (t + 1) * np.arange(1, inner + 1, dtype=np.float64)
        s = w.sum()
        o = out[t * inner:(t + 1) * inner]
        recovered = np.rint((o - w) * s / (t + 1)).astype(int) - 1
        assert sorted(recovered) == list(range(inner))


@pytest.mark.parametrize("N", [1, 2, 64, 256])
def test_icv_table_openmp_values(N):
    teams = 3
    rec = oracle.icv_table(teams, N, nested_request=4)
    for t in range(teams):
        # prologue on the main thread: thread 0 of 1, level 0, not in parallel
        assert list(rec[t, 0]) == [0, 1, 0, 0, 0, t, teams]
        for k in range(N):
            active = 1 if N > 1 else 0
            assert list(rec[t, 1 + k]) == [k, N, 1, active, active, t, teams]
            # nested parallel: serialized -> thread 0 of 1, level 2, active level unchanged
            assert list(rec[t, 1 + N + k]) == [0, 1, 2, active, active, t, teams]
            # after the nested region the thread's environment is the outer one again
            assert list(rec[t, 1 + 2 * N + k]) == [k, N, 1, active, active, t, teams]


def _recover_perm(teams, inner, t):
    """perm of team t recovered from the oracle's outputs: with in = 1..n, w[k] = (t+1)(k+1)
    and out[j] = w[perm[j]]/s + w[j], so perm[j] = (out[j] - w[j]) s/(t+1) - 1."""
    inp = np.tile(np.arange(1, inner + 1, dtype=np.float64), teams)
    out, _, _ = oracle.generic_team(teams, 64, inner, inp)
    w = (t + 1) * np.arange(1, inner + 1, dtype=np.float64)
    o = out[t * inner:(t + 1) * inner]
    return np.rint((o - w) * w.sum() / (t + 1)).astype(int) - 1


def test_generic_perm_hand_derived_golden():
    """The prologue's permutation (App. A.4, reading R-A1: perm[k] = (17k + t) mod n) at
    hand-derived entries (tests/golden/generic_perm.txt), recovered from the oracle's
    outputs -- a wrong bijection (another multiplier or offset) fails here."""
    import os
    rows = np.loadtxt(os.path.join(os.path.dirname(__file__), "golden", "generic_perm.txt"),
                      dtype=np.int64, comments="#")
    cache = {}
    for t, n, k, p in rows:
        key = (int(t), int(n))
        if key not in cache:
            cache[key] = _recover_perm(int(t) + 1, int(n), int(t))
        assert cache[key][k] == p, (t, n, k)
