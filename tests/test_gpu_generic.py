"""GPU parity: generic mode (P:87, P:92 state machine, P:110-112 alloc_shared stack with
global fallback) and ICV queries with/without thread ICV states."""
import numpy as np
import pytest
import torch

import gen
import oracle

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def _generic(rt, fn, teams, N, inner, flags=0, post=False):
    inp = gen.generic_inputs(teams, inner)
    out = torch.full((max(teams * inner, 1),), float("nan"), dtype=torch.float64, device=DEV)
    owner = torch.full((max(teams * inner, 1),), -1, dtype=torch.int32, device=DEV)
    pst = torch.zeros(teams, dtype=torch.float64, device=DEV) if post else None
    fn(teams, N, inner, torch.from_numpy(inp).to(DEV), out, owner, pst,
       flags | (rt.OMPRT_POSTLOGUE if post else 0))
    torch.cuda.synchronize()
    return (inp, out.cpu().numpy()[: teams * inner], owner.cpu().numpy()[: teams * inner],
            pst.cpu().numpy() if post else None)


# odd inner_n: rows start 8 mod 16 B for odd teams (the prologue's bulk-copied span then
# starts one element early and its last element is read separately); 513 spans 3 chunks
@pytest.mark.parametrize("teams,N,inner", [(64, 256, 256), (64, 96, 256), (64, 33, 256),
                                           (4096, 256, 256), (7, 64, 100), (3, 128, 1),
                                           (9, 64, 33), (5, 64, 513)])
@pytest.mark.parametrize("variant", ["custom", "general", "twin", "custom_assume"])
def test_generic_bit_exact(rt, teams, N, inner, variant):
    if variant == "custom_assume" and inner > N:
        pytest.skip("assumption needs inner_n <= threads")
    if variant == "twin" and inner > 256:
        pytest.skip("the CUDA twin supports inner_n <= 256")
    flags = {"custom": 0, "general": rt.OMPRT_GENERAL_SM, "twin": 0,
             "custom_assume": rt.OMPRT_ASSUME_OVERSUB}[variant]
    fn = rt.omprt_cuda_generic_team if variant == "twin" else rt.omprt_generic_team
    inp, out, owner, _ = _generic(rt, fn, teams, N, inner, flags)
    o_ref, own_ref, _ = oracle.generic_team(teams, N, inner, inp)
    assert (out == o_ref).all()
    assert (owner == own_ref).all()


@pytest.mark.parametrize("variant", ["custom", "general", "twin"])
def test_generic_postlogue_join_visibility(rt, variant):
    teams, N, inner = 64, 96, 256
    flags = rt.OMPRT_GENERAL_SM if variant == "general" else 0
    fn = rt.omprt_cuda_generic_team if variant == "twin" else rt.omprt_generic_team
    inp, out, owner, post = _generic(rt, fn, teams, N, inner, flags, post=True)
    o_ref, _, p_ref = oracle.generic_team(teams, N, inner, inp)
    assert (out == o_ref).all()
    assert (post == p_ref).all()  # the main thread summed the region's writes after the join


@pytest.mark.parametrize("stack", ["4K", "2K", "0"])
@pytest.mark.parametrize("sm", ["custom", "general"])
def test_fallback_transparency(rt, stack, sm):
    """a full stack spills to global memory transparently -- identical bits."""
    flags = {"4K": 0, "2K": rt.OMPRT_SMALL_STACK, "0": rt.OMPRT_NO_STACK}[stack]
    flags |= rt.OMPRT_GENERAL_SM if sm == "general" else 0
    inp, out, owner, _ = _generic(rt, rt.omprt_generic_team, 64, 256, 256, flags)
    o_ref, own_ref, _ = oracle.generic_team(64, 256, 256, inp)
    assert (out == o_ref).all() and (owner == own_ref).all()


def test_large_inner_spills_to_pool(rt):
    """inner_n = 1000 needs 12 KiB of globalized arrays: stack + pool."""
    inp, out, owner, post = _generic(rt, rt.omprt_generic_team, 16, 128, 1000, 0, post=True)
    o_ref, own_ref, p_ref = oracle.generic_team(16, 128, 1000, inp)
    assert (out == o_ref).all() and (owner == own_ref).all() and (post == p_ref).all()


def test_pool_exhaustion_is_reported(rt):
    with pytest.raises(rt.OmprtError) as e:
        _generic(rt, rt.omprt_generic_team, 4, 128, 65536, rt.OMPRT_NO_STACK)
    assert e.value.code == rt.OMPRT_E_STACK


def test_threads_assumption_rejected(rt):
    with pytest.raises(rt.OmprtError) as e:
        _generic(rt, rt.omprt_generic_team, 4, 64, 256, rt.OMPRT_ASSUME_OVERSUB)
    assert e.value.code == rt.OMPRT_E_INVAL


@pytest.mark.parametrize("N", [1, 2, 64, 256])
@pytest.mark.parametrize("variant", ["plain", "thread_states", "general", "debug_ts"])
def test_icv_probe(rt, N, variant):
    teams, nested = 4, 4
    flags = {"plain": 0, "thread_states": rt.OMPRT_THREAD_STATES, "general": rt.OMPRT_GENERAL_SM,
             "debug_ts": rt.OMPRT_THREAD_STATES | rt.OMPRT_DEBUG_BUILD}[variant]
    rec = torch.full((teams * (1 + 3 * N) * 7,), -7, dtype=torch.int32, device=DEV)
    rt.omprt_icv_probe(teams, N, nested, rec, flags)
    torch.cuda.synchronize()
    got = rec.cpu().numpy().reshape(teams, 1 + 3 * N, 7)
    ref = oracle.icv_table(teams, N, nested)
    assert (got == ref).all()


@pytest.mark.parametrize("teams,N,inner", [(64, 256, 256), (64, 96, 256), (7, 64, 100),
                                           (4096, 256, 256)])
@pytest.mark.parametrize("variant", ["spmdize", "spmdize_assume", "deglob", "deglob_assume",
                                     "deglob_general"])
@pytest.mark.parametrize("post", [False, True])
def test_spmdized_and_deglobalized(rt, teams, N, inner, variant, post):
    """NEXT f1 / f2: the SPMDized (guarded prologue, no state machine) and deglobalized
    (static team-local arrays, no stack) forms of C2 give the generic-mode results."""
    if "assume" in variant and inner > N:
        pytest.skip("assumption needs inner_n <= threads")
    flags = {"spmdize": rt.OMPRT_SPMDIZE,
             "spmdize_assume": rt.OMPRT_SPMDIZE | rt.OMPRT_ASSUME_OVERSUB,
             "deglob": rt.OMPRT_DEGLOBALIZE,
             "deglob_assume": rt.OMPRT_DEGLOBALIZE | rt.OMPRT_ASSUME_OVERSUB,
             "deglob_general": rt.OMPRT_DEGLOBALIZE | rt.OMPRT_GENERAL_SM}[variant]
    inp, out, owner, pst = _generic(rt, rt.omprt_generic_team, teams, N, inner, flags, post=post)
    o_ref, own_ref, p_ref = oracle.generic_team(teams, N, inner, inp)
    assert (out == o_ref).all() and (owner == own_ref).all()
    if post:
        assert (pst == p_ref).all()
