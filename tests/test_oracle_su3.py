"""Oracle pins: SU(3) link multiply (GridMini-shaped P:268)."""
import math

import numpy as np

import gen
import oracle


def test_identity_gives_a_exactly():
    A, B = gen.su3_inputs(257, "identity")
    C = oracle.su3_mult(A, B, 257)
    assert (C == A).all()


def test_one_third_closed_form():
    """A = 1+0i, B = 1/3+0i: three fmas of 1*(1/3) land on the tie 1-2^-54 -> 1.0 exactly."""
    n = 100
    A, B = gen.su3_inputs(n, "third")
    C = oracle.su3_mult(A, B, n)
    re = C.reshape(n, 4, 3, 3, 2)[..., 0]
    im = C.reshape(n, 4, 3, 3, 2)[..., 1]
    assert (re == 1.0).all() and (im == 0.0).all()
    assert oracle.sum_f64(re.reshape(-1)) == 36.0 * n


def test_random_against_einsum():
    n = 1000
    A, B = gen.su3_inputs(n)
    C = oracle.su3_mult(A, B, n, threads=3)
    a = A.reshape(n, 4, 3, 3, 2)
    b = B.reshape(4, 3, 3, 2)
    ac = a[..., 0] + 1j * a[..., 1]
    bc = b[..., 0] + 1j * b[..., 1]
    ref = np.einsum("slrm,lmc->slrc", ac, bc)
    c = C.reshape(n, 4, 3, 3, 2)
    err = np.abs(c[..., 0] + 1j * c[..., 1] - ref).max()
    assert err < 1e-14
    # transposed-operand mutation would be caught: B^T gives a different product
    ref_t = np.einsum("slrm,lcm->slrc", ac, bc)
    assert np.abs(ref_t - ref).max() > 1e-3


def test_checksum_tolerance_reference():
    n = 4096
    A, B = gen.su3_inputs(n)
    C = oracle.su3_mult(A, B, n)
    re = C.reshape(-1)[0::2]
    assert abs(oracle.sum_f64(re) - math.fsum(re)) <= 1e-15 * oracle.sum_abs_f64(re)


def test_su3_input_shards_tile_the_lattice():
    """A rank's shard of the inputs (first_site) is the same slice of the one lattice."""
    import gen
    A, B = gen.su3_inputs(100)
    for s0, n in [(0, 40), (40, 35), (75, 25)]:
        a, b = gen.su3_inputs(n, first_site=s0)
        assert (a == A[s0 * 72:(s0 + n) * 72]).all() and (b == B).all()
