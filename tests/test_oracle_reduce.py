"""Oracle pins: C1 axpy + sum (BASELINE configs[0]) and the reduction semantics."""
import math
from fractions import Fraction

import numpy as np

import gen
import oracle


def test_axpy_integer_valued_closed_form():
    """SURVEY §8(c) C2 pin (i): x=2, b=i mod 1024, c=1 -> sum = 2*sum(i mod 1024) + n = 2^30."""
    n = 1 << 20
    x, b, c = gen.axpy_inputs(n, exact=True)
    a = oracle.axpy(x, b, c)
    assert (a == 2 * (np.arange(n) % 1024) + 1).all()
    assert oracle.sum_f64(a) == float(1 << 30)
    assert oracle.sum_f64(a, 5.0) == float((1 << 30) + 5)


def test_axpy_is_single_rounding_fma():
    """a = fma(x,b,c): the exact x*b+c rounded once (Fraction -> float is correctly rounded)."""
    x, b, c = gen.axpy_inputs(4096)
    a = oracle.axpy(x, b, c)
    for i in range(0, 4096, 7):
        exact = Fraction(x) * Fraction(float(b[i])) + Fraction(float(c[i]))
        assert a[i] == float(exact)
    # and differs from the twice-rounded form somewhere (the pin can fail)
    assert (a != (x * b) + c).any()


def test_sum_against_exact_fsum_and_long_double():
    x, b, c = gen.axpy_inputs((1 << 20) + 7)
    a = oracle.axpy(x, b, c)
    exact = math.fsum(a)  # correctly rounded sum
    assert oracle.sum_f64(a) == exact
    assert abs(float(oracle.sum_f64_ld(a)) - exact) <= 1e-15 * exact
    # init value is added (OpenMP reduction: orig (+) partials)
    assert oracle.sum_f64(a, 1.25) == math.fsum(list(a) + [1.25])
    assert abs(oracle.sum_abs_f64(-a) - exact) <= 1e-12 * exact


def test_reduce_u64_wraps_and_ops():
    rng = np.random.default_rng(1)
    v = rng.integers(0, 2**63, size=10001, dtype=np.uint64) * np.uint64(3)
    s = (sum(int(t) for t in v) + 12345) % 2**64
    assert oracle.reduce_u64(v, oracle.OP_ADD, 12345) == s
    w = np.array([3, 5, 7], np.uint64)
    assert oracle.reduce_u64(w, oracle.OP_MUL, 2) == 210
    assert oracle.reduce_u64(v, oracle.OP_MIN, 2**64 - 1) == int(v.min())
    assert oracle.reduce_u64(v, oracle.OP_MAX, 0) == int(v.max())
    assert oracle.reduce_u64(v[:0], oracle.OP_ADD, 9) == 9  # empty: orig only


def test_reduce_f64_ops():
    v = gen.uniform(7, 999, -2.0, 3.0)
    assert oracle.reduce_f64(v, oracle.OP_ADD, 0.5) == math.fsum(list(v) + [0.5])
    assert oracle.reduce_f64(v, oracle.OP_MIN, 10.0) == v.min()
    assert oracle.reduce_f64(v, oracle.OP_MAX, -10.0) == v.max()
    assert oracle.reduce_f64(v, oracle.OP_MIN, -10.0) == -10.0
    assert oracle.reduce_f64(np.array([2.0, 0.5, 4.0]), oracle.OP_MUL, 3.0) == 12.0
