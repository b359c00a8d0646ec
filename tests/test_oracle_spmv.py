"""Pins for oracle O4 (Dot2 parity SpMV) and O4' (plain timed SpMV).

Each pin is independent of the oracle's own arithmetic: dense brute force on integer data
(every summation order exact), exact rational arithmetic (fractions), identity and
permutation matrices, math.fsum row sums, scipy.sparse.
"""
import math
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp
import torch

import oracle
import synth

U64 = 2.0 ** -53


def _rand_csr(n, m, density, seed, integer=False):
    rng = np.random.default_rng(seed)
    A = (rng.random((n, m)) < density)
    vals = rng.integers(-8, 9, (n, m)).astype(np.float64) if integer else rng.uniform(-1, 1, (n, m))
    A = np.where(A, vals, 0.0)
    A[A == 0.0] = 0.0
    csr = sp.csr_matrix(A)
    csr.sort_indices()
    return A, csr.indptr.astype(np.int32), csr.indices.astype(np.int32), csr.data.copy()


@pytest.mark.parametrize("seed", range(4))
def test_dense_bruteforce_integer_exact(seed):
    A, rp, ci, v = _rand_csr(64, 48, 0.3, seed, integer=True)
    x = np.random.default_rng(100 + seed).integers(-8, 9, 48).astype(np.float64)
    y, den = oracle.spmv(rp, ci, v, x)
    ref = np.array([sum(int(A[i, j]) * int(x[j]) for j in range(48)) for i in range(64)],
                   dtype=np.float64)
    assert np.array_equal(y, ref)
    assert np.array_equal(den, np.abs(A) @ np.abs(x))


@pytest.mark.parametrize("seed", range(3))
def test_exact_rational_float(seed):
    A, rp, ci, v = _rand_csr(40, 300, 0.5, seed)
    x = np.random.default_rng(7 + seed).uniform(-1, 1, 300)
    y, den = oracle.spmv(rp, ci, v, x)
    for i in range(40):
        exact = sum(Fraction(float(v[k])) * Fraction(float(x[ci[k]])) for k in range(rp[i], rp[i + 1]))
        err = abs(Fraction(float(y[i])) - exact)
        # Dot2: |err| <= u|s| + gamma_n^2 sum|a b|   (Ogita-Rump-Oishi, n <= 300)
        assert err <= U64 * abs(exact) + Fraction(1e-26) * Fraction(float(den[i])), i


def test_adversarial_equal_long_row():
    # 0.1 summed 1e5 times: a plain sequential sum is off by 1.9e-12 relative (SURVEY
    # Appendix A); the parity oracle must be accurate to ~u.
    L = 100_000
    rp = np.array([0, L], np.int32)
    ci = np.zeros(L, np.int32)
    v = np.full(L, 0.1)
    x = np.ones(1)
    y, _ = oracle.spmv(rp, ci, v, x)
    exact = Fraction(0.1) * L
    assert abs(Fraction(float(y[0])) - exact) <= U64 * exact
    yp = oracle.spmv_plain(rp, ci, v, x)
    assert abs(float(yp[0]) - 1e4) > 1e-9  # the plain path really is inaccurate here


def test_identity_and_permutation_bitwise():
    n = 1000
    x = synth.vector(n, 5).numpy()
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    y, _ = oracle.spmv(rp, ci, np.ones(n), x)
    assert np.array_equal(y, x)
    perm = np.random.default_rng(3).permutation(n).astype(np.int32)
    y, _ = oracle.spmv(rp, perm, None, x)  # pattern matrix P: y = P x
    assert np.array_equal(y, x[perm])


def test_row_sums_A_times_ones():
    rp, ci = synth.rmat_csr(10)
    rp, ci = rp.numpy(), ci.numpy()
    v = synth.values(ci.size, 9).numpy()
    y, den = oracle.spmv(rp, ci, v, np.ones(1 << 10))
    for i in range(1 << 10):
        s = math.fsum(v[rp[i]:rp[i + 1]])
        assert abs(y[i] - s) <= U64 * abs(s) + 1e-300
        assert den[i] == pytest.approx(math.fsum(np.abs(v[rp[i]:rp[i + 1]])), rel=1e-15)


def test_scipy_crosscheck_rmat14():
    rp, ci = synth.rmat_csr(14)
    rp, ci = rp.numpy(), ci.numpy()
    n = rp.size - 1
    v = synth.values(ci.size, 1014).numpy()
    x = synth.vector(n, 2014).numpy()
    y, den = oracle.spmv(rp, ci, v, x)
    ys = sp.csr_matrix((v, ci, rp), shape=(n, n)) @ x
    assert np.all(np.abs(y - ys) <= 1e-12 * den)
    empty = np.diff(rp) == 0
    assert np.all(y[empty] == 0.0) and not np.any(np.signbit(y[empty]))


def test_fp32_rounded_once():
    A, rp, ci, v = _rand_csr(50, 200, 0.4, 11)
    v32 = v.astype(np.float32)
    x32 = np.random.default_rng(2).uniform(-1, 1, 200).astype(np.float32)
    y, den = oracle.spmv(rp, ci, v32, x32)
    assert y.dtype == np.float32
    for i in range(50):
        exact = sum(Fraction(float(v32[k])) * Fraction(float(x32[ci[k]])) for k in range(rp[i], rp[i + 1]))
        # correctly rounded to float32 (ties aside): within half an ulp of fp32
        ulp = np.spacing(np.float32(abs(float(exact)) if exact != 0 else 1e-38))
        assert abs(Fraction(float(y[i])) - exact) <= Fraction(float(ulp)) * Fraction(1, 2) * Fraction(1001, 1000)


def test_row_end_slack_equals_standard():
    rp, ci = synth.rmat_csr(12)
    v = synth.values(ci.numel(), 3)
    rb, re, cap, c2, v2 = synth.with_slack(rp, ci, v)
    x = synth.vector(1 << 12, 4).numpy()
    y1, _ = oracle.spmv(rp.numpy(), ci.numpy(), v.numpy(), x)
    y2, _ = oracle.spmv(rb.numpy(), c2.numpy(), v2.numpy(), x, row_end=re.numpy())
    assert np.array_equal(y1, y2)


def test_empty_matrix_and_plain_threads():
    y, den = oracle.spmv(np.zeros(1, np.int32), np.zeros(0, np.int32), np.zeros(0), np.zeros(3))
    assert y.size == 0
    rp, ci = synth.rmat_csr(12)
    rp, ci = rp.numpy(), ci.numpy()
    v = synth.values(ci.size, 3).numpy()
    x = synth.vector(1 << 12, 4).numpy()
    y1 = oracle.spmv_plain(rp, ci, v, x, threads=1)
    y4 = oracle.spmv_plain(rp, ci, v, x, threads=4)
    assert np.array_equal(y1, y4)  # same per-row order regardless of threads
    yd, den = oracle.spmv(rp, ci, v, x)
    assert np.all(np.abs(y1 - yd) <= 1e-12 * den)


# ---------------------------------------------------------------------- fp32 pins (round 2)
def _rand_csr32(n, m, density, seed, integer):
    A, rp, ci, v = _rand_csr(n, m, density, seed, integer=integer)
    return A.astype(np.float32), rp, ci, v.astype(np.float32)


@pytest.mark.parametrize("seed", range(3))
def test_fp32_den_exact_on_integer_data(seed):
    """oracle_spmv_f32's den (the denominator of every fp32 parity bar, reading Q16) equals
    |A| @ |x| exactly on integer data (every partial sum is an exact small integer)."""
    A, rp, ci, v = _rand_csr32(64, 48, 0.3, seed, integer=True)
    x = np.random.default_rng(300 + seed).integers(-8, 9, 48).astype(np.float32)
    y, den = oracle.spmv(rp, ci, v, x)
    assert np.array_equal(den, np.abs(A.astype(np.float64)) @ np.abs(x.astype(np.float64)))
    ref = np.array([sum(int(A[i, j]) * int(x[j]) for j in range(48)) for i in range(64)], np.float32)
    assert np.array_equal(y, ref)


@pytest.mark.parametrize("seed", range(3))
def test_fp32_den_matches_fsum_on_float_data(seed):
    """den on U(-1,1) float data: the exact sum of |a||x| (fractions) within n*u relative
    (it is a plain double accumulation of exact non-negative products)."""
    A, rp, ci, v = _rand_csr32(30, 400, 0.5, seed, integer=False)
    x = np.random.default_rng(9 + seed).uniform(-1, 1, 400).astype(np.float32)
    _, den = oracle.spmv(rp, ci, v, x)
    for i in range(30):
        ex = sum(abs(Fraction(float(v[k])) * Fraction(float(x[ci[k]]))) for k in range(rp[i], rp[i + 1]))
        assert abs(Fraction(float(den[i])) - ex) <= Fraction(400) * Fraction(U64) * ex, i


@pytest.mark.parametrize("seed", range(3))
def test_fp32_plain_is_double_sum_rounded_once(seed):
    """oracle_spmv_plain_f32 (the bitwise checker of the GPU's fp32 window rows): float
    products are exact in double, summed in double, rounded once to float.  Pinned
    against the exact rational row sum: |y - exact| <= ulp32(exact)/2 + n u64 sum|p|."""
    A, rp, ci, v = _rand_csr32(40, 300, 0.5, seed, integer=False)
    x = np.random.default_rng(21 + seed).uniform(-1, 1, 300).astype(np.float32)
    y = oracle.spmv_plain(rp, ci, v, x)
    assert y.dtype == np.float32
    for i in range(40):
        terms = [Fraction(float(v[k])) * Fraction(float(x[ci[k]])) for k in range(rp[i], rp[i + 1])]
        ex = sum(terms, Fraction(0))
        absum = sum((abs(t) for t in terms), Fraction(0))
        half_ulp = Fraction(float(np.spacing(np.float32(abs(float(ex)))))) / 2
        assert abs(Fraction(float(y[i])) - ex) <= half_ulp * Fraction(1001, 1000) + len(terms) * Fraction(U64) * absum, i


def test_fp32_plain_integer_exact_and_in_element_order():
    """Integer data: exact.  Element order: with p = (2^60, 1, -2^60) a left-to-right double
    sum gives 0 (2^60 + 1 rounds to 2^60), while (2^60, -2^60, 1) gives 1 -- IEEE facts,
    so the in-order reading of the window-row checker is pinned, not re-typed."""
    A, rp, ci, v = _rand_csr32(64, 48, 0.3, 5, integer=True)
    x = np.random.default_rng(305).integers(-8, 9, 48).astype(np.float32)
    y = oracle.spmv_plain(rp, ci, v, x)
    assert np.array_equal(y, (A.astype(np.float64) @ x.astype(np.float64)).astype(np.float32))
    big = np.float32(2.0 ** 60)
    rp2 = np.array([0, 3, 6], np.int32)
    ci2 = np.zeros(6, np.int32)
    v2 = np.array([big, 1, -big, big, -big, 1], np.float32)
    y2 = oracle.spmv_plain(rp2, ci2, v2, np.ones(1, np.float32))
    assert y2[0] == 0.0 and y2[1] == 1.0
    y64 = oracle.spmv_plain(rp2, ci2, v2.astype(np.float64), np.ones(1))
    assert y64[0] == 0.0 and y64[1] == 1.0
