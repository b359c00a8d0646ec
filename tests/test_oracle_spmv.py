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
