"""Pins of O1 (oracle/ref: the plain definition y = A·x) to things other
than itself: exact rational arithmetic, closed forms, an ill-conditioned case that
defeats naive summation, and scipy's CSR product.  CPU only."""
from fractions import Fraction

import numpy as np
import pytest
import scipy.sparse as sp

import synth
from oracle import ref


def _exact(csr, x):
    out = []
    for i in range(csr.m):
        s = Fraction(0)
        for k in range(csr.row_ptr[i], csr.row_ptr[i + 1]):
            s += Fraction(float(csr.val[k])) * Fraction(float(x[csr.col[k]]))
        out.append(s)
    return out


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("seed", range(8))
def test_against_exact_rationals(seed, dtype):
    a = synth.random_tiny(seed, m=20, n=23, density=0.6, dtype=dtype, integer=False)
    x = synth.make_x(a.n, dtype, "uniform", seed)
    y, b = ref.spmv(a.row_ptr, a.col, a.val, x)
    ex = _exact(a, x)
    u = 2.0 ** -53
    for i in range(a.m):
        err = abs(Fraction(y[i]) - ex[i])
        # Dot2: |err| <= u|y| + gamma_{n}^2 bound  (Ogita-Rump-Oishi 2005, Thm 4.7)
        assert err <= Fraction(u) * abs(ex[i]) + Fraction(1e-28) * Fraction(b[i]) + Fraction(1e-300)


def test_ill_conditioned_row_needs_compensation():
    # 1e16 + 1 - 1e16: naive fp64 summation returns 0, the exact value is 1
    rp = np.array([0, 3], dtype=np.int64)
    col = np.array([0, 1, 2], dtype=np.int32)
    val = np.array([1e16, 1.0, -1e16])
    y, b = ref.spmv(rp, col, val, np.ones(3))
    assert y[0] == 1.0
    assert b[0] == 2e16 + 1.0


def test_laplacian_row_sums_closed_form():
    a = synth.laplacian_2d(64)
    y, _ = ref.spmv(a.row_ptr, a.col, a.val, np.ones(a.n))
    g = y.reshape(64, 64)
    # Dirichlet 5-point rows sum to 4 - (#neighbours): 0 inside, 1 on edges, 2 at corners
    expect = np.zeros((64, 64))
    expect[0, :] += 1; expect[-1, :] += 1; expect[:, 0] += 1; expect[:, -1] += 1
    assert np.array_equal(g, expect)
    assert a.nnz == 20224


def test_rank_one_dense():
    rng = np.random.default_rng(3)
    u = rng.integers(-5, 6, size=37).astype(np.float64)
    v = rng.integers(-5, 6, size=41).astype(np.float64)
    A = np.outer(u, v)
    rp = np.arange(0, 37 * 41 + 1, 41, dtype=np.int64)
    col = np.tile(np.arange(41, dtype=np.int32), 37)
    x = rng.integers(-3, 4, size=41).astype(np.float64)
    y, _ = ref.spmv(rp, col, A.reshape(-1), x)
    assert np.array_equal(y, u * float(v @ x))


@pytest.mark.parametrize("dtype", [np.float32, np.float64])
def test_matches_scipy(dtype):
    a = synth.webbase_like(m=20000, dtype=dtype)
    x = synth.make_x(a.n, dtype, "unit", 1)
    y, b = ref.spmv(a.row_ptr, a.col, a.val, x)
    S = sp.csr_matrix((a.val.astype(np.float64), a.col, a.row_ptr), shape=(a.m, a.n))
    ys = S @ x.astype(np.float64)
    assert np.all(np.abs(y - ys) <= 1e-14 * b + 1e-300)
    assert np.allclose(b, abs(S) @ np.abs(x.astype(np.float64)), rtol=1e-14, atol=0)


def test_rows_subset_and_tolerance_helper():
    a = synth.fem_like("cantilever")
    x = synth.make_x(a.n, np.float32, "uniform", 2)
    y, b = ref.spmv(a.row_ptr, a.col, a.val, x)
    rows = np.array([0, 5, 777, a.m - 1])
    ys, bs = ref.spmv_rows(rows, a.row_ptr, a.col, a.val, x)
    assert np.array_equal(ys, y[rows]) and np.array_equal(bs, b[rows])
    ok, worst = ref.check_tolerance(y.astype(np.float32), y, b, np.float32)
    assert ok and worst <= 0.1          # rounding to fp32 costs <= 2^-24 |y| <= 6e-8 bound
    bad = y.copy(); bad[3] += 1e-3 * b[3]
    assert not ref.check_tolerance(bad, y, b, np.float32)[0]
