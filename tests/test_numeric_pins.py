"""Pins of the numeric-factorization oracle (oracle/numeric.py, Alg. 2).

Each check is independent of Alg. 2's loop structure: the dense product L U, SciPy's LAPACK LU,
a closed form, the Thomas recurrence, and structural zeros of a dense elimination.
"""
import numpy as np
import pytest
import scipy.linalg

import oracle
from oracle import numeric
from inputs import gen
from tests import pins


def _factor(rp, ci, seed):
    val_a = gen.dominant_values(rp, ci, seed)
    r = oracle.fill2(rp, ci)
    As = numeric.scatter(rp, ci, val_a, r["row_ptr"], r["col_idx"])
    out = numeric.factor(r["row_ptr"], r["col_idx"], As)
    A = np.zeros((len(rp) - 1,) * 2)
    for i in range(len(rp) - 1):
        A[i, ci[rp[i]:rp[i + 1]]] = val_a[rp[i]:rp[i + 1]]
    return A, r, out


def test_lu_product_reconstructs_a():
    """L U == A (dense product, any plausible slip in Alg. 2 — a dropped update, a wrong
    operand, the division on the wrong side — breaks it)."""
    rng = np.random.default_rng(7)
    for case in range(150):
        n = int(rng.integers(1, 36))
        rp, ci = gen.random_pattern(n, float(rng.uniform(0.5, 3.5)), seed=1000 + case,
                                    zero_free_diag=True, sym_frac=float(rng.uniform(0, 1)))
        A, r, out = _factor(rp, ci, case)
        L, U = numeric.to_dense_lu(r["row_ptr"], r["col_idx"], out)
        np.testing.assert_allclose(L @ U, A, rtol=0, atol=1e-12 * max(1.0, np.abs(A).max()))


def test_matches_lapack_lu_without_pivots():
    """Column-diagonally-dominant A: LAPACK's partial pivoting picks no swap (P = I), so its
    L and U are the pivot-free factors Alg. 2 computes."""
    for case, (rp, ci) in enumerate([gen.lap2d(6), gen.lap3d(3), gen.arrow_first(12),
                                     gen.arrow_last(12), gen.band(20, 3),
                                     gen.random_pattern(30, 2.5, seed=3, zero_free_diag=True,
                                                        sym_frac=0.3)]):
        A, r, out = _factor(rp, ci, 50 + case)
        P, Lr, Ur = scipy.linalg.lu(A)
        assert np.array_equal(P, np.eye(len(A)))
        L, U = numeric.to_dense_lu(r["row_ptr"], r["col_idx"], out)
        np.testing.assert_allclose(L, Lr, rtol=1e-12, atol=1e-13)
        np.testing.assert_allclose(U, Ur, rtol=1e-12, atol=1e-12 * np.abs(A).max())


def test_two_by_two_closed_form():
    rp = np.array([0, 2, 4], dtype=np.int64)
    ci = np.array([0, 1, 0, 1], dtype=np.int32)
    a, b, c, d = 4.0, 2.0, 3.0, 5.0
    out = numeric.factor(rp, ci, np.array([a, b, c, d]))
    assert out[0] == a and out[1] == b
    assert out[2] == pytest.approx(c / a, rel=1e-15)
    assert out[3] == pytest.approx(d - c * b / a, rel=1e-15)


def test_tridiagonal_thomas_recurrence():
    """Tridiagonal A: U(i,i) = b_i - a_i c_{i-1} / U(i-1,i-1), L(i,i-1) = a_i / U(i-1,i-1),
    U(i,i+1) = c_i (the Thomas algorithm)."""
    n = 40
    rp, ci = gen.tridiag(n)
    A, r, out = _factor(rp, ci, 9)
    L, U = numeric.to_dense_lu(r["row_ptr"], r["col_idx"], out)
    d = A[0, 0]
    assert U[0, 0] == d
    for i in range(1, n):
        l = A[i, i - 1] / d
        d = A[i, i] - l * A[i - 1, i]
        assert L[i, i - 1] == pytest.approx(l, rel=1e-14)
        assert U[i, i] == pytest.approx(d, rel=1e-14)
        assert U[i - 1, i] == A[i - 1, i]


def test_dense_elimination_zeros_outside_pattern():
    """Dense Gaussian elimination with generic values leaves exact zeros outside the symbolic
    pattern (Theorem 1) — ties the numeric oracle's output support to fill2's."""
    for seed in range(20):
        rp, ci = gen.random_pattern(25, 2.0, seed=seed, zero_free_diag=True, sym_frac=0.5)
        A, r, out = _factor(rp, ci, seed)
        _, Lr, Ur = scipy.linalg.lu(A)
        S = pins.to_dense(r["row_ptr"], r["col_idx"], len(A))
        assert np.all((Lr - np.eye(len(A)))[~S.astype(bool)] == 0)
        assert np.all(Ur[~S.astype(bool)] == 0)


def test_pattern_not_closed_raises():
    """Alg. 2 on a pattern missing a fill entry: the update (1,2) has nowhere to go."""
    rp = np.array([0, 3, 5, 7], dtype=np.int64)           # (0,*) full; (1,0),(1,1); (2,0),(2,2)
    ci = np.array([0, 1, 2, 0, 1, 0, 2], dtype=np.int32)  # fill (1,2) and (2,1) absent
    with pytest.raises(ValueError):
        numeric.factor(rp, ci, np.array([4.0, 1, 1, 1, 4, 1, 4]))


def test_zero_pivot_raises():
    rp = np.array([0, 1, 2], dtype=np.int64)
    ci = np.array([0, 1], dtype=np.int32)
    with pytest.raises(ZeroDivisionError):
        numeric.factor(rp, ci, np.array([0.0, 1.0]))
