"""Pins of the oracle's restarted GMRES(m) and of the identity-preconditioner
option ("further batched Krylov solvers and
preconditioners"; the paper implements "several preconditionable iterative
solvers").  Each test checks the oracle against something
other than itself: exact linear algebra (numpy solve / lstsq), Saad's
residual identity, the minimal polynomial of a diagonal matrix, scipy's
GMRES / BiCGSTAB, and exact power-of-two scaling.
"""
import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.linalg as spla

import oracle as O
import xgcgen as X

from test_oracle import dense_pattern, rand_dd_dense


def _dense_csr(A):
    n = A.shape[0]
    rp, ci = dense_pattern(n)
    return rp, ci, A.ravel().copy()


# ------------------------------------------------------------------ G1 --
@pytest.mark.parametrize("n", [4, 5, 8])
@pytest.mark.parametrize("precond", [O.PREC_JACOBI, O.PREC_NONE])
def test_gmres_finite_termination(n, precond):
    """GMRES(m >= n) reaches the exact solution after at most n Krylov steps
    (the Krylov space is then all of R^n); with rounding, the stop test
    fires at <= n steps and x equals numpy's solve.  Also for matrices that
    are NOT diagonally dominant."""
    rng = np.random.default_rng(7 + n + 10 * precond)
    for trial in range(30):
        A = rand_dd_dense(rng, n) if trial % 2 == 0 else rng.standard_normal((n, n)) + 3 * np.eye(n)
        if abs(np.linalg.det(A)) < 1e-3:
            continue
        b = rng.standard_normal(n)
        rp, ci, v = _dense_csr(A)
        x, R = O.gmres(rp, ci, v, b, restart=n, tol=1e-12, maxiter=10 * n, precond=precond)
        assert R.status == O.CONVERGED
        assert R.iters <= n
        np.testing.assert_allclose(x, np.linalg.solve(A, b), rtol=1e-9, atol=1e-10)


# ------------------------------------------------------------------ G2 --
def test_gmres_givens_estimate_equals_true_residual():
    """Saad Prop. 6.9: after k Krylov steps |g_{k+1}| = ||b - A x_k|| where
    x_k = x0 + M^-1 V_k y_k is formed explicitly: pins H, the rotations and
    the back substitution at every step of every restart cycle."""
    B = X.make_batch(0, 2)
    p = B.pattern
    for j in range(2):
        bn = np.linalg.norm(B.b[j])
        x, R, tr = O.gmres(p.row_ptr, p.col_idx, B.values[j], B.b[j], restart=8, trace=True)
        assert R.status == O.CONVERGED and tr.shape[0] == R.iters
        assert np.all(np.abs(tr[:, 0] - tr[:, 1]) <= 1e-12 * bn)


# ------------------------------------------------------------------ G3 --
def test_gmres_minimal_residual_brute_force():
    """The first cycle's x_k minimises ||b - A x|| over x0 + M^-1 K_k(A M^-1, r0):
    compare the oracle's residual with numpy's least squares over an
    explicitly built (orthonormalised) Krylov basis, k = 1..6."""
    rng = np.random.default_rng(3)
    n = 12
    A = rand_dd_dense(rng, n, margin=0.2)
    b = rng.standard_normal(n)
    x0 = rng.standard_normal(n)
    rp, ci, v = _dense_csr(A)
    d = 1.0 / np.diag(A)
    AM = A * d[None, :]
    r0 = b - A @ x0
    for k in range(1, 7):
        K = np.empty((n, k))
        K[:, 0] = r0
        for i in range(1, k):
            K[:, i] = AM @ K[:, i - 1]
        Q, _ = np.linalg.qr(K)
        y, *_ = np.linalg.lstsq(AM @ Q, r0, rcond=None)
        best = np.linalg.norm(r0 - AM @ Q @ y)
        x, R = O.gmres(rp, ci, v, b, x0=x0, restart=20, tol=0.0, maxiter=k)
        assert R.iters == k
        got = np.linalg.norm(b - A @ x)
        assert abs(got - best) <= 1e-10 * np.linalg.norm(r0), (k, got, best)


# ------------------------------------------------------------------ G4 --
def test_gmres_diagonal_matrices():
    """Jacobi-preconditioned GMRES on a diagonal A: A M^-1 = I -> exactly one
    Krylov step and x = b / diag.  Without preconditioner the number of steps
    equals the degree of the minimal polynomial = number of DISTINCT
    diagonal values (3 here)."""
    n = 30
    diag = np.array([2.0, 5.0, -7.0])[np.arange(n) % 3]
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    b = np.random.default_rng(1).standard_normal(n)
    x, R = O.gmres(rp, ci, diag, b, restart=10)
    assert R.iters == 1 and R.status == O.CONVERGED
    np.testing.assert_allclose(x, b / diag, rtol=1e-15)
    x, R = O.gmres(rp, ci, diag, b, restart=10, precond=O.PREC_NONE, tol=1e-13)
    assert R.iters == 3 and R.status == O.CONVERGED
    np.testing.assert_allclose(x, b / diag, rtol=1e-12)


# ------------------------------------------------------------------ G5 --
def test_gmres_edge_cases():
    B = X.make_batch(0, 2)
    p = B.pattern
    v, b = B.values[1], B.b[1]
    xd = O.banded_solve(p.row_ptr, p.col_idx, v, b)
    x, R = O.gmres(p.row_ptr, p.col_idx, v, b, x0=xd)            # x0 = x*
    assert R.iters == 0 and R.status == O.CONVERGED and np.array_equal(x, xd)
    x, R = O.gmres(p.row_ptr, p.col_idx, v, np.zeros(p.n))       # b = 0
    assert R.iters == 0 and np.all(x == 0)
    x0 = np.ones(p.n)
    x, R = O.gmres(p.row_ptr, p.col_idx, v, b, x0=x0, maxiter=0)  # maxiter = 0
    assert R.iters == 0 and R.status == O.MAXITER and np.array_equal(x, x0)
    x, R = O.gmres(p.row_ptr, p.col_idx, v, b, maxiter=5)         # not converged
    assert R.iters == 5 and R.status == O.MAXITER
    x1, R1 = O.gmres(p.row_ptr, p.col_idx, v, b)                  # x0 NULL == zeros
    x2, R2 = O.gmres(p.row_ptr, p.col_idx, v, b, x0=np.zeros(p.n))
    assert np.array_equal(x1, x2) and R1.iters == R2.iters
    with pytest.raises(ValueError):
        O.gmres(p.row_ptr, p.col_idx, v, b, restart=0)


# ------------------------------------------------------------------ G6 --
@pytest.mark.parametrize("m", [4, 8, 16])
def test_gmres_vs_scipy_and_direct(m):
    """Solutions agree with scipy's restarted GMRES (Jacobi M) and with the
    banded LU; the true relative residual meets the tolerance."""
    B = X.make_batch(0, 4)
    p = B.pattern
    out = O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b, solver=O.SOLVER_GMRES, restart=m)
    xd = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b)
    for j in range(4):
        bn = np.linalg.norm(B.b[j])
        assert out["status"][j] == O.CONVERGED
        assert out["resnorm"][j] / bn < 1e-10
        assert np.linalg.norm(out["x"][j] - xd[j]) / np.linalg.norm(xd[j]) <= 1e-8
        if j < 2:
            A = sp.csr_matrix((B.values[j], p.col_idx, p.row_ptr), shape=(p.n, p.n))
            M = sp.diags(1.0 / A.diagonal())
            xs, info = spla.gmres(A, B.b[j], rtol=1e-13, atol=0.0, restart=m, M=M, maxiter=2000)
            assert info == 0
            assert np.linalg.norm(out["x"][j] - xs) / np.linalg.norm(xs) <= 1e-8
        x1, R1 = O.gmres(p.row_ptr, p.col_idx, B.values[j], B.b[j], restart=m)
        assert np.array_equal(x1, out["x"][j]) and R1.iters == out["iters"][j]


# ------------------------------------------------------------------ G7 --
@pytest.mark.parametrize("k", [-3, 5])
@pytest.mark.parametrize("precond", [O.PREC_JACOBI, O.PREC_NONE])
def test_gmres_power_of_two_scaling_bitwise(k, precond):
    """(2^k A, 2^k b): every quantity scales exactly -> bitwise equal x and
    iteration count (REL_B stop)."""
    B = X.make_batch(0, 2)
    p = B.pattern
    c = 2.0 ** k
    for j in range(2):
        x1, R1 = O.gmres(p.row_ptr, p.col_idx, B.values[j], B.b[j], precond=precond)
        x2, R2 = O.gmres(p.row_ptr, p.col_idx, c * B.values[j], c * B.b[j], precond=precond)
        assert np.array_equal(x1, x2) and R1.iters == R2.iters


# ------------------------------------------------------------------ G8 --
def test_bicgstab_without_preconditioner_vs_scipy():
    """PREC_NONE BiCGSTAB (M = I) agrees with scipy's unpreconditioned
    BiCGSTAB and with the direct solve; Jacobi is the default (bitwise equal
    to the precond-less entry point)."""
    B = X.make_batch(0, 2)
    p = B.pattern
    for j in range(2):
        A = sp.csr_matrix((B.values[j], p.col_idx, p.row_ptr), shape=(p.n, p.n))
        xs, info = spla.bicgstab(A, B.b[j], rtol=1e-13, atol=0.0, maxiter=2000)
        assert info == 0
        x, R = O.bicgstab(p.row_ptr, p.col_idx, B.values[j], B.b[j], precond=O.PREC_NONE)
        assert R.status == O.CONVERGED
        assert np.linalg.norm(x - xs) / np.linalg.norm(xs) <= 1e-8
        xj, Rj = O.bicgstab(p.row_ptr, p.col_idx, B.values[j], B.b[j])
        out = O.batch_bicgstab(p.row_ptr, p.col_idx, B.values[j:j + 1], B.b[j:j + 1])
        assert np.array_equal(xj, out["x"][0])
