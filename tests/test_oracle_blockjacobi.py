"""Pins of the oracle's block-Jacobi preconditioner ("block-
Jacobi"; R30): M = block diagonal of A with blocks of bs consecutive
rows, each solved exactly (dgetf2/dgetrs order).  Every check compares against
something other than the oracle itself: numpy's dense solve of the explicit
block-diagonal matrix, the exact-inverse special case (one iteration), the
scalar-Jacobi path in an exactly representable case, scipy's BiCGSTAB with the
same M, and the direct (banded LU) solution."""
import numpy as np
import pytest
import scipy.sparse as sp
import scipy.sparse.linalg as spla

import oracle as O
import xgcgen as X


def dense(row_ptr, col_idx, val):
    n = len(row_ptr) - 1
    A = np.zeros((n, n))
    rows = np.repeat(np.arange(n), np.diff(row_ptr))
    np.add.at(A, (rows, col_idx), val)
    return A


def block_diag_part(A, bs):
    M = np.zeros_like(A)
    for r0 in range(0, A.shape[0], bs):
        r1 = min(A.shape[0], r0 + bs)
        M[r0:r1, r0:r1] = A[r0:r1, r0:r1]
    return M


@pytest.mark.parametrize("bs", [1, 3, 8, 32])
def test_apply_equals_dense_block_solve_xgc(bs):
    """B1: M^-1 y = numpy.linalg.solve(blockdiag(A), y) on an XGC electron."""
    B = X.make_batch(1, 1)
    p = B.pattern
    M = block_diag_part(dense(p.row_ptr, p.col_idx, B.values[0]), bs)
    y = np.random.default_rng(bs).standard_normal(p.n)
    out = O.precond_apply(p.row_ptr, p.col_idx, B.values[0], y, O.block_jacobi(bs))
    ref = np.linalg.solve(M, y)
    assert np.linalg.norm(out - ref) <= 1e-13 * np.linalg.norm(ref)


def test_apply_with_pivoting_blocks():
    """B1': random blocks with tiny diagonals force row interchanges inside
    the block factorisation (partial pivoting); still the exact block solve."""
    rp, ci = X.random_pattern(40, 9, seed=5, density=0.9)
    rng = np.random.default_rng(3)
    v = rng.standard_normal(len(ci))
    rows = np.repeat(np.arange(40), np.diff(rp))
    v[ci == rows] *= 1e-3
    M = block_diag_part(dense(rp, ci, v), 8)
    y = rng.standard_normal(40)
    out = O.precond_apply(rp, ci, v, y, O.block_jacobi(8))
    ref = np.linalg.solve(M, y)
    assert np.linalg.norm(out - ref) <= 1e-10 * np.linalg.norm(ref)


def test_default_block_size_is_8():
    B = X.make_batch(0, 1)
    p = B.pattern
    y = np.linspace(-1, 1, p.n)
    a = O.precond_apply(p.row_ptr, p.col_idx, B.values[0], y, O.PREC_BLOCK_JACOBI)
    b = O.precond_apply(p.row_ptr, p.col_idx, B.values[0], y, O.block_jacobi(8))
    assert np.array_equal(a, b)


def test_singular_block_is_identity():
    """R30: a block with an exactly zero pivot is used as the identity."""
    A = np.array([[1., 1, 1, 0], [1, 1, 0, 1], [1, 0, 2, 0], [0, 1, 0, 2]])
    rp = np.array([0, 3, 6, 8, 10], np.int32)
    ci = np.array([0, 1, 2, 0, 1, 3, 0, 2, 1, 3], np.int32)
    v = A[np.repeat(np.arange(4), np.diff(rp)), ci]
    y = np.array([3.0, -5.0, 4.0, 6.0])
    out = O.precond_apply(rp, ci, v, y, O.block_jacobi(2))
    assert np.array_equal(out, [3.0, -5.0, 2.0, 3.0])


def _block_diagonal_system(bs, seed=0):
    """XGC electron values with every coupling across blocks of bs rows removed."""
    B = X.make_batch(1, 1, seed=seed)
    p = B.pattern
    rows = np.repeat(np.arange(p.n), np.diff(p.row_ptr))
    v = np.where(rows // bs == p.col_idx // bs, B.values[0], 0.0)
    return p, v, B.b[0]


@pytest.mark.parametrize("bs", [8, 32])
def test_exact_inverse_one_iteration(bs):
    """B2 (P3 analogue): A block diagonal with the preconditioner's blocks ->
    M^-1 = A^-1, p^ = A^-1 r0, v = r0, alpha = 1, s = 0: exactly one
    iteration, exit at stop test 2, x = A^-1 b; GMRES: one Krylov step."""
    p, v, b = _block_diagonal_system(bs)
    x, R = O.bicgstab(p.row_ptr, p.col_idx, v, b, precond=O.block_jacobi(bs))
    xe = np.linalg.solve(dense(p.row_ptr, p.col_idx, v), b)
    assert R.iters == 1 and R.exit_kind == 2 and R.status == O.CONVERGED
    assert np.linalg.norm(x - xe) <= 1e-13 * np.linalg.norm(xe)
    xg, Rg = O.gmres(p.row_ptr, p.col_idx, v, b, precond=O.block_jacobi(bs), restart=4)
    assert Rg.iters == 1 and Rg.status == O.CONVERGED
    assert np.linalg.norm(xg - xe) <= 1e-12 * np.linalg.norm(xe)


def test_block_size_one_is_scalar_jacobi_bitwise():
    """B3: with power-of-two diagonals (1 / a_ii exact) the 1 x 1 block solve
    y / a_ii and scalar Jacobi's (1 / a_ii) y are the same bits, so the whole
    iteration agrees bit for bit."""
    B = X.make_batch(0, 4)
    p = B.pattern
    rows = np.repeat(np.arange(p.n), np.diff(p.row_ptr))
    for k in range(4):
        v = B.values[k].copy()
        dg = rows == p.col_idx
        v[dg] = 2.0 ** np.ceil(np.log2(v[dg]))
        x1, R1 = O.bicgstab(p.row_ptr, p.col_idx, v, B.b[k], precond=O.PREC_JACOBI)
        x2, R2 = O.bicgstab(p.row_ptr, p.col_idx, v, B.b[k], precond=O.block_jacobi(1))
        assert np.array_equal(x1, x2) and R1.iters == R2.iters


def test_fewer_iterations_and_direct_agreement_on_xgc():
    """B4: on XGC ion/electron systems and the ill-conditioned electrons
    (cross = 0, margin 1e-2) block-Jacobi(8) converges to the direct solution
    (1e-8, TRUE residual < 1e-10) in fewer iterations than scalar Jacobi."""
    for electron in (X.ELECTRON, X.Species(X.ELECTRON_K, cross=0.0, margin=1e-2)):
        B = X.make_batch(0, 16, electron=electron)
        p = B.pattern
        oj = O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b, maxiter=3000)
        ob = O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b, precond=O.block_jacobi(8),
                            maxiter=3000)
        xd = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b)
        assert np.all(ob["status"] == 0)
        fwd = np.linalg.norm(ob["x"] - xd, axis=1) / np.linalg.norm(xd, axis=1)
        assert fwd.max() <= 1e-8
        assert np.all(ob["resnorm"] < 1e-10 * np.linalg.norm(B.b, axis=1))
        e = slice(1, None, 2)
        assert ob["iters"][e].mean() <= 0.85 * oj["iters"][e].mean(), (ob["iters"], oj["iters"])


def test_scipy_bicgstab_with_the_same_block_preconditioner():
    """B5: scipy's BiCGSTAB with M = blockdiag(A)^-1 reaches the same solution."""
    B = X.make_batch(1, 2)
    p = B.pattern
    for k in range(2):
        A = sp.csr_matrix((B.values[k], p.col_idx, p.row_ptr), shape=(p.n, p.n))
        Md = block_diag_part(A.toarray(), 8)
        Minv = spla.LinearOperator(A.shape, matvec=lambda y: np.linalg.solve(Md, y))
        xs, info = spla.bicgstab(A, B.b[k], M=Minv, rtol=1e-12, atol=0.0, maxiter=500)
        assert info == 0
        x, R = O.bicgstab(p.row_ptr, p.col_idx, B.values[k], B.b[k], precond=O.block_jacobi(8))
        assert np.linalg.norm(x - xs) <= 1e-8 * np.linalg.norm(xs)


def test_gmres_block_jacobi_converges_to_direct():
    """B7: GMRES(7) + block-Jacobi(8) on XGC systems: direct solution, fewer
    Krylov steps than with scalar Jacobi on the electrons."""
    B = X.make_batch(0, 8)
    p = B.pattern
    og = O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b, solver=O.SOLVER_GMRES, restart=7)
    ob = O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b, solver=O.SOLVER_GMRES, restart=7,
                        precond=O.block_jacobi(8))
    xd = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b)
    assert np.all(ob["status"] == 0)
    assert (np.linalg.norm(ob["x"] - xd, axis=1) / np.linalg.norm(xd, axis=1)).max() <= 1e-8
    assert ob["iters"][1::2].mean() < og["iters"][1::2].mean()
