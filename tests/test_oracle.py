"""Pins for the CPU oracle (oracle/oracle.c) against things other than itself.

Each test names the pin
and the passage it follows.  None of these tests re-types the oracle's
formulas: they check closed forms, library routines (numpy/LAPACK gesv,
LAPACK gbsv through scipy, scipy's BiCGSTAB), brute force on tiny inputs,
invariants and hand-derived special cases.
"""
import json
import os

import numpy as np
import pytest
import scipy.linalg as sla
import scipy.sparse as sp
import scipy.sparse.linalg as spla

import oracle as O
import xgcgen as X

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def dense_of(rp, ci, v, n):
    return sp.csr_matrix((v, ci, rp), shape=(n, n)).toarray()


def dense_pattern(n):
    rp = np.arange(0, n * n + 1, n, dtype=np.int32)
    ci = np.tile(np.arange(n, dtype=np.int32), n)
    return rp, ci


def rand_dd_dense(rng, n, margin=1.0):
    A = rng.uniform(-1, 1, (n, n))
    np.fill_diagonal(A, 0.0)
    sgn = np.where(rng.uniform(-1, 1, n) < 0, -1.0, 1.0)
    A += np.diag((np.abs(A).sum(1) + margin) * sgn)
    return A


# ------------------------------------------------------------------ P1 --
def test_dense_ge_hand_example():
    """Closed form: A x = b with x = (1, 2, 3) chosen by hand."""
    A = np.array([[4.0, -1, 0], [-1, 4, -1], [0, -1, 4]])
    b = np.array([2.0, 4.0, 10.0])
    np.testing.assert_allclose(O.dense_solve(A, b), [1.0, 2.0, 3.0], rtol=0, atol=1e-15)


def test_dense_ge_needs_pivoting_vs_lapack():
    """Zero leading pivot: only partial pivoting solves it; vs LAPACK gesv."""
    rng = np.random.default_rng(5)
    for n in (2, 3, 6, 11):
        A = rng.standard_normal((n, n))
        A[0, 0] = 0.0
        b = rng.standard_normal(n)
        np.testing.assert_allclose(O.dense_solve(A, b), np.linalg.solve(A, b), rtol=1e-11, atol=1e-12)


@pytest.mark.parametrize("nx,ny", [(3, 3), (5, 5), (4, 3)])
def test_banded_vs_brute_force_ge(nx, ny):
    """P1: banded LU == dense GE with partial pivoting on tiny 9-point grids."""
    pat = X.stencil_pattern(nx, ny)
    vals = X.random_dd_values(pat.row_ptr, pat.col_idx, 6, seed=nx * 10 + ny)
    bs = X.random_rhs(6, pat.n, seed=1)
    for k in range(6):
        A = dense_of(pat.row_ptr, pat.col_idx, vals[k], pat.n)
        xb = O.banded_solve(pat.row_ptr, pat.col_idx, vals[k], bs[k])
        xd = O.dense_solve(A, bs[k])
        np.testing.assert_allclose(xb, xd, rtol=1e-13, atol=1e-14)


def test_banded_pivoting_non_dominant():
    """Banded LU on a matrix that forces row interchanges, vs numpy gesv."""
    pat = X.stencil_pattern(5, 4)
    rng = np.random.default_rng(9)
    v = rng.standard_normal(pat.nnz)
    for i in range(pat.n):                  # make diagonal tiny -> pivots move
        for e in range(pat.row_ptr[i], pat.row_ptr[i + 1]):
            if pat.col_idx[e] == i:
                v[e] = 1e-3 * v[e]
    b = rng.standard_normal(pat.n)
    A = dense_of(pat.row_ptr, pat.col_idx, v, pat.n)
    np.testing.assert_allclose(O.banded_solve(pat.row_ptr, pat.col_idx, v, b),
                               np.linalg.solve(A, b), rtol=1e-9, atol=1e-10)


def test_banded_vs_lapack_gbsv_full_size():
    """P1: vs LAPACK gbsv (scipy.linalg.solve_banded) at n = 992, kl = ku = 33."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    assert O.bandwidth(pat.row_ptr, pat.col_idx) == (33, 33)
    kl = ku = 33
    for k in range(2):
        A = dense_of(pat.row_ptr, pat.col_idx, B.values[k], pat.n)
        ab = np.zeros((kl + ku + 1, pat.n))
        for j in range(pat.n):
            for i in range(max(0, j - ku), min(pat.n, j + kl + 1)):
                ab[ku + i - j, j] = A[i, j]
        ref = sla.solve_banded((kl, ku), ab, B.b[k])
        x = O.banded_solve(pat.row_ptr, pat.col_idx, B.values[k], B.b[k])
        assert np.linalg.norm(x - ref) / np.linalg.norm(ref) <= 1e-12


@pytest.mark.parametrize("nx,ny,scale", [(5, 4, 1e-3), (8, 6, 1e-2), (32, 31, 1e-3)])
def test_banded_pivots_vs_lapack_dgbtrf(nx, ny, scale):
    """P1 (f4 pivots): the row interchanges of the oracle's dgbtf2 equal those
    of LAPACK dgbtrf (scipy.linalg.lapack) on matrices with tiny diagonals,
    where most steps swap; x matches LAPACK's dgbtrs.  ipiv is what the GPU
    banded solver is compared with bit for bit (PAPER.md:97-99 dgbsv)."""
    from scipy.linalg import lapack
    pat = X.stencil_pattern(nx, ny)
    kl, ku = O.bandwidth(pat.row_ptr, pat.col_idx)
    rng = np.random.default_rng(nx * 100 + ny)
    for _ in range(3):
        v = rng.standard_normal(pat.nnz)
        diag = pat.col_idx == np.repeat(np.arange(pat.n), np.diff(pat.row_ptr))
        v[diag] *= scale
        b = rng.standard_normal(pat.n)
        A = dense_of(pat.row_ptr, pat.col_idx, v, pat.n)
        ab = np.zeros((2 * kl + ku + 1, pat.n))
        for j in range(pat.n):
            for i in range(max(0, j - ku), min(pat.n, j + kl + 1)):
                ab[kl + ku + i - j, j] = A[i, j]
        lu, piv, info = lapack.dgbtrf(ab, kl, ku)
        assert info == 0
        xr, info2 = lapack.dgbtrs(lu, kl, ku, b, piv)
        x, oinfo, opiv = O.banded_factor_solve(pat.row_ptr, pat.col_idx, v, b)
        assert oinfo == 0
        assert np.array_equal(opiv, piv), np.nonzero(opiv != piv)
        assert np.count_nonzero(opiv != np.arange(pat.n)) > pat.n // 4  # pivoting happened
        np.testing.assert_allclose(x, xr, rtol=1e-9, atol=1e-9 * np.abs(xr).max())


def test_banded_zero_pivot_info():
    """LAPACK convention: info = j+1 for the first exactly-zero pivot column
    (a zero column j makes every candidate of step j zero)."""
    pat = X.stencil_pattern(4, 4)
    v = X.random_dd_values(pat.row_ptr, pat.col_idx, 1, seed=3)[0].copy()
    v[pat.col_idx == 6] = 0.0               # column 6 of A is zero
    b = np.ones(pat.n)
    _, info, piv = O.banded_factor_solve(pat.row_ptr, pat.col_idx, v, b)
    assert info == 7 and piv[6] == 6


def test_spmv_vs_dense():
    pat = X.stencil_pattern(7, 5)
    v = X.random_dd_values(pat.row_ptr, pat.col_idx, 1, seed=4)[0]
    x = np.random.default_rng(0).standard_normal(pat.n)
    A = dense_of(pat.row_ptr, pat.col_idx, v, pat.n)
    np.testing.assert_allclose(O.spmv(pat.row_ptr, pat.col_idx, v, x), A @ x, rtol=1e-14, atol=1e-14)


# ------------------------------------------------------------------ P2 --
def test_manufactured_solution():
    """P2: b = A x_true (numpy dense product); direct error <= 1e-12 kappa,
    BiCGSTAB error <= kappa * tol (forward error bound of a residual test)."""
    B = X.make_batch(0, 4)
    pat = B.pattern
    rng = np.random.default_rng(11)
    for k in range(4):
        A = dense_of(pat.row_ptr, pat.col_idx, B.values[k], pat.n)
        xt = rng.standard_normal(pat.n)
        b = A @ xt
        kappa = np.linalg.cond(A)
        xd = O.banded_solve(pat.row_ptr, pat.col_idx, B.values[k], b)
        assert np.linalg.norm(xd - xt) / np.linalg.norm(xt) <= 1e-12 * kappa
        xi, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[k], b, tol=1e-10)
        assert R.status == O.CONVERGED
        assert np.linalg.norm(xi - xt) / np.linalg.norm(xt) <= kappa * 1e-10


# ------------------------------------------------------------------ P3 --
def test_diagonal_matrix_one_iteration_stop2():
    """P3: A diagonal => Jacobi is exact: p^ = A^-1 r0, v = r0, alpha = 1,
    s = 0, so exactly ONE iteration with exit at stop test 2,
    x = A^-1 b.  Pins Jacobi, alpha (R3), the mid-loop exit and the
    iteration-count convention (R8)."""
    n = 17
    rp = np.arange(n + 1, dtype=np.int32)
    ci = np.arange(n, dtype=np.int32)
    rng = np.random.default_rng(2)
    dv = rng.uniform(0.5, 3.0, n) * np.where(rng.random(n) < 0.5, -1, 1)
    b = rng.standard_normal(n)
    x, R = O.bicgstab(rp, ci, dv, b, tol=1e-10)
    assert R.iters == 1 and R.exit_kind == 2 and R.status == O.CONVERGED
    np.testing.assert_allclose(x, b / dv, rtol=1e-15, atol=0)


def test_diagonal_values_in_stencil_pattern():
    """P3 on the full 992-row pattern with all off-diagonal values zero."""
    pat = X.stencil_pattern()
    v = np.zeros(pat.nnz)
    diag_e = [e for i in range(pat.n) for e in range(pat.row_ptr[i], pat.row_ptr[i + 1])
              if pat.col_idx[e] == i]
    v[diag_e] = np.linspace(1.0, 40.0, pat.n)
    b = np.cos(np.arange(pat.n))
    x, R = O.bicgstab(pat.row_ptr, pat.col_idx, v, b)
    assert R.iters == 1 and R.exit_kind == 2
    np.testing.assert_allclose(x, b / v[diag_e], rtol=1e-15)


# ------------------------------------------------------------------ P4 --
def test_exact_initial_guess_zero_iterations():
    """P4: x0 = x* (direct solve) => stop test 1 at i = 0, x unchanged."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    for k in range(2):
        xs = O.banded_solve(pat.row_ptr, pat.col_idx, B.values[k], B.b[k])
        x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[k], B.b[k], x0=xs)
        assert R.iters == 0 and R.exit_kind == 1 and R.status == O.CONVERGED
        assert np.array_equal(x, xs)


def test_zero_rhs():
    """P4: b = 0 => x = 0, iters = 0, converged, resnorm 0 (R5)."""
    B = X.make_batch(0, 1)
    pat = B.pattern
    x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[0], np.zeros(pat.n),
                      x0=np.ones(pat.n))
    assert R.iters == 0 and R.status == O.CONVERGED and R.resnorm == 0.0
    assert not np.any(x)


def test_maxiter_zero():
    """maxiter = 0 => x = x0, iters = 0, status maxiter, resnorm = ||b - A x0||."""
    B = X.make_batch(1, 1)
    pat = B.pattern
    x0 = np.full(pat.n, 0.25)
    x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[0], B.b[0], x0=x0, maxiter=0)
    A = dense_of(pat.row_ptr, pat.col_idx, B.values[0], pat.n)
    assert R.iters == 0 and R.status == O.MAXITER
    assert np.array_equal(x, x0)
    assert R.resnorm == pytest.approx(np.linalg.norm(B.b[0] - A @ x0), rel=1e-13)


def test_forced_nonconvergence():
    """maxiter below the needed count => status maxiter, iters == maxiter."""
    B = X.make_batch(1, 1)
    pat = B.pattern
    x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[0], B.b[0], maxiter=5)
    assert R.iters == 5 and R.status == O.MAXITER
    assert R.resnorm > 1e-10 * np.linalg.norm(B.b[0])


def test_breakdown_hand_example():
    """R10, derived by hand: A = [[0,1],[1,0]] (zero diagonal -> d = 1, R11),
    b = (1, 0): r = r^ = b, rho = 1, p^ = r, v = A p^ = (0, 1), r^.v = 0 ->
    breakdown after the first SpMV: iters = 1, status 2, x stays 0."""
    rp = np.array([0, 2, 4], np.int32)
    ci = np.array([0, 1, 0, 1], np.int32)
    v = np.array([0.0, 1.0, 1.0, 0.0])
    x, R = O.bicgstab(rp, ci, v, np.array([1.0, 0.0]))
    assert R.status == O.BREAKDOWN and R.iters == 1
    assert not np.any(x)


# ------------------------------------------------------------------ P5 --
@pytest.mark.parametrize("k", [-3, 5])
def test_power_of_two_scaling_bitwise(k):
    """P5: (2^k A, 2^k b) gives bitwise identical x and iteration count
    in REL_B mode (all scalings in Alg. 1 are exact in fp64)."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    c = 2.0 ** k
    for j in range(2):
        x1, R1 = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j])
        x2, R2 = O.bicgstab(pat.row_ptr, pat.col_idx, c * B.values[j], c * B.b[j])
        assert R1.iters == R2.iters and np.array_equal(x1, x2)


# ------------------------------------------------------------------ P6 --
def test_recursive_vs_true_residual_invariant():
    """P6: ||r_rec - (b - A x)|| / ||b|| <= 1e-12 at every iteration."""
    B = X.make_batch(0, 4)
    pat = B.pattern
    for j in range(4):
        x, R, tr = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j], trace=True)
        full = tr[~np.isnan(tr)]
        assert full.size >= 1
        assert np.max(full) / np.linalg.norm(B.b[j]) <= 1e-12


# ------------------------------------------------------------------ P7 --
def test_bicgstab_matches_direct_on_generated_systems():
    """P7: BiCGSTAB vs banded LU within 1e-8; true rel residual <= 1e-10;
    iteration counts in the calibrated bands (ion ~5-6, electron ~31)."""
    B = X.make_batch(0, 16)
    pat = B.pattern
    out = O.batch_bicgstab(pat.row_ptr, pat.col_idx, B.values, B.b)
    xd = O.batch_banded(pat.row_ptr, pat.col_idx, B.values, B.b)
    for j in range(16):
        assert out["status"][j] == O.CONVERGED
        assert out["resnorm"][j] / np.linalg.norm(B.b[j]) <= 1e-10
        assert np.linalg.norm(out["x"][j] - xd[j]) / np.linalg.norm(xd[j]) <= 1e-8
    ion, ele = out["iters"][0::2], out["iters"][1::2]
    assert 3 <= ion.min() and ion.max() <= 8
    assert 25 <= ele.min() and ele.max() <= 40


@pytest.mark.parametrize("n", [4, 5, 8])
def test_finite_termination_dense(n):
    """Exact-arithmetic BiCGSTAB terminates in <= n steps (BiCG polynomial
    annihilates r0 once the Krylov space is exhausted, van der Vorst [18]);
    with rounding we allow n + 1.  A wrong beta/alpha/omega or an updated
    shadow residual breaks this bound (checked against mutants offline)."""
    rng = np.random.default_rng(100 + n)
    rp, ci = dense_pattern(n)
    worst = 0
    for _ in range(40):
        A = rand_dd_dense(rng, n)
        b = rng.standard_normal(n)
        x, R = O.bicgstab(rp, ci, A.ravel(), b, tol=1e-10, maxiter=200)
        assert R.status == O.CONVERGED
        np.testing.assert_allclose(x, np.linalg.solve(A, b), rtol=1e-8, atol=1e-9)
        worst = max(worst, R.iters)
    assert worst <= n + 1


# ------------------------------------------------------------------ P8 --
def test_vs_scipy_bicgstab():
    """P8: solution agreement with scipy's BiCGSTAB (Templates algorithm,
    Jacobi as M); iteration counts are not compared."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    for j in range(2):
        A = sp.csr_matrix((B.values[j], pat.col_idx, pat.row_ptr), shape=(pat.n, pat.n))
        M = sp.diags(1.0 / A.diagonal())
        xs, info = spla.bicgstab(A, B.b[j], rtol=1e-13, atol=0.0, M=M, maxiter=1000)
        assert info == 0
        x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j])
        assert np.linalg.norm(x - xs) / np.linalg.norm(xs) <= 1e-8


# ------------------------------------------------------------------ P9 --
def test_null_x0_equals_zero_x0_bitwise():
    B = X.make_batch(0, 2)
    pat = B.pattern
    for j in range(2):
        x1, R1 = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j])
        x2, R2 = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j], x0=np.zeros(pat.n))
        assert R1.iters == R2.iters and np.array_equal(x1, x2)


# ----------------------------------------------------------------- P10 --
def test_symmetric_permutation():
    """P10: P A P^T (P x) = P b gives the permuted x within 1e-8, iters +-2."""
    B = X.make_batch(0, 2)
    pat = B.pattern
    perm = np.random.default_rng(3).permutation(pat.n)
    inv = np.argsort(perm)
    for j in range(2):
        A = sp.csr_matrix((B.values[j], pat.col_idx, pat.row_ptr), shape=(pat.n, pat.n))
        Ap = A[perm][:, perm].tocsr()
        Ap.sort_indices()
        x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j])
        xp, Rp = O.bicgstab(Ap.indptr, Ap.indices, Ap.data, B.b[j][perm])
        assert np.linalg.norm(xp[inv] - x) / np.linalg.norm(x) <= 1e-8
        assert abs(R.iters - Rp.iters) <= 2


# ---------------------------------------------------------- true residual --
def test_true_residual_guard_restarts_ill_conditioned():
    """R4: at kappa ~ 1e5 (cross = 0, margin 1e-3 electrons) the recursive
    residual drifts from the true one; the guard restarts and the final TRUE
    residual meets tau, which it may not without the guard."""
    ill = X.Species(X.ELECTRON_K, cross=0.0, margin=1e-3)
    B = X.make_batch(1, 6, electron=ill)
    pat = B.pattern
    rest = 0
    for j in range(6):
        bn = np.linalg.norm(B.b[j])
        x, R = O.bicgstab(pat.row_ptr, pat.col_idx, B.values[j], B.b[j], maxiter=2000)
        assert R.status == O.CONVERGED and R.resnorm < 1e-10 * bn
        rest += R.restarts
        xd = O.banded_solve(pat.row_ptr, pat.col_idx, B.values[j], B.b[j])
        assert np.linalg.norm(x - xd) / np.linalg.norm(xd) <= 1e-8
    assert rest >= 1


# -------------------------------------------------------------- layouts --
def test_paper_storage_numbers():
    """Storage formulas for the paper's 992-row 9-point pattern."""
    facts = json.load(open(os.path.join(GOLD, "paper_facts.json")))
    pat = X.stencil_pattern(facts["grid"]["nx"], facts["grid"]["ny"])
    assert pat.n == facts["rows"]["value"]
    assert pat.max_row_nnz == facts["max_nnz_per_row"]["value"]
    assert pat.nnz == facts["csr_nnz_9pt_32x31"]["value"]
    ell_col, src = X.ell_layout(pat.row_ptr, pat.col_idx)
    assert ell_col.size == facts["ell_slots_9pt_32x31"]["value"]
    assert int(np.sum(src < 0)) == facts["ell_padding_slots"]["value"]


def test_paper_vector_planner_accounting():
    """The paper's SMEM planner (Sec. IV-D): the BiCGSTAB vectors
    (9 of n doubles, the 4 SpMV vectors first) go to shared memory in priority
    order while they fit the per-block budget, the rest to global memory.  On
    the V100 with the default 48 KiB budget and n = 992 that is 6 + 3
    (golden).  The same byte accounting with B200's 227 KB opt-in
    budget places all 9 (71.4 KB) on chip; the B200 plan goes further and
    keeps them off the SMEM data pipe altogether (registers, TMEM; DESIGN.md
    Kernels 12), so no planner is needed there."""
    facts = json.load(open(os.path.join(GOLD, "paper_facts.json")))
    nvec = facts["bicgstab_vectors"]["value"]
    n = facts["rows"]["value"]
    vec_bytes = 8 * n
    def plan(budget):
        smem = 0
        for _ in range(nvec):  # priority order; each vector whole or not at all
            if (smem + 1) * vec_bytes <= budget:
                smem += 1
        return smem, nvec - smem
    v100 = facts["v100_smem_split"]
    assert plan(v100["budget_bytes"]) == (v100["smem"], v100["global"])
    assert plan(232448) == (9, 0)  # B200: 227 KB dynamic SMEM per CTA (opt-in)
