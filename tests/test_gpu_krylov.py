"""GPU parity of the further Krylov solvers and preconditioners (SURVEY.md
8(f) f3; "several preconditionable iterative solvers"):
restarted GMRES(m) and the identity preconditioner, C-ABI CUDA path vs the
oracle's GMRES / BiCGSTAB on the same seeded inputs, with the parity bar of
BASELINE.json (true relative residual <= 1e-10, forward error vs the banded LU
<= 1e-8, |iters - oracle iters| <= 2, equal status).
"""
import numpy as np
import pytest
import torch

import oracle as O
import xgcgen as X
from gpu_common import compare, gpu_solve
from paper_conf_ipps_kashinksla22_b200 import BsolveError, Solver

pytestmark = pytest.mark.gpu

_PREC = {"jacobi": O.PREC_JACOBI, "none": O.PREC_NONE}


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.fail("GPU tests need a CUDA device")


def _oracle(p, B, solver, precond="jacobi", restart=7, x0=None, maxiter=1000, stop=O.STOP_REL_B,
            tol=1e-10):
    return O.batch_krylov(p.row_ptr, p.col_idx, B.values, B.b,
                          solver=O.SOLVER_GMRES if solver == "gmres" else O.SOLVER_BICGSTAB,
                          precond=_PREC[precond], restart=restart, x0=x0, maxiter=maxiter,
                          stop=stop, tol=tol)


@pytest.mark.parametrize("restart", [7, 4, 1])
@pytest.mark.parametrize("nx,ny", [(32, 31), (31, 32)])
def test_gmres_line_kernel(restart, nx, ny):
    """GMRES(m) on the paper's grid and its transpose, ion + electron mix."""
    B = X.make_batch(0, 48, nx=nx, ny=ny)
    p = B.pattern
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", restart=restart,
                  maxiter=4000)
    assert g["info"]["solver"] == 1 and g["info"]["restart"] == restart
    assert g["info"]["kernel_mode"] == 4
    o = _oracle(p, B, "gmres", restart=restart, maxiter=4000)
    compare(p.row_ptr, p.col_idx, B.values, B.b, g, o=o)


@pytest.mark.parametrize("nx,ny,restart", [(40, 25, 7), (24, 40, 4), (5, 7, 7), (100, 10, 3)])
def test_gmres_generic_width(nx, ny, restart):
    """GMRES(m) on grid widths other than the compiled 31 / 32: the generic-
    width instance of the 2-CTA line kernel (width mod 8 compiled)."""
    B = X.make_batch(0, 32, nx=nx, ny=ny)
    p = B.pattern
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", restart=restart,
                  maxiter=4000)
    i = g["info"]
    assert i["solver"] == 1 and i["kernel_mode"] == 4 and i["line_generic"] == 1, i
    assert i["line_width"] == nx
    o = _oracle(p, B, "gmres", restart=restart, maxiter=4000)
    compare(p.row_ptr, p.col_idx, B.values, B.b, g, o=o)


@pytest.mark.parametrize("nx,ny", [(32, 31), (31, 32)])
def test_gmres_generic_equals_compiled_width_bitwise(nx, ny, monkeypatch):
    B = X.make_batch(0, 32, nx=nx, ny=ny)
    p = B.pattern
    outs = []
    for knob in ("0", "1"):
        monkeypatch.setenv("BSOLVE_LINE_GENERIC", knob)
        outs.append(gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", restart=5))
        assert outs[-1]["info"]["line_generic"] == int(knob)
    for k in ("x", "iters", "resnorm", "status"):
        assert np.array_equal(outs[0][k], outs[1][k]), k


def test_gmres_warm_start_maxiter_and_edge_cases():
    B = X.make_batch(0, 40, picard=2)
    p = B.pattern
    x0 = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b) * (1 + 1e-4)
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, x0=x0, solver="gmres")
    compare(p.row_ptr, p.col_idx, B.values, B.b, g, o=_oracle(p, B, "gmres", x0=x0))
    # maxiter cut mid-cycle: every system stops at exactly maxiter, status 1
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", maxiter=10)
    o = _oracle(p, B, "gmres", maxiter=10)
    assert np.array_equal(g["iters"], o["iters"]) and np.all(g["iters"][1::2] == 10)
    assert np.array_equal(g["status"], o["status"])
    # x0 = x*: zero iterations; b = 0: x = 0
    xd = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b)
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, x0=xd, solver="gmres")
    assert np.all(g["iters"] == 0) and np.all(g["status"] == 0)
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, np.zeros_like(B.b), solver="gmres")
    assert np.all(g["iters"] == 0) and np.all(g["x"] == 0)


def test_gmres_unpreconditioned_and_abs_stop():
    B = X.make_batch(0, 24)
    p = B.pattern
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", precond="none",
                  maxiter=4000)
    compare(p.row_ptr, p.col_idx, B.values, B.b, g,
            o=_oracle(p, B, "gmres", precond="none", maxiter=4000))
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres", stop="abs", tol=1e-9)
    o = _oracle(p, B, "gmres", stop=O.STOP_ABS, tol=1e-9)
    assert np.abs(g["iters"].astype(int) - o["iters"].astype(int)).max() <= 2
    assert np.all(g["resnorm"] < 1e-9)


def test_gmres_deterministic_and_slicing_independent():
    B = X.make_batch(0, 64)
    p = B.pattern
    g1 = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, solver="gmres")
    g2 = gpu_solve(p.row_ptr, p.col_idx, B.values[10:], B.b[10:], solver="gmres")
    for k in ("x", "iters", "resnorm", "status"):
        assert np.array_equal(g1[k][10:], g2[k])


@pytest.mark.parametrize("placement,block_threads", [("auto", 0), ("smem", 256), ("tmem", 0),
                                                     ("stream", 0)])
def test_bicgstab_without_preconditioner(placement, block_threads):
    """precond = none (d = 1) in every kernel family against the oracle's
    unpreconditioned Algorithm 1."""
    B = X.make_batch(0, 24)
    p = B.pattern
    g = gpu_solve(p.row_ptr, p.col_idx, B.values, B.b, precond="none", placement=placement,
                  block_threads=block_threads, maxiter=3000)
    assert g["info"]["precond"] == 1
    compare(p.row_ptr, p.col_idx, B.values, B.b, g,
            o=_oracle(p, B, "bicgstab", precond="none", maxiter=3000))


def test_bicgstab_without_preconditioner_random_pattern():
    rp, ci = X.random_pattern(300, 7, seed=11)
    vals = X.random_dd_values(rp, ci, 16, seed=12)
    # positive diagonal: Gershgorin discs in the right half plane, so the
    # unpreconditioned iteration converges smoothly (with mixed-sign diagonals
    # it is erratic and its count is rounding-order sensitive)
    for i in range(300):
        e = rp[i] + int(np.nonzero(ci[rp[i]:rp[i + 1]] == i)[0][0])
        vals[:, e] = np.abs(vals[:, e])
    b = X.random_rhs(16, 300, seed=13)
    g = gpu_solve(rp, ci, vals, b, precond="none", maxiter=3000)
    o = O.batch_krylov(rp, ci, vals, b, precond=O.PREC_NONE, maxiter=3000)
    compare(rp, ci, vals, b, g, o=o)


def test_solver_option_errors():
    rp, ci = X.random_pattern(200, 6, seed=4)
    with pytest.raises(BsolveError) as e:
        Solver(rp, ci, 2, solver="gmres")
    assert e.value.code == -3
    p = X.stencil_pattern(32, 31)
    for m in (0, 8):
        with pytest.raises(BsolveError) as e:
            Solver(p.row_ptr, p.col_idx, 2, solver="gmres", restart=m)
        assert e.value.code == -1
