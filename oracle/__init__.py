"""CPU oracle for the batched Jacobi-preconditioned BiCGSTAB (ctypes wrapper).

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
cpu_baseline / ``--impl reference`` legs of bench.py may import this package.
The product package (paper_conf_ipps_kashinksla22_b200) never imports it and
shares no code with it (see oracle.c for the algorithm and its citations).

Functions mirror oracle.c:
  spmv, dense_solve, banded_solve, banded_factor_solve (with pivots),
  bandwidth, bicgstab (one system, with
  optional invariant trace), gmres (restarted GMRES(m)),
  batch_bicgstab, batch_krylov, batch_banded (host threads).
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

STOP_REL_B = 0
STOP_ABS = 1
PREC_JACOBI, PREC_NONE = 0, 1
PREC_BLOCK_JACOBI = 2  # blocks of 8 consecutive rows; block_jacobi(bs) for other sizes


def block_jacobi(bs: int = 8) -> int:
    """precond code of block-Jacobi with blocks of bs consecutive rows (R30)."""
    return PREC_BLOCK_JACOBI | (int(bs) << 8)
SOLVER_BICGSTAB, SOLVER_GMRES = 0, 2
CONVERGED, MAXITER, BREAKDOWN = 0, 1, 2

_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (no BLAS, no CUDA, IEEE fp64, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-D_GNU_SOURCE", "-ffp-contract=off", "-fno-fast-math",
               "-fPIC", "-shared", "-o", _LIB + ".tmp", _SRC, "-lpthread", "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class Result(C.Structure):
    _fields_ = [("iters", C.c_int32), ("status", C.c_int32), ("restarts", C.c_int32),
                ("exit_kind", C.c_int32), ("resnorm", C.c_double),
                ("recursive", C.c_double), ("tau", C.c_double)]


_P = C.c_void_p


def lib():
    global _lib
    with _lock:
        if _lib is None:
            L = C.CDLL(build())
            L.oracle_spmv_csr.argtypes = [C.c_int, _P, _P, _P, _P, _P]
            L.oracle_spmv_csr.restype = None
            L.oracle_dense_solve.argtypes = [C.c_int, _P, _P]
            L.oracle_dense_solve.restype = C.c_int
            L.oracle_bandwidth.argtypes = [C.c_int, _P, _P, C.POINTER(C.c_int), C.POINTER(C.c_int)]
            L.oracle_bandwidth.restype = None
            L.oracle_banded_solve.argtypes = [C.c_int, _P, _P, _P, _P, _P]
            L.oracle_banded_solve.restype = C.c_int
            L.oracle_banded_solve_piv.argtypes = [C.c_int, _P, _P, _P, _P, _P, _P]
            L.oracle_banded_solve_piv.restype = C.c_int
            L.oracle_bicgstab.argtypes = [C.c_int, _P, _P, _P, _P, _P, C.c_double, C.c_int,
                                          C.c_int, C.c_int, _P, C.POINTER(Result), _P]
            L.oracle_bicgstab.restype = C.c_int
            L.oracle_batch_bicgstab.argtypes = [C.c_int, C.c_int, C.c_int, _P, _P, _P, _P, _P,
                                                C.c_double, C.c_int, C.c_int, C.c_int,
                                                _P, _P, _P, _P, _P, C.c_int]
            L.oracle_batch_bicgstab.restype = C.c_int
            L.oracle_bicgstab_p.argtypes = [C.c_int, _P, _P, _P, _P, _P, C.c_double, C.c_int,
                                            C.c_int, C.c_int, C.c_int, _P, C.POINTER(Result),
                                            _P]
            L.oracle_bicgstab_p.restype = C.c_int
            L.oracle_gmres.argtypes = [C.c_int, _P, _P, _P, _P, _P, C.c_double, C.c_int,
                                       C.c_int, C.c_int, C.c_int, _P, C.POINTER(Result), _P]
            L.oracle_gmres.restype = C.c_int
            L.oracle_batch_krylov.argtypes = [C.c_int, C.c_int, C.c_int, C.c_int, C.c_int,
                                              C.c_int, _P, _P, _P, _P, _P, C.c_double, C.c_int,
                                              C.c_int, C.c_int, _P, _P, _P, _P, _P, C.c_int]
            L.oracle_batch_krylov.restype = C.c_int
            L.oracle_batch_banded.argtypes = [C.c_int, C.c_int, C.c_int, _P, _P, _P, _P, _P,
                                              _P, C.c_int]
            L.oracle_batch_banded.restype = C.c_int
            L.oracle_precond_apply.argtypes = [C.c_int, _P, _P, _P, C.c_int, _P, _P]
            L.oracle_precond_apply.restype = C.c_int
            _lib = L
    return _lib


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _ptr(a):
    return None if a is None else a.ctypes.data


def spmv(row_ptr, col_idx, val, x):
    rp, ci, v, xx = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(x)
    n = rp.size - 1
    y = np.empty(n)
    lib().oracle_spmv_csr(n, _ptr(rp), _ptr(ci), _ptr(v), _ptr(xx), _ptr(y))
    return y


def dense_solve(A, b):
    A = np.array(A, dtype=np.float64, order="C")
    x = np.array(b, dtype=np.float64)
    info = lib().oracle_dense_solve(A.shape[0], _ptr(A), _ptr(x))
    if info:
        raise np.linalg.LinAlgError(f"zero pivot at {info - 1}")
    return x


def bandwidth(row_ptr, col_idx):
    rp, ci = _i32(row_ptr), _i32(col_idx)
    kl, ku = C.c_int(), C.c_int()
    lib().oracle_bandwidth(rp.size - 1, _ptr(rp), _ptr(ci), C.byref(kl), C.byref(ku))
    return kl.value, ku.value


def banded_solve(row_ptr, col_idx, val, b):
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(b)
    x = np.empty(rp.size - 1)
    info = lib().oracle_banded_solve(rp.size - 1, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb), _ptr(x))
    if info:
        raise np.linalg.LinAlgError(f"banded LU: zero pivot / error {info}")
    return x


def banded_factor_solve(row_ptr, col_idx, val, b):
    """dgbtf2 + dgbtrs on one system without raising: (x, info, ipiv).
    info = 0 or j+1 for the first zero pivot (x is then not written: NaN);
    ipiv[j] = 0-based row interchanged with row j."""
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(b)
    n = rp.size - 1
    x = np.full(n, np.nan)
    piv = np.empty(n, np.int32)
    info = lib().oracle_banded_solve_piv(n, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb), _ptr(x),
                                         _ptr(piv))
    if info < 0:
        raise MemoryError("oracle_banded_solve_piv")
    return x, int(info), piv


def bicgstab(row_ptr, col_idx, val, b, x0=None, tol=1e-10, maxiter=1000, stop=STOP_REL_B,
             true_res_check=True, trace=False, precond=PREC_JACOBI):
    """One system through Algorithm 1.  Returns (x, Result[, trace])."""
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(b)
    n = rp.size - 1
    x0a = None if x0 is None else _f64(x0)
    x = np.empty(n)
    R = Result()
    tr = np.full(max(maxiter, 1), np.nan) if trace else None
    rc = lib().oracle_bicgstab_p(n, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb), _ptr(x0a),
                                 float(tol), int(maxiter), int(stop), int(bool(true_res_check)),
                                 int(precond), _ptr(x), C.byref(R), _ptr(tr))
    if rc:
        raise MemoryError("oracle_bicgstab")
    if trace:
        return x, R, tr[: R.iters]
    return x, R


def precond_apply(row_ptr, col_idx, val, y, precond=PREC_JACOBI):
    """M^-1 y for one system (the preconditioner alone, oracle.c precond_apply)."""
    rp, ci, v, yy = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(y)
    out = np.empty(rp.size - 1)
    if lib().oracle_precond_apply(rp.size - 1, _ptr(rp), _ptr(ci), _ptr(v), int(precond),
                                  _ptr(yy), _ptr(out)):
        raise MemoryError("oracle_precond_apply")
    return out


def batch_bicgstab(row_ptr, col_idx, values, b, x0=None, tol=1e-10, maxiter=1000,
                   stop=STOP_REL_B, true_res_check=True, threads=0):
    """Alg. 1 on every system (values [batch, nnz] CSR order).
    Returns dict(x, iters, resnorm, status, restarts)."""
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(values), _f64(b)
    batch, nnz = v.shape
    n = rp.size - 1
    x0a = None if x0 is None else _f64(x0)
    out = dict(x=np.empty((batch, n)), iters=np.empty(batch, np.int32),
               resnorm=np.empty(batch), status=np.empty(batch, np.int32),
               restarts=np.empty(batch, np.int32))
    rc = lib().oracle_batch_bicgstab(n, nnz, batch, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb),
                                     _ptr(x0a), float(tol), int(maxiter), int(stop),
                                     int(bool(true_res_check)), _ptr(out["x"]),
                                     _ptr(out["iters"]), _ptr(out["resnorm"]),
                                     _ptr(out["status"]), _ptr(out["restarts"]), int(threads))
    if rc:
        raise MemoryError("oracle_batch_bicgstab")
    return out


def batch_banded(row_ptr, col_idx, values, b, threads=0):
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(values), _f64(b)
    batch, nnz = v.shape
    n = rp.size - 1
    x = np.empty((batch, n))
    st = np.empty(batch, np.int32)
    rc = lib().oracle_batch_banded(n, nnz, batch, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb),
                                   _ptr(x), _ptr(st), int(threads))
    if rc or np.any(st != 0):
        raise np.linalg.LinAlgError("batch banded LU failed")
    return x


def gmres(row_ptr, col_idx, val, b, x0=None, tol=1e-10, maxiter=1000, restart=8,
          stop=STOP_REL_B, precond=PREC_JACOBI, trace=False):
    """One system through restarted GMRES(restart) (oracle.c oracle_gmres).
    Returns (x, Result[, trace (iters, 2): |g_{k+1}|, ||b - A x_k||])."""
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(val), _f64(b)
    n = rp.size - 1
    x0a = None if x0 is None else _f64(x0)
    x = np.empty(n)
    R = Result()
    tr = np.full(2 * max(maxiter, 1), np.nan) if trace else None
    rc = lib().oracle_gmres(n, _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb), _ptr(x0a), float(tol),
                            int(maxiter), int(restart), int(stop), int(precond), _ptr(x),
                            C.byref(R), _ptr(tr))
    if rc:
        raise ValueError("oracle_gmres: allocation failure or restart < 1")
    if trace:
        return x, R, tr[: 2 * R.iters].reshape(-1, 2)
    return x, R


def batch_krylov(row_ptr, col_idx, values, b, solver=SOLVER_BICGSTAB, precond=PREC_JACOBI,
                 restart=8, x0=None, tol=1e-10, maxiter=1000, stop=STOP_REL_B,
                 true_res_check=True, threads=0):
    """BiCGSTAB or GMRES(restart) with Jacobi, block-Jacobi (R30) or no
    preconditioner on every system.  Returns dict(x, iters, resnorm, status, restarts)."""
    rp, ci, v, bb = _i32(row_ptr), _i32(col_idx), _f64(values), _f64(b)
    batch, nnz = v.shape
    n = rp.size - 1
    x0a = None if x0 is None else _f64(x0)
    out = dict(x=np.empty((batch, n)), iters=np.empty(batch, np.int32),
               resnorm=np.empty(batch), status=np.empty(batch, np.int32),
               restarts=np.empty(batch, np.int32))
    rc = lib().oracle_batch_krylov(int(solver), int(precond), int(restart), n, nnz, batch,
                                   _ptr(rp), _ptr(ci), _ptr(v), _ptr(bb), _ptr(x0a), float(tol),
                                   int(maxiter), int(stop), int(bool(true_res_check)),
                                   _ptr(out["x"]), _ptr(out["iters"]), _ptr(out["resnorm"]),
                                   _ptr(out["status"]), _ptr(out["restarts"]), int(threads))
    if rc:
        raise ValueError("oracle_batch_krylov failed")
    return out
