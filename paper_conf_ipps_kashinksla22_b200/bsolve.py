"""Thin ctypes binding of libbsolve.so (include/bsolve.h).

Argument marshalling only: every step of the solve runs in the library's
CUDA kernels.  PyTorch provides device memory and the current CUDA stream.
There is no CPU fallback: if the library cannot be loaded, import fails.
"""
from __future__ import annotations

import ctypes as C
import os
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libbsolve.so")

OK = 0
ERR_INVALID, ERR_PATTERN, ERR_UNSUPPORTED, ERR_CUDA, ERR_NOMEM = -1, -2, -3, -4, -5
FMT_AUTO, FMT_CSR, FMT_ELL = 0, 1, 2
PLACE_AUTO, PLACE_SMEM, PLACE_STREAM, PLACE_REGS, PLACE_CLUSTER, PLACE_TMEM = 0, 1, 2, 3, 4, 5
STOP_REL_B, STOP_ABS = 0, 1
SOLVER_BICGSTAB, SOLVER_GMRES = 0, 1
PREC_JACOBI, PREC_NONE, PREC_BLOCK_JACOBI = 0, 1, 2
MAX_RESTART = 7
SYS_CONVERGED, SYS_MAXITER, SYS_BREAKDOWN, SYS_DIRECT = 0, 1, 2, 3

_FMT = {"auto": FMT_AUTO, "csr": FMT_CSR, "ell": FMT_ELL}
_PLACE = {"auto": PLACE_AUTO, "smem": PLACE_SMEM, "stream": PLACE_STREAM, "regs": PLACE_REGS,
          "cluster": PLACE_CLUSTER, "tmem": PLACE_TMEM}
_STOP = {"rel_b": STOP_REL_B, "rel": STOP_REL_B, "abs": STOP_ABS}
_SOLVER = {"bicgstab": SOLVER_BICGSTAB, "gmres": SOLVER_GMRES}
_PREC = {"jacobi": PREC_JACOBI, "none": PREC_NONE, "block_jacobi": PREC_BLOCK_JACOBI}


class BsolveError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"bsolve error {code}: {msg}")
        self.code = code


class Options(C.Structure):
    _fields_ = [("format", C.c_int), ("placement", C.c_int), ("stop", C.c_int),
                ("true_residual_check", C.c_int), ("device", C.c_int),
                ("block_threads", C.c_int), ("reg_slots", C.c_int), ("solver", C.c_int),
                ("precond", C.c_int), ("restart", C.c_int), ("direct_fallback", C.c_int)]


class Info(C.Structure):
    _fields_ = [(f, C.c_int) for f in (
        "n", "nnz", "batch", "ell_width", "format", "placement", "block_threads",
        "rows_per_thread", "smem_bytes", "ctas_per_sm", "num_sms", "grid", "kl", "ku", "device",
        "kernel_mode", "cluster", "solver", "precond", "restart", "banded_launches",
        "regs_per_thread", "occupancy_api", "line_width", "line_generic",
        "max_active_clusters")]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


_lock = threading.Lock()
_lib = None
_P = C.c_void_p


def lib():
    """Load libbsolve.so (build it with __graft_entry__.build() first)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(LIB_PATH):
                raise ImportError(f"{LIB_PATH} missing: run python -c 'import __graft_entry__ as g; g.build()'")
            L = C.CDLL(LIB_PATH)
            L.bsolve_default_options.argtypes = [C.POINTER(Options)]
            L.bsolve_default_options.restype = None
            L.bsolve_create.argtypes = [C.POINTER(_P), C.c_int, C.c_int, _P, _P, C.POINTER(Options)]
            L.bsolve_run.argtypes = [_P, _P, _P, _P, C.c_double, C.c_int, _P, _P, _P, _P, _P]
            L.bsolve_run_host.argtypes = [_P, _P, _P, _P, C.c_double, C.c_int, _P, _P, _P, _P]
            L.bsolve_spmv.argtypes = [_P, _P, _P, _P, C.c_int, _P]
            L.bsolve_csr_to_ell.argtypes = [_P, _P, _P, C.c_int, _P]
            L.bsolve_query.argtypes = [_P, C.POINTER(Info)]
            L.bsolve_ell_map.argtypes = [_P, _P, _P]
            L.bsolve_banded_solve.argtypes = [_P, _P, _P, _P, _P, _P, _P]
            L.bsolve_banded_solve_host.argtypes = [_P, _P, _P, _P, _P]
            L.bsolve_ell_layout.argtypes = [C.c_int, _P, _P, C.POINTER(C.c_int32), _P, _P]
            L.bsolve_destroy.argtypes = [_P]
            L.bsolve_last_error.argtypes = []
            L.bsolve_last_error.restype = C.c_char_p
            L.bsolve_probe_smem_bandwidth.argtypes = [C.c_int, C.POINTER(C.c_double),
                                                      C.POINTER(C.c_double)]
            L.bsolve_probe_fp64.argtypes = [C.c_int, C.POINTER(C.c_double), C.POINTER(C.c_double)]
            for f in ("bsolve_create", "bsolve_run", "bsolve_run_host", "bsolve_spmv",
                      "bsolve_csr_to_ell", "bsolve_query", "bsolve_ell_map", "bsolve_destroy",
                      "bsolve_ell_layout", "bsolve_banded_solve", "bsolve_banded_solve_host",
                      "bsolve_probe_smem_bandwidth", "bsolve_probe_fp64"):
                getattr(L, f).restype = C.c_int
            _lib = L
    return _lib


def check(rc: int):
    if rc != OK:
        raise BsolveError(rc, lib().bsolve_last_error().decode(errors="replace"))


def _stream_ptr(stream, device=None):
    """cudaStream_t of `stream`, default: the current stream of the handle's device."""
    import torch
    s = torch.cuda.current_stream(device) if stream is None else stream
    return s.cuda_stream


def ell_layout(row_ptr, col_idx):
    """Host-only ELL slot map of a pattern: (W, cols[W*n], src[W*n])."""
    rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
    ci = np.ascontiguousarray(col_idx, dtype=np.int32)
    n = rp.size - 1
    w = C.c_int32()
    check(lib().bsolve_ell_layout(n, rp.ctypes.data, ci.ctypes.data, C.byref(w), None, None))
    cols = np.empty(w.value * n, np.int32)
    src = np.empty(w.value * n, np.int32)
    check(lib().bsolve_ell_layout(n, rp.ctypes.data, ci.ctypes.data, C.byref(w),
                                  cols.ctypes.data, src.ctypes.data))
    return w.value, cols, src


def ell_values(csr_values, src):
    """[batch, nnz] CSR-ordered values -> [batch, W*n] ELL values given `src`."""
    v = np.asarray(csr_values, dtype=np.float64)
    out = np.zeros((v.shape[0], src.size), np.float64)
    ok = src >= 0
    out[:, ok] = v[:, src[ok]]
    return out


def probe_smem_bandwidth(device: int = -1):
    bw, hz = C.c_double(), C.c_double()
    check(lib().bsolve_probe_smem_bandwidth(int(device), C.byref(bw), C.byref(hz)))
    return bw.value, hz.value


def probe_fp64(device: int = -1):
    """(FP64 flop/s, SM clock Hz) of a DFMA loop over all SMs."""
    fl, hz = C.c_double(), C.c_double()
    check(lib().bsolve_probe_fp64(int(device), C.byref(fl), C.byref(hz)))
    return fl.value, hz.value


class Solver:
    """Batched preconditioned Krylov solve over one shared sparsity pattern.

    Solver(row_ptr, col_idx, batch, format="ell", placement="auto",
           stop="rel_b", true_residual_check=True, device=None,
           solver="bicgstab" | "gmres",
           precond="jacobi" | "none" | "block_jacobi" (8-row blocks, R30), restart=7,
           direct_fallback=False)
    .run(values, b, x0=None, tol=1e-10, maxiter=1000) -> (x, iters, resnorm, status)
    """

    def __init__(self, row_ptr, col_idx, batch: int, *, format: str = "ell",
                 placement: str = "auto", stop: str = "rel_b", true_residual_check: bool = True,
                 device: int | None = None, block_threads: int = 0, reg_slots: int = 0,
                 solver: str = "bicgstab", precond: str = "jacobi", restart: int = MAX_RESTART,
                 direct_fallback: bool = False):
        L = lib()
        rp = np.ascontiguousarray(row_ptr, dtype=np.int32)
        ci = np.ascontiguousarray(col_idx, dtype=np.int32)
        self.n = int(rp.size - 1)
        self.batch = int(batch)
        opt = Options()
        L.bsolve_default_options(C.byref(opt))
        opt.format = _FMT[format]
        opt.placement = _PLACE[placement]
        opt.stop = _STOP[stop]
        opt.true_residual_check = int(bool(true_residual_check))
        opt.device = -1 if device is None else int(device)
        opt.block_threads = int(block_threads)
        opt.reg_slots = int(reg_slots)
        opt.solver = _SOLVER[solver]
        opt.precond = _PREC[precond]
        opt.restart = int(restart)
        opt.direct_fallback = int(bool(direct_fallback))
        h = _P()
        check(L.bsolve_create(C.byref(h), self.n, self.batch, rp.ctypes.data, ci.ctypes.data,
                              C.byref(opt)))
        self._h = h
        self.info = self.query()
        self.device = self.info["device"]
        self.format = "ell" if self.info["format"] == FMT_ELL else "csr"
        self.width = self.info["ell_width"]
        self.nnz = self.info["nnz"]
        self.values_per_system = self.width * self.n if self.format == "ell" else self.nnz

    def query(self) -> dict:
        inf = Info()
        check(lib().bsolve_query(self._h, C.byref(inf)))
        return inf.as_dict()

    def ell_map(self):
        """(cols, src): the handle's ELL slot map, each [W*n] int32 column-major."""
        cols = np.empty(self.width * self.n, np.int32)
        src = np.empty(self.width * self.n, np.int32)
        check(lib().bsolve_ell_map(self._h, cols.ctypes.data, src.ctypes.data))
        return cols, src

    def ell_values(self, csr_values) -> np.ndarray:
        """Host-side re-layout of CSR-ordered values [batch, nnz] into this
        handle's ELL layout [batch, W*n] (pure permutation, zero padding)."""
        return ell_values(csr_values, self.ell_map()[1])

    def close(self):
        if getattr(self, "_h", None):
            lib().bsolve_destroy(self._h)
            self._h = None

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    # ------------------------------------------------------------ device --
    def _dev_check(self, t, name, shape, dtype):
        import torch
        if not isinstance(t, torch.Tensor) or not t.is_cuda:
            raise TypeError(f"{name} must be a CUDA tensor")
        if t.dtype != dtype or not t.is_contiguous():
            raise TypeError(f"{name} must be contiguous {dtype}")
        if t.numel() != int(np.prod(shape)):
            raise ValueError(f"{name} has {t.numel()} elements, expected {shape}")
        if t.device.index != self.device:
            raise ValueError(f"{name} lives on cuda:{t.device.index}, the handle on cuda:{self.device}")

    def alloc_outputs(self):
        import torch
        dev = torch.device("cuda", self.device)
        return (torch.empty((self.batch, self.n), dtype=torch.float64, device=dev),
                torch.empty(self.batch, dtype=torch.int32, device=dev),
                torch.empty(self.batch, dtype=torch.float64, device=dev),
                torch.empty(self.batch, dtype=torch.int8, device=dev))

    def run(self, values, b, x0=None, tol: float = 1e-10, maxiter: int = 1000, out=None,
            stream=None):
        """Asynchronous solve on the current (or given) CUDA stream."""
        import torch
        self._dev_check(values, "values", (self.batch, self.values_per_system), torch.float64)
        self._dev_check(b, "b", (self.batch, self.n), torch.float64)
        if x0 is not None:
            self._dev_check(x0, "x0", (self.batch, self.n), torch.float64)
        x, it, res, st = self.alloc_outputs() if out is None else out
        check(lib().bsolve_run(self._h, values.data_ptr(), b.data_ptr(),
                               None if x0 is None else x0.data_ptr(), float(tol), int(maxiter),
                               x.data_ptr(), it.data_ptr(), res.data_ptr(),
                               None if st is None else st.data_ptr(), _stream_ptr(stream, self.device)))
        return x, it, res, st

    def spmv(self, values, x, out=None, stream=None):
        import torch
        batch = int(x.shape[0]) if x.dim() > 0 else 0
        self._dev_check(x, "x", (batch, self.n), torch.float64)
        self._dev_check(values, "values", (batch, self.values_per_system), torch.float64)
        y = torch.empty_like(x) if out is None else out
        self._dev_check(y, "out", (batch, self.n), torch.float64)
        check(lib().bsolve_spmv(self._h, values.data_ptr(), x.data_ptr(), y.data_ptr(), int(batch),
                                _stream_ptr(stream, self.device)))
        return y

    def banded_solve(self, values, b, out=None, ipiv: bool = False, stream=None):
        """Batched banded LU with partial pivoting + solve (dgbsv analogue,
        SURVEY.md 8(f) f4): returns (x, info) or (x, info, ipiv)."""
        import torch
        self._dev_check(values, "values", (self.batch, self.values_per_system), torch.float64)
        self._dev_check(b, "b", (self.batch, self.n), torch.float64)
        dev = torch.device("cuda", self.device)
        if out is None:
            x = torch.empty((self.batch, self.n), dtype=torch.float64, device=dev)
            info = torch.empty(self.batch, dtype=torch.int32, device=dev)
        else:
            x, info = out
        piv = torch.empty((self.batch, self.n), dtype=torch.int32, device=dev) if ipiv else None
        check(lib().bsolve_banded_solve(self._h, values.data_ptr(), b.data_ptr(), x.data_ptr(),
                                        info.data_ptr(), None if piv is None else piv.data_ptr(),
                                        _stream_ptr(stream, self.device)))
        return (x, info, piv) if ipiv else (x, info)

    def csr_to_ell(self, csr_values, out=None, stream=None):
        import torch
        batch = int(csr_values.shape[0]) if csr_values.dim() > 0 else 0
        self._dev_check(csr_values, "csr_values", (batch, self.nnz), torch.float64)
        y = (torch.empty((batch, self.width * self.n), dtype=torch.float64,
                         device=csr_values.device) if out is None else out)
        self._dev_check(y, "out", (batch, self.width * self.n), torch.float64)
        check(lib().bsolve_csr_to_ell(self._h, csr_values.data_ptr(), y.data_ptr(), int(batch),
                                      _stream_ptr(stream, self.device)))
        return y

    # -------------------------------------------------------------- host --
    def run_host(self, values, b, x0=None, tol: float = 1e-10, maxiter: int = 1000, out=None):
        """Synchronous solve from HOST numpy arrays (pinned memory overlaps best)."""
        v = np.ascontiguousarray(values, dtype=np.float64)
        bb = np.ascontiguousarray(b, dtype=np.float64)
        assert v.size == self.batch * self.values_per_system and bb.size == self.batch * self.n
        xx0 = None if x0 is None else np.ascontiguousarray(x0, dtype=np.float64)
        if out is None:
            out = (np.empty((self.batch, self.n)), np.empty(self.batch, np.int32),
                   np.empty(self.batch), np.empty(self.batch, np.int8))
        x, it, res, st = out
        check(lib().bsolve_run_host(self._h, _np_ptr(v), _np_ptr(bb), _np_ptr(xx0), float(tol),
                                    int(maxiter), _np_ptr(x), _np_ptr(it), _np_ptr(res),
                                    _np_ptr(st)))
        return x, it, res, st

    def banded_solve_host(self, values, b, out=None):
        """Synchronous banded LU solve from HOST arrays (chunked H2D / solve /
        D2H pipeline; pinned memory overlaps best): returns (x, info)."""
        v = np.ascontiguousarray(values, dtype=np.float64)
        bb = np.ascontiguousarray(b, dtype=np.float64)
        assert v.size == self.batch * self.values_per_system and bb.size == self.batch * self.n
        if out is None:
            out = (np.empty((self.batch, self.n)), np.empty(self.batch, np.int32))
        x, info = out
        check(lib().bsolve_banded_solve_host(self._h, _np_ptr(v), _np_ptr(bb), _np_ptr(x),
                                             _np_ptr(info)))
        return x, info


def _np_ptr(a):
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        return a.data_ptr()
    return a.ctypes.data
