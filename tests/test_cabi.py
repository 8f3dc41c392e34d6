"""CPU-side checks of the C-ABI boundary (no GPU needed): the library loads,
exports every symbol include/bsolve.h declares, and rejects bad arguments and
bad patterns with the documented codes BEFORE any CUDA call."""
import ctypes as C
import os
import re

import numpy as np
import pytest

import paper_conf_ipps_kashinksla22_b200 as pkg
from paper_conf_ipps_kashinksla22_b200 import bsolve as B

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "bsolve.h")


def header_symbols():
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(bsolve_[a-z_]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    syms = header_symbols()
    for s in ("bsolve_create", "bsolve_run", "bsolve_destroy", "bsolve_last_error",
              "bsolve_run_host", "bsolve_spmv", "bsolve_csr_to_ell", "bsolve_query"):
        assert s in syms


def test_library_exports_every_header_symbol():
    L = C.CDLL(pkg.LIB_PATH)
    for s in header_symbols():
        assert hasattr(L, s), s


def test_library_built_for_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "-lelf", pkg.LIB_PATH], capture_output=True, text=True)
    assert "sm_100a" in out.stdout


def _create(n, rp, ci, **kw):
    L = B.lib()
    opt = B.Options()
    L.bsolve_default_options(C.byref(opt))
    for k, v in kw.items():
        setattr(opt, k, v)
    h = C.c_void_p()
    rpa = np.ascontiguousarray(rp, np.int32)
    cia = np.ascontiguousarray(ci, np.int32)
    rc = L.bsolve_create(C.byref(h), n, 4, rpa.ctypes.data, cia.ctypes.data, C.byref(opt))
    return rc, L.bsolve_last_error().decode()


def test_pattern_errors():
    # missing diagonal
    rc, msg = _create(2, [0, 1, 2], [1, 0])
    assert rc == B.ERR_PATTERN and "diagonal" in msg
    # column out of range
    rc, msg = _create(2, [0, 1, 2], [0, 5])
    assert rc == B.ERR_PATTERN and "range" in msg
    # unsorted / duplicate
    rc, _ = _create(2, [0, 2, 3], [1, 0, 1])
    assert rc == B.ERR_PATTERN
    rc, _ = _create(2, [0, 2, 3], [0, 0, 1])
    assert rc == B.ERR_PATTERN
    # row_ptr not starting at 0 / decreasing
    rc, _ = _create(2, [1, 2, 3], [0, 1, 1])
    assert rc == B.ERR_PATTERN
    rc, _ = _create(2, [0, 2, 1], [0, 1])
    assert rc == B.ERR_PATTERN


def test_invalid_arguments():
    L = B.lib()
    h = C.c_void_p()
    rp = np.array([0, 1], np.int32)
    ci = np.array([0], np.int32)
    assert L.bsolve_create(None, 1, 1, rp.ctypes.data, ci.ctypes.data, None) == B.ERR_INVALID
    assert L.bsolve_create(C.byref(h), 0, 1, rp.ctypes.data, ci.ctypes.data, None) == B.ERR_INVALID
    assert L.bsolve_create(C.byref(h), 1, -1, rp.ctypes.data, ci.ctypes.data, None) == B.ERR_INVALID
    assert L.bsolve_create(C.byref(h), 1, 1, None, ci.ctypes.data, None) == B.ERR_INVALID
    rc, _ = _create(1, rp, ci, format=7)
    assert rc == B.ERR_INVALID
    rc, _ = _create(1, rp, ci, placement=9)
    assert rc == B.ERR_INVALID
    rc, _ = _create(1, rp, ci, placement=6)
    assert rc == B.ERR_INVALID
    rc, _ = _create(1, rp, ci, stop=3)
    assert rc == B.ERR_INVALID
    rc, _ = _create(1, rp, ci, block_threads=100)
    assert rc == B.ERR_INVALID
    # NULL handle on every entry point
    assert L.bsolve_run(None, None, None, None, 1e-10, 10, None, None, None, None, None) == B.ERR_INVALID
    assert L.bsolve_run_host(None, None, None, None, 1e-10, 10, None, None, None, None) == B.ERR_INVALID
    assert L.bsolve_spmv(None, None, None, None, 1, None) == B.ERR_INVALID
    assert L.bsolve_csr_to_ell(None, None, None, 1, None) == B.ERR_INVALID
    assert L.bsolve_query(None, None) == B.ERR_INVALID
    assert L.bsolve_destroy(None) == B.OK


def test_unsupported_row_width():
    n = 20
    rp = np.arange(0, n * n + 1, n, dtype=np.int32)   # dense 20x20: 20 entries per row
    ci = np.tile(np.arange(n, dtype=np.int32), n)
    rc, msg = _create(n, rp, ci)
    assert rc == B.ERR_UNSUPPORTED and "entries" in msg


def test_fails_loudly_without_library(monkeypatch):
    monkeypatch.setattr(B, "_lib", None)
    monkeypatch.setattr(B, "LIB_PATH", "/nonexistent/libbsolve.so")
    with pytest.raises(ImportError):
        B.lib()


def test_product_never_touches_oracle():
    pkgdir = os.path.dirname(pkg.__file__)
    for dp, _, fs in os.walk(pkgdir):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert not re.search(r"^\s*(import|from)\s+oracle\b", txt, re.M), f
                assert "oracle.c" not in txt and "liboracle" not in txt, f


# ------------------------------------------------------------ ELL slot map --
def _check_map(rp, ci, W, cols, src):
    n = len(rp) - 1
    seen = np.zeros(rp[-1], np.int32)
    for k in range(W):
        for i in range(n):
            e = src[k * n + i]
            if e >= 0:
                assert rp[i] <= e < rp[i + 1]          # entry belongs to row i
                assert cols[k * n + i] == ci[e]
                seen[e] += 1
            else:
                assert 0 <= cols[k * n + i] < n         # padding reads a valid column
    assert np.all(seen == 1)                            # every CSR entry exactly once


def test_ell_map_is_a_valid_permutation():
    import xgcgen as X
    for (nx, ny) in [(32, 31), (31, 32), (5, 5), (1, 1), (64, 63)]:
        pat = X.stencil_pattern(nx, ny)
        W, cols, src = pkg.ell_layout(pat.row_ptr, pat.col_idx)
        assert W == pat.max_row_nnz
        _check_map(pat.row_ptr, pat.col_idx, W, cols, src)
        assert int(np.sum(src < 0)) == W * pat.n - pat.nnz  # 374 pads at 32x31
    for seed in range(3):
        rp, ci = X.random_pattern(300, 12, seed=seed)
        W, cols, src = pkg.ell_layout(rp, ci)
        _check_map(rp, ci, W, cols, src)


def _excess_wavefronts(cols, n, W):
    """Bank-conflict excess of the gather LDS.64 of each (warp, slot): lanes
    of a half-warp hitting the same 8-byte bank pair at different addresses."""
    excess = 0
    for k in range(W):
        for w0 in range(0, n, 32):
            for h0 in (w0, w0 + 16):
                addr = [cols[k * n + i] for i in range(h0, min(h0 + 16, n))]
                banks = {}
                for a in set(addr):
                    banks.setdefault(a % 16, set()).add(a)
                excess += max(len(v) for v in banks.values()) - 1 if banks else 0
    return excess


def test_ell_map_conflict_free_gathers_on_stencil():
    """the library's slot assignment makes the 9-point
    gathers conflict-free, where the CSR-order slot assignment is not."""
    import xgcgen as X
    pat = X.stencil_pattern(32, 31)
    W, cols, src = pkg.ell_layout(pat.row_ptr, pat.col_idx)
    csr_cols, _ = X.ell_layout(pat.row_ptr, pat.col_idx)
    assert _excess_wavefronts(cols, pat.n, W) == 0
    assert _excess_wavefronts(csr_cols, pat.n, W) > 0


def test_ell_layout_rejects_bad_pattern():
    with pytest.raises(B.BsolveError) as e:
        pkg.ell_layout([0, 1, 2], [1, 0])
    assert e.value.code == B.ERR_PATTERN


def test_ell_map_slot0_diagonal_and_stencil_offsets():
    """Slot 0 holds the diagonal in every row (any pattern); for stencils each
    slot has one column offset (the kernel's DIA addressing)."""
    import xgcgen as X
    pats = [X.stencil_pattern(32, 31), X.stencil_pattern(5, 5), X.stencil_pattern(64, 32)]
    for pat in pats:
        W, cols, src = pkg.ell_layout(pat.row_ptr, pat.col_idx)
        n = pat.n
        assert np.all(cols[:n] == np.arange(n)) and np.all(src[:n] >= 0)
        for k in range(W):
            offs = {int(cols[k * n + i]) - i for i in range(n) if src[k * n + i] >= 0}
            assert len(offs) == 1
    rp, ci = X.random_pattern(200, 9, seed=7)
    W, cols, src = pkg.ell_layout(rp, ci)
    assert np.all(cols[:200] == np.arange(200)) and np.all(src[:200] >= 0)


def _header_struct_fields(name):
    txt = re.sub(r"/\*.*?\*/", "", open(HEADER).read(), flags=re.S)
    body = re.search(r"typedef struct " + name + r" \{(.*?)\}", txt, flags=re.S).group(1)
    fields = []
    for decl in body.split(";"):
        decl = decl.strip()
        if decl:
            fields += [f.strip() for f in decl.split(None, 1)[1].split(",")]
    return fields


def test_binding_structs_match_the_header():
    """The ctypes mirrors of bsolve_options / bsolve_info list the header's
    int fields in the header's order (a mismatch would shift every option)."""
    assert [f for f, _ in B.Options._fields_] == _header_struct_fields("bsolve_options")
    assert [f for f, _ in B.Info._fields_] == _header_struct_fields("bsolve_info")


def test_direct_fallback_needs_status():
    """direct_fallback selects the systems to re-solve from status[]: a NULL
    status is rejected before any CUDA call."""
    rp = np.array([0, 1], np.int32)
    ci = np.array([0], np.int32)
    L = B.lib()
    opt = B.Options()
    L.bsolve_default_options(C.byref(opt))
    assert opt.direct_fallback == 0
    opt.direct_fallback = 1
    h = B._P()
    rc = L.bsolve_create(C.byref(h), 1, 1, rp.ctypes.data, ci.ctypes.data, C.byref(opt))
    if rc != B.OK:  # no GPU in this container: create fails at the device query
        pytest.skip("bsolve_create needs a CUDA device")
    d = C.c_void_p(1)
    rc = L.bsolve_run(h, d, d, None, 1e-10, 10, d, d, d, None, None)
    L.bsolve_destroy(h)
    assert rc == B.ERR_INVALID


def test_direct_fallback_wide_band_rejected_before_cuda():
    """direct_fallback needs a banded-kernel instance for the pattern: a band
    wider than 65 is UNSUPPORTED at create time, before any CUDA call."""
    n = 100
    rp, ci = [0], []
    for i in range(n):
        ci += sorted({i, (i + 70) % n})
        rp.append(len(ci))
    rp, ci = np.array(rp, np.int32), np.array(ci, np.int32)
    L = B.lib()
    opt = B.Options()
    L.bsolve_default_options(C.byref(opt))
    opt.direct_fallback = 1
    h = B._P()
    assert L.bsolve_create(C.byref(h), n, 2, rp.ctypes.data, ci.ctypes.data, C.byref(opt)) == \
        B.ERR_UNSUPPORTED
    assert "direct_fallback" in L.bsolve_last_error().decode()
