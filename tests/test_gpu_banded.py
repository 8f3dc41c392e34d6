"""GPU parity of the batched banded LU solver (bsolve_banded_solve, the dgbsv
analogue of SURVEY.md 8(f) f4) against the
oracle's dgbtf2 + dgbtrs (oracle/oracle.c oracle_banded_solve_piv).

Bar (f4 rows):
  * ipiv (integer): bit-exact.  Both sides pick the pivot in fp64 from values
    that agree to rounding; the test inputs have no near-ties.
  * info (integer): equal.
  * x: ||x_gpu - x_oracle|| / ||x_oracle|| <= FWD (kernel: fused multiply-add
    and the multiplier folded as a_kj * (u_jc / u_jj), R25), with
    FWD = 1e-12 on the well-conditioned XGC systems and a condition-scaled
    bound on the pivoting-heavy random ones.
"""
import numpy as np
import pytest
import torch

import oracle as O
import xgcgen as X
from paper_conf_ipps_kashinksla22_b200 import Solver

pytestmark = pytest.mark.gpu


def to_dev(a, dtype=torch.float64):
    return torch.as_tensor(np.ascontiguousarray(a)).to(device="cuda", dtype=dtype)


def gpu_banded(row_ptr, col_idx, csr_values, b, fmt="ell"):
    batch = csr_values.shape[0]
    S = Solver(row_ptr, col_idx, batch, format=fmt)
    vals = S.ell_values(csr_values) if S.format == "ell" else csr_values
    x, info, piv = S.banded_solve(to_dev(vals), to_dev(b), ipiv=True)
    torch.cuda.synchronize()
    out = x.cpu().numpy(), info.cpu().numpy(), piv.cpu().numpy()
    S.close()
    return out


def oracle_banded(row_ptr, col_idx, csr_values, b):
    xs, infos, pivs = [], [], []
    for k in range(csr_values.shape[0]):
        x, info, piv = O.banded_factor_solve(row_ptr, col_idx, csr_values[k], b[k])
        xs.append(x)
        infos.append(info)
        pivs.append(piv)
    return np.array(xs), np.array(infos), np.array(pivs)


def check(row_ptr, col_idx, vals, b, fmt="ell", fwd=1e-12):
    xg, ig, pg = gpu_banded(row_ptr, col_idx, vals, b, fmt)
    xo, io, po = oracle_banded(row_ptr, col_idx, vals, b)
    assert np.array_equal(ig, io), (ig, io)
    assert np.array_equal(pg, po), np.argwhere(pg != po)[:5]
    ok = io == 0
    rel = np.linalg.norm(xg[ok] - xo[ok], axis=1) / np.linalg.norm(xo[ok], axis=1)
    assert rel.max(initial=0.0) <= fwd, rel.max()
    return xg, pg


@pytest.mark.parametrize("fmt", ["ell", "csr"])
def test_xgc_pair(fmt):
    """configs[0]: the ion + electron pair at 32 x 31 (kl = ku = 33, KB = 33)."""
    B = X.make_batch(0, 2)
    p = B.pattern
    xg, pg = check(p.row_ptr, p.col_idx, B.values, B.b, fmt)
    # the direct solution also satisfies the 1e-10 relative residual bar
    for k in range(2):
        r = B.b[k] - O.spmv(p.row_ptr, p.col_idx, B.values[k], xg[k])
        assert np.linalg.norm(r) / np.linalg.norm(B.b[k]) <= 1e-13


def test_xgc_batch_many_waves():
    """configs[1] size (1280 systems): more systems than resident CTAs, so
    every CTA of the persistent grid solves several (workspace reuse)."""
    B = X.make_batch(0, 1280)
    p = B.pattern
    check(p.row_ptr, p.col_idx, B.values, B.b)


@pytest.mark.parametrize("nx,ny", [(3, 3), (5, 4), (7, 5), (12, 9), (17, 6), (32, 31)])
@pytest.mark.parametrize("fmt", ["ell", "csr"])
def test_pivoting_random(nx, ny, fmt):
    """Random 9-point values with tiny diagonals: most steps interchange rows,
    exercising the swap path of every instance (KB = 4, 8, 16, 33) and n not a
    multiple of the unroll (ragged last block)."""
    pat = X.stencil_pattern(nx, ny)
    rng = np.random.default_rng(nx * 1000 + ny)
    batch = 40
    v = rng.standard_normal((batch, pat.nnz))
    diag = pat.col_idx == np.repeat(np.arange(pat.n), np.diff(pat.row_ptr))
    v[:, diag] *= 1e-2
    b = rng.standard_normal((batch, pat.n))
    xo, io, po = oracle_banded(pat.row_ptr, pat.col_idx, v, b)
    assert np.all(io == 0)
    assert np.mean(po != np.arange(pat.n)) > 0.2
    # condition-scaled bound: kappa_1 estimate of each system
    kap = max(np.linalg.cond(X_dense(pat, v[k]), 1) for k in range(min(batch, 8)))
    check(pat.row_ptr, pat.col_idx, v, b, fmt, fwd=max(1e-12, 1e-15 * kap * pat.n))


def X_dense(pat, v):
    A = np.zeros((pat.n, pat.n))
    for i in range(pat.n):
        for e in range(pat.row_ptr[i], pat.row_ptr[i + 1]):
            A[i, pat.col_idx[e]] = v[e]
    return A


def test_tridiagonal_and_tiny():
    """kl = ku = 1 (KB = 4 instance) at n = 1, 2, 3, 50; diagonal n = 1."""
    for n in (1, 2, 3, 50):
        rp = [0]
        ci = []
        for i in range(n):
            for j in (i - 1, i, i + 1):
                if 0 <= j < n:
                    ci.append(j)
            rp.append(len(ci))
        rp, ci = np.array(rp, np.int32), np.array(ci, np.int32)
        rng = np.random.default_rng(n)
        v = rng.standard_normal((5, ci.size))
        b = rng.standard_normal((5, n))
        check(rp, ci, v, b, fwd=1e-10)


def test_singular_info():
    """A zero column j gives info = j+1 (LAPACK), same as the oracle; the
    other systems of the batch are unaffected."""
    pat = X.stencil_pattern(32, 31)
    v = X.random_dd_values(pat.row_ptr, pat.col_idx, 3, seed=11).copy()
    v[1, pat.col_idx == 500] = 0.0
    b = X.random_rhs(3, pat.n, seed=2)
    xg, ig, pg = gpu_banded(pat.row_ptr, pat.col_idx, v, b)
    xo, io, po = oracle_banded(pat.row_ptr, pat.col_idx, v, b)
    assert list(ig) == [0, 501, 0] and np.array_equal(ig, io)
    assert np.array_equal(pg, po)
    for k in (0, 2):
        assert np.linalg.norm(xg[k] - xo[k]) / np.linalg.norm(xo[k]) <= 1e-12


def test_large_grid_kb65():
    """configs[4] grid 64 x 63 (n = 4032, kl = ku = 65: KB = 65 instance)."""
    B = X.make_batch(0, 6, nx=64, ny=63)
    p = B.pattern
    check(p.row_ptr, p.col_idx, B.values, B.b)


def test_bandwidth_too_large_is_unsupported():
    """A pattern with kl > 65 has no instance: UNSUPPORTED, nothing launched."""
    from paper_conf_ipps_kashinksla22_b200.bsolve import BsolveError, ERR_UNSUPPORTED
    n = 100
    rp, ci = [0], []
    for i in range(n):
        cols = sorted({i, (i + 70) % n})
        ci += cols
        rp.append(len(ci))
    S = Solver(np.array(rp, np.int32), np.array(ci, np.int32), 2, format="csr")
    v = torch.ones((2, len(ci)), dtype=torch.float64, device="cuda")
    b = torch.ones((2, n), dtype=torch.float64, device="cuda")
    with pytest.raises(BsolveError) as e:
        S.banded_solve(v, b)
    assert e.value.code == ERR_UNSUPPORTED


# ------------------------------------------- direct fallback in bsolve_run --
def _run(p, vals, b, **kw):
    maxiter = kw.pop("maxiter", 1000)
    S = Solver(p.row_ptr, p.col_idx, vals.shape[0], **kw)
    ev = to_dev(S.ell_values(vals))
    x, it, res, st = S.run(ev, to_dev(b), maxiter=maxiter)
    torch.cuda.synchronize()
    out = x.cpu().numpy(), it.cpu().numpy(), res.cpu().numpy(), st.cpu().numpy()
    return S, out


def test_direct_fallback_replaces_non_converged():
    """maxiter = 6: ions converge (status 0, untouched), electrons do not
    (status 1) and are re-solved by the banded LU: status DIRECT (3), x = the
    oracle's banded solution, resnorm = its true residual, iters kept."""
    B = X.make_batch(0, 300)
    p = B.pattern
    _, (x0, it0, r0, s0) = _run(p, B.values, B.b, maxiter=6)
    assert np.any(s0 == 0) and np.any(s0 == 1)
    _, (x1, it1, r1, s1) = _run(p, B.values, B.b, maxiter=6, direct_fallback=True)
    conv = s0 == 0
    assert np.array_equal(s1[conv], s0[conv]) and np.array_equal(x1[conv], x0[conv])
    assert np.array_equal(r1[conv], r0[conv])
    assert np.all(s1[~conv] == 3) and np.array_equal(it1, it0)
    xo, io, _ = oracle_banded(p.row_ptr, p.col_idx, B.values[~conv], B.b[~conv])
    assert np.all(io == 0)
    rel = np.linalg.norm(x1[~conv] - xo, axis=1) / np.linalg.norm(xo, axis=1)
    assert rel.max() <= 1e-12
    bn = np.linalg.norm(B.b[~conv], axis=1)
    tr = np.array([np.linalg.norm(B.b[k] - O.spmv(p.row_ptr, p.col_idx, B.values[k], x1[k]))
                   for k in np.nonzero(~conv)[0]])
    assert np.all(r1[~conv] <= 1e-13 * bn) and np.allclose(r1[~conv], tr, rtol=0.5, atol=1e-14 * bn.max())


def test_direct_fallback_singular_keeps_iterative_result_and_host_path():
    """A singular band cannot be solved directly: that system keeps its
    iterative x, resnorm and status; run_host gives the same outputs."""
    pat = X.stencil_pattern(32, 31)
    v = X.random_dd_values(pat.row_ptr, pat.col_idx, 4, seed=11).copy()
    v[2, pat.col_idx == 500] = 0.0          # column 500 of A_2 is zero: singular
    b = X.random_rhs(4, pat.n, seed=2)
    _, (x0, it0, r0, s0) = _run(pat, v, b, maxiter=2)
    S, (x1, it1, r1, s1) = _run(pat, v, b, maxiter=2, direct_fallback=True)
    assert s0[2] != 0 and s1[2] == s0[2] and np.array_equal(x1[2], x0[2]) and r1[2] == r0[2]
    others = [0, 1, 3]
    assert np.all(s1[others] == 3)
    xh, ih, rh, sh = S.run_host(S.ell_values(v), b, maxiter=2)
    assert np.array_equal(sh, s1) and np.array_equal(xh, x1) and np.array_equal(rh, r1)


def test_direct_fallback_rejects_wide_band_at_create():
    """direct_fallback on a pattern the banded kernels cannot cover fails in
    bsolve_create (UNSUPPORTED), not later inside bsolve_run."""
    from paper_conf_ipps_kashinksla22_b200.bsolve import BsolveError, ERR_UNSUPPORTED
    n = 100
    rp, ci = [0], []
    for i in range(n):
        ci += sorted({i, (i + 70) % n})
        rp.append(len(ci))
    with pytest.raises(BsolveError) as e:
        Solver(np.array(rp, np.int32), np.array(ci, np.int32), 2, format="csr",
               direct_fallback=True)
    assert e.value.code == ERR_UNSUPPORTED


def test_host_pipeline_banded_and_fallback_many_chunks():
    """bsolve_banded_solve_host (3 streams, one workspace per pipeline slot)
    equals the device path bit for bit over several chunks; run_host with
    direct_fallback (banded re-solves on concurrent streams) equals run."""
    B = X.make_batch(0, 3000)
    p = B.pattern
    S = Solver(p.row_ptr, p.col_idx, 3000)
    ev = S.ell_values(B.values)
    xd, infod = S.banded_solve(to_dev(ev), to_dev(B.b))
    xh, infoh = S.banded_solve_host(ev, B.b)
    torch.cuda.synchronize()
    assert np.array_equal(xh, xd.cpu().numpy()) and np.array_equal(infoh, infod.cpu().numpy())
    F = Solver(p.row_ptr, p.col_idx, 3000, direct_fallback=True)
    x1, it1, r1, s1 = F.run(to_dev(ev), to_dev(B.b), maxiter=6)
    torch.cuda.synchronize()
    x2, it2, r2, s2 = F.run_host(ev, B.b, maxiter=6)
    assert np.any(s2 == 3) and np.array_equal(s2, s1.cpu().numpy())
    assert np.array_equal(x2, x1.cpu().numpy()) and np.array_equal(r2, r1.cpu().numpy())


def test_direct_fallback_with_gmres():
    """direct_fallback also covers the GMRES(m) solver's non-converged systems."""
    B = X.make_batch(0, 64)
    p = B.pattern
    _, (x0, it0, r0, s0) = _run(p, B.values, B.b, maxiter=5, solver="gmres")
    _, (x1, it1, r1, s1) = _run(p, B.values, B.b, maxiter=5, solver="gmres", direct_fallback=True)
    bad = s0 != 0
    assert np.any(bad) and np.all(s1[bad] == 3) and np.array_equal(x1[~bad], x0[~bad])
    xo, _, _ = oracle_banded(p.row_ptr, p.col_idx, B.values[bad], B.b[bad])
    assert np.max(np.linalg.norm(x1[bad] - xo, axis=1) / np.linalg.norm(xo, axis=1)) <= 1e-12


def test_direct_fallback_csr_resnorm_is_true_residual():
    """CSR values + direct_fallback: the DIRECT systems' resnorm is the true
    ||b - A x|| (the residual reads each value with its own column: ADVICE r1)."""
    B = X.make_batch(0, 64)
    p = B.pattern
    S = Solver(p.row_ptr, p.col_idx, 64, format="csr", direct_fallback=True)
    x, it, res, st = S.run(to_dev(B.values), to_dev(B.b), maxiter=6)
    torch.cuda.synchronize()
    x, res, st = x.cpu().numpy(), res.cpu().numpy(), st.cpu().numpy()
    assert np.any(st == 3) and np.any(st == 0)
    for k in np.nonzero(st == 3)[0]:
        tr = np.linalg.norm(B.b[k] - O.spmv(p.row_ptr, p.col_idx, B.values[k], x[k]))
        bn = np.linalg.norm(B.b[k])
        assert res[k] <= 1e-13 * bn and abs(res[k] - tr) <= 0.5 * tr + 1e-15 * bn, (k, res[k], tr)
    assert S.query()["banded_launches"] == 2  # compaction + one fused solve launch


def test_direct_fallback_no_failures_is_cheap():
    """All systems converge: the fallback launches still run (compaction +
    an immediately-exiting solve) and change nothing, bit for bit."""
    B = X.make_batch(0, 600)
    p = B.pattern
    _, (x0, it0, r0, s0) = _run(p, B.values, B.b)
    _, (x1, it1, r1, s1) = _run(p, B.values, B.b, direct_fallback=True)
    assert np.all(s0 == 0)
    for a, b in ((x0, x1), (it0, it1), (r0, r1), (s0, s1)):
        assert np.array_equal(a, b)


def test_banded_large_grid_backsub_smem():
    """64 x 127 grid (n = 8128, kb = 65): the split back substitution sizes its
    per-warp x arrays to the device's SMEM limit."""
    pat = X.stencil_pattern(64, 127)
    B = X.make_batch(0, 3, pattern=pat)
    S = Solver(pat.row_ptr, pat.col_idx, 3)
    x, info = S.banded_solve(to_dev(S.ell_values(B.values)), to_dev(B.b))
    torch.cuda.synchronize()
    x, info = x.cpu().numpy(), info.cpu().numpy()
    assert np.all(info == 0)
    xo, io, _ = oracle_banded(pat.row_ptr, pat.col_idx, B.values, B.b)
    assert np.max(np.linalg.norm(x - xo, axis=1) / np.linalg.norm(xo, axis=1)) <= 1e-12


@pytest.mark.parametrize("nx,ny,pivot", [(32, 31, False), (32, 31, True), (12, 9, True),
                                         (17, 6, True), (5, 4, True), (31, 32, False)])
def test_warp_kernel_bitwise_equals_cta_kernel(nx, ny, pivot, monkeypatch):
    """The one-warp-per-system factorisation (banded_lu_warp_kernel, default in
    split mode) does every column's operations in the CTA kernel's order, so x,
    info and ipiv agree bit for bit with BSOLVE_BANDED_WARP=0 (instances KB =
    4, 16, 33; pivoting-heavy and XGC values), and both match the oracle."""
    pat = X.stencil_pattern(nx, ny)
    if pivot:
        rng = np.random.default_rng(nx * 7 + ny)
        v = rng.standard_normal((24, pat.nnz))
        v[:, pat.col_idx == np.repeat(np.arange(pat.n), np.diff(pat.row_ptr))] *= 1e-2
        b = rng.standard_normal((24, pat.n))
    else:
        B = X.make_batch(0, 24, nx=nx, ny=ny)
        v, b = B.values, B.b
    outs = []
    for knob in (None, "0"):
        if knob is None:
            monkeypatch.delenv("BSOLVE_BANDED_WARP", raising=False)
        else:
            monkeypatch.setenv("BSOLVE_BANDED_WARP", knob)
        outs.append(gpu_banded(pat.row_ptr, pat.col_idx, v, b))
    for a, c in zip(outs[0], outs[1]):
        assert np.array_equal(a, c)
    xo, io, po = oracle_banded(pat.row_ptr, pat.col_idx, v, b)
    assert np.array_equal(outs[0][1], io) and np.array_equal(outs[0][2], po)
