"""Parity at BASELINE.json's full size, in the launch configuration bench.py
times (10^5 XGC systems of 992 rows, 50/50 ion/electron, x0 = 0, one launch):
sampled systems against the oracle one by one, and properties that hold at
any size over every system.

  * BiCGSTAB (default plan, the bench kernel): every 1999th system vs the
    oracle's Algorithm 1 (|d iters| <= 2, equal status) and banded LU
    (||x - x_direct|| / ||x_direct|| <= 1e-8); all systems: converged, the
    reported TRUE residual <= 1e-10 ||b||, iteration counts in the species
    bands of SURVEY.md 8(d).
  * Banded LU (bsolve_banded_solve, f4): sampled systems vs the oracle's
    dgbtf2 + dgbtrs (ipiv bit-exact, x <= 1e-12 relative); all systems: info 0.
"""
import os
import sys
import types

import numpy as np
import pytest
import torch

import oracle as O
import xgcgen as X
from paper_conf_ipps_kashinksla22_b200 import Solver

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402  (input generator of the bench workload)

pytestmark = pytest.mark.gpu

BATCH = 100_000
STRIDE = 1999


@pytest.fixture(scope="module")
def workload():
    args = types.SimpleNamespace(nx=32, ny=31, format="ell", seed=X.DEFAULT_SEED)
    pat, vals_h, b_h = bench.make_inputs(0, BATCH, args, pinned=True)
    idx = np.arange(0, BATCH, STRIDE)
    idx = np.unique(np.concatenate([idx, idx + 1, [BATCH - 1]]))  # ions and electrons
    idx = idx[idx < BATCH]
    # the sampled systems regenerated one by one in CSR order for the oracle
    samples = [X.make_batch(int(g), 1, pattern=pat) for g in idx]
    return pat, vals_h, b_h, idx, samples


def test_bicgstab_full_size_sampled(workload):
    pat, vals_h, b_h, idx, samples = workload
    S = Solver(pat.row_ptr, pat.col_idx, BATCH)
    assert S.info["kernel_mode"] == 4  # the bench plan (line-tiled TMEM)
    vals, b = vals_h.cuda(), b_h.cuda()
    x, it, res, st = S.run(vals, b, tol=1e-10, maxiter=1000)
    torch.cuda.synchronize()
    it, res, st = it.cpu().numpy(), res.cpu().numpy(), st.cpu().numpy()
    bn = torch.linalg.norm(b, dim=1).cpu().numpy()
    assert np.all(st == 0)
    assert np.all(res <= 1e-10 * bn)
    assert 2 <= it[0::2].min() and it[0::2].max() <= 12       # ions
    assert 15 <= it[1::2].min() and it[1::2].max() <= 45      # electrons
    xs = x[torch.as_tensor(idx, device="cuda")].cpu().numpy()
    for k, g in enumerate(idx):
        B = samples[k]
        o = O.batch_bicgstab(pat.row_ptr, pat.col_idx, B.values, B.b)
        xd = O.banded_solve(pat.row_ptr, pat.col_idx, B.values[0], B.b[0])
        assert abs(int(it[g]) - int(o["iters"][0])) <= 2, (g, it[g], o["iters"][0])
        assert int(st[g]) == int(o["status"][0])
        assert np.linalg.norm(xs[k] - xd) / np.linalg.norm(xd) <= 1e-8


def test_banded_full_size_sampled(workload):
    pat, vals_h, b_h, idx, samples = workload
    S = Solver(pat.row_ptr, pat.col_idx, BATCH)
    vals, b = vals_h.cuda(), b_h.cuda()
    x, info, piv = S.banded_solve(vals, b, ipiv=True)
    torch.cuda.synchronize()
    assert int((info != 0).sum().item()) == 0
    sel = torch.as_tensor(idx, device="cuda")
    xs, ps = x[sel].cpu().numpy(), piv[sel].cpu().numpy()
    for k in range(len(idx)):
        B = samples[k]
        xo, io, po = O.banded_factor_solve(pat.row_ptr, pat.col_idx, B.values[0], B.b[0])
        assert io == 0 and np.array_equal(ps[k], po)
        assert np.linalg.norm(xs[k] - xo) / np.linalg.norm(xo) <= 1e-12


def test_literal_three_round_schedule(monkeypatch):
    """The 3-CTA line kernel with Alg. 1's literal schedule (rho = r^.r and
    ||r|| from a third reduction, BSOLVE_ROUNDS=3; the default takes them
    from the omega round, R29): same parity bar."""
    monkeypatch.setenv("BSOLVE_ROUNDS", "3")
    B = X.make_batch(0, 300)
    p = B.pattern
    S = Solver(p.row_ptr, p.col_idx, 300)
    assert S.info["kernel_mode"] == 4
    vals = torch.from_numpy(S.ell_values(B.values)).cuda()
    x, it, res, st = S.run(vals, torch.from_numpy(B.b).cuda())
    torch.cuda.synchronize()
    o = O.batch_bicgstab(p.row_ptr, p.col_idx, B.values, B.b)
    assert np.array_equal(st.cpu().numpy(), o["status"])
    assert np.abs(it.cpu().numpy().astype(int) - o["iters"].astype(int)).max() <= 2
    xd = O.batch_banded(p.row_ptr, p.col_idx, B.values, B.b)
    xg = x.cpu().numpy()
    assert np.max(np.linalg.norm(xg - xd, axis=1) / np.linalg.norm(xd, axis=1)) <= 1e-8


