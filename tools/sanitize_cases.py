"""Small solves through every kernel family, for compute-sanitizer runs:
  compute-sanitizer --tool {memcheck,racecheck,synccheck} python tools/sanitize_cases.py
Exits non-zero if any result fails the parity bar against the direct solve."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle as O  # noqa: E402  (test infrastructure: checks the results)
import xgcgen as X  # noqa: E402
from paper_conf_ipps_kashinksla22_b200 import Solver  # noqa: E402

# (name, grid, Solver options[, developer env knobs read by bsolve_create])
CASES = [
    ("line-tiled tmem (bench default)", dict(nx=32, ny=31), dict()),
    ("line-tiled tmem, grid 31x32", dict(nx=31, ny=32), dict()),
    ("line-tiled generic width 40x25", dict(nx=40, ny=25), dict()),
    ("line-tiled generic width 5x7", dict(nx=5, ny=7), dict()),
    ("line-tiled GMRES(7)", dict(nx=32, ny=31), dict(solver="gmres")),
    ("line-tiled + direct fallback", dict(nx=32, ny=31), dict(direct_fallback=True)),
    ("strided tmem (line off)", dict(nx=32, ny=31), dict(), {"BSOLVE_TMEM_LINE": "0"}),
    ("tmem values, unaligned block (5x5)", dict(nx=5, ny=5), dict(placement="tmem")),
    ("hybrid 128x8 DIA, 4 reg slots", dict(nx=32, ny=31), dict(block_threads=128, reg_slots=4)),
    ("smem 256x4 DIA", dict(nx=32, ny=31), dict(block_threads=256)),
    ("csr smem", dict(nx=32, ny=31), dict(format="csr")),
    ("stream ell", dict(nx=32, ny=31), dict(placement="stream")),
    ("persistent regs", dict(nx=32, ny=31), dict(placement="regs")),
    ("cluster C=3 (n=2112)", dict(nx=64, ny=33), dict()),
    ("line-tiled cluster C=4 (n=4032)", dict(nx=64, ny=63), dict()),
    ("line-tiled cluster C=4, halo exchange", dict(nx=64, ny=63), dict(),
     {"BSOLVE_CLUSTER_SYNC": "halo"}),
    ("line-tiled block-Jacobi", dict(nx=32, ny=31), dict(precond="block_jacobi")),
    ("line-tiled cluster C=4 block-Jacobi", dict(nx=64, ny=63), dict(precond="block_jacobi")),
    ("strided cluster C=4 (st.async)", dict(nx=64, ny=63), dict(), {"BSOLVE_CLUSTER_LINE": "0"}),
]


def banded_cases():
    """f4 banded LU (bsolve_banded_solve): XGC systems (KB = 33), pivoting-heavy
    random values (KB = 8, swaps every step), more systems than CTAs."""
    bad = 0
    for name, grid, pivot, batch, knob in (
            ("banded 32x31 (KB=33), warp kernel", dict(nx=32, ny=31), False, 3, None),
            ("banded 32x31 (KB=33), CTA kernel", dict(nx=32, ny=31), False, 3, "0"),
            ("banded 7x5 pivoting (KB=8), warp", dict(nx=7, ny=5), True, 5, None),
            ("banded 7x5 pivoting (KB=8), CTA", dict(nx=7, ny=5), True, 5, "0")):
        # BSOLVE_BANDED_WARP is read at launch: 0 = the multi-warp CTA kernel
        if knob is None:
            os.environ.pop("BSOLVE_BANDED_WARP", None)
        else:
            os.environ["BSOLVE_BANDED_WARP"] = knob
        pat = X.stencil_pattern(**grid)
        B = X.make_batch(0, batch, pattern=pat)
        vals = B.values.copy()
        if pivot:
            rng = np.random.default_rng(1)
            vals = rng.standard_normal(vals.shape)
            diag = pat.col_idx == np.repeat(np.arange(pat.n), np.diff(pat.row_ptr))
            vals[:, diag] *= 1e-2
        S = Solver(pat.row_ptr, pat.col_idx, batch)
        x, info, piv = S.banded_solve(torch.from_numpy(S.ell_values(vals)).cuda(),
                                      torch.from_numpy(B.b).cuda(), ipiv=True)
        torch.cuda.synchronize()
        x, piv = x.cpu().numpy(), piv.cpu().numpy()
        err, same = 0.0, True
        for k in range(batch):
            xo, io, po = O.banded_factor_solve(pat.row_ptr, pat.col_idx, vals[k], B.b[k])
            err = max(err, np.linalg.norm(x[k] - xo) / np.linalg.norm(xo))
            same = same and np.array_equal(piv[k], po)
        os.environ.pop("BSOLVE_BANDED_WARP", None)
        ok = err <= 1e-10 and same and int(info.abs().sum()) == 0
        bad += not ok
        print(f"{name:32s} fwd_err_vs_oracle={err:.2e} ipiv_equal={same} {'ok' if ok else 'FAIL'}",
              flush=True)
    return bad


def main():
    batch = int(os.environ.get("SAN_BATCH", "3"))
    only = os.environ.get("SAN_CASES")
    bad = banded_cases() if not only or "banded" in only else 0
    if os.environ.get("SAN_ONLY_BANDED"):
        sys.exit(1 if bad else 0)
    # SAN_CASES: comma-separated substrings of case names ("banded": the f4 cases)
    for case in CASES:
        name, grid, opts = case[:3]
        if only and not any(k in name for k in only.split(",")):
            continue
        env = case[3] if len(case) > 3 else {}
        saved = {k: os.environ.get(k) for k in env}
        os.environ.update(env)
        pat = X.stencil_pattern(**grid)
        B = X.make_batch(0, batch, pattern=pat)
        S = Solver(pat.row_ptr, pat.col_idx, batch, **opts)
        for k, v in saved.items():  # knobs are read at create time only
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v
        vals = S.ell_values(B.values) if S.format == "ell" else B.values
        x, it, res, st = S.run(torch.from_numpy(vals).cuda(), torch.from_numpy(B.b).cuda())
        torch.cuda.synchronize()
        x = x.cpu().numpy()
        xd = O.batch_banded(pat.row_ptr, pat.col_idx, B.values, B.b)
        err = np.max(np.linalg.norm(x - xd, axis=1) / np.linalg.norm(xd, axis=1))
        ok = err <= 1e-8 and bool(np.all(st.cpu().numpy() == 0))
        bad += not ok
        print(f"{name:32s} iters={it.cpu().tolist()} fwd_err={err:.2e} {'ok' if ok else 'FAIL'}",
              flush=True)
    sys.exit(1 if bad else 0)


if __name__ == "__main__":
    main()
