"""Iteration-count sensitivity of BiCGSTAB on the ill-conditioned electrons
(BASELINE.json configs[4]; R28).

For each margin (kappa ~ 1.2e3, 1.4e4, 1.4e5 at the 32 x 31 grid, cross = 0)
and N electron systems:
  * oracle       : oracle/ Algorithm 1 on A, b                (the reference count)
  * oracle_ulp   : the same oracle on A perturbed by ONE ulp per value
                   (a_ij * (1 +- 2^-52), random sign): the spread of counts an
                   input change far below any modelling accuracy produces
  * gpu          : the C-ABI CUDA path (only with --gpu)
and the histogram of iteration differences vs the oracle, the fraction within
+-2, and the forward error of x against the oracle's banded LU (which stays
<= 1e-8 whatever the count).  Writes one JSON document.

  python tools/iter_sensitivity.py [--gpu] [--n 1000] [--out profiles/r2_iter_sensitivity.json]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import oracle as O  # noqa: E402  (test infrastructure)
import xgcgen as X  # noqa: E402

MARGINS = (1e-1, 1e-2, 1e-3)


def hist(d):
    u, c = np.unique(d, return_counts=True)
    return {int(k): int(v) for k, v in zip(u, c)}


def summary(d):
    a = np.abs(d)
    return {"hist": hist(d), "frac_within_2": float(np.mean(a <= 2)),
            "median_abs": float(np.median(a)), "q95_abs": float(np.quantile(a, 0.95)),
            "max_abs": int(a.max())}


def electrons(margin, n, nx=32, ny=31, seed=X.DEFAULT_SEED):
    ill = X.Species(X.ELECTRON_K, cross=0.0, margin=margin)
    pat = X.stencil_pattern(nx, ny)
    B = X.make_batch(1, 2 * n, pattern=pat, electron=ill, seed=seed)
    return pat, B.values[0::2].copy(), B.b[0::2].copy()   # odd g = electrons


def perturb_ulp(vals, seed=0):
    rng = np.random.default_rng(seed)
    return vals * (1.0 + rng.choice([-1.0, 1.0], size=vals.shape) * 2.0 ** -52)


def gpu_solve(pat, vals, b, maxiter):
    import torch
    from paper_conf_ipps_kashinksla22_b200 import Solver
    S = Solver(pat.row_ptr, pat.col_idx, vals.shape[0])
    x, it, res, st = S.run(torch.from_numpy(S.ell_values(vals)).cuda(),
                           torch.from_numpy(b).cuda(), maxiter=maxiter)
    torch.cuda.synchronize()
    out = {"x": x.cpu().numpy(), "iters": it.cpu().numpy(), "status": st.cpu().numpy(),
           "resnorm": res.cpu().numpy(), "plan": S.info}
    S.close()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=1000)
    ap.add_argument("--gpu", action="store_true")
    ap.add_argument("--maxiter", type=int, default=3000)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    doc = {"what": "iteration-count differences vs the oracle on ill-conditioned electrons "
                   "(32x31, cross = 0); oracle_ulp = oracle on A perturbed by one ulp",
           "n_per_margin": a.n, "margins": {}}
    for m in MARGINS:
        pat, vals, b = electrons(m, a.n)
        o = O.batch_bicgstab(pat.row_ptr, pat.col_idx, vals, b, maxiter=a.maxiter)
        ou = O.batch_bicgstab(pat.row_ptr, pat.col_idx, perturb_ulp(vals), b, maxiter=a.maxiter)
        xd = O.batch_banded(pat.row_ptr, pat.col_idx, vals, b)
        nrm = np.linalg.norm(xd, axis=1)
        rec = {"oracle_iters_mean": float(o["iters"].mean()),
               "oracle_iters_range": [int(o["iters"].min()), int(o["iters"].max())],
               "oracle_all_converged": bool(np.all(o["status"] == 0)),
               "oracle_ulp_vs_oracle": summary(ou["iters"].astype(int) - o["iters"].astype(int)),
               "oracle_fwd_err_max": float(np.max(np.linalg.norm(o["x"] - xd, axis=1) / nrm))}
        if a.gpu:
            g = gpu_solve(pat, vals, b, a.maxiter)
            rec["gpu_vs_oracle"] = summary(g["iters"].astype(int) - o["iters"].astype(int))
            rec["gpu_status_equal"] = bool(np.array_equal(g["status"], o["status"]))
            rec["gpu_fwd_err_max"] = float(np.max(np.linalg.norm(g["x"] - xd, axis=1) / nrm))
            rec["gpu_true_rel_res_max"] = float(np.max(g["resnorm"] / np.linalg.norm(b, axis=1)))
            rec["gpu_plan"] = {k: g["plan"][k] for k in ("placement", "kernel_mode", "block_threads")}
        doc["margins"][f"{m:g}"] = rec
        print(f"margin {m:g}: {json.dumps(rec)}", flush=True)
    if a.out:
        with open(a.out, "w") as f:
            json.dump(doc, f, indent=1)


if __name__ == "__main__":
    main()
