"""Time the batched SpMV y_i = A_i x_i (bsolve_spmv; the paper's Fig. 7
microbenchmark) on the bench workload with CUDA events;
prints one JSON line with the HBM roofline fraction.

    python tools/spmv_bench.py [--batch 100000] [--fmt ell|csr] [--reps 10]
"""
import argparse
import json
import os
import sys
import types

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_ipps_kashinksla22_b200 import Solver  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=100000)
    ap.add_argument("--fmt", default="ell")
    ap.add_argument("--reps", type=int, default=10)
    a = ap.parse_args()
    args = types.SimpleNamespace(nx=32, ny=31, format=a.fmt, seed=20220530)
    pat, vals_h, b_h = bench.make_inputs(0, a.batch, args, pinned=True)
    S = Solver(pat.row_ptr, pat.col_idx, a.batch, format=a.fmt)
    vals, x = vals_h.cuda(), b_h.cuda()
    y = torch.empty_like(x)
    s = torch.cuda.current_stream()
    for _ in range(3):
        S.spmv(vals, x, out=y)
    torch.cuda.synchronize()
    ts = []
    for _ in range(a.reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        S.spmv(vals, x, out=y)
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts))
    nbytes = vals.numel() * 8 + x.numel() * 8 + y.numel() * 8
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:  # noqa: BLE001
        pass
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    # parity spot check: system 0 and the last one against a host product
    import scipy.sparse as sp
    import xgcgen as X
    yy = y.cpu().numpy()
    err = 0.0
    for g in (0, 1, a.batch - 1):
        B = X.make_batch(g, 1, pattern=pat)
        A = sp.csr_matrix((B.values[0], pat.col_idx, pat.row_ptr), shape=(pat.n, pat.n))
        ref = A @ b_h[g].numpy()
        err = max(err, float(np.max(np.abs(yy[g] - ref)) / np.max(np.abs(ref))))
    print(json.dumps({"metric": "batched SpMV systems/s", "value": a.batch / ms * 1e3, "ms": ms,
                      "fmt": a.fmt, "batch": a.batch, "bytes_per_system": nbytes / a.batch,
                      "hbm_gbs": nbytes / ms / 1e6, "hbm_peak_gbs": hbm,
                      "frac": nbytes / ms / 1e6 / hbm, "max_rel_err_vs_scipy": err,
                      "plan": S.info}))


if __name__ == "__main__":
    main()
