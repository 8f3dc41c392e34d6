"""Time the batched banded LU solver (bsolve_banded_solve)
on the bench workload (XGC 32x31 9-point systems, 50/50 ion/electron) with
CUDA events on the launching stream; prints one JSON line.

    python tools/banded_bench.py [--batch 100000] [--reps 5] [--fmt ell|csr]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import xgcgen as X  # noqa: E402
from paper_conf_ipps_kashinksla22_b200 import Solver  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--batch", type=int, default=100000)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--fmt", default="ell")
    ap.add_argument("--nx", type=int, default=32)
    ap.add_argument("--ny", type=int, default=31)
    a = ap.parse_args()
    B = X.make_batch(0, a.batch, nx=a.nx, ny=a.ny)
    p = B.pattern
    S = Solver(p.row_ptr, p.col_idx, a.batch, format=a.fmt)
    vals = torch.from_numpy(S.ell_values(B.values) if S.format == "ell" else B.values).cuda()
    b = torch.from_numpy(B.b).cuda()
    x = torch.empty_like(b)
    info = torch.empty(a.batch, dtype=torch.int32, device="cuda")
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    s = torch.cuda.current_stream()
    for _ in range(2):
        S.banded_solve(vals, b, out=(x, info))
    torch.cuda.synchronize()
    ts = []
    for _ in range(a.reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        S.banded_solve(vals, b, out=(x, info))
        e1.record(s)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ms = float(np.median(ts))
    n, kl = p.n, 33
    flops = 2.0 * n * kl * (2 * kl + 1)  # dgbtf2 updates on the padded window (FMA = 2)
    print(json.dumps({"metric": "banded LU systems/s", "value": a.batch / ms * 1e3,
                      "ms": ms, "ms_all": ts, "batch": a.batch, "fmt": a.fmt, "n": n,
                      "info_nonzero": int((info != 0).sum().item()),
                      "window_gflops": flops * a.batch / ms / 1e6}))


if __name__ == "__main__":
    main()
