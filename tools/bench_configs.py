#!/usr/bin/env python
"""Measure BASELINE.json configs[0..2] (and [4] when supported) on one B200.

bench.py reports the headline (configs[3]: 1e5 systems).  This script fills
the other configs' tables in DESIGN.md:
  c0  batch = 2 (ion + electron pair): latency per batch
  c1  batch = 1280 (640 mesh nodes x 2 species): zero guess vs Picard warm start
      p = 0..4 (x0 = previous GPU solution), time per step, iterations per species
  c2  batch sweep 2^10..2^17 x {ELL (auto plan), CSR} x {SMEM-staged, HBM-streamed}
  c4  n = 4032 (64x63 grid) 9-point systems + ill-conditioned electrons
Timing: CUDA events on the launching stream, warm-up first; between timed
launches a 256 MB buffer is rewritten so inputs smaller than L2 start cold.
Writes one JSON line per measurement to --out (default gpurun_out/configs.jsonl).
"""
import argparse
import json
import os
import statistics
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import xgcgen as X  # noqa: E402
from paper_conf_ipps_kashinksla22_b200 import BsolveError, Solver  # noqa: E402

FLUSH = None


def flush_l2():
    global FLUSH
    if FLUSH is None:
        FLUSH = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    FLUSH.fill_(1)


def timed(fn, reps=5, warm=2, flush=True):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        if flush:
            flush_l2()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts), ts


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def emit(rec, out):
    s = json.dumps(rec)
    print(s, flush=True)
    with open(out, "a") as f:
        f.write(s + "\n")


def solver_inputs(B, fmt="ell", placement="auto", **kw):
    p = B.pattern
    S = Solver(p.row_ptr, p.col_idx, B.count, format=fmt, placement=placement, **kw)
    vals = S.ell_values(B.values) if S.format == "ell" else B.values
    return S, dev(vals), dev(B.b)


def c0(out):
    B = X.make_batch(0, 2)
    S, v, b = solver_inputs(B)
    o = S.alloc_outputs()
    ms, _ = timed(lambda: S.run(v, b, out=o), reps=20, warm=5)
    msb, _ = timed(lambda: S.banded_solve(v, b), reps=20, warm=5)
    emit({"config": "c0 pair (batch 2)", "us_per_batch": ms * 1e3,
          "us_per_batch_banded_lu": msb * 1e3,
          "iters": o[1].cpu().tolist(), "plan": S.info}, out)


def c1(out, batch=1280):
    xprev = None
    tot_zero = tot_warm = 0.0
    for pcd in range(5):
        B = X.make_batch(0, batch, picard=pcd)
        S, v, b = solver_inputs(B)
        o = S.alloc_outputs()
        ms0, _ = timed(lambda: S.run(v, b, out=o))
        msb, _ = timed(lambda: S.banded_solve(v, b))
        it0 = o[1].cpu().numpy()
        if xprev is None:
            msw, itw = ms0, it0
            S.run(v, b, out=o)
        else:
            x0 = dev(xprev)
            msw, _ = timed(lambda: S.run(v, b, x0=x0, out=o))
            itw = o[1].cpu().numpy()
        torch.cuda.synchronize()
        xprev = o[0].cpu().numpy()
        tot_zero += ms0
        tot_warm += msw
        emit({"config": f"c1 picard p={pcd} (batch {batch})", "ms_zero_guess": ms0,
              "ms_warm_start": msw, "ms_banded_lu": msb, "sys_per_s_warm": batch / (msw * 1e-3),
              "iters_zero": {"ion": float(it0[0::2].mean()), "electron": float(it0[1::2].mean())},
              "iters_warm": {"ion": float(itw[0::2].mean()), "electron": float(itw[1::2].mean())},
              "paper_table3": {"ion": [5, 4, 3, 2, 2][pcd], "electron": [30, 28, 20, 16, 12][pcd]}},
             out)
    emit({"config": f"c1 cumulative 5 Picard solves (batch {batch})", "ms_zero_guess": tot_zero,
          "ms_warm_start": tot_warm, "speedup_warm_over_zero": tot_zero / tot_warm,
          "paper": "ELL 1.2-1.6x on A100 (PAPER.md:1085-1090)"}, out)


def c2(out, exps=(10, 12, 14, 16, 17)):
    pat = X.stencil_pattern()
    for e in exps:
        batch = 1 << e
        B = X.make_batch(0, batch, pattern=pat)
        for fmt, placements in (("ell", ("auto", "smem", "stream")),
                                ("csr", ("auto", "smem", "stream"))):
            for placement in placements:
                S, v, b = solver_inputs(B, fmt=fmt, placement=placement)
                o = S.alloc_outputs()
                ms, _ = timed(lambda: S.run(v, b, out=o), reps=3, warm=1)
                its = o[1].cpu().numpy()
                emit({"config": f"c2 sweep", "batch": batch, "format": fmt,
                      "placement": placement, "ms": ms, "sys_per_s": batch / (ms * 1e-3),
                      "us_per_system": ms * 1e3 / batch, "iters_mean": float(its.mean()),
                      "kernel_mode": S.info["kernel_mode"],
                      "block_threads": S.info["block_threads"]}, out)
                if placement == "auto" and fmt == "ell":
                    msb, _ = timed(lambda: S.banded_solve(v, b), reps=3, warm=1)
                    emit({"config": "c2 sweep", "batch": batch, "format": fmt,
                          "placement": "banded LU", "ms": msb, "sys_per_s": batch / (msb * 1e-3)},
                         out)
                del S, v, o
        del B
        torch.cuda.empty_cache()


def c4(out, batch=16384):
    pat = X.stencil_pattern(64, 63)
    mixes = {"ion+electron": (X.ION, X.ELECTRON)}
    for m in (1e-1, 1e-2, 1e-3):
        mixes[f"ion+ill-electron margin {m:g}"] = (X.ION, X.Species(X.ELECTRON_K, margin=m))
    for name, (ion, ele) in mixes.items():
        B = X.make_batch(0, batch, pattern=pat, ion=ion, electron=ele)
        try:
            S, v, b = solver_inputs(B)
        except BsolveError as ex:
            emit({"config": f"c4 n=4032 {name}", "unsupported": str(ex)}, out)
            return
        o = S.alloc_outputs()
        ms, _ = timed(lambda: S.run(v, b, out=o, maxiter=2000), reps=3, warm=1)
        its, st = o[1].cpu().numpy(), o[3].cpu().numpy()
        emit({"config": f"c4 n=4032 {name}", "batch": batch, "ms": ms,
              "sys_per_s": batch / (ms * 1e-3), "iters_mean_ion": float(its[0::2].mean()),
              "iters_mean_electron": float(its[1::2].mean()),
              "all_converged": bool(np.all(st == 0)), "plan": S.info}, out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/configs.jsonl")
    ap.add_argument("--only", default="c0,c1,c2,c4")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    open(a.out, "w").close()
    for c in a.only.split(","):
        globals()[c](a.out)


if __name__ == "__main__":
    main()
