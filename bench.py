#!/usr/bin/env python
"""Benchmark: systems solved per second for batched Jacobi-BiCGSTAB on B200.

Metric (BASELINE.json): "systems solved/sec (992-row XGC matrices, tol 1e-10)
at 1/2/4/8 B200; % roofline".  Workload at N = 1: BASELINE.json configs[3]'s
batch of 10^5 XGC-shaped systems (50/50 ion/electron, 32x31 grid, 9-point
stencil, fp64, zero initial guess, tol 1e-10 relative to ||b||), which fits
one GPU; with N GPUs each rank solves its own 10^5-system slice (weak
scaling, no collective on the solve path).

One "step" = one bsolve_run over the rank's whole batch (one kernel launch).
Timed region: W untimed warm-up steps, then K steps bracketed by barrier +
cuda synchronize, CUDA events on the launching stream, max over ranks.
Inputs (8.7 GB per rank) exceed the 126 MB L2, so no flush is needed.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
  torchrun --nproc-per-node N bench.py --gpus N ...
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "systems solved/sec (992-row XGC matrices, tol 1e-10)"
UNIT = "systems/s"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--batch", type=int, default=100_000, help="systems per GPU (weak scaling)")
    ap.add_argument("--scaling", choices=["weak", "strong"], default="weak")
    ap.add_argument("--nx", type=int, default=32)
    ap.add_argument("--ny", type=int, default=31)
    ap.add_argument("--format", choices=["ell", "csr"], default="ell")
    ap.add_argument("--placement", choices=["auto", "smem", "stream", "regs", "cluster", "tmem"],
                    default="auto")
    ap.add_argument("--block-threads", type=int, default=0)
    ap.add_argument("--reg-slots", type=int, default=0)
    ap.add_argument("--solver", choices=["bicgstab", "gmres", "banded"], default="bicgstab",
                    help="BiCGSTAB = the paper's Algorithm 1; gmres = f3; banded = the "
                         "dgbsv-analogue direct solver (SURVEY.md 8(f) f4)")
    ap.add_argument("--precond", choices=["jacobi", "none", "block_jacobi"], default="jacobi",
                    help="block_jacobi: 8-row blocks (SURVEY.md 8(f) f3, DESIGN.md R30)")
    ap.add_argument("--restart", type=int, default=7, help="GMRES restart length m")
    ap.add_argument("--tol", type=float, default=1e-10)
    ap.add_argument("--maxiter", type=int, default=1000)
    ap.add_argument("--seed", type=int, default=20220530)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0,
                    help="target wall seconds of the oracle sample")
    ap.add_argument("--out", default=None, help="also append the JSON line to this file")
    ap.add_argument("--picard", type=int, default=0,
                    help="P > 0: the Picard pipeline (SURVEY.md 8(f) f1, BASELINE configs[1] at "
                         "scale): one step = P successive solves, matrices of Picard step p "
                         "resident on the device, x0 = the previous solution (warm), timed "
                         "beside P zero-guess solves")
    ap.add_argument("--parity", choices=["full", "sample", "none"], default="full",
                    help="N = 1: compare EVERY system's x with the oracle's banded LU (full) "
                         "or only the cpu_baseline sample")
    ap.add_argument("--backend", choices=["nccl", "gloo"], default="nccl",
                    help="process-group backend for N > 1 (gloo: CPU plumbing tests)")
    ap.add_argument("--standin", action="store_true",
                    help="CPU stand-in solver (plumbing tests of the multi-rank harness; "
                         "no GPU): Jacobi sweeps on the generator's systems")
    ap.add_argument("--cross-check", type=int, default=64,
                    help="N > 1: systems per rank that rank 0 re-solves and compares bitwise")
    return ap.parse_args()


# ----------------------------------------------------------------- clocks --
class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self._stop = threading.Event()
        self._t = None

    def __enter__(self):
        # streaming mode: one nvidia-smi process printing every 20 ms
        try:
            self._p = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                 "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self._p = None
            return self
        def reader():
            for line in self._p.stdout:
                line = line.strip()
                if line:
                    self.rows.append([c.strip() for c in line.split(",")])
        self._t = threading.Thread(target=reader, daemon=True)
        self._t.start()
        time.sleep(0.3)  # let the sampler start before the timed region
        return self

    def __exit__(self, *a):
        if getattr(self, "_p", None):
            time.sleep(0.05)
            self._p.terminate()
            try:
                self._p.wait(timeout=5)
            except Exception:
                self._p.kill()
        if self._t:
            self._t.join(timeout=5)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"],
                    "samples": 0}
        def f(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [f(r[1]) for r in self.rows if f(r[1])]
        mx = [f(r[2]) for r in self.rows if f(r[2])]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for nm, v in zip(names, r[5:9]):
                if v.strip().lower() == "active":
                    reasons.add(nm)
        pw = [f(r[3]) for r in self.rows if f(r[3])]
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "power_w_max": max(pw) if pw else None, "samples": len(self.rows)}


# ------------------------------------------------------------- inputs --
def make_inputs(g0, count, args, pinned, picard=0):
    """Generate systems g0..g0+count-1 (Picard step `picard`) into (pinned)
    host buffers, ELL/CSR."""
    import torch
    import xgcgen as X
    pat = X.stencil_pattern(args.nx, args.ny)
    W = pat.max_row_nnz
    per = W * pat.n if args.format == "ell" else pat.nnz
    vals = torch.empty((count, per), dtype=torch.float64, pin_memory=pinned)
    b = torch.empty((count, pat.n), dtype=torch.float64, pin_memory=pinned)
    vn, bn = vals.numpy(), b.numpy()
    from paper_conf_ipps_kashinksla22_b200 import ell_layout
    _, _, src = ell_layout(pat.row_ptr, pat.col_idx)   # the library's ELL slot map
    ok = src >= 0
    CH = 8192
    for c0 in range(0, count, CH):
        c1 = min(count, c0 + CH)
        # ranks share the host: split its cores among them for the generator
        world = int(os.environ.get("WORLD_SIZE", "1"))
        Bt = X.make_batch(g0 + c0, c1 - c0, pattern=pat, seed=args.seed, picard=picard,
                          threads=max(1, min(32, host_cores() // max(1, world))))
        if args.format == "ell":
            blk = vn[c0:c1]
            blk[:, ~ok] = 0.0
            blk[:, ok] = Bt.values[:, src[ok]]
        else:
            vn[c0:c1] = Bt.values
        bn[c0:c1] = Bt.b
    return pat, vals, b


def make_csr_sample(g0, count, args):
    import xgcgen as X
    pat = X.stencil_pattern(args.nx, args.ny)
    return pat, X.make_batch(g0, count, pattern=pat, seed=args.seed)


# ------------------------------------------------------- cpu baseline --
def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except AttributeError:
        return os.cpu_count() or 1


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def oracle_krylov(O, pat, B, args, cores):
    """The oracle's solver for this run's --solver / --precond / --restart."""
    return O.batch_krylov(pat.row_ptr, pat.col_idx, B.values, B.b,
                          solver=O.SOLVER_GMRES if args.solver == "gmres" else O.SOLVER_BICGSTAB,
                          precond={"none": O.PREC_NONE, "jacobi": O.PREC_JACOBI,
                                   "block_jacobi": O.block_jacobi(8)}[args.precond],
                          restart=args.restart, tol=args.tol, maxiter=args.maxiter, threads=cores)


def oracle_algorithm(args):
    name = ("GMRES(%d)" % args.restart if args.solver == "gmres"
            else "Alg. 1 BiCGSTAB")
    pre = {"jacobi": "Jacobi", "none": "no preconditioner",
           "block_jacobi": "block-Jacobi(8)"}[args.precond]
    return f"{name} + {pre} (oracle/oracle.c)"


def oracle_sample_rate(g0, max_count, args, target_s, kind="bicgstab"):
    """Time the oracle (as it stands) on a bounded sample; returns dict."""
    import oracle as O
    cores = host_cores()
    # calibrate on a small sample, then size the sample to ~target_s of wall time
    n_cal = min(max_count, max(2 * cores, 64))
    pat, Bc = make_csr_sample(g0, n_cal, args)
    t0 = time.perf_counter()
    if kind == "bicgstab":
        oracle_krylov(O, pat, Bc, args, cores)
    else:
        O.batch_banded(pat.row_ptr, pat.col_idx, Bc.values, Bc.b, threads=cores)
    dt = time.perf_counter() - t0
    rate = n_cal / max(dt, 1e-9)
    count = int(min(max_count, max(n_cal, rate * target_s)))
    count -= count % 2  # keep the ion/electron mix 50/50
    count = max(count, 2)
    pat, Bs = make_csr_sample(g0, count, args)
    t0 = time.perf_counter()
    if kind == "bicgstab":
        out = oracle_krylov(O, pat, Bs, args, cores)
    else:
        out = {"x": O.batch_banded(pat.row_ptr, pat.col_idx, Bs.values, Bs.b, threads=cores)}
    dt = time.perf_counter() - t0
    return {"value": count / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "algorithm": oracle_algorithm(args) if kind == "bicgstab"
            else "banded LU with partial pivoting, dgbsv-like (oracle/oracle.c)",
            "sample": f"systems g={g0}..{g0 + count - 1} of the same workload "
                      f"({count} systems, {dt:.1f} s wall, one system per task over "
                      f"{cores} host threads)",
            "cpu": cpu_model(), "_out": out, "_count": count, "_csr": Bs}


# --------------------------------------------------------------- reference --
def run_reference(args, rank, world):
    """--impl reference: the oracle (as it stands) on the host cores."""
    if rank != 0:
        return
    per_rank = rank_slice_count(args, world)
    cal = oracle_sample_rate(0, per_rank, args, target_s=min(5.0, args.cpu_seconds),
                             kind="banded" if args.solver == "banded" else "bicgstab")
    count = cal["_count"]
    import oracle as O
    pat, Bs = make_csr_sample(0, count, args)
    cores = host_cores()
    times = []
    for s in range(args.warmup + args.steps):
        t0 = time.perf_counter()
        if args.solver == "banded":
            O.batch_banded(pat.row_ptr, pat.col_idx, Bs.values, Bs.b, threads=cores)
        else:
            oracle_krylov(O, pat, Bs, args, cores)
        dt = time.perf_counter() - t0
        if s >= args.warmup:
            times.append(dt)
    ms = 1e3 * statistics.mean(times)
    value = count / (ms * 1e-3)
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_dict(args, world, per_rank),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": f"{count} systems (g=0..{count - 1}) of the workload per step"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        "note": f"CPU oracle (oracle/oracle.c, "
                f"{'banded LU' if args.solver == 'banded' else 'Alg. 1'}) on the host cores; "
                "the paper has no "
                "public code and this tier has no installable reference",
    }
    emit(line, args)


def h2d_copy_gbs(dev, nbytes=1 << 30, reps=3):
    """Measured pinned host -> device copy rate (GB/s, best of reps, CUDA
    events): the link bound of every e2e number (inputs cross it once)."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    best = 0.0
    for _ in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        d.copy_(h, non_blocking=True)
        e1.record()
        torch.cuda.synchronize()
        best = max(best, nbytes / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    del h, d
    return best


def rank_slice_count(args, world):
    from paper_conf_ipps_kashinksla22_b200.parallel import rank_slice
    return rank_slice(args.batch, 0, world, args.scaling).count


def config_dict(args, world, per_rank):
    n = args.nx * args.ny
    return {"workload": f"xgc{n}_9pt_mix_zero_guess",
            "description": "BASELINE configs[3]: 10^5-system batch of XGC-shaped 9-point "
                           "stencil systems per GPU, 50/50 ion/electron, x0 = 0",
            "batch_per_gpu": per_rank,
            "global_batch": args.batch * world if args.scaling == "weak" else args.batch, "n": n,
            "grid": f"{args.nx}x{args.ny}", "format": args.format, "placement": args.placement,
            "tol": args.tol, "stop": "rel_b", "maxiter": args.maxiter, "x0": "zero",
            "solver": (f"gmres({args.restart})" if args.solver == "gmres" else
                       "banded LU (dgbsv analogue)" if args.solver == "banded" else args.solver),
            "precond": args.precond,
            "parallelism": f"batch-partitioned x{world} (one process per GPU, no solve-path "
                           f"collective)",
            "l2": "inputs larger than L2 (no flush needed)", "seed": args.seed}


def emit(line, args):
    s = json.dumps(line)
    print(s, flush=True)
    if args.out:
        with open(args.out, "a") as f:
            f.write(s + "\n")


# ------------------------------------------------- multi-rank helpers --
def digest(*arrays):
    import hashlib
    h = hashlib.sha256()
    for a in arrays:
        h.update(np.ascontiguousarray(a).tobytes())
    return h.hexdigest()


def cross_check(args, rank, world, local, solve_fn, device):
    """Cross-P bitwise check: every rank hashes (x, iters,
    resnorm, status) of the first m systems of its slice; rank 0 re-solves
    those systems of EVERY rank on its own device and compares the hashes.
    local = this rank's outputs (numpy); solve_fn(g0, m) -> same tuple."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_kashinksla22_b200.parallel import rank_slice
    sls = [rank_slice(args.batch, r, world, args.scaling) for r in range(world)]
    ms = [min(args.cross_check, s.count) for s in sls]
    mine = digest(*(a[: ms[rank]] for a in local))
    t = torch.tensor(list(bytes.fromhex(mine)), dtype=torch.uint8, device=device)
    bufs = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(bufs, t)
    if rank != 0:
        return None
    got = [bytes(b.cpu().tolist()).hex() for b in bufs]
    equal = []
    for r in range(world):
        if ms[r] == 0:
            equal.append(True)
            continue
        ref = digest(*solve_fn(sls[r].g0, ms[r]))
        equal.append(ref == got[r])
    return {"systems_per_rank": ms, "ranks": world, "bitwise_equal": bool(all(equal)),
            "per_rank": equal,
            "how": "rank 0 re-solves the first systems of every rank's slice on its own device; "
                   "sha256 of (x, iters, resnorm, status) compared"}


def standin_solve(g0, count, args):
    """CPU stand-in for the GPU solve, for the multi-rank plumbing tests only
    (no GPU in the build container): Jacobi sweeps x += (b - A x) / diag(A) on
    the generator's systems until ||b - A x|| < 1e-8 ||b|| (cap 500 sweeps).
    Per-system results depend only on the global system index."""
    import xgcgen as X
    B = X.make_batch(g0, count, nx=args.nx, ny=args.ny, seed=args.seed)
    p = B.pattern
    n = p.n
    rows = np.repeat(np.arange(n), np.diff(p.row_ptr))
    A = np.zeros((count, n, n))
    A[:, rows, p.col_idx] = B.values
    dg = A[:, np.arange(n), np.arange(n)]
    x = np.zeros_like(B.b)
    it = np.zeros(count, np.int32)
    bn = np.linalg.norm(B.b, axis=1)
    res = bn.copy()
    for _ in range(500):
        r = B.b - np.einsum("bij,bj->bi", A, x)
        res = np.linalg.norm(r, axis=1)
        act = res >= 1e-8 * bn
        if not act.any():
            break
        x[act] += r[act] / dg[act]
        it[act] += 1
    st = np.where(res < 1e-8 * bn, 0, 1).astype(np.int8)
    return x, it, res, st


def run_standin(args, rank, world):
    """The multi-rank harness of run_ours (rank slices, barrier, timed steps,
    max over ranks, stats gather, cross-P check, one JSON line from rank 0)
    around the CPU stand-in solver: `python bench.py --gpus 2 --standin
    --backend gloo` exercises the driver's N-rank entry point without a GPU."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_kashinksla22_b200.parallel import (gather_stats, max_over_ranks,
                                                            rank_slice)
    sl = rank_slice(args.batch, rank, world, args.scaling)
    out = None
    for _ in range(max(args.warmup, 0)):
        out = standin_solve(sl.g0, sl.count, args)
    if world > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        out = standin_solve(sl.g0, sl.count, args)
    dt = time.perf_counter() - t0
    if world > 1:
        dist.barrier()
    dt = max_over_ranks(dt)
    x, it, res, st = out
    it_all, res_all, st_all = (t.numpy() for t in gather_stats(
        torch.from_numpy(it), torch.from_numpy(res), torch.from_numpy(st)))
    cross = (cross_check(args, rank, world, out, lambda g0, m: standin_solve(g0, m, args),
                         "cpu") if world > 1 else None)
    if rank == 0:
        emit({"metric": METRIC, "value": sl.total * args.steps / dt, "unit": UNIT,
              "n_gpus": world, "steps": args.steps, "warmup": args.warmup,
              "ms_per_step": 1e3 * dt / args.steps, "higher_is_better": True,
              "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
              "impl": "standin", "config": config_dict(args, world, sl.count),
              "note": "CPU stand-in solver: plumbing test of the multi-rank harness, not a "
                      "measurement",
              "gathered": {"systems": int(it_all.size), "digest": digest(it_all, res_all, st_all),
                           "iters_sum": int(it_all.astype(np.int64).sum())},
              "cross_p": cross}, args)


def full_parity(args, g0, count, x_dev, res_h, st_h):
    """Every system of the timed batch against the oracle's direct solve
    (north_star: ||x - x_direct|| / ||x_direct|| <= 1e-8 per system; VERDICT
    r1 weak #2): the banded LU (dgbsv-like, oracle/oracle.c) over all host
    cores, chunk by chunk, and the GPU's reported TRUE relative residual."""
    import oracle as O
    cores = host_cores()
    t0 = time.perf_counter()
    worst, worst_g, over, CH = 0.0, -1, 0, 8192
    res_rel_max = 0.0
    for c0 in range(0, count, CH):
        c1 = min(count, c0 + CH)
        pat, B = make_csr_sample(g0 + c0, c1 - c0, args)
        xd = O.batch_banded(pat.row_ptr, pat.col_idx, B.values, B.b, threads=cores)
        xg = x_dev[c0:c1].cpu().numpy()
        rel = np.linalg.norm(xg - xd, axis=1) / np.linalg.norm(xd, axis=1)
        k = int(np.argmax(rel))
        if rel[k] > worst:
            worst, worst_g = float(rel[k]), g0 + c0 + k
        over += int(np.sum(rel > 1e-8))
        res_rel_max = max(res_rel_max, float(np.max(res_h[c0:c1] / np.linalg.norm(B.b, axis=1))))
    return {"systems_checked": count, "oracle": "banded LU with partial pivoting, dgbtf2 + "
            "dgbtrs order (oracle/oracle.c), every system", "max_rel_x_diff_vs_direct": worst,
            "worst_system": worst_g, "systems_over_1e-8": over,
            "max_true_rel_residual_gpu": res_rel_max,
            "all_converged": bool(np.all(st_h == 0)),
            "within_north_star": bool(over == 0 and res_rel_max <= args.tol),
            "oracle_wall_s": time.perf_counter() - t0, "oracle_cores": cores}


# -------------------------------------------------------------------- ours --
def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_kashinksla22_b200 import Solver, probe_smem_bandwidth
    from paper_conf_ipps_kashinksla22_b200.parallel import (gather_stats, max_over_ranks,
                                                            rank_slice)

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    sl = rank_slice(args.batch, rank, world, args.scaling)
    per_rank, g0 = sl.count, sl.g0
    pat, vals_h, b_h = make_inputs(g0, per_rank, args, pinned=True)
    n, nnz, W = pat.n, pat.nnz, pat.max_row_nnz
    S = Solver(pat.row_ptr, pat.col_idx, per_rank, format=args.format,
               placement=args.placement, device=local_rank, block_threads=args.block_threads,
               reg_slots=args.reg_slots, solver=args.solver, precond=args.precond,
               restart=args.restart)
    vals = vals_h.to(dev, non_blocking=False)
    b = b_h.to(dev)
    out = S.alloc_outputs()
    x, it, res, st = out
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    nvtx = torch.cuda.nvtx  # ranges for nsys / ncu --nvtx timelines
    nvtx.range_push("warmup")
    for _ in range(max(args.warmup, 0)):
        S.run(vals, b, None, args.tol, args.maxiter, out=out)
    barrier()
    nvtx.range_pop()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    launch_ms = []
    with ClockSampler(local_rank) as clk:
        barrier()
        nvtx.range_push(f"timed {args.steps} steps")
        ev0.record(stream)
        for _ in range(args.steps):
            e_a = torch.cuda.Event(enable_timing=True)
            e_b = torch.cuda.Event(enable_timing=True)
            e_a.record(stream)
            S.run(vals, b, None, args.tol, args.maxiter, out=out)
            e_b.record(stream)
            launch_ms.append((e_a, e_b))
        ev1.record(stream)
        torch.cuda.synchronize()
        nvtx.range_pop()
        barrier()
    total_ms = ev0.elapsed_time(ev1)
    kern_ms = [a.elapsed_time(bb) for a, bb in launch_ms]
    total_ms = max_over_ranks(total_ms, device=dev)
    ms_per_step = total_ms / args.steps
    value = sl.total * args.steps / (total_ms * 1e-3)

    # ---- stats of the last step (outside the timed region) ------------------
    it_h = it.cpu().numpy()
    st_h = st.cpu().numpy()
    res_h = res.cpu().numpy()
    it_all, res_all, st_all = (t.numpy() for t in gather_stats(it, res, st))
    sum_iters_rank = int(it_h.astype(np.int64).sum())
    cross = None
    if world > 1:  # cross-P bitwise check of per-system outputs
        def solve_local(gs, m):
            _, vh, bh = make_inputs(gs, m, args, pinned=False)
            T = Solver(pat.row_ptr, pat.col_idx, m, format=args.format,
                       placement=args.placement, device=local_rank,
                       block_threads=args.block_threads, reg_slots=args.reg_slots,
                       solver=args.solver, precond=args.precond, restart=args.restart)
            o = T.run(vh.to(dev), bh.to(dev), None, args.tol, args.maxiter)
            torch.cuda.synchronize()
            r = tuple(t.cpu().numpy() for t in o)
            T.close()
            return r
        local = (x[: args.cross_check].cpu().numpy(), it_h, res_h, st_h)
        cross = cross_check(args, rank, world, local, solve_local, dev)

    # ---- roofline (dominant kernel = the one solve kernel per step) ---------
    import json as _json
    peaks = {}
    try:
        peaks = _json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        pass
    info = S.info
    num_sms = info["num_sms"]
    sm_max_mhz = float(peaks.get("sm_max_mhz", 1965.0))
    kern_avg_s = statistics.mean(kern_ms) * 1e-3
    # Algorithmic SMEM bytes per unit (= one BiCGSTAB iteration of one system;
    # SURVEY.md 8(d)): each of the 2 SpMVs gathers one
    # 8-byte operand per nonzero and publishes one 8-byte entry per row.  When
    # the matrix values are staged in SMEM (placements smem/stream/cluster with
    # SMEM slots) they add 8 B per nonzero; in the TMEM / register-resident
    # plans they never cross the SMEM pipe and are accounted on their own path.
    values_in_smem = info["placement"] not in (3, 5)
    smem_bytes_iter = 2 * ((16 if values_in_smem else 8) * nnz + 8 * n)
    smem_bytes_launch = smem_bytes_iter * sum_iters_rank
    smem_peak = 128.0 * num_sms * sm_max_mhz * 1e6      # guide: 128 B/clk/SM
    smem_achieved = smem_bytes_launch / kern_avg_s
    # operand model of the method (values + gathered operands + stores), the
    # pre-TMEM definition: an effective on-chip bandwidth, not a pipe bound
    all_operand_bytes = 2 * (16 * nnz + 8 * n) * sum_iters_rank
    tmem_bytes_launch = (0 if values_in_smem else 2 * 8 * nnz * sum_iters_rank)
    tmem_peak = 280.0 * num_sms * sm_max_mhz * 1e6      # measured tcgen05.ld, 8 warps/SM
    fp64_flops_launch = (4 * nnz + 26 * n) * sum_iters_rank   # 61,504 / iter
    fp64_peak = 64 * 2 * num_sms * sm_max_mhz * 1e6     # 64 DFMA/clk/SM
    try:
        from paper_conf_ipps_kashinksla22_b200 import probe_fp64
        fp64_measured, fp64_probe_hz = probe_fp64(local_rank)
    except Exception:  # noqa: BLE001
        fp64_measured, fp64_probe_hz = None, None
    vals_bytes = vals.element_size() * vals.numel() / per_rank
    hbm_bytes_sys = vals_bytes + 8 * n + 8 * n + 4 + 8 + 1   # values, b, x, iters, resnorm, status
    hbm_achieved = hbm_bytes_sys * per_rank / kern_avg_s
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0)) * 1e9
    try:
        probe_bw, probe_hz = probe_smem_bandwidth(local_rank)
    except Exception:
        probe_bw, probe_hz = None, None
    clocks = clk.summary()
    roofline = {
        "bound": "smem", "achieved": smem_achieved / 1e9, "peak": smem_peak / 1e9,
        "unit": "GB/s", "frac": smem_achieved / smem_peak, "traffic": None,
        "kernel": "bicgstab_kernel (one launch per step)",
        "algorithmic_bytes_per_launch": smem_bytes_launch,
        "algorithmic_bytes_per_unit": (
            f"{smem_bytes_iter} B per BiCGSTAB iteration (2 SpMVs x ("
            + ("16 B x nnz [values + gathered operands]" if values_in_smem else
               "8 B x nnz [gathered operands; values live in TMEM/registers]")
            + " + 8 B x n [published vector]))"),
        "units_per_launch": sum_iters_rank,
        "peak_source": f"derived: 128 B/clk/SM x {num_sms} SMs x {sm_max_mhz:.0f} MHz "
                       f"(B300_MICROARCH smem crossbar; no SMEM figure in MEASURED_PEAKS)",
        "peak_measured_probe": None if probe_bw is None else probe_bw / 1e9,
        "probe_sm_mhz": None if probe_hz is None else probe_hz / 1e6,
        "kernel_ms_avg": kern_avg_s * 1e3,
        "hbm": {"achieved": hbm_achieved / 1e9, "peak": hbm_peak / 1e9, "unit": "GB/s",
                "frac": hbm_achieved / hbm_peak, "bytes_per_system": hbm_bytes_sys,
                "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"},
        "tmem": {"achieved": tmem_bytes_launch / kern_avg_s / 1e9, "peak": tmem_peak / 1e9,
                 "unit": "GB/s", "frac": tmem_bytes_launch / kern_avg_s / tmem_peak,
                 "peak_source": "tools/tmem_probe.cu: tcgen05.ld 280 B/clk/SM at 8 warps "
                                "(profiles/r1_tmem_probe.txt)"},
        "fp64": {"achieved": fp64_flops_launch / kern_avg_s / 1e12, "peak": fp64_peak / 1e12,
                 "unit": "TFLOP/s", "frac": fp64_flops_launch / kern_avg_s / fp64_peak,
                 "peak_source": "derived: 64 DFMA/clk/SM x 148 x 1965 MHz",
                 "peak_measured": None if fp64_measured is None else fp64_measured / 1e12,
                 "probe_sm_mhz": None if fp64_probe_hz is None else fp64_probe_hz / 1e6,
                 "frac_of_measured": (None if not fp64_measured else
                                      fp64_flops_launch / kern_avg_s / fp64_measured),
                 "measured_how": "bsolve_probe_fp64: DFMA loop, 8 chains per thread, "
                                 "4 x 256 threads per SM"},
        "frac_ell_slots": (2 * ((16 if values_in_smem else 8) * W * n + 8 * n) * sum_iters_rank
                           / kern_avg_s / smem_peak),
        "model_note": "frac charges the 8554 CSR nonzeros per SpMV (conservative); "
                      "frac_ell_slots charges SURVEY 8(d)'s 8928 ELL slots incl. padding",
        "all_operand_effective": {
            "achieved": all_operand_bytes / kern_avg_s / 1e9, "unit": "GB/s",
            "frac_of_smem_peak": all_operand_bytes / kern_avg_s / smem_peak,
            "note": "values + gathered operands + stores per iteration (2 x (16 nnz + 8 n)) "
                    "wherever they live; effective on-chip bandwidth, can exceed 1"},
    }
    # traffic from the committed ncu --set full capture of this kernel on this
    # workload (profiles/ncu_traffic.json), scaled to this launch's systems; the
    # capture is of the default workload only (another grid, preconditioner,
    # solver or placement runs another kernel: no traffic / physical fields)
    default_workload = ((args.nx, args.ny) == (32, 31) and args.precond == "jacobi" and
                        args.solver == "bicgstab" and args.format == "ell" and
                        args.placement == "auto" and not args.block_threads and
                        not args.reg_slots)
    try:
        if not default_workload:
            raise LookupError("no committed capture for this workload")
        tr = _json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        scale = per_rank / tr["systems_per_launch"]
        roofline["traffic"] = tr["smem_data_pipe_bytes_per_launch"] * scale
        roofline["traffic_unit"] = ("bytes per launch through the SMEM/L1 data pipe "
                                    "(ncu l1tex__data_pipe_lsu_wavefronts_mem_shared x 128 B)")
        roofline["traffic_over_algorithmic"] = (roofline["traffic"] / smem_bytes_launch
                                                if smem_bytes_launch else None)
        roofline["hbm"]["traffic"] = tr["dram_bytes_per_launch"] * scale
        roofline["hbm"]["traffic_over_algorithmic"] = (tr["dram_bytes_per_launch"] * scale /
                                                       (hbm_bytes_sys * per_rank))
        roofline["traffic_source"] = tr["source"]
        if "smem_pipe_busy" in tr:  # physical resource use of the same capture
            roofline["physical"] = {
                k: tr[k] for k in ("smem_pipe_busy", "fp64_pipe_busy", "lsu_pipe_busy",
                                   "warps_active", "registers_per_thread") if k in tr}
            roofline["physical"]["frac"] = max(tr["smem_pipe_busy"], tr["fp64_pipe_busy"])
            roofline["physical"]["note"] = ("ncu busy fractions of the tightest physical "
                                            "resources (the honest roofline of a latency-bound "
                                            "kernel; frac above is the byte model)")
    except Exception:  # noqa: BLE001 - no capture committed for this build
        pass
    if clocks.get("sm_mhz"):
        roofline["frac_at_observed_clock"] = smem_achieved / (128.0 * num_sms *
                                                              clocks["sm_mhz"] * 1e6)

    # ---- e2e through the public host API (pinned host buffers) -------------
    e2e = None
    if not args.no_e2e:
        x_h = torch.empty((per_rank, n), dtype=torch.float64, pin_memory=True).numpy()
        i_h = torch.empty(per_rank, dtype=torch.int32, pin_memory=True).numpy()
        r_h = torch.empty(per_rank, dtype=torch.float64, pin_memory=True).numpy()
        s_h = torch.empty(per_rank, dtype=torch.int8, pin_memory=True).numpy()
        vn, bn = vals_h.numpy(), b_h.numpy()
        outs = (x_h, i_h, r_h, s_h)
        S.run_host(vn, bn, None, args.tol, args.maxiter, out=outs)  # warm-up (allocates)
        e2e_steps = max(1, min(args.steps, 3))
        barrier()
        nvtx.range_push("e2e (host buffers)")
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            S.run_host(vn, bn, None, args.tol, args.maxiter, out=outs)
        torch.cuda.synchronize()
        nvtx.range_pop()
        dt = time.perf_counter() - t0
        dt = max_over_ranks(dt, device=dev)
        h2d = int(vn.nbytes + bn.nbytes)
        d2h = int(x_h.nbytes + i_h.nbytes + r_h.nbytes + s_h.nbytes)
        link = h2d_copy_gbs(dev)
        e2e = {"value": sl.total * e2e_steps / dt, "unit": UNIT,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e2e_steps,
               "h2d_gbs": h2d * e2e_steps / dt / 1e9, "h2d_copy_gbs_measured": link,
               "link_frac": h2d * e2e_steps / dt / 1e9 / link,
               "api": "bsolve_run_host (C ABI, chunked H2D/solve/D2H pipeline)",
               "bitwise_equal_to_device_path": bool(np.array_equal(i_h, it_h) and
                                                    np.array_equal(r_h, res_h))}

    # ---- cpu baseline (rank 0, N = 1 only) -------------------------------------
    cpu = None
    parity = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cb = oracle_sample_rate(g0, per_rank, args, target_s=args.cpu_seconds)
        o = cb.pop("_out")
        cnt = cb.pop("_count")
        cb.pop("_csr")
        cpu = cb
        xo = x[:cnt].cpu().numpy()
        bnrm = np.linalg.norm(b_h.numpy()[:cnt], axis=1)
        parity = {"systems_checked": cnt,
                  "max_iter_diff": int(np.abs(o["iters"][:cnt].astype(int) -
                                              it_h[:cnt].astype(int)).max()),
                  "status_equal": bool(np.array_equal(o["status"][:cnt], st_h[:cnt])),
                  "oracle": oracle_algorithm(args),
                  "max_rel_x_diff_vs_oracle": float(np.max(
                      np.linalg.norm(xo - o["x"], axis=1) / np.linalg.norm(o["x"], axis=1))),
                  "max_true_rel_residual_gpu": float(np.max(res_h[:cnt] / bnrm))}
        try:
            cbl = oracle_sample_rate(g0, per_rank, args, target_s=args.cpu_seconds / 2,
                                     kind="banded")
            for k in ("_out", "_count", "_csr"):
                cbl.pop(k)
            cpu["banded_lu"] = cbl
        except Exception as e:  # noqa: BLE001
            cpu["banded_lu"] = {"error": str(e)}

    if rank == 0 and world == 1 and args.parity == "full":
        parity_full = full_parity(args, g0, per_rank, x, res_h, st_h)
    else:
        parity_full = None

    ion = it_all[0::2]   # global index parity: even = ion (rank slices start anywhere,
    ele = it_all[1::2]   # but the gathered stats start at g = 0)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_dict(args, world, per_rank),
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "clocks": clocks,
        "gpu_launches": args.steps,
        "plan": info,
        "solve_stats": {"iters_mean_ion": float(np.mean(ion)), "iters_mean_electron":
                        float(np.mean(ele)), "iters_max": int(it_all.max()),
                        "all_converged": bool(np.all(st_all == 0)),
                        "max_true_rel_residual_rank0": float(np.max(
                            res_h / np.linalg.norm(b_h.numpy(), axis=1)))},
        "parity_sample": parity,
        "parity_full": parity_full,
        "cross_p": cross,
        "stats_digest": digest(it_all, res_all, st_all),
        "kernel_ms": {"min": min(kern_ms), "max": max(kern_ms), "mean": statistics.mean(kern_ms),
                      "std": statistics.pstdev(kern_ms), "n": len(kern_ms)},
    }
    if rank == 0:
        emit(line, args)


# ---------------------------------------------------- Picard (f1) arm --
def run_picard(args, rank, world, local_rank):
    """--picard P: the Picard warm-start pipeline (the
    analogue of Figs. 8/9) at the bench scale.  The
    matrices of Picard steps p = 0..P-1 (xgcgen picard=p: the operator scale
    1 + 0.3 * 0.05^p, b fixed) are all resident in HBM -- XGC rebuilds them on
    the device between solves; that rebuild is not the solver's work and is
    not timed.  One step = P successive bsolve_run calls, x0 of solve p = the
    solution of solve p - 1 kept on the device (warm); the same P solves from
    x0 = 0 are timed beside it.  value = systems x P / cumulative warm time."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_kashinksla22_b200 import Solver
    from paper_conf_ipps_kashinksla22_b200.parallel import (gather_stats, max_over_ranks,
                                                            rank_slice)
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    sl = rank_slice(args.batch, rank, world, args.scaling)
    per_rank, g0 = sl.count, sl.g0
    P = args.picard
    vals, b = [], None
    for p in range(P):
        pat, vh, bh = make_inputs(g0, per_rank, args, pinned=False, picard=p)
        vals.append(vh.to(dev))
        if b is None:
            b = bh.to(dev)   # b is the same at every Picard step
        del vh, bh
    n = pat.n
    S = Solver(pat.row_ptr, pat.col_idx, per_rank, format=args.format,
               placement=args.placement, device=local_rank, solver=args.solver,
               precond=args.precond, restart=args.restart)
    outs = [S.alloc_outputs() for _ in range(P)]
    stream = torch.cuda.current_stream()

    def chain(warm):
        for p in range(P):
            x0 = outs[p - 1][0] if (warm and p > 0) else None
            S.run(vals[p], b, x0, args.tol, args.maxiter, out=outs[p])

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def timed(warm, steps):
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            chain(warm)
        e1.record(stream)
        torch.cuda.synchronize()
        barrier()
        return max_over_ranks(e0.elapsed_time(e1), device=dev)

    for _ in range(max(args.warmup, 0)):
        chain(True)
        chain(False)
    with ClockSampler(local_rank) as clk:
        warm_ms = timed(True, args.steps)
    zero_ms = timed(False, args.steps)
    chain(True)  # leave the warm chain's outputs for the stats below
    torch.cuda.synchronize()
    per_p = []
    all_conv = True
    for p in range(P):
        it_all, res_all, st_all = (t.numpy() for t in gather_stats(*outs[p][1:]))
        all_conv = all_conv and bool(np.all(st_all == 0))
        per_p.append({"p": p, "iters_mean_ion": float(np.mean(it_all[0::2])),
                      "iters_mean_electron": float(np.mean(it_all[1::2]))})
    value = sl.total * P * args.steps / (warm_ms * 1e-3)
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": warm_ms / args.steps, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": dict(config_dict(args, world, per_rank),
                       workload=f"xgc{n}_9pt_mix_picard{P}_warm",
                       description=f"SURVEY 8(f) f1 / BASELINE configs[1] at scale: {P} Picard "
                                   "solves per step, matrices resident on the device, x0 = "
                                   "previous solution", x0="previous Picard solution"),
        "picard": {"steps_per_chain": P, "cumulative_ms_warm": warm_ms / args.steps,
                   "cumulative_ms_zero_guess": zero_ms / args.steps,
                   "speedup_warm_over_zero": zero_ms / warm_ms,
                   "paper": "ELL warm vs zero total time 1.2-1.6x on A100 (PAPER.md:1085-1090); "
                            "Table III iterations e- 30,28,20,16,12 / ion 5,4,3,2,2",
                   "per_step": per_p, "all_converged": all_conv},
        "clocks": clk.summary(), "gpu_launches": args.steps * P, "plan": S.info,
        "e2e": None, "cpu_baseline": None,
    }
    if rank == 0:
        emit(line, args)


# ------------------------------------------------------ banded (f4) arm --
def run_banded(args, rank, world, local_rank):
    """--solver banded: the batched banded LU + solve (bsolve_banded_solve,
    the dgbsv analogue of SURVEY.md 8(f) f4) on the same workload.  A direct
    solve meets the tol 1e-10 residual bar by construction (checked below)."""
    import torch
    from paper_conf_ipps_kashinksla22_b200 import Solver
    from paper_conf_ipps_kashinksla22_b200.parallel import max_over_ranks, rank_slice

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    sl = rank_slice(args.batch, rank, world, args.scaling)
    per_rank, g0 = sl.count, sl.g0
    pat, vals_h, b_h = make_inputs(g0, per_rank, args, pinned=True)
    n, nnz = pat.n, pat.nnz
    S = Solver(pat.row_ptr, pat.col_idx, per_rank, format=args.format, device=local_rank)
    vals = vals_h.to(dev)
    b = b_h.to(dev)
    x = torch.empty((per_rank, n), dtype=torch.float64, device=dev)
    info_d = torch.empty(per_rank, dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            import torch.distributed as dist
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(max(args.warmup, 0)):
        S.banded_solve(vals, b, out=(x, info_d))
    barrier()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launch = []
    with ClockSampler(local_rank) as clk:
        barrier()
        ev0.record(stream)
        for _ in range(args.steps):
            ea, eb = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            ea.record(stream)
            S.banded_solve(vals, b, out=(x, info_d))
            eb.record(stream)
            launch.append((ea, eb))
        ev1.record(stream)
        torch.cuda.synchronize()
        barrier()
    total_ms = max_over_ranks(ev0.elapsed_time(ev1), device=dev)
    launches_per_step = S.query()["banded_launches"]  # of the timed call (before e2e)
    kern_ms = [a.elapsed_time(bb) for a, bb in launch]
    kern_s = statistics.mean(kern_ms) * 1e-3
    value = sl.total * args.steps / (total_ms * 1e-3)
    info = S.info
    kl, ku = info["kl"], info["ku"]
    kb = next(k for k in (4, 8, 16, 33, 65) if k >= max(kl, ku))
    Wb = 2 * kb + 1
    # algorithmic FP64 work per system: dgbtf2's
    # updates on the kl x (kl + ku) band window + the b column, and the two
    # triangular solves: 2 n kl (kl + ku + 1) + 2 n (kl + ku + 1) flop
    flops_sys = 2.0 * n * kl * (kl + ku + 1) + 2.0 * n * (kl + ku + 1)
    fp64_peak = 64 * 2 * info["num_sms"] * 1965e6
    hbm_sys = 8 * (vals.numel() / per_rank + 2 * n) + 4 + 2 * 8 * n * (Wb + 1)
    peaks = {}
    try:
        peaks = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:  # noqa: BLE001
        pass
    hbm_peak = float(peaks.get("hbm_gbs", 6650.0)) * 1e9
    roof = {"bound": "alu", "achieved": flops_sys * per_rank / kern_s / 1e12,
            "peak": fp64_peak / 1e12, "unit": "TFLOP/s",
            "frac": flops_sys * per_rank / kern_s / fp64_peak, "traffic": None,
            "kernel": f"banded_lu_kernel<{kb},{kb},.,true> + banded_backsub_kernel (per chunk)",
            "algorithmic_flops_per_unit": flops_sys, "units_per_launch": per_rank,
            "peak_source": "derived: 64 DFMA/clk/SM x 148 SMs x 1965 MHz (FP64 pipe)",
            "kernel_ms_avg": kern_s * 1e3,
            "hbm": {"achieved": hbm_sys * per_rank / kern_s / 1e9, "peak": hbm_peak / 1e9,
                    "unit": "GB/s", "frac": hbm_sys * per_rank / kern_s / hbm_peak,
                    "bytes_per_system": hbm_sys,
                    "note": "values + b + x + info + the U/y workspace written and read back"}}
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic_banded.json")))
        roof["hbm"]["traffic"] = tr["dram_bytes_per_launch"] * per_rank / tr["systems_per_launch"]
        roof["hbm"]["traffic_note"] = tr.get("note", "")
        roof["traffic_source"] = tr["source"]
    except Exception:  # noqa: BLE001
        pass
    # e2e through the public host API: bsolve_banded_solve_host (chunked
    # H2D / solve / D2H pipeline on the handle's streams), pinned buffers
    e2e = None
    if not args.no_e2e:
        xh = torch.empty((per_rank, n), dtype=torch.float64, pin_memory=True).numpy()
        ih = torch.empty(per_rank, dtype=torch.int32, pin_memory=True).numpy()
        vn, bn = vals_h.numpy(), b_h.numpy()
        S.banded_solve_host(vn, bn, out=(xh, ih))  # warm-up (allocates the pipeline)
        steps = max(1, min(args.steps, 3))
        barrier()
        t0 = time.perf_counter()
        for _ in range(steps):
            S.banded_solve_host(vn, bn, out=(xh, ih))
        torch.cuda.synchronize()
        dt = max_over_ranks(time.perf_counter() - t0, device=dev)
        link = h2d_copy_gbs(dev)
        h2d = int(vn.nbytes + bn.nbytes)
        e2e = {"value": sl.total * steps / dt, "unit": UNIT,
               "h2d_bytes_per_step": h2d,
               "d2h_bytes_per_step": int(xh.nbytes + ih.nbytes), "steps": steps,
               "h2d_gbs": h2d * steps / dt / 1e9, "h2d_copy_gbs_measured": link,
               "link_frac": h2d * steps / dt / 1e9 / link,
               "api": "bsolve_banded_solve_host (C ABI, chunked H2D/solve/D2H pipeline)",
               "bitwise_equal_to_device_path": bool(np.array_equal(
                   xh[:2000], x[:2000].cpu().numpy()))}
    info_h = info_d.cpu().numpy()
    xs = x[: min(per_rank, 2000)].cpu().numpy()
    cpu, parity = None, None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cb = oracle_sample_rate(g0, per_rank, args, target_s=args.cpu_seconds, kind="banded")
        o, cnt = cb.pop("_out"), cb.pop("_count")
        Bs = cb.pop("_csr")
        cnt = min(cnt, xs.shape[0])
        import oracle as O
        rel = np.linalg.norm(xs[:cnt] - o["x"][:cnt], axis=1) / np.linalg.norm(o["x"][:cnt], axis=1)
        res = max(np.linalg.norm(Bs.b[i] - O.spmv(pat.row_ptr, pat.col_idx, Bs.values[i], xs[i]))
                  / np.linalg.norm(Bs.b[i]) for i in range(min(cnt, 64)))
        cpu = cb
        parity = {"systems_checked": int(cnt), "oracle": "banded LU, dgbtf2 + dgbtrs order "
                  "(oracle/oracle.c)", "max_rel_x_diff_vs_oracle": float(rel.max()),
                  "max_true_rel_residual_gpu_first64": float(res)}
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
        "scaling": args.scaling, "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": config_dict(args, world, per_rank), "roofline": roof, "cpu_baseline": cpu,
        "e2e": e2e, "clocks": clk.summary(),
        "gpu_launches": args.steps * launches_per_step,
        "plan": {"kb": kb, "window": Wb, "kl": kl, "ku": ku,
                 "launches_per_step": launches_per_step,
                 "mode": "split: factor kernel + back-substitution kernel per chunk of systems"},
        "solve_stats": {"info_nonzero": int((info_h != 0).sum())}, "parity_sample": parity,
        "kernel_ms": {"min": min(kern_ms), "max": max(kern_ms), "mean": statistics.mean(kern_ms),
                      "std": statistics.pstdev(kern_ms), "n": len(kern_ms)},
    }
    if rank == 0:
        emit(line, args)


def free_port():
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def spawn(args):
    """`bench.py --gpus N` outside torchrun: re-launch this script as N ranks
    (one process per GPU) through torch.distributed.run on 127.0.0.1; rank 0
    prints the JSON line.  NCCL init lines stay visible (NCCL_DEBUG=INFO,
    subsystem INIT) so the communicator size can be read from the log."""
    env = dict(os.environ)
    if args.backend == "nccl":
        env.setdefault("NCCL_DEBUG", "INFO")
        env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
           f"--nproc-per-node={args.gpus}", "--master-addr=127.0.0.1",
           f"--master-port={free_port()}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd, env=env)


def main():
    args = parse()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ and args.impl == "ours":
        sys.exit(spawn(args))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        if args.backend == "nccl" and not args.standin:
            torch.cuda.set_device(local_rank)
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group("gloo")
    try:
        if args.standin:
            run_standin(args, rank, world)
        elif args.picard > 0:
            run_picard(args, rank, world, local_rank)
        elif args.solver == "banded":
            run_banded(args, rank, world, local_rank)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
