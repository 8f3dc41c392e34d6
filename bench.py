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
    ap.add_argument("--precond", choices=["jacobi", "none"], default="jacobi")
    ap.add_argument("--restart", type=int, default=7, help="GMRES restart length m")
    ap.add_argument("--tol", type=float, default=1e-10)
    ap.add_argument("--maxiter", type=int, default=1000)
    ap.add_argument("--seed", type=int, default=20220530)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0,
                    help="target wall seconds of the oracle sample")
    ap.add_argument("--out", default=None, help="also append the JSON line to this file")
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
def make_inputs(g0, count, args, pinned):
    """Generate systems g0..g0+count-1 into (pinned) host buffers, ELL/CSR."""
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
        Bt = X.make_batch(g0 + c0, c1 - c0, pattern=pat, seed=args.seed)
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
                          precond=O.PREC_NONE if args.precond == "none" else O.PREC_JACOBI,
                          restart=args.restart, tol=args.tol, maxiter=args.maxiter, threads=cores)


def oracle_algorithm(args):
    name = ("GMRES(%d)" % args.restart if args.solver == "gmres"
            else "Alg. 1 BiCGSTAB")
    return f"{name} + {'Jacobi' if args.precond == 'jacobi' else 'no preconditioner'} (oracle/oracle.c)"


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

    for _ in range(max(args.warmup, 0)):
        S.run(vals, b, None, args.tol, args.maxiter, out=out)
    barrier()
    ev0 = torch.cuda.Event(enable_timing=True)
    ev1 = torch.cuda.Event(enable_timing=True)
    launch_ms = []
    with ClockSampler(local_rank) as clk:
        barrier()
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
    it_all, _, st_all = (t.numpy() for t in gather_stats(it, res, st))
    sum_iters_rank = int(it_h.astype(np.int64).sum())

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
                 "peak_source": "derived: 64 DFMA/clk/SM x 148 x 1965 MHz"},
        "all_operand_effective": {
            "achieved": all_operand_bytes / kern_avg_s / 1e9, "unit": "GB/s",
            "frac_of_smem_peak": all_operand_bytes / kern_avg_s / smem_peak,
            "note": "values + gathered operands + stores per iteration (2 x (16 nnz + 8 n)) "
                    "wherever they live; effective on-chip bandwidth, can exceed 1"},
    }
    # traffic from the committed ncu --set full capture of this kernel on this
    # workload (profiles/ncu_traffic.json), scaled to this launch's systems
    try:
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
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            S.run_host(vn, bn, None, args.tol, args.maxiter, out=outs)
        torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        dt = max_over_ranks(dt, device=dev)
        h2d = int(vn.nbytes + bn.nbytes)
        d2h = int(x_h.nbytes + i_h.nbytes + r_h.nbytes + s_h.nbytes)
        e2e = {"value": sl.total * e2e_steps / dt, "unit": UNIT,
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h, "steps": e2e_steps,
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

    ion = it_all[0::2] if (g0 % 2 == 0) else it_all[1::2]
    ele = it_all[1::2] if (g0 % 2 == 0) else it_all[0::2]
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
        "kernel_ms": {"min": min(kern_ms), "max": max(kern_ms), "mean": statistics.mean(kern_ms),
                      "std": statistics.pstdev(kern_ms), "n": len(kern_ms)},
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
        e2e = {"value": sl.total * steps / dt, "unit": UNIT,
               "h2d_bytes_per_step": int(vn.nbytes + bn.nbytes),
               "d2h_bytes_per_step": int(xh.nbytes + ih.nbytes), "steps": steps,
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


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        if args.solver == "banded":
            run_banded(args, rank, world, local_rank)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
