// gmres.cuh -- restarted, right-preconditioned GMRES(m) for ONE system per
// CTA (the paper implements "several preconditionable
// iterative solvers"; BiCGSTAB is its headline).
//
// Same algorithm and conventions as DESIGN.md "GMRES" (Saad,
// "Iterative Methods for Sparse Linear Systems", Alg. 6.9 / 6.11 / 9.5):
//   * every restart cycle starts from the TRUE residual r = b - A x and the
//     solve stops when ||r|| < tau (tau = tol ||b|| or tol, strict);
//   * inside a cycle the Givens estimate |g_{j+1}| ends the cycle early;
//   * iters counts the Krylov products w = A z_j;
//   * breakdown: non-finite or zero rotation denominator -> status 2 with the
//     x of the cycle start.
// GPU design (DESIGN.md "Kernels" 11):
//   * the Krylov basis v_0 .. v_{m-1} lives in SHARED MEMORY, element (i, row
//     j of thread t) at sV[(i R + j) NT + t]: every access is one conflict-free
//     LDS/STS per row; w, z, x, b and d stay in registers;
//   * Arnoldi by classical Gram-Schmidt with one re-orthogonalisation (CGS2):
//     all j + 1 projections of a pass are ONE fused block reduction (instead
//     of the j + 1 dependent reductions of modified Gram-Schmidt); the second
//     pass also reduces ||w'||^2, so h_{j+1,j}^2 = ||w'||^2 - sum c_i^2 needs no
//     third barrier (exact for orthonormal v_i; the correction c is O(eps)).
//     CGS2 and MGS build the same Arnoldi basis in exact arithmetic; the
//     rounding differs from an MGS implementation (parity is tolerance-based);
//   * the small Hessenberg / Givens state (<= kMaxRestart columns) is computed
//     redundantly and identically by every thread from the reduced values
//     (uniform control flow, no broadcast), with compile-time indices only
//     (selects on the runtime column index, no local memory); thread 0 keeps
//     the triangular factor R in SMEM for the back substitution.
#pragma once
#include "kernels.cuh"

namespace bsolve {

template <int R, int NT, int M, class Comm, class SpMV>
__device__ __forceinline__ void gmres_core(const SolveParams &P, long long sys, double (&x)[R],
                                           const double (&bv)[R], const double (&d)[R],
                                           const bool (&act)[R], double *sV, double *sR,
                                           Comm &comm, SpMV &&spmv) {
  static_assert(M >= 1 && M + 1 <= 8, "block_sum reduces at most 8 values");
  const int n = P.n;
  const int m = P.restart;  // 1 .. M (validated on the host)
  const int tid = threadIdx.x;
  auto V = [&](int i, int j) -> double & { return sV[(i * R + j) * NT + tid]; };

  double bb[1];
  bb[0] = rows_sum<R>([&](int j) { return bv[j] * bv[j]; });
  comm.template sum<1>(bb);
  const double bnorm = sqrt(bb[0]);
  const double tau = (P.stop == STOP_ABS) ? P.tol : P.tol * bnorm;
  double *xout = P.x + sys * n;
  if (P.stop == STOP_REL_B && bnorm == 0.0) {
#pragma unroll
    for (int j = 0; j < R; ++j)
      if (act[j]) xout[comm.grow(j)] = 0.0;
    if (comm.leader()) {
      P.iters[sys] = 0;
      P.resnorm[sys] = 0.0;
      if (P.status) P.status[sys] = SYS_CONVERGED;
    }
    return;
  }

  int it = 0, st = -1;
  double rnorm = 0.0;
  for (;;) {
    // ---- true residual r = b - A x; converged? ------------------------------
#pragma unroll
    for (int j = 0; j < R; ++j) comm.publish(j, x[j]);
    comm.sync();
    double q[R];
    spmv(x, q);
    double r[R];
#pragma unroll
    for (int j = 0; j < R; ++j) r[j] = act[j] ? bv[j] - q[j] : 0.0;
    double rr[1];
    rr[0] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
    comm.template sum<1>(rr);
    rnorm = sqrt(rr[0]);
    if (rnorm < tau) break;
    if (it >= P.maxiter) break;
    if (!isfinite(rnorm)) { st = SYS_BREAKDOWN; break; }
    // ---- v_0 = r / beta, g = beta e_1 --------------------------------------
    const double rinv = 1.0 / rnorm;
#pragma unroll
    for (int j = 0; j < R; ++j) V(0, j) = r[j] * rinv;
    double g[M + 1], cs[M], sn[M];
#pragma unroll
    for (int i = 0; i <= M; ++i) g[i] = 0.0;
#pragma unroll
    for (int i = 0; i < M; ++i) cs[i] = sn[i] = 0.0;
    g[0] = rnorm;
    int k = 0;
    bool brk = false;
#pragma unroll 1
    for (int jj = 0; jj < m && it < P.maxiter; ++jj) {
      // z = M^-1 v_jj, w = A z (v_jj was stored by this thread: no barrier
      // needed before reading it; the publish is fenced by comm.sync)
      double z[R];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        z[j] = d[j] * V(jj, j);
        comm.publish(j, z[j]);
      }
      comm.sync();
      double w[R];
      spmv(z, w);
      ++it;
      // ---- CGS pass 1: h_i = (w, v_i), i <= jj -------------------------------
      double h[M];
#pragma unroll
      for (int i = 0; i < M; ++i)
        h[i] = (i <= jj) ? rows_sum<R>([&](int j) { return w[j] * V(i, j); }) : 0.0;
      comm.template sum<M>(h);
#pragma unroll
      for (int i = 0; i < M; ++i)
        if (i <= jj) {
#pragma unroll
          for (int j = 0; j < R; ++j) w[j] = w[j] - h[i] * V(i, j);
        }
      // ---- CGS pass 2 (re-orthogonalisation) + ||w'||^2 ----------------------
      double c[M + 1];
#pragma unroll
      for (int i = 0; i < M; ++i)
        c[i] = (i <= jj) ? rows_sum<R>([&](int j) { return w[j] * V(i, j); }) : 0.0;
      c[M] = rows_sum<R>([&](int j) { return w[j] * w[j]; });
      comm.template sum<M + 1>(c);
      double cc = 0.0;
#pragma unroll
      for (int i = 0; i < M; ++i)
        if (i <= jj) {
          h[i] += c[i];
          cc += c[i] * c[i];
#pragma unroll
          for (int j = 0; j < R; ++j) w[j] = w[j] - c[i] * V(i, j);
        }
      const double hn2 = c[M] - cc;
      const double hn = hn2 > 0.0 ? sqrt(hn2) : 0.0;  // h_{jj+1,jj}; 0: lucky breakdown
      // ---- Hessenberg column jj: previous rotations, new rotation -------------
      double hc[M + 1];
#pragma unroll
      for (int i = 0; i <= M; ++i) {
        hc[i] = (i == jj + 1) ? hn : 0.0;
        if (i < M) {
          if (i <= jj) hc[i] = h[i];
        }
      }
#pragma unroll
      for (int i = 0; i < M; ++i)
        if (i < jj) {
          const double a = hc[i], b = hc[i + 1];
          hc[i] = cs[i] * a + sn[i] * b;
          hc[i + 1] = -sn[i] * a + cs[i] * b;
        }
      double a = 0.0, b = 0.0, gj = 0.0;
#pragma unroll
      for (int i = 0; i <= M; ++i) {
        if (i == jj) { a = hc[i]; gj = g[i]; }
        if (i == jj + 1) b = hc[i];
      }
      const double den = sqrt(a * a + b * b);
      if (den == 0.0 || !isfinite(den) || !isfinite(hn)) { brk = true; break; }
      const double cj = a / den, sj = b / den;
      double gn = 0.0;
#pragma unroll
      for (int i = 0; i <= M; ++i) {
        if (i < M && i == jj) { cs[i] = cj; sn[i] = sj; g[i] = cj * gj; }
        if (i == jj + 1) { g[i] = -sj * gj; gn = g[i]; }
      }
      if (comm.leader()) {  // column jj of the triangular factor
#pragma unroll
        for (int i = 0; i < M; ++i)
          if (i < jj) sR[i * M + jj] = hc[i];
        sR[jj * M + jj] = den;
      }
      k = jj + 1;
      if (fabs(gn) < tau || hn == 0.0) break;
      if (jj + 1 < m) {
        const double hinv = 1.0 / hn;
#pragma unroll
        for (int j = 0; j < R; ++j) V(jj + 1, j) = w[j] * hinv;
      }
    }
    if (brk) { st = SYS_BREAKDOWN; break; }
    // ---- y = R^-1 g (every thread, R from SMEM); x += M^-1 V y --------------
    comm.barrier();  // thread 0's writes of R visible (CTA only)
    double y[M];
#pragma unroll
    for (int i = M - 1; i >= 0; --i) {
      y[i] = 0.0;
      if (i < k) {
        double s = g[i];
#pragma unroll
        for (int l = i + 1; l < M; ++l)
          if (l < k) s -= sR[i * M + l] * y[l];
        y[i] = s / sR[i * M + i];
      }
    }
#pragma unroll
    for (int j = 0; j < R; ++j) {
      double s = 0.0;
#pragma unroll
      for (int i = 0; i < M; ++i)
        if (i < k) s += V(i, j) * y[i];
      x[j] = x[j] + d[j] * s;
    }
    // (the basis is thread-private: no barrier; the next publish of x follows
    // the reductions above, so every reader of the gather buffer and of R has
    // passed a barrier since)
  }
  if (st != SYS_BREAKDOWN) st = rnorm < tau ? SYS_CONVERGED : SYS_MAXITER;
#pragma unroll
  for (int j = 0; j < R; ++j)
    if (act[j]) xout[comm.grow(j)] = x[j];
  if (comm.leader()) {
    P.iters[sys] = it;
    P.resnorm[sys] = rnorm;
    if (P.status) P.status[sys] = static_cast<int8_t>(st);
  }
}

}  // namespace bsolve
