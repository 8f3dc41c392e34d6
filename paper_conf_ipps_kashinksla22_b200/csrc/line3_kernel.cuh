// line3_kernel.cuh -- the line-tiled TMEM plan at THREE CTAs per SM
// (DESIGN.md "Kernels" 12; round-2 redesign of bicgstab_tmem_line_kernel).
//
// What it computes: Algorithm 1 of the paper (Sec. IV-D),
// BiCGSTAB right-preconditioned with scalar Jacobi, one CTA per system, each
// system stopping on its own -- the same schedule, stop
// tests, breakdown and true-residual guard as bicgstab_core (kernels.cuh,
// readings R1-R10 of DESIGN.md); only WHERE the per-row state lives changes.
//
// Why: the 2-CTA line kernel (252 registers x 128 threads) is latency-bound
// (round-1 ncu: 12.4% warps active, "wait" and "short scoreboard" stalls,
// SMEM pipe 39% busy).  A third resident CTA needs <= 168 registers per
// thread (65,536 / 384).  The register diet:
//   * registers: only r (then s), p, v and d = 1/a_ii, 8 rows each;
//   * tensor memory: besides the 8 off-diagonal values of each row (128
//     columns, as before) a SECOND allocation of 32 columns per CTA holds the
//     shadow residual r^ (columns 0-15) and the diagonal a_ii (16-31):
//     3 x (128 + 32) = 480 <= 512 columns per SM;
//   * shared memory: the iterate x, thread-private (double2 layout, every
//     access conflict-free): read and written once per iteration;
//   * the SpMV operand of the thread's own rows, d_j * p_j (or d_j * s_j), is
//     recomputed where it is needed instead of being kept: the same product
//     the publish stored, so the same bits;
//   * one TMEM row (16 columns) in flight at a time, a sliding window of
//     gathered operands.
#pragma once
#include "line_kernel.cuh"

namespace bsolve {

// SMEM layout of one CTA: [gather planes R*S][reduction scratch 16*NWARP]
// [x: R*NT][PRE = 1: block-Jacobi factors 22*NT][2 TMEM base slots].
template <int NX, int PRE = 0>
struct Line3Geom {
  static constexpr int R = 8, NT = 128, NWARP = 4;
  using L = LineGeom<NX, NT, R>;
  static constexpr int OFF_RED = R * L::S;
  static constexpr int OFF_X = ((OFF_RED + 16 * NWARP) + 1) & ~1;  // 16-byte aligned
  static constexpr int OFF_F = OFF_X + R * NT;
  static constexpr int NF = PRE ? 22 : 0;  // l_1..7, 1/u_0..7, a_(j,j+1) j = 0..6
  static constexpr int SMEM_BYTES = (OFF_F + NF * NT) * 8 + 16;
};

__device__ __forceinline__ void tmem_ld2(uint32_t taddr, uint32_t (&r)[2]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x2.b32 {%0,%1}, [%2];"
               : "=r"(r[0]), "=r"(r[1])
               : "r"(taddr));
}
__device__ __forceinline__ void tmem_regs_ready2(uint32_t (&r)[2]) {
  asm volatile("" : "+r"(r[0]), "+r"(r[1]));
}

// y = A (d .* g) for rows 8t .. 8t+7 with the operands of the thread's own
// rows recomputed as d_j * g_j; values from TMEM, diagonal a_jj from the aux
// TMEM columns; neighbours gathered from the published planes.  One row at a
// time: its TMEM loads, the two plane operands it is the first to need
// (a sliding window: registers), wait, then three independent partial sums
// (line above | own line | line below) added at the end -- the 9-term FMA
// chain of one row was the latency bound (ncu "wait" stalls; DESIGN.md perf
// log).  The row sum is a fixed order, so results are deterministic.
// Grid width: NX at compile time (NXG = NX, A = 0), or -- the generic-width
// instances -- NX = B = width mod 8 with A = width / 8 at run time and the
// plane geometry of the widest grid NXG: row 8t + o with o = +-(8A + B) + d
// sits at idx(+-B + d) +- A (idx(8k + x) = idx(x) + k), so only the column
// shift of the two neighbour lines is a run-time offset.
template <int NX, int NXG = NX>
__device__ __forceinline__ void line3_spmv(uint32_t tval, uint32_t ta0, const double *gq,
                                           const double (&dd)[8], const double (&g)[8],
                                           double (&y)[8], int A = 0) {
  constexpr int R = 8;
  using L = LineGeom<NXG, 128, R>;
  uint32_t w[16], aw[2];
  double gm[R + 2], gp[R + 2], gr = 0.0;
  const double *gqm = gq - A, *gqp = gq + A;  // the line below / above
#pragma unroll
  for (int e = 0; e < 3; ++e) {
    gm[e] = gqm[L::idx(-NX + e - 1)];
    gp[e] = gqp[L::idx(NX + e - 1)];
  }
  const double gl = gq[L::idx(-1)];
#pragma unroll
  for (int j = 0; j < R; ++j) {
    tmem_ld16(tval + 16 * j, w);
    tmem_ld2(ta0 + 2 * j, aw);
    if (j > 0) {  // the two operands row j is the first to need
      gm[j + 2] = gqm[L::idx(-NX + j + 1)];
      gp[j + 2] = gqp[L::idx(NX + j + 1)];
    }
    if (j == R - 1) gr = gq[L::idx(R)];
    tmem_wait_ld();
    tmem_regs_ready(w);
    tmem_regs_ready2(aw);
    const double a0 = __hiloint2double(static_cast<int>(aw[1]), static_cast<int>(aw[0]));
    const double own = dd[j] * g[j];
    const double left = j == 0 ? gl : dd[j == 0 ? 0 : j - 1] * g[j == 0 ? 0 : j - 1];
    const double right = j == R - 1 ? gr : dd[j == R - 1 ? j : j + 1] * g[j == R - 1 ? j : j + 1];
    double c0 = tmem_f64(w, 0) * gm[j];
    double c1 = a0 * own;
    double c2 = tmem_f64(w, 5) * gp[j];
    c0 = fma(tmem_f64(w, 1), gm[j + 1], c0);
    c1 = fma(tmem_f64(w, 3), left, c1);
    c2 = fma(tmem_f64(w, 6), gp[j + 1], c2);
    c0 = fma(tmem_f64(w, 2), gm[j + 2], c0);
    c1 = fma(tmem_f64(w, 4), right, c1);
    c2 = fma(tmem_f64(w, 7), gp[j + 2], c2);
    y[j] = (c0 + c1) + c2;  // rows >= n: zero values and diagonal -> 0
  }
}

// Algorithm 1 for one system on this CTA's rows (the whole system for the
// single-CTA kernel, rows grow0 .. grow0 + 1023 of it on a cluster): every
// global row index is grow0 + 8 t + j; the communication policy Comm
// (LineComm: CTA-local; Line3ClusterComm: halo rows and reduction partials
// through distributed shared memory) publishes, synchronises and reduces.
template <int NX, int ROUNDS, int PRE, class Comm, int NXG = NX>
__device__ __forceinline__ void line3_solve(const SolveParams &P, long long sys, int grow0,
                                            bool leader, const bool (&act)[8], Comm &comm,
                                            double *sf, double2 *sx2, uint32_t tval,
                                            uint32_t trh, uint32_t ta0, int A = 0) {
  constexpr int R = 8, NT = 128;
  const int n = P.n;
  const int row0 = grow0 + R * threadIdx.x;  // global index of this thread's first row
  const double *gval = P.values + sys * P.sys_stride;
  // ---- this thread's rows: values -> TMEM, diagonal -> TMEM + d ------------
  double d[R];
  double bdiag[PRE ? R : 1], blo[PRE ? R : 1], bup[PRE ? R : 1];  // block-Jacobi block
  {
    const bool vec = !P.vidx && ((n & 1) == 0) && ((reinterpret_cast<uintptr_t>(gval) & 15u) == 0) &&
                     row0 + R <= n;
    uint32_t aw[16];
#pragma unroll
    for (int j = 0; j < R; j += 2) {
      double a0p[2], vv[2][8];
      if (vec) {
        const double2 dg = __ldg(reinterpret_cast<const double2 *>(gval + row0 + j));
        a0p[0] = dg.x;
        a0p[1] = dg.y;
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          const int k = P.c2s[c];
          double2 v = make_double2(0.0, 0.0);
          if (k >= 0) v = __ldg(reinterpret_cast<const double2 *>(gval + (long long)k * n + row0 + j));
          vv[0][c] = v.x;
          vv[1][c] = v.y;
        }
      } else {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const bool a = act[j + h];
          const int row = row0 + j + h;
          if (P.vidx) {  // CSR values: the handle's (row, canonical slot) -> CSR index table
            const int e0 = a ? __ldg(P.vidx + 8 * n + row) : -1;
            a0p[h] = e0 >= 0 ? __ldg(gval + e0) : 0.0;
#pragma unroll
            for (int c = 0; c < 8; ++c) {
              const int e = a ? __ldg(P.vidx + c * n + row) : -1;
              vv[h][c] = e >= 0 ? __ldg(gval + e) : 0.0;
            }
          } else {
            a0p[h] = a ? __ldg(gval + row) : 0.0;
#pragma unroll
            for (int c = 0; c < 8; ++c) {
              const int k = P.c2s[c];
              vv[h][c] = (a && k >= 0) ? __ldg(gval + (long long)k * n + row) : 0.0;
            }
          }
        }
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        uint32_t w[16];
#pragma unroll
        for (int c = 0; c < 8; ++c) {
          w[2 * c] = static_cast<uint32_t>(__double2loint(vv[h][c]));
          w[2 * c + 1] = static_cast<uint32_t>(__double2hiint(vv[h][c]));
        }
        tmem_st16(tval + 16 * (j + h), w);
        d[j + h] = jacobi_inv(P.precond, a0p[h]);
        if constexpr (PRE == 1) {  // canonical offsets 3 = -1, 4 = +1 (line_kernel.cuh)
          bdiag[j + h] = a0p[h];
          blo[j + h] = vv[h][3];
          bup[j + h] = vv[h][4];
        }
        aw[2 * (j + h)] = static_cast<uint32_t>(__double2loint(a0p[h]));
        aw[2 * (j + h) + 1] = static_cast<uint32_t>(__double2hiint(a0p[h]));
      }
    }
    tmem_st16(ta0, aw);
  }
  if constexpr (PRE == 1) {
    // Thomas factorisation of the thread's tridiagonal block (rows >= n: the
    // identity, so their entries stay 0)
    double l[R], u[R];
    bool ok = true;
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const bool a = act[j];
      l[j] = (j > 0 && a) ? blo[j] / u[j - 1] : 0.0;
      u[j] = a ? bdiag[j] - l[j] * (j > 0 ? bup[j - 1] : 0.0) : 1.0;
      ok = ok && u[j] != 0.0 && isfinite(u[j]) && isfinite(l[j]);
    }
#pragma unroll
    for (int j = 0; j < R; ++j) {
      if (j > 0) sf[(j - 1) * NT] = ok ? l[j] : 0.0;
      sf[(7 + j) * NT] = ok ? 1.0 / u[j] : 1.0;
      if (j < R - 1) sf[(15 + j) * NT] = (ok && act[j + 1]) ? bup[j] : 0.0;
    }
  }
  const double *bsys = P.b + sys * n;
  double r[R], p[R], v[R];
#pragma unroll
  for (int j = 0; j < R; ++j) r[j] = act[j] ? __ldg(bsys + row0 + j) : 0.0;
  tmem_wait_st();

  const double one[R] = {1, 1, 1, 1, 1, 1, 1, 1};
  auto spmv = [&](const double(&dd)[R], const double(&g)[R], double(&y)[R]) {
    line3_spmv<NX, NXG>(tval, ta0, comm.gq, dd, g, y, A);
  };
  auto x_load = [&](double(&xx)[R]) {
#pragma unroll
    for (int k = 0; k < R / 2; ++k) {
      const double2 q = sx2[k * NT];
      xx[2 * k] = q.x;
      xx[2 * k + 1] = q.y;
    }
  };
  auto x_store = [&](const double(&xx)[R]) {
#pragma unroll
    for (int k = 0; k < R / 2; ++k) sx2[k * NT] = make_double2(xx[2 * k], xx[2 * k + 1]);
  };
  auto rh_store = [&](const double(&q)[R]) {
    uint32_t w[16];
#pragma unroll
    for (int j = 0; j < R; ++j) {
      w[2 * j] = static_cast<uint32_t>(__double2loint(q[j]));
      w[2 * j + 1] = static_cast<uint32_t>(__double2hiint(q[j]));
    }
    tmem_st16(trh, w);
    tmem_wait_st();
  };
  auto rh_load = [&](uint32_t(&w)[16]) {
    tmem_ld16(trh, w);
    tmem_wait_ld();
    tmem_regs_ready(w);
  };
  // z = M^-1 y for the thread's block (PRE = 1): forward then back substitution
  auto bj_apply = [&](const double(&y)[R], double(&z)[R]) {
    z[0] = y[0];
#pragma unroll
    for (int j = 1; j < R; ++j) z[j] = fma(-sf[(j - 1) * NT], z[j - 1], y[j]);
    z[R - 1] = z[R - 1] * sf[(7 + R - 1) * NT];
#pragma unroll
    for (int j = R - 2; j >= 0; --j) z[j] = fma(-sf[(15 + j) * NT], z[j + 1], z[j]) * sf[(7 + j) * NT];
  };

  // ---- a3: x = x0 (or 0), r = b - A x0, r^ = r, ||b|| ----------------------
  double red3[2] = {0.0, 0.0};
#pragma unroll
  for (int j = 0; j < R; ++j) red3[0] += r[j] * r[j];  // b.b
  {
    double xx[R];
#pragma unroll
    for (int j = 0; j < R; ++j) xx[j] = (act[j] && P.x0) ? __ldg(P.x0 + sys * n + row0 + j) : 0.0;
    x_store(xx);
    if (P.x0) {
#pragma unroll
      for (int j = 0; j < R; ++j) comm.publish(j, xx[j]);
      comm.sync();
      spmv(one, xx, v);
#pragma unroll
      for (int j = 0; j < R; ++j) r[j] = r[j] - v[j];
    }
  }
#pragma unroll
  for (int j = 0; j < R; ++j) {
    p[j] = 0.0;
    v[j] = 0.0;
    red3[1] += r[j] * r[j];
  }
  rh_store(r);
  comm.template sum_x<2>(red3, r, 2, d);  // (+ boundary r and d: the halo state)
  const double bnorm = sqrt(red3[0]);
  const double tau = (P.stop == STOP_ABS) ? P.tol : P.tol * bnorm;
  const double tau2 = tau * tau;
  const bool sq = tau2 > 1e-300 && tau2 < 1e300;  // R7: squared-norm stop tests
  auto below = [&](double nrm2) { return sq ? nrm2 < tau2 : sqrt(nrm2) < tau; };
  double rnorm2 = red3[1];
  double rho = red3[1];  // r^.r with r^ = r

  double *xout = P.x + sys * n;
  if (P.stop == STOP_REL_B && bnorm == 0.0) {
#pragma unroll
    for (int j = 0; j < R; ++j)
      if (act[j]) xout[row0 + j] = 0.0;
    if (leader) {
      P.iters[sys] = 0;
      P.resnorm[sys] = 0.0;
      if (P.status) P.status[sys] = SYS_CONVERGED;
    }
  } else {
    // true residual ||b - A x||^2 into q (publishes x; one more barrier)
    auto true_residual = [&](double(&q)[R]) -> double {
      double xx[R];
      x_load(xx);
#pragma unroll
      for (int j = 0; j < R; ++j) comm.publish(j, xx[j]);
      comm.sync();
      spmv(one, xx, q);
      double tr[1] = {0.0};
#pragma unroll
      for (int j = 0; j < R; ++j) {
        const double bj = act[j] ? __ldg(bsys + row0 + j) : 0.0;
        q[j] = act[j] ? bj - q[j] : 0.0;
        tr[0] += q[j] * q[j];
      }
      comm.template sum_x<1>(tr, q, 3, q);  // (+ boundary q: the restart's halo r)
      return tr[0];
    };

    int it = 0, st = -1, exit_kind = 0;
    double alpha = 1.0, omega = 1.0;
    double beta_c = 1.0;  // alpha / (rho' omega): beta = rho * beta_c (R2)
    double final_res = -1.0;
    for (;;) {
      exit_kind = 0;
      while (true) {
        if (below(rnorm2)) { exit_kind = 1; break; }        // stop test 1
        if (it >= P.maxiter) break;
        if (bad(rho)) { st = SYS_BREAKDOWN; break; }
        // R2: beta = (rho / rho') (alpha / omega), the division done after the
        // previous omega; ROUNDS == 2 keeps beta itself in beta_c (R29)
        const double beta = ROUNDS == 2 ? beta_c : rho * beta_c;
        // a5: p = r + beta (p - omega v); publish p^ = PRECOND(p)
        double ph[PRE ? R : 1];  // block-Jacobi: p^ (scalar Jacobi recomputes d p)
        if constexpr (PRE == 1) {
#pragma unroll
          for (int j = 0; j < R; ++j) p[j] = r[j] + beta * (p[j] - omega * v[j]);
          bj_apply(p, ph);
#pragma unroll
          for (int j = 0; j < R; ++j) comm.publish(j, ph[j]);
        } else {
#pragma unroll
          for (int j = 0; j < R; ++j) {
            p[j] = r[j] + beta * (p[j] - omega * v[j]);
            comm.publish(j, d[j] * p[j]);
          }
        }
        if constexpr (Comm::kHalo2) {
          comm.halo_p(beta, omega);  // the neighbours' boundary rows, recomputed here
          comm.sync_local();
        } else {
          comm.sync();
        }
        if constexpr (PRE == 1) spmv(one, ph, v);           // a6: v = A p^
        else spmv(d, p, v);
        ++it;
        double rv[1];
        {
          uint32_t hw[16];
          rh_load(hw);
          rv[0] = rows_sum<R>([&](int j) { return tmem_f64(hw, j) * v[j]; });
        }
        comm.template sum_x<1>(rv, v, 1, v);                // a7: r^.v (+ boundary v)
        if (bad(rv[0])) { st = SYS_BREAKDOWN; break; }
        alpha = rho / rv[0];                                // R3
        // s = r - alpha v (kept in r); publish s^ = PRECOND(s)
        double sh[PRE ? R : 1];
        if constexpr (PRE == 1) {
          // x + alpha p^ now (p^ dies here): the first half of x's update, in
          // the oracle's order (x + alpha p^) + omega s^, and stop test 2's x
          double xx[R];
          x_load(xx);
#pragma unroll
          for (int j = 0; j < R; ++j) xx[j] = xx[j] + alpha * ph[j];
          x_store(xx);
#pragma unroll
          for (int j = 0; j < R; ++j) r[j] = r[j] - alpha * v[j];
          bj_apply(r, sh);
#pragma unroll
          for (int j = 0; j < R; ++j) comm.publish(j, sh[j]);
        } else {
#pragma unroll
          for (int j = 0; j < R; ++j) {
            r[j] = r[j] - alpha * v[j];
            comm.publish(j, d[j] * r[j]);
          }
        }
        if constexpr (Comm::kHalo2) {
          comm.halo_s(alpha);
          comm.sync_local();
        } else {
          comm.sync();
        }
        // ROUNDS == 3: t.s, t.t, s.s here and ||r||^2, r^.r in a third round.
        // ROUNDS == 2 (R29): + r^.s, r^.t, so that rho_{i+1} =
        // r^.s - omega r^.t and ||r_{i+1}||^2 = s.s - omega t.s come from this
        // round (exact identities for r = s - omega t, omega = t.s / t.t); the
        // third round runs only when an identity cancels more than 8 digits.
        constexpr int KT = ROUNDS == 2 ? 5 : 3;
        double ts[KT];
        ts[2] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
        if constexpr (ROUNDS == 2) {
          uint32_t hw[16];
          rh_load(hw);
          ts[3] = rows_sum<R>([&](int j) { return tmem_f64(hw, j) * r[j]; });
        }
        double t[R];
        if constexpr (PRE == 1) spmv(one, sh, t);           // a9: t = A s^ (speculative)
        else spmv(d, r, t);
        ts[0] = rows_sum<R>([&](int j) { return t[j] * r[j]; });
        ts[1] = rows_sum<R>([&](int j) { return t[j] * t[j]; });
        if constexpr (ROUNDS == 2) {
          uint32_t hw[16];
          rh_load(hw);
          ts[4] = rows_sum<R>([&](int j) { return tmem_f64(hw, j) * t[j]; });
        }
        comm.template sum_x<KT>(ts, t, 4, t);               // (+ boundary t)
        if (below(ts[2])) {                                 // stop test 2
          if constexpr (PRE == 0) {  // (block-Jacobi: x + alpha p^ is stored already)
            double xx[R];
            x_load(xx);
#pragma unroll
            for (int j = 0; j < R; ++j) xx[j] = xx[j] + alpha * (d[j] * p[j]);
            x_store(xx);
          }
          exit_kind = 2;
          break;
        }
        if (bad(ts[1])) { st = SYS_BREAKDOWN; break; }
        omega = ts[0] / ts[1];
        if (bad(omega)) { st = SYS_BREAKDOWN; break; }
        if constexpr (ROUNDS == 3) beta_c = alpha / (rho * omega);  // rho becomes rho' below
        {
          double xx[R];
          x_load(xx);
          if constexpr (PRE == 1) {
#pragma unroll
            for (int j = 0; j < R; ++j) xx[j] = xx[j] + omega * sh[j];
          } else {
#pragma unroll
            for (int j = 0; j < R; ++j) xx[j] = xx[j] + alpha * (d[j] * p[j]) + omega * (d[j] * r[j]);
          }
          x_store(xx);
        }
#pragma unroll
        for (int j = 0; j < R; ++j) r[j] = r[j] - omega * t[j];   // r = s - omega t
        if constexpr (Comm::kHalo2) comm.halo_r(omega);
        bool explicit_round = ROUNDS == 3;
        if constexpr (ROUNDS == 2) {
          const double rho_n = ts[3] - omega * ts[4];
          const double rr2 = ts[2] - omega * ts[0];
          explicit_round = !(rr2 > 1e-8 * ts[2]) ||
                           !(fabs(rho_n) > 1e-8 * (fabs(ts[3]) + fabs(omega * ts[4])));
          if (!explicit_round) {
            // beta_{i+1} = (rho_{i+1} / rho_i)(alpha / omega) with rho_{i+1} t.t =
            // r^.s t.t - t.s r^.t: one division, independent of omega's
            beta_c = alpha * (ts[3] * ts[1] - ts[0] * ts[4]) / (rho * ts[0]);
            rnorm2 = rr2;
            rho = rho_n;
          }
        }
        if (explicit_round) {
          double rr[2];
          rr[0] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
          {
            uint32_t hw[16];
            rh_load(hw);
            rr[1] = rows_sum<R>([&](int j) { return tmem_f64(hw, j) * r[j]; });
          }
          comm.template sum<2>(rr);                         // ||r||^2, r^.r
          if constexpr (ROUNDS == 2) beta_c = rr[1] * alpha / (rho * omega);
          rnorm2 = rr[0];
          rho = rr[1];
        }
      }
      if (st == SYS_BREAKDOWN || exit_kind == 0 || !P.trc) break;
      // ---- a11: true-residual guard (R4) ------------------------
      double q[R];
      const double tr2 = true_residual(q);
      final_res = sqrt(tr2);
      if (final_res < tau || it >= P.maxiter) break;
#pragma unroll
      for (int j = 0; j < R; ++j) {  // restart from the true residual, keep counting
        r[j] = q[j];
        p[j] = 0.0;
        v[j] = 0.0;
      }
      if constexpr (Comm::kHalo2) comm.halo_restart();
      rh_store(q);
      alpha = omega = beta_c = 1.0;
      rnorm2 = tr2;
      rho = tr2;
      final_res = -1.0;
    }
    if (final_res < 0.0) {
      comm.barrier();  // earlier gathers of this CTA done before x is published
      double q[R];
      final_res = sqrt(true_residual(q));
    }
    if (st != SYS_BREAKDOWN) {
      if (P.trc) st = final_res < tau ? SYS_CONVERGED : SYS_MAXITER;
      else st = exit_kind != 0 ? SYS_CONVERGED : SYS_MAXITER;
    }
    double xx[R];
    x_load(xx);
#pragma unroll
    for (int j = 0; j < R; ++j)
      if (act[j]) xout[row0 + j] = xx[j];
    if (leader) {
      P.iters[sys] = it;
      P.resnorm[sys] = final_res;
      if (P.status) P.status[sys] = static_cast<int8_t>(st);
    }
  }
}

// PRE = 0: PRECOND(y) = d .* y (scalar Jacobi, or none).
// PRE = 1: block-Jacobi with one block per thread = its 8 consecutive rows
// (R30).  On an NX >= 9 wide 9-point grid the
// block A[8t..8t+7, 8t..8t+7] is tridiagonal (only the +-1 couplings fall
// inside it); it is factored once per system without pivoting (Thomas,
// l_j = a_(j,j-1) / u_(j-1), u_j = a_jj - l_j a_(j-1,j); a zero or non-finite
// pivot makes the block the identity) into thread-private SMEM, and every
// application is a forward and a back substitution in registers.
// NXG > NX: a generic-width instance (NX = width mod 8, A = P.line_a = width
// / 8, any width <= NXG; see line3_spmv).
template <int NX, int ROUNDS = 2, int PRE = 0, int NXG = NX>
__global__ void __launch_bounds__(128, 3) bicgstab_line3_kernel(const SolveParams P) {
  using G3 = Line3Geom<NXG, PRE>;
  constexpr int R = G3::R, NT = G3::NT;
  using L = typename G3::L;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sg = reinterpret_cast<double *>(smem_raw);
  double *sred = sg + G3::OFF_RED;
  double2 *sx2 = reinterpret_cast<double2 *>(sg + G3::OFF_X) + threadIdx.x;  // x pair k at [k*NT]
  double *sf = sg + G3::OFF_F + threadIdx.x;  // block-Jacobi factor k at sf[k * NT]
  uint32_t *tbase_s = reinterpret_cast<uint32_t *>(sg + G3::OFF_F + G3::NF * NT);

  const int tid = threadIdx.x, warp = tid >> 5;
  const int n = P.n;
  const long long sys = blockIdx.x;
  const int row0 = R * tid;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s)),
                 "n"(128));
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s + 1)),
                 "n"(32));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  for (int i = tid; i < R * (L::S - NT); i += NT) {  // zero guard columns
    const int pl = i / (L::S - NT), q = i % (L::S - NT);
    sg[pl * L::S + (q < L::GQ ? q : q + NT)] = 0.0;
  }
  if (tid == 0 && P.pf_ahead > 0 && sys + P.pf_ahead < P.batch) {  // L2 prefetch, as line kernel
    const long long ns = sys + P.pf_ahead;
    const void *va = P.values + ns * P.sys_stride;
    const void *ba = P.b + ns * n;
    if (((reinterpret_cast<uintptr_t>(va) | reinterpret_cast<uintptr_t>(ba)) & 15u) == 0) {
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(va),
                   "r"(static_cast<uint32_t>(P.sys_stride * 8) & ~15u)
                   : "memory");
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(ba),
                   "r"(static_cast<uint32_t>(n * 8) & ~15u)
                   : "memory");
      const void *xa = P.x0 ? P.x0 + ns * n : nullptr;
      if (xa && (reinterpret_cast<uintptr_t>(xa) & 15u) == 0)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(xa),
                     "r"(static_cast<uint32_t>(n * 8) & ~15u)
                     : "memory");
    }
  }
  bool act[R];
#pragma unroll
  for (int j = 0; j < R; ++j) act[j] = row0 + j < n;
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t lane_hi = static_cast<uint32_t>(32 * warp) << 16;
  const uint32_t tval = tbase_s[0] + lane_hi;  // 8 rows x 16 columns of values
  const uint32_t trh = tbase_s[1] + lane_hi;   // r^ (8 doubles)
  const uint32_t ta0 = trh + 16;               // a_jj (8 doubles)

  LineComm<NXG, NT, R> comm(sg, sred, act);
  line3_solve<NX, ROUNDS, PRE, LineComm<NXG, NT, R>, NXG>(P, sys, 0, tid == 0, act, comm, sf, sx2,
                                                          tval, trh, ta0,
                                                          NXG == NX ? 0 : P.line_a);
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase_s[1]), "n"(32));
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase_s[0]), "n"(128));
  }
}

// ------------------------------------------------ the 3-CTA plan on a cluster --
// Systems larger than one CTA (n > 1024, e.g. the 63 x 64 grid, n = 4032:
// SURVEY.md 8(f) f2, BASELINE configs[4]) on a cluster of C CTAs of 1024
// consecutive rows each, every CTA running line3_solve on its rows.  The
// exchange is BARRIER-based: publishing row li also stores it (st.shared::
// cluster) into the left neighbour's right guard (li < NX + 1) or the right
// neighbour's left guard (li >= nloc - NX - 1); sync() is a cluster barrier
// (arrive.release / wait.acquire), after which every CTA's SpMV reads only
// its own planes.  Reductions push each warp's partial into every CTA's
// scratch and pass one cluster barrier.  WAR safety: a CTA rewrites its
// planes (and its neighbours' guards) only after a reduction barrier that
// every CTA reaches after its previous SpMV; reduction scratch alternates
// between two halves.  No mbarrier, no transaction counting: racecheck
// models these barriers.
__device__ __forceinline__ void st_cluster_f64(uint32_t addr, double v) {
  asm volatile("st.shared::cluster.f64 [%0], %1;" ::"r"(addr), "d"(v) : "memory");
}
// Bulk copy of `bytes` (multiple of 16, 16-byte aligned) from this CTA's
// shared memory to a peer's (shared::cluster address), completing the bytes on
// the peer's mbarrier.
__device__ __forceinline__ void bulk_s2c(uint32_t dst, uint32_t src, uint32_t bytes, uint32_t rbar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(dst), "r"(src), "r"(bytes), "r"(rbar)
      : "memory");
}
__device__ __forceinline__ void cluster_barrier() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}

// MB = 1 (default): point-to-point transaction barriers instead of cluster
// barriers -- halo rows and reduction partials travel by st.async, each
// completing 8 bytes on the RECEIVER's mbarrier; the receiver's thread 0 arms
// the expected byte count, everyone waits with acquire.cluster semantics.  No
// cluster-wide barrier (and no membar) per exchange.  Ordering (the same
// transitive argument as DESIGN.md Kernels 8): a neighbour pushes the next
// halo into my guards only after a reduction that needs my partial, which I
// push after my SpMV read those guards; racecheck does not model that chain,
// so MB = 0 (BSOLVE_CLUSTER_SYNC=barrier) is kept as the checkable reference.
template <int NX, int C, int MB, int H2 = 0>
struct Line3ClusterComm {
  static constexpr int R = 8, NT = 128, NWARP = 4, RPC = R * NT, G = NX + 1;
  // H2 = 1 (MB = 1 only; DESIGN.md Kernels 14): two exchanges per iteration
  // instead of four.  The p^ and s^ halos are not sent: every CTA keeps the
  // state (d, p, r|s, v, t) of its neighbours' G boundary rows next to its
  // guards and updates it with the owner's expressions (the same source
  // expressions, so the same contraction into the same fma sequence: the
  // guard values are the owner's bits -- checked bitwise against the
  // exchanging variants by the tests); the owner's new v and t for those rows
  // ride along with the two reductions that follow the SpMVs.
  static constexpr bool kHalo2 = H2 != 0;
  static constexpr int HS = 66;  // halo state: [side][field][HS], sides L = 0, R = 1
  static_assert(G <= HS && (HS * 8) % 16 == 0, "halo state rows: bulk-copy granules");
  // r and d adjacent: the pair pushed together is one bulk copy
  enum { F_R = 0, F_D = 1, F_P = 2, F_V0 = 3, F_V1 = 4, F_T = 5, NF = 6 };
  static constexpr int NP = C * NWARP;  // partials per reduced value
  using L = LineGeom<NX, NT, R>;
  double *gq;    // sg + GQ + threadIdx.x
  double *sred;  // scratch [2][8][NWARP + C]: warp partials, CTA partials
  // this thread's rows j < nleft go to the left neighbour's right guard, rows
  // j >= rfirst to the right neighbour's left guard: row j of thread t sits
  // in plane j, column GQ + t + 128 (left) or GQ + t - 128 (right) there
  uint32_t lbase = 0, rbase = 0, sred_s;
  int nleft = 0, rfirst = R, buf = 0, rank;
  // MB = 1: [0] halo, [1], [2] reduction halves; the neighbours' halo barriers
  uint64_t *bars;
  uint32_t lhbar = 0, rhbar = 0, phases = 0;  // phases: bit 0/1 reduction halves, bit 2 halo
  uint32_t lseg = 0, rseg = 0;  // MB = 1: bulk-copy destinations (plane 0) in the neighbours
  int n;
  double *hst = nullptr;        // H2: halo state (this CTA's copy of the neighbours' rows)
  double *stg = nullptr;        // H2: outgoing boundary rows [2 halves][2 sides][2 * HS]
  int vk = 0;                   // H2: v exchanges so far (v is double-buffered by parity)
  __device__ __forceinline__ Line3ClusterComm(double *sg, double *sred_, uint64_t *bars_, int rank_,
                                              int n_, double *hst_ = nullptr)
      : gq(sg + L::GQ + threadIdx.x), sred(sred_), rank(rank_), bars(bars_), n(n_), hst(hst_),
        stg(hst_ ? hst_ + 2 * NF * HS : nullptr) {
    const uint32_t sg_s = smem_addr(sg);
    const int t = threadIdx.x;
    const uint32_t bars_s = smem_addr(bars);
    if (MB) {  // halo by bulk copies, issued by threads 0..7 (left) and 32..39 (right)
      if (rank > 0 && t < 8) {
        lseg = mapa_u32(sg_s, rank - 1) + 8u * static_cast<uint32_t>(L::GQ + NT);
        lhbar = mapa_u32(bars_s, rank - 1);
      }
      static_assert(L::GQ >= 10 && NX + 1 <= 80, "halo segments: 10 columns cover the reach");
      if (rank < C - 1 && t >= 32 && t < 40) {
        rseg = mapa_u32(sg_s, rank + 1) + 8u * static_cast<uint32_t>(L::GQ - 10);
        rhbar = mapa_u32(bars_s, rank + 1);
      }
    } else {
      if (rank > 0 && R * t < G) {
        lbase = mapa_u32(sg_s, rank - 1) + 8u * static_cast<uint32_t>(L::GQ + t + NT);
        nleft = min(R, G - R * t);
      }
      if (rank < C - 1 && R * t + R > RPC - G) {  // (only the last CTA has nloc < RPC)
        rbase = mapa_u32(sg_s, rank + 1) + 8u * static_cast<uint32_t>(L::GQ + t - NT);
        rfirst = max(0, RPC - G - R * t);
      }
    }
    sred_s = smem_addr(sred);
    if (H2) init_push();
  }
  // halo bytes this CTA receives: G rows from each neighbour (the right
  // neighbour's first G rows; the left neighbour's last G rows)
  __device__ __forceinline__ uint32_t halo_bytes() const {  // 8 segments per neighbour
    return 8u * SEG * static_cast<uint32_t>((rank > 0 ? 1 : 0) + (rank < C - 1 ? 1 : 0));
  }
  __device__ __forceinline__ void push(uint32_t addr, double v, uint32_t rbar) {
    st_async_f64(addr, v, rbar);
  }
  // MB = 0 stores through generic pointers to the peer's shared memory
  // (cooperative_groups map_shared_rank), the form compute-sanitizer tracks
  __device__ __forceinline__ static double *peer(double *local, int r) {
    return cooperative_groups::this_cluster().map_shared_rank(local, r);
  }
  __device__ __forceinline__ void publish(int j, double v) {
    gq[j * L::S] = v;
    if (MB) {
      // (the halo leaves in sync(), by bulk copies)
    } else {
      if (j < nleft) peer(gq, rank - 1)[NT + j * L::S] = v;
      if (j >= rfirst) peer(gq, rank + 1)[j * L::S - NT] = v;
    }
  }
  // MB = 1: one 80-byte bulk copy per plane and side moves the halo: my rows
  // 0..64 (plane j, columns GQ..GQ+9) into the left neighbour's right guard
  // (columns GQ+128..), my rows 959..1023 (columns GQ+118..GQ+127) into the
  // right neighbour's left guard (columns 0..9); the extra rows copied are
  // never read (the stencil reaches 65 rows).  S and GQ are even, so every
  // segment is 16-byte aligned.
  static constexpr uint32_t SEG = 80;
  __device__ __forceinline__ void sync() {
    if (MB) {
      fence_proxy_async_smem();  // my plane stores before the async-proxy copies read them
      if (threadIdx.x == 0) mbar_arrive_expect_tx(bars, halo_bytes());
      __syncthreads();
      const int t = threadIdx.x;
      if (t < 8 && rank > 0) {  // thread t copies plane t to the left
        const uint32_t src = smem_addr(gq - t) + 8u * static_cast<uint32_t>(t * L::S);
        bulk_s2c(lseg + 8u * static_cast<uint32_t>(t * L::S), src, SEG, lhbar);
      } else if (t >= 32 && t < 40 && rank < C - 1) {  // thread 32 + j: plane j to the right
        const int j = t - 32;
        const uint32_t src = smem_addr(gq - t) + 8u * static_cast<uint32_t>(j * L::S + NT - 10);
        bulk_s2c(rseg + 8u * static_cast<uint32_t>(j * L::S), src, SEG, rhbar);
      }
      // only the warps whose gathers reach a guard wait for the halo (threads
      // t <= 8 and t >= 119 with the stencil reach G = NX + 1 <= 72); the
      // middle warps start their SpMV while the copies are in flight
      const int w = threadIdx.x >> 5;
      if (w == 0 || w == NWARP - 1) mbar_wait_parity_cluster(bars, (phases >> 2) & 1u);
      phases ^= 4u;
    } else {
      cooperative_groups::this_cluster().sync();
    }
  }
  // before a publish that follows no exchange: the CTA's own readers only
  // (every peer's earlier SpMV is ordered by the last reduction)
  __device__ __forceinline__ void barrier() {
    if (MB) __syncthreads();
    else cooperative_groups::this_cluster().sync();
  }
  template <int K>
  __device__ __forceinline__ void sum(double (&v)[K]) {
    const double none[R] = {0, 0, 0, 0, 0, 0, 0, 0};
    sum_x<K>(v, none, 0, none);
  }
  __device__ __forceinline__ int nloc() const { return min(RPC, n - rank * RPC); }
  // H2: the rows this thread owns that a neighbour keeps as halo state (the
  // first G rows for the left neighbour, the last G for the right one; nleft /
  // rfirst, set by init_push) are staged in stg and leave as ONE bulk copy per
  // side and exchange (thread 32: left, thread 64: right) into the
  // neighbour's state field, completing on its reduction barrier.  The
  // staging is double-buffered by reduction half: half h is rewritten two
  // exchanges later, after a reduction that needed the neighbour's partial,
  // which it pushed only after its wait for this copy returned.
  uint32_t hl = 0, hr = 0, hlb = 0, hrb = 0;  // remote state sides / barriers (threads 32, 64)
  int roff = 0;                               // staging index of this thread's row 0 (right side)
  __device__ __forceinline__ void init_push() {
    const int t = threadIdx.x, nl = nloc();
    if (rank > 0 && R * t < G) nleft = min(R, G - R * t);
    if (rank < C - 1 && R * t + R > nl - G && R * t < nl) {
      rfirst = max(0, nl - G - R * t);
      roff = R * t - (nl - G);
    }
    if (t == 32 && rank > 0) {
      hl = mapa_u32(smem_addr(hst + HS * NF), rank - 1);
      hlb = mapa_u32(smem_addr(bars + 1), rank - 1);
    }
    if (t == 64 && rank < C - 1) {
      hr = mapa_u32(smem_addr(hst), rank + 1);
      hrb = mapa_u32(smem_addr(bars + 1), rank + 1);
    }
  }
  __device__ __forceinline__ void stage_rows(const double (&a)[R], int slot) {
    double *sl = stg + buf * (4 * HS) + slot * HS;
    double *sr = sl + 2 * HS;
#pragma unroll
    for (int j = 0; j < R; ++j) {
      if (j < nleft) sl[R * threadIdx.x + j] = a[j];
      if (j >= rfirst) sr[roff + j] = a[j];
    }
  }
  __device__ __forceinline__ void send_rows(int f, int nfield) {
    const uint32_t bytes = static_cast<uint32_t>(8 * HS * nfield);
    const uint32_t fo = 8u * static_cast<uint32_t>(f * HS), bo = 8u * static_cast<uint32_t>(buf);
    if (hl) bulk_s2c(hl + fo, smem_addr(stg + buf * (4 * HS)), bytes, hlb + bo);
    if (hr) bulk_s2c(hr + fo, smem_addr(stg + buf * (4 * HS) + 2 * HS), bytes, hrb + bo);
  }
  // Cluster-wide sum of K values in two stages (every exchange variant uses
  // the same order, so all give the same bits): warp butterflies, the 4 warp
  // partials of the CTA added by lane q of warp 0 (value q), that CTA partial
  // pushed to every CTA, then the C CTA partials added in rank order.
  // what: 0 nothing, 1 v, 4 t, 2 r and d (xb), 3 r (restart): the boundary
  // rows pushed with the reduction (H2)
  template <int K>
  __device__ __forceinline__ void sum_x(double (&v)[K], const double (&xa)[R], int what,
                                        const double (&xb)[R]) {
    static_assert(K >= 1 && K <= 8, "cluster sum supports 1..8 values");
    uint32_t hbytes = 0;
    int hf = 0;
    if (H2 && what) {
      const int nb = (rank > 0 ? 1 : 0) + (rank < C - 1 ? 1 : 0);
      hbytes = static_cast<uint32_t>(8 * HS * nb * (what == 2 ? 2 : 1));
      hf = what == 1 ? ((vk & 1) ? F_V1 : F_V0) : what == 4 ? F_T : F_R;
      if (nleft || rfirst < R) {
        stage_rows(xa, 0);
        if (what == 2) stage_rows(xb, 1);  // d right after r (F_D = F_R + 1)
        fence_proxy_async_smem();          // staged rows before the async-proxy copy reads them
      }
      if (what == 1) ++vk;
    }
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int KP = K <= 1 ? 1 : K <= 2 ? 2 : K <= 4 ? 4 : 8;
    constexpr int SPAN = 32 / KP;
    double a[KP];
#pragma unroll
    for (int i = 0; i < KP; ++i) a[i] = i < K ? v[i] : 0.0;
#pragma unroll
    for (int cnt = KP, o = 16; cnt > 1; cnt >>= 1, o >>= 1) {  // recursive halving
      const bool hi = lane & o;
#pragma unroll
      for (int i = 0; i < cnt / 2; ++i) {
        const double send = hi ? a[i] : a[i + cnt / 2];
        const double keep = hi ? a[i + cnt / 2] : a[i];
        a[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
      }
    }
#pragma unroll
    for (int o = SPAN / 2; o > 0; o >>= 1) a[0] += __shfl_xor_sync(0xffffffffu, a[0], o);
    double *Wb = sred + buf * (8 * (NWARP + C));  // [8][NWARP] warp partials
    double *Sb = Wb + 8 * NWARP;                  // [8][C] CTA partials (pushed by peers)
    const int q = lane / SPAN;
    if ((lane % SPAN) == 0 && q < K) Wb[q * NWARP + warp] = a[0];
    if (MB && threadIdx.x == 0)
      mbar_arrive_expect_tx(bars + 1 + buf, static_cast<uint32_t>(K * C * 8) + hbytes);
    __syncthreads();
    if (H2 && what) send_rows(hf, what == 2 ? 2 : 1);
    if (threadIdx.x < K) {  // lane k of warp 0: the CTA partial of value k, to every CTA
      const double2 w01 = reinterpret_cast<const double2 *>(Wb + threadIdx.x * NWARP)[0];
      const double2 w23 = reinterpret_cast<const double2 *>(Wb + threadIdx.x * NWARP)[1];
      const double cp = (w01.x + w01.y) + (w23.x + w23.y);
      const uint32_t off = static_cast<uint32_t>((Sb - sred + threadIdx.x * C + rank) * 8);
#pragma unroll
      for (int r = 0; r < C; ++r) {
        if (MB) push(mapa_u32(sred_s + off, r), cp, mapa_u32(smem_addr(bars + 1 + buf), r));
        else peer(sred, r)[off / 8] = cp;
      }
    }
    if (MB) {
      const uint32_t bit = 1u << buf;
      mbar_wait_parity_cluster(bars + 1 + buf, (phases & bit) ? 1u : 0u);
      phases ^= bit;
    } else {
      cooperative_groups::this_cluster().sync();
    }
#pragma unroll
    for (int k = 0; k < K; ++k) {
      double part[C];
#pragma unroll
      for (int r = 0; r < C; ++r) part[r] = Sb[k * C + r];
      v[k] = tree_sum<C>(part);
    }
    buf ^= 1;
  }
  // ---- H2 halo state updates (threads t < G, one row per side each) --------
  // guard slot of halo row i of side s in this CTA's planes
  __device__ __forceinline__ double *guard(int side, int i) const {
    const int x = side == 0 ? i - G : nloc() + i;  // local row index (< 0 or >= nloc)
    const int q = x >= 0 ? x / R : -((-x + R - 1) / R);
    return gq - threadIdx.x + (x - R * q) * L::S + q;
  }
  __device__ __forceinline__ bool side_ok(int side) const {
    return side == 0 ? rank > 0 : rank < C - 1;
  }
  __device__ __forceinline__ double &hv(int side, int f, int i) const {
    return hst[side * (HS * NF) + f * HS + i];
  }
  __device__ __forceinline__ void halo_p(double beta, double omega) {  // p = r + beta (p - omega v)
    const int i = threadIdx.x;
    if (!H2 || i >= G) return;
    const int fv = ((vk - 1) & 1) ? F_V1 : F_V0;
#pragma unroll
    for (int sd = 0; sd < 2; ++sd)
      if (side_ok(sd)) {
        const double pn = hv(sd, F_R, i) + beta * (hv(sd, F_P, i) - omega * hv(sd, fv, i));
        hv(sd, F_P, i) = pn;
        *guard(sd, i) = hv(sd, F_D, i) * pn;
      }
  }
  __device__ __forceinline__ void halo_s(double alpha) {  // s = r - alpha v
    const int i = threadIdx.x;
    if (!H2 || i >= G) return;
    const int fv = ((vk - 1) & 1) ? F_V1 : F_V0;
#pragma unroll
    for (int sd = 0; sd < 2; ++sd)
      if (side_ok(sd)) {
        const double sn = hv(sd, F_R, i) - alpha * hv(sd, fv, i);
        hv(sd, F_R, i) = sn;
        *guard(sd, i) = hv(sd, F_D, i) * sn;
      }
  }
  __device__ __forceinline__ void halo_r(double omega) {  // r = s - omega t
    const int i = threadIdx.x;
    if (!H2 || i >= G) return;
#pragma unroll
    for (int sd = 0; sd < 2; ++sd)
      if (side_ok(sd)) hv(sd, F_R, i) = hv(sd, F_R, i) - omega * hv(sd, F_T, i);
  }
  __device__ __forceinline__ void halo_restart() {  // p = v = 0 (r came with the residual)
    const int i = threadIdx.x;
    if (!H2 || i >= G) return;
#pragma unroll
    for (int sd = 0; sd < 2; ++sd) {
      hv(sd, F_P, i) = 0.0;
      hv(sd, F_V0, i) = 0.0;
      hv(sd, F_V1, i) = 0.0;
    }
  }
  __device__ __forceinline__ void sync_local() { __syncthreads(); }
};

template <int NX, int C, int PRE = 0>
struct Line3ClusterGeom {
  using G3 = Line3Geom<NX, 0>;
  static constexpr int R = 8, NT = 128;
  static constexpr int OFF_RED = G3::OFF_RED;                         // [2][8][C*4]
  static constexpr int OFF_X = (OFF_RED + 2 * 8 * (4 + C) + 1) & ~1;  // scratch [2][8][4 + C]
  static constexpr int OFF_HS = OFF_X + R * NT;  // halo state [2][6][66], staging [2][2][2][66] (H2)
  static constexpr int OFF_F = OFF_HS + 2 * 6 * 66 + 8 * 66;  // PRE = 1: block-Jacobi factors [22][NT]
  static constexpr int OFF_BAR = OFF_F + (PRE ? 22 * NT : 0);  // 3 mbarriers (MB = 1)
  static constexpr int SMEM_BYTES = (OFF_BAR + 3) * 8 + 16;
};

// One system per cluster of C CTAs x 1024 rows (blockIdx.x / C = system).
// PRE = 1: block-Jacobi (R30) with the thread's 8 rows as its block, as in the
// single-CTA kernel; the guards then hold p^ = M^-1 p and s^ = M^-1 s, which
// a neighbour cannot recompute from the row state alone, so PRE = 1 runs the
// halo exchange (H2 = 0).
template <int NX, int C, int MB = 1, int H2 = 1, int ROUNDS = 2, int PRE = 0>
__global__ void __launch_bounds__(128, 3) bicgstab_line3_cluster_kernel(const SolveParams P) {
  static_assert(!(PRE && H2), "block-Jacobi guards are exchanged, not recomputed");
  using CG = Line3ClusterGeom<NX, C, PRE>;
  constexpr int R = 8, NT = 128;
  using L = LineGeom<NX, NT, R>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sg = reinterpret_cast<double *>(smem_raw);
  double *sred = sg + CG::OFF_RED;
  double2 *sx2 = reinterpret_cast<double2 *>(sg + CG::OFF_X) + threadIdx.x;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sg + CG::OFF_BAR);
  double *hst = sg + CG::OFF_HS;
  uint32_t *tbase_s = reinterpret_cast<uint32_t *>(sg + CG::OFF_BAR + 3);
  uint32_t crank;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(crank));
  const int rank = static_cast<int>(crank);
  const int tid = threadIdx.x, warp = tid >> 5;
  const int n = P.n;
  const long long sys = blockIdx.x / C;
  const int grow0 = rank * 1024;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s)),
                 "n"(128));
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s + 1)),
                 "n"(32));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  for (int i = tid; i < R * (L::S - NT); i += NT) {  // guards: global edges stay 0
    const int pl = i / (L::S - NT), q = i % (L::S - NT);
    sg[pl * L::S + (q < L::GQ ? q : q + NT)] = 0.0;
  }
  if (H2)
    for (int i = tid; i < 2 * 6 * 66 + 8 * 66; i += NT) hst[i] = 0.0;  // state + staging
  if (rank == 0 && tid == 0 && P.pf_ahead > 0 && sys + P.pf_ahead < P.batch) {
    const long long ns = sys + P.pf_ahead;
    const void *va = P.values + ns * P.sys_stride;
    const void *ba = P.b + ns * n;
    if (((reinterpret_cast<uintptr_t>(va) | reinterpret_cast<uintptr_t>(ba)) & 15u) == 0) {
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(va),
                   "r"(static_cast<uint32_t>(P.sys_stride * 8) & ~15u)
                   : "memory");
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(ba),
                   "r"(static_cast<uint32_t>(n * 8) & ~15u)
                   : "memory");
    }
  }
  if (MB && tid == 32) {
    for (int i = 0; i < 3; ++i) mbar_init(bars + i, 1);
    fence_mbar_init();
  }
  bool act[R];
#pragma unroll
  for (int j = 0; j < R; ++j) act[j] = grow0 + R * tid + j < n;
  asm volatile("tcgen05.fence::before_thread_sync;");
  // TMEM addresses published; every CTA's guards zeroed and mbarriers
  // initialised before any peer pushes into them
  cluster_barrier();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t lane_hi = static_cast<uint32_t>(32 * warp) << 16;
  const uint32_t tval = tbase_s[0] + lane_hi;
  const uint32_t trh = tbase_s[1] + lane_hi;
  const uint32_t ta0 = trh + 16;
  Line3ClusterComm<NX, C, MB, H2> comm(sg, sred, bars, rank, n, hst);
  line3_solve<NX, ROUNDS, PRE>(P, sys, grow0, rank == 0 && tid == 0, act, comm,
                               PRE ? sg + CG::OFF_F + tid : nullptr, sx2, tval, trh, ta0);
  asm volatile("tcgen05.fence::before_thread_sync;");
  // no CTA leaves while a peer may still store into its SMEM.  MB = 1: the
  // last exchange is a reduction whose pushes into this CTA all completed on
  // its barrier before the wait above returned -- a CTA barrier suffices
  if (MB) __syncthreads();
  else cluster_barrier();
  if (warp == 0) {
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase_s[1]), "n"(32));
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tbase_s[0]), "n"(128));
  }
}

}  // namespace bsolve
