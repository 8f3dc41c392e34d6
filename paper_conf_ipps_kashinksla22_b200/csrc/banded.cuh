// banded.cuh -- sm_100a batched banded LU with partial pivoting + solve
// (the GPU analogue of LAPACK dgbsv, the paper's CPU
// solver for the XGC collision systems, PAPER.md:97-99 [I], 556-559 [III],
// 915-925 [V-A]; the direct comparator next to Algorithm 1).
//
// What one CTA computes for one system (persistent grid, systems strided by
// gridDim.x): the factorisation P A = L U of LAPACK dgbtf2 (for j = 0..n-1:
// pivot = first row of max |a_kj| among rows j..j+kl, swap rows, eliminate
// the kl rows below with multipliers a_kj / a_jj), the forward substitution
// of dgbtrs applied to b as an extra column during the factorisation (same
// operations, same order), and the back substitution with U in the column
// order of dgbtrs (x_j = y_j / u_jj, then y_i -= u_ij x_j for i < j).
//
// B200 design:
//  * the active window of the band -- rows j..j+KL, columns j..j+KL+KU -- is
//    held in REGISTERS: thread t owns every column c = t (mod W) in turn, one
//    double per window row, v[k] = row j+k.  The elimination update writes
//    row j+k into v[k-1], so the window slides by one row per step through
//    the FMA destinations: every register index is static (no local memory)
//    and the step loop stays rolled (small code: the instruction cache holds
//    it, which an unrolled-by-(KL+1) loop of ~50k instructions did not).
//  * thread W owns the right-hand side as one more column.
//  * per step the pivot column's thread finds the pivot (first index of the
//    largest |a_kj|: a cheap "is the diagonal the maximum" test, then a tree
//    argmax only when it is not), publishes the pivot row index, 1/pivot and the column to
//    SMEM (double-buffered, ONE __syncthreads per step); every thread then
//    swaps (warp-uniform branch, rare) and applies
//        a_kc -= a_kj * (u_jc / u_jj)                            k = 1..KL
//    i.e. the multiplier l_kj = a_kj / u_jj of dgbtf2 is folded into the
//    column thread's scalar (one DMUL per column instead of KL per step).
//  * rows enter the window KL+1 steps before they are pivot candidates: idle
//    "loader" lanes cp.async the next rows' pattern entries (values in the
//    handle's CSR or ELL layout, b) into a zeroed SMEM row ring D steps ahead.
//  * U (row j: 1/u_jj, u_j,j+1 .. u_j,j+W-1; coalesced stores) and y go to a
//    per-CTA global workspace (HBM/L2).  The back substitution runs in ONE
//    warp: lane l keeps the accumulators of the rows = l (mod 32) still in
//    the band and x_j travels by shuffle (no CTA barrier per step).
#pragma once
#include <cstdint>
#include <type_traits>
#include <cuda_runtime.h>

#ifndef BBAND_LDS64
#define BBAND_LDS64 0  // 1: 8-byte multiplier loads (same SMEM wavefronts, measured 0.895 vs 0.903)
#endif

namespace bband {

struct BandParams {
  const double *values;   // [batch][sys_stride] in the handle's CSR or ELL layout
  const double *b;        // [batch][n]
  const int32_t *bnd;     // [E][n]: (value index << 8) | (col mod W), -1 = none
  double *x;              // [batch][n] out
  int32_t *info;          // [batch] out or nullptr: 0, or j+1 if u_jj == 0 (LAPACK)
  int32_t *ipiv;          // [batch][n] out or nullptr: row swapped with row j (0-based)
  const int32_t *cols;    // [E][n] column of entry e of row r (residual in fallback mode)
  int8_t *only;           // fallback mode: [batch] status of the iterative solve; systems
                          // with 0 (converged) are skipped, the others get x = the direct
                          // solution, resnorm = its true residual, only[i] = 3 (DIRECT);
                          // a singular band (info > 0) leaves x, resnorm and status as
                          // they were.  nullptr: solve every system.
  double *resnorm;        // fallback mode: [batch] out
  double *ws;             // per CTA: U [n][W] (row j: 1/u_jj, u_j,j+1 ..) then y [n]
  const int32_t *list;    // fallback mode: indices of the systems to solve (compacted
                          // on the device by fallback_compact_kernel), nullptr: all
  const int32_t *list_len;  // device: number of entries in `list`
  long long sys_stride;
  int E, n, batch;
};

__device__ __forceinline__ uint32_t saddr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void cp_async8(void *dst, const void *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"(saddr(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// Window geometry of a kernel instance.
template <int KL, int KU>
struct Geo {
  static constexpr int R = KL + 1;            // window rows = register slots per column
  static constexpr int W = KL + KU + 1;       // window columns (U row length)
  static constexpr int NTF = ((W + 2 + 31) / 32) * 32;  // factor warps: + RHS thread + >= 1 loader
  static constexpr int NT = NTF + 32;                    // + the back-substitution warp
  static constexpr int D = R - 2 < 4 ? R - 2 : 4;      // row prefetch distance (steps)
  static constexpr int RB = W + 2;            // row ring stride: W columns, b, a dummy slot
  static constexpr int smem_bytes = R * RB * 8;
  static_assert(D >= 1, "KL must be >= 2");
};

// Loader lane e (< E: pattern entry e of the row; == E: b) issues the cp.async
// that brings row rr into ring slot `slot`: the entry of column c goes to
// position c mod W (precomputed in pk's low byte), b to position W.
// pk = P.bnd[e][rr], loaded one step ahead.
template <int KL, int KU>
__device__ __forceinline__ void load_entry(const BandParams &P, const double *val, const double *bb,
                                           double *ring, int slot, int rr, int e, int pk) {
  using G = Geo<KL, KU>;
  if (rr >= P.n || e > P.E) return;
  double *row = ring + slot * G::RB;
  if (e == P.E) cp_async8(row + G::W, bb + rr);
  else if (pk >= 0) cp_async8(row + (pk & 255), val + (pk >> 8));
}
__device__ __forceinline__ int load_pk(const BandParams &P, int rr, int e) {
  return (rr < P.n && e < P.E) ? __ldg(P.bnd + (size_t)e * P.n + rr) : -1;
}

// First index of the largest |a_k|, k = 0..N-1 (dgbtf2's IDAMAX): a tree
// that keeps the left operand unless the right one is strictly larger.
__device__ __forceinline__ void bar_factor(int nthreads) {  // named barrier 1: factor warps only
  asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");
}
__device__ __forceinline__ void mbar_init1(uint64_t *bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive1(uint64_t *bar) {
  asm volatile("{\n.reg .b64 st;\nmbarrier.arrive.release.cta.shared::cta.b64 st, [%0];\n}" ::"r"(
                   saddr(bar))
               : "memory");
}
// try_wait with a suspend-time hint: the back-substitution warp waits most
// of the time (the factorisation is the long pole); the hint lets the
// hardware park the warp until the phase flips instead of spinning on issue
// slots the factor warps need (a __nanosleep back-off still woke ~20 times
// per elimination step)
__device__ __forceinline__ void mbar_wait_sleep(uint64_t *bar, uint32_t parity) {
  uint32_t ok;
  do {
    asm volatile(
        "{\n.reg .pred p;\nmbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2, %3;\n"
        "selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(saddr(bar)), "r"(parity), "r"(1000000u)
        : "memory");
  } while (!ok);
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred p;\nW%=:\n"
      "mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra W%=;\n}" ::"r"(saddr(bar)),
      "r"(parity)
      : "memory");
}

template <int N>
__device__ __forceinline__ int argmax_abs(const double (&a)[N]) {
  double bv[N];
  int bi[N];
#pragma unroll
  for (int k = 0; k < N; ++k) {
    bv[k] = a[k];
    bi[k] = k;
  }
#pragma unroll
  for (int s = 1; s < N; s *= 2)
#pragma unroll
    for (int k = 0; k + s < N; k += 2 * s)
      if (fabs(bv[k + s]) > fabs(bv[k])) {
        bv[k] = bv[k + s];
        bi[k] = bi[k + s];
      }
  return bi[0];
}

// Back substitution of one system by one warp (dgbtrs U part, column order):
// lane l holds the accumulators of rows r0 - 32m (m < NA), r0 = the largest
// row <= j with r0 = l (mod 32).  Step j: the owner lane (l = j mod 32) forms
// x_j = y_j * (1/u_jj) and broadcasts it by shuffle; every other row i in
// the band gets y_i -= u_ij x_j.  u_ij is read from the row-major U
// (L1-cached: each lane walks its rows backwards), PF steps ahead.
template <int W>
__device__ __forceinline__ void backsub_system(const BandParams &P, const double *U,
                                               long long sys, int l, bool skip) {
  constexpr int NA = (W + 31) / 32;
  const int n = P.n;
      const double *Y = U + (size_t)n * W;
      constexpr int PF = 8;  // U entries are loaded PF steps ahead
      double a[NA], q[PF][NA];
      const int r0 = (n - 1) - ((n - 1 - l) & 31);
#pragma unroll
      for (int m = 0; m < NA; ++m) a[m] = r0 - 32 * m >= 0 ? Y[r0 - 32 * m] : 0.0;
      double ynext = r0 - 32 * NA >= 0 ? Y[r0 - 32 * NA] : 0.0;
      auto uload = [&](int jj, int m) -> double {  // u_{i,jj}, i = the lane's m-th row at step jj
        const int d = ((jj - l) & 31) + 32 * m;
        const int i = jj - d;
        return (jj >= 0 && i >= 0 && d < W) ? U[(size_t)i * W + d] : 0.0;
      };
#pragma unroll
      for (int s = 0; s < PF; ++s)
#pragma unroll
        for (int m = 0; m < NA; ++m) q[s][m] = uload(n - 1 - s, m);
      double *xs = P.x + sys * n;
#pragma unroll 1
      for (int jb0 = skip ? -1 : n - 1; jb0 >= 0; jb0 -= PF) {
#pragma unroll
        for (int s = 0; s < PF; ++s) {
          const int j = jb0 - s;
          double u[NA];
#pragma unroll
          for (int m = 0; m < NA; ++m) {
            u[m] = q[s][m];
            q[s][m] = uload(j - PF, m);
          }
          if (j >= 0) {  // uniform
            const bool own = l == (j & 31);
            const double xo = a[0] * u[0];  // owner: x_j = y_j / u_jj
            const double x = __shfl_sync(0xffffffffu, xo, j & 31);
            if (own) {
              xs[j] = x;
              u[0] = 0.0;
            }
#pragma unroll
            for (int m = 0; m < NA; ++m) a[m] = fma(-u[m], x, a[m]);
            if (own) {  // row j is done: the lane takes row j - 32 NA
#pragma unroll
              for (int m = 0; m + 1 < NA; ++m) a[m] = a[m + 1];
              a[NA - 1] = ynext;
              const int rn = j - 32 * (NA + 1);
              ynext = rn >= 0 ? Y[rn] : 0.0;
            }
          }
        }
      }
  __syncwarp();
}

// Fallback mode: true residual ||b - A x||_2 of the direct solution, status
// DIRECT (one warp; x re-read from L2).
__device__ __forceinline__ void fallback_residual(const BandParams &P, long long sys, int l) {
  const int n = P.n;
  double *xs = P.x + sys * n;
      {
        // true residual ||b - A x||_2 of the direct solution (plain sum of
        // squares per lane, then a butterfly), x re-read from L2
        const double *val = P.values + sys * P.sys_stride;
        const double *bb = P.b + sys * n;
        double ss = 0.0;
        for (int r = l; r < n; r += 32) {
          double acc = __ldg(bb + r);
          for (int e = 0; e < P.E; ++e) {
            const int pk = __ldg(P.bnd + (size_t)e * n + r);
            if (pk >= 0) acc -= __ldg(val + (pk >> 8)) * __ldcg(xs + __ldg(P.cols + (size_t)e * n + r));
          }
          ss += acc * acc;
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) ss += __shfl_xor_sync(0xffffffffu, ss, o);
        if (l == 0) {
          P.resnorm[sys] = sqrt(ss);
          P.only[sys] = 3;  // BSOLVE_SYS_DIRECT
        }
      }
}

// SPLIT = false: factor warps + the back-substitution warp in one kernel
// (per-CTA double-buffered workspace, mbarrier hand-off).  SPLIT = true: the
// factor warps only (NTF threads: more CTAs per SM); U and y of system i go to
// workspace slot i and banded_backsub_kernel finishes the systems afterwards.
template <int KL, int KU, int MINB, bool SPLIT = false>
__global__ void __launch_bounds__(SPLIT ? Geo<KL, KU>::NTF : Geo<KL, KU>::NT, MINB)
    banded_lu_kernel(const BandParams P) {
  using G = Geo<KL, KU>;
  constexpr int R = G::R, W = G::W, NTF = G::NTF, D = G::D, RB = G::RB;
  extern __shared__ __align__(16) double ring[];  // [R][RB]
  constexpr int RP = (R + 1) & ~1;
  __shared__ __align__(16) double colbuf[2][RP];  // pivot column rows 1..KL (index k-1)
  __shared__ double s_rp[2];
  __shared__ int s_p[2];
  __shared__ int s_info;
  // workspace hand-off factor warps -> back-substitution warp (2 buffers)
  __shared__ __align__(8) uint64_t full_bar[2], empty_bar[2];
  __shared__ int s_info_buf[2];  // info of the system in workspace buffer b

  const int t = threadIdx.x;
  const int n = P.n;
  const size_t ws_sys = (size_t)n * W + n;  // U [n][W] then y [n]
  double *ws = P.ws + (SPLIT ? 0 : (size_t)blockIdx.x * 2 * ws_sys);

  if (!SPLIT && t == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init1(&full_bar[i]);
      mbar_init1(&empty_bar[i]);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (int i = t; i < R * RB; i += (SPLIT ? NTF : G::NT)) ring[i] = 0.0;
  __syncthreads();

  if (!SPLIT && t >= NTF) {
    // ======== back-substitution warp (dgbtrs U part, column order) =========
    // lane l holds the accumulators of rows r0 - 32m (m < NA), r0 = the
    // largest row <= j with r0 = l (mod 32).  Step j: the owner lane
    // (l = j mod 32) forms x_j = y_j * (1/u_jj) and broadcasts it by shuffle;
    // every other row i in the band gets y_i -= u_ij x_j.  u_ij is read from
    // the row-major U (L1-cached: each lane walks its rows backwards).
    const int l = t - NTF;
    int k = 0;
    const long long cnt = P.list ? *P.list_len : P.batch;
    for (long long it = blockIdx.x; it < cnt; it += gridDim.x) {
      const long long sys = P.list ? P.list[it] : it;
      if (P.only && P.only[sys] == 0) continue;  // converged iteratively (same test as below)
      const int b = k & 1;
      mbar_wait_sleep(&full_bar[b], (k >> 1) & 1);
      const bool skip = P.only && s_info_buf[b] != 0;  // singular: keep the iterative result
      backsub_system<W>(P, ws + b * ws_sys, sys, l, skip);
      if (l == 0) mbar_arrive1(&empty_bar[b]);  // buffer b may be overwritten
      if (P.only && !skip) fallback_residual(P, sys, l);
      ++k;
    }
    return;
  }

  // ======== factor warps: dgbtf2 + the L part of dgbtrs on b ================
  const bool owns = t <= W;  // column thread (t < W) or RHS thread (t == W)
  const bool loader = t > W;
  const int lidx = t - W - 1;  // loader lane = pattern entry (needs NTF - W - 1 > E)
  int k = 0;
  const long long cnt = P.list ? *P.list_len : P.batch;
  for (long long it = blockIdx.x; it < cnt; it += gridDim.x) {
    const long long sys = P.list ? P.list[it] : it;
    if (P.only && P.only[sys] == 0) continue;  // converged iteratively
    const int b = k & 1;
    if (!SPLIT && k >= 2) mbar_wait(&empty_bar[b], ((k >> 1) - 1) & 1);  // back subst. k-2 done
    double *U = SPLIT ? ws + (size_t)sys * ws_sys : ws + b * ws_sys;
    double *Y = U + (size_t)n * W;
    const double *val = P.values + sys * P.sys_stride;
    const double *bb = P.b + sys * n;
    if (t == 0) s_info = 0;
    // ---- prologue: rows 0..KL straight into the registers -----------------
    if (loader) {
#pragma unroll 1
      for (int r = 0; r < R; ++r) load_entry<KL, KU>(P, val, bb, ring, r, r, lidx, load_pk(P, r, lidx));
      cp_commit();
      cp_wait<0>();
    }
    bar_factor(NTF);
    double v[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      v[r] = owns ? ring[r * RB + t] : 0.0;
      if (owns) ring[r * RB + t] = 0.0;
    }
    bar_factor(NTF);
    // rows KL+1..KL+D into ring slots 0..D-1, one commit group per row
    int pk = -1;  // loader: pattern entry of the row the next step issues
    if (loader) {
#pragma unroll
      for (int d = 1; d <= D; ++d) {
        load_entry<KL, KU>(P, val, bb, ring, (KL + d) % R, KL + d, lidx, load_pk(P, KL + d, lidx));
        cp_commit();
      }
      pk = load_pk(P, KL + 1 + D, lidx);
    }
    int pos = owns ? (t == W ? W : t) : -1;  // column j + pos (RHS: W; loaders -1)
    const int rcol = owns ? t : W + 1;       // ring column read (loaders: dummy slot)
    int jr = 0;                              // j mod R: ring slot of row j+KL+1
    double *Urow = U;                        // row j of U
    // v[k] holds window row j+k of the thread's column; the update writes row
    // j+k into v[k-1], so the window slides by register renaming
#pragma unroll 1
    for (int j = 0; j < n; ++j) {
      const int jb = j & 1;
      if (pos == 0) {
        // pivot: IDAMAX over rows j..j+KL.  Fast test first: the diagonal is
        // the (first) largest iff |a_jj| >= |a_kj| for all k (ties keep k=0)
        bool diag_max[4] = {true, true, true, true};
#pragma unroll
        for (int kk = 1; kk < R; ++kk)
          diag_max[kk & 3] = diag_max[kk & 3] && (fabs(v[0]) >= fabs(v[kk]));
        int p = 0;
        if (!(diag_max[0] && diag_max[1] && diag_max[2] && diag_max[3])) p = argmax_abs<R>(v);
        double pv = v[0];
        double2 *cbw = reinterpret_cast<double2 *>(colbuf[jb]);
#pragma unroll
        for (int kk = 1; kk < R; kk += 2)
          cbw[(kk - 1) / 2] = make_double2(v[kk], kk + 1 < R ? v[kk + 1] : 0.0);
        if (p != 0) {
          pv = colbuf[jb][p - 1];
          colbuf[jb][p - 1] = v[0];  // row swap in the published column
        }
        const double rp = pv != 0.0 ? __drcp_rn(pv) : 0.0;
        s_p[jb] = p;
        s_rp[jb] = rp;
        Urow[0] = rp;
        if (P.ipiv) P.ipiv[sys * n + j] = j + p;
        if (pv == 0.0 && s_info == 0) s_info = j + 1;
      }
      if (loader) {
        int slot = jr + D;
        if (slot >= R) slot -= R;
        load_entry<KL, KU>(P, val, bb, ring, slot, j + KL + 1 + D, lidx, pk);
        pk = load_pk(P, j + KL + 2 + D, lidx);
        cp_commit();
        cp_wait<D>();
      }
      bar_factor(NTF);
      {  // every factor thread (loader lanes hold zeros and use the dummy slot)
        const int p = s_p[jb];
        const double rp = s_rp[jb];
        if (p != 0) {  // row swap j <-> j+p (uniform branch)
          const double a = v[0];
          double bsel = a;
#pragma unroll
          for (int kk = 1; kk < R; ++kk) bsel = (p == kk) ? v[kk] : bsel;
#pragma unroll
          for (int kk = 1; kk < R; ++kk) v[kk] = (p == kk) ? a : v[kk];
          v[0] = bsel;
        }
        const double uc = v[0];
        // u_jc (c = j + pos) or y_j: one predicated store, no branch
        double *dst = pos == W ? Y + j : Urow + pos;
        if (pos == W || (pos >= 1 && pos < n - j)) *dst = uc;
        // the pivot thread's column equals the published one, so w = 1 turns
        // its registers into exact zeros: it takes column j + W next
        const double w = pos == 0 ? 1.0 : uc * rp;
#if BBAND_LDS64
        // 8-byte broadcast loads of the multipliers: one SMEM wavefront each
        // (a 16-byte broadcast load costs as many wavefronts as a full one)
        const double *cb = colbuf[jb];
#pragma unroll
        for (int kk = 1; kk < R; ++kk) {
          v[kk - 1] = fma(-cb[kk - 1], w, v[kk]);
          if ((kk - 1) % 12 == 11) asm volatile("" ::: "memory");
        }
#else
        const double2 *cb = reinterpret_cast<const double2 *>(colbuf[jb]);
#pragma unroll
        for (int kk = 1; kk < R; kk += 2) {
          const double2 m = cb[(kk - 1) / 2];
          v[kk - 1] = fma(-m.x, w, v[kk]);
          if (kk + 1 < R) v[kk] = fma(-m.y, w, v[kk + 1]);
          // keep at most 6 multiplier pairs in flight (register pressure)
          if ((kk - 1) % 12 == 10) asm volatile("" ::: "memory");
        }
#endif
        // row j leaves; row j+KL+1 (ring slot j mod R) enters as window row KL
        // (loader lanes own no column: they keep zeros and leave the ring alone)
        if (owns) {
          v[KL] = ring[jr * RB + rcol];
          ring[jr * RB + rcol] = 0.0;
        }
        pos = t < W ? (pos == 0 ? W - 1 : pos - 1) : pos;
      }
      jr = (jr + 1 == R) ? 0 : jr + 1;
      Urow += W;
    }
    if (loader) cp_wait<0>();
    bar_factor(NTF);  // every U / y store of this system issued; s_info final
    if (t == 0) {
      if (P.info) P.info[sys] = s_info;
      if (!SPLIT) {
        s_info_buf[b] = s_info;
        __threadfence_block();
        mbar_arrive1(&full_bar[b]);  // release: U, y of buffer b are complete
      }
    }
    ++k;
  }
}

// ---- one warp per system (split mode factorisation) --
// The same dgbtf2 step as banded_lu_kernel, with the W + 1 "virtual column
// threads" vt = 0..W (vt = W: b) folded onto NCL lanes, CPL columns per lane
// (vt = lane + NCL s, s < CPL).  One multiplier load then feeds CPL columns,
// the step needs no CTA barrier (one __syncwarp), and every SMEM broadcast
// reaches one warp instead of ceil((W + 2) / 32): per elimination step of a
// K = 33 system 17 LDS.128 + 17 STS.128 instead of 51 + 17.  The pivot
// column vt = j mod W is warp-uniform, so the lane and slot are known to all;
// its lane runs the IDAMAX test and publishes as before.  Lanes e <= E load
// pattern entry e of the rows entering the ring (E + 1 <= 32).
// (A look-ahead variant -- the next pivot column updated first and its test
// overlapped with the other columns' FMAs -- needs ~20 more registers than
// the 255 this one uses and spilled: 0.73 vs 0.94 M sys/s; DESIGN.md f4 log.)
template <int KL, int KU>
struct WGeo {
  static constexpr int R = KL + 1, W = KL + KU + 1;
  static constexpr int CPL = (W + 1 + 31) / 32;           // columns per lane
  static constexpr int NCL = (W + 1 + CPL - 1) / CPL;     // lanes owning columns
  static constexpr int D = R - 2 < 4 ? R - 2 : 4;         // row prefetch distance
  static constexpr int RB = W + 2;                        // ring stride (+ a dummy slot)
  static constexpr int RP = (R + 1) & ~1;
  static constexpr int OFF_CB = (R * RB + 1) & ~1;        // colbuf [2][RP] (16-byte aligned)
  static constexpr int smem_bytes = (OFF_CB + 2 * RP + 3) * 8;  // + s_p[2], s_rp[2]
  static_assert(NCL <= 32 && D >= 1, "one warp per system");
};

template <int KL, int KU, int MINB>
__global__ void __launch_bounds__(32, MINB) banded_lu_warp_kernel(const BandParams P) {
  using G = WGeo<KL, KU>;
  constexpr int R = G::R, W = G::W, CPL = G::CPL, NCL = G::NCL, D = G::D, RB = G::RB;
  constexpr int RP = G::RP;
  extern __shared__ __align__(16) double wsm[];
  double *ring = wsm;                 // [R][RB]
  double *colbuf = wsm + G::OFF_CB;   // [2][RP]: pivot column rows 1..KL (index k-1)
  int *s_p = reinterpret_cast<int *>(colbuf + 2 * RP);
  double *s_rp = colbuf + 2 * RP + 1;  // [2]
  const int l = threadIdx.x;
  const int n = P.n;
  const size_t ws_sys = (size_t)n * W + n;
  for (int i = l; i < R * RB; i += 32) ring[i] = 0.0;
  __syncwarp();
  int vt[CPL];
#pragma unroll
  for (int s = 0; s < CPL; ++s) vt[s] = l + NCL * s <= W && l < NCL ? l + NCL * s : -1;
  const bool loader = l <= P.E;  // pattern entry l (l == E: b)
  const long long cnt = P.list ? *P.list_len : P.batch;
  for (long long it = blockIdx.x; it < cnt; it += gridDim.x) {
    const long long sys = P.list ? P.list[it] : it;
    if (P.only && P.only[sys] == 0) continue;  // converged iteratively
    double *U = P.ws + (size_t)sys * ws_sys;
    double *Y = U + (size_t)n * W;
    const double *val = P.values + sys * P.sys_stride;
    const double *bb = P.b + sys * n;
    int info = 0;  // this lane's first zero pivot (j + 1)
    // ---- prologue: rows 0..KL straight into the registers -----------------
    if (loader) {
#pragma unroll 1
      for (int r = 0; r < R; ++r) load_entry<KL, KU>(P, val, bb, ring, r, r, l, load_pk(P, r, l));
      cp_commit();
      cp_wait<0>();
    }
    __syncwarp();
    double v[CPL][R];
#pragma unroll
    for (int s = 0; s < CPL; ++s)
#pragma unroll
      for (int r = 0; r < R; ++r) {
        v[s][r] = vt[s] >= 0 ? ring[r * RB + vt[s]] : 0.0;
        if (vt[s] >= 0) ring[r * RB + vt[s]] = 0.0;
      }
    __syncwarp();
    int pk = -1;
    if (loader) {
#pragma unroll
      for (int d = 1; d <= D; ++d) {
        load_entry<KL, KU>(P, val, bb, ring, (KL + d) % R, KL + d, l, load_pk(P, KL + d, l));
        cp_commit();
      }
      pk = load_pk(P, KL + 1 + D, l);
    }
    int pos[CPL];
#pragma unroll
    for (int s = 0; s < CPL; ++s) pos[s] = vt[s];  // column j + pos (b: W; unused: -1)
    int jr = 0;       // j mod R
    int pt = 0;       // pivot virtual thread j mod W
    double *Urow = U;
#pragma unroll 1
    for (int j = 0; j < n; ++j) {
      const int jb = j & 1;
      const int pl = pt % NCL, ps = pt / NCL;  // pivot lane and slot (warp-uniform)
      if (l == pl) {
#pragma unroll
        for (int s = 0; s < CPL; ++s) {
          if (s != ps) continue;
          bool diag_max[4] = {true, true, true, true};
#pragma unroll
          for (int kk = 1; kk < R; ++kk)
            diag_max[kk & 3] = diag_max[kk & 3] && (fabs(v[s][0]) >= fabs(v[s][kk]));
          int p = 0;
          if (!(diag_max[0] && diag_max[1] && diag_max[2] && diag_max[3])) p = argmax_abs<R>(v[s]);
          double pv = v[s][0];
          double2 *cbw = reinterpret_cast<double2 *>(colbuf + jb * RP);
#pragma unroll
          for (int kk = 1; kk < R; kk += 2)
            cbw[(kk - 1) / 2] = make_double2(v[s][kk], kk + 1 < R ? v[s][kk + 1] : 0.0);
          if (p != 0) {
            pv = colbuf[jb * RP + p - 1];
            colbuf[jb * RP + p - 1] = v[s][0];  // row swap in the published column
          }
          const double rp = pv != 0.0 ? __drcp_rn(pv) : 0.0;
          s_p[jb] = p;
          s_rp[jb] = rp;
          Urow[0] = rp;
          if (P.ipiv) P.ipiv[sys * n + j] = j + p;
          if (pv == 0.0 && info == 0) info = j + 1;
        }
      }
      if (loader) {
        int slot = jr + D;
        if (slot >= R) slot -= R;
        load_entry<KL, KU>(P, val, bb, ring, slot, j + KL + 1 + D, l, pk);
        pk = load_pk(P, j + KL + 2 + D, l);
        cp_commit();
        cp_wait<D>();
      }
      __syncwarp();
      const int p = s_p[jb];
      const double rp = s_rp[jb];
      if (p != 0) {  // row swap j <-> j+p (uniform branch)
#pragma unroll
        for (int s = 0; s < CPL; ++s) {
          const double a = v[s][0];
          double bsel = a;
#pragma unroll
          for (int kk = 1; kk < R; ++kk) bsel = (p == kk) ? v[s][kk] : bsel;
#pragma unroll
          for (int kk = 1; kk < R; ++kk) v[s][kk] = (p == kk) ? a : v[s][kk];
          v[s][0] = bsel;
        }
      }
      double w[CPL];
#pragma unroll
      for (int s = 0; s < CPL; ++s) {
        const double uc = v[s][0];
        double *dst = pos[s] == W ? Y + j : Urow + pos[s];
        if (pos[s] == W || (pos[s] >= 1 && pos[s] < n - j)) *dst = uc;
        w[s] = pos[s] == 0 ? 1.0 : uc * rp;  // pivot column: exact zeros
      }
      const double2 *cb = reinterpret_cast<const double2 *>(colbuf + jb * RP);
#pragma unroll
      for (int kk = 1; kk < R; kk += 2) {
        const double2 m = cb[(kk - 1) / 2];
#pragma unroll
        for (int s = 0; s < CPL; ++s) {
          v[s][kk - 1] = fma(-m.x, w[s], v[s][kk]);
          if (kk + 1 < R) v[s][kk] = fma(-m.y, w[s], v[s][kk + 1]);
        }
        if ((kk - 1) % 6 == 4) asm volatile("" ::: "memory");  // <= 3 multiplier pairs in flight
      }
      // row j+KL+1 (ring slot j mod R) enters as window row KL
#pragma unroll
      for (int s = 0; s < CPL; ++s) {
        if (vt[s] >= 0) {
          v[s][KL] = ring[jr * RB + vt[s]];
          ring[jr * RB + vt[s]] = 0.0;
        } else {
          v[s][KL] = 0.0;
        }
        pos[s] = (vt[s] >= 0 && vt[s] < W) ? (pos[s] == 0 ? W - 1 : pos[s] - 1) : pos[s];
      }
      jr = (jr + 1 == R) ? 0 : jr + 1;
      pt = (pt + 1 == W) ? 0 : pt + 1;
      Urow += W;
    }
    if (loader) cp_wait<0>();
    __syncwarp();  // every ring read of this system done before the next prologue
    const unsigned first = __reduce_min_sync(0xffffffffu, info ? static_cast<unsigned>(info) : ~0u);
    if (l == 0 && P.info) P.info[sys] = first == ~0u ? 0 : static_cast<int>(first);
  }
}

// Split mode, second launch: one warp per system, ROW-oriented back
// substitution on the row-major U that the factor kernel wrote with
// coalesced stores:  x_j = (y_j - sum_d u_j,j+d x_j+d) / u_jj, the sum split
// over the lanes (d = l, l+32, l+64 ..) and closed by a butterfly; each step
// reads one contiguous U row (prefetched PF steps ahead).  x is kept in a
// per-warp SMEM array (zero beyond n).  Many warps per SM hide the per-step
// reduction latency; P.info holds the factorisation's info (fallback mode:
// singular systems keep their iterative result).
template <int KL, int KU>
__global__ void __launch_bounds__(128, 6) banded_backsub_kernel(const BandParams P) {
  constexpr int W = Geo<KL, KU>::W;
  constexpr int NA = (W + 31) / 32;
  constexpr int PF = 4;
  extern __shared__ __align__(16) double xsm[];  // [4 warps][n + W]
  const int l = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int n = P.n;
  double *xw = xsm + (size_t)wi * (n + W);
  const size_t ws_sys = (size_t)n * W + n;
  const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long sys = (long long)blockIdx.x * (blockDim.x >> 5) + wi; sys < P.batch; sys += nw) {
    if (P.only && (P.only[sys] == 0 || P.info[sys] != 0)) continue;  // converged / singular
    const double *U = P.ws + (size_t)sys * ws_sys;
    const double *Y = U + (size_t)n * W;
    for (int i = l; i < W; i += 32) xw[n + i] = 0.0;  // x beyond n is zero
    __syncwarp();
    auto uload = [&](int jj, int m) -> double {  // u_jj,jj+d, d = l + 32 m (d = 0: 1/u_jj)
      // entries of columns >= n are never written by the factor kernel (the
      // workspace is not cleared): never read them, x beyond n is zero anyway
      const int d = l + 32 * m;
      return (jj >= 0 && d < W && jj + d < n) ? U[(size_t)jj * W + d] : 0.0;
    };
    double q[PF][NA], yq[PF];
#pragma unroll
    for (int s = 0; s < PF; ++s) {
#pragma unroll
      for (int m = 0; m < NA; ++m) q[s][m] = uload(n - 1 - s, m);
      yq[s] = n - 1 - s >= 0 ? Y[n - 1 - s] : 0.0;
    }
    double *xs = P.x + sys * n;
#pragma unroll 1
    for (int jb0 = n - 1; jb0 >= 0; jb0 -= PF) {
#pragma unroll
      for (int s = 0; s < PF; ++s) {
        const int j = jb0 - s;
        double u[NA];
#pragma unroll
        for (int m = 0; m < NA; ++m) {
          u[m] = q[s][m];
          q[s][m] = uload(j - PF, m);
        }
        const double yj = yq[s];
        yq[s] = j - PF >= 0 ? Y[j - PF] : 0.0;
        if (j >= 0) {  // uniform
          double part = 0.0;
#pragma unroll
          for (int m = 0; m < NA; ++m) {
            const int d = l + 32 * m;
            if (d >= 1 && d < W) part = fma(u[m], xw[j + d], part);
          }
#pragma unroll
          for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
          const double rp = __shfl_sync(0xffffffffu, u[0], 0);  // lane 0 holds d = 0
          const double xj = (yj - part) * rp;
          if (l == 0) {
            xw[j] = xj;
            xs[j] = xj;
          }
          __syncwarp();
        }
      }
    }
    if (P.only) fallback_residual(P, sys, l);
    __syncwarp();
  }
}
// Fallback mode, first launch: list the systems whose iterative status is not
// CONVERGED (their order in the list is irrelevant: every system is solved
// independently, bit for bit the same wherever it lands).  *len must be 0 on
// entry (cudaMemsetAsync on the same stream).
static __global__ void __launch_bounds__(256) fallback_compact_kernel(const int8_t *status, long long batch,
                                                               int32_t *list, int32_t *len) {
  const int lane = threadIdx.x & 31;
  // warp-uniform trip count: the ballot needs all 32 lanes
  for (long long i0 = blockIdx.x * 256LL + (threadIdx.x & ~31); i0 < batch; i0 += gridDim.x * 256LL) {
    const long long i = i0 + lane;
    const bool need = i < batch && status[i] != 0;
    const unsigned m = __ballot_sync(0xffffffffu, need);
    if (m == 0) continue;
    int base = 0;
    if (lane == __ffs(m) - 1) base = atomicAdd(len, __popc(m));
    base = __shfl_sync(0xffffffffu, base, __ffs(m) - 1);
    if (need) list[base + __popc(m & ((1u << lane) - 1))] = static_cast<int32_t>(i);
  }
}
}  // namespace bband
