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
//    double per window row; window row r sits in register slot r mod (KL+1).
//    The step loop is unrolled by KL+1, so every slot index is static (no
//    local memory) while the window slides one row/column per step.
//  * thread W owns the right-hand side as one more column.
//  * per step the pivot column's thread finds the pivot (tree argmax, first
//    index on ties), publishes the pivot row index, 1/pivot and the column to
//    SMEM (double-buffered, ONE __syncthreads per step); every thread then
//    swaps (warp-uniform branch, rare) and applies
//        a_kc -= a_kj * (u_jc / u_jj)                            k = 1..KL
//    i.e. the multiplier l_kj = a_kj / u_jj of dgbtf2 is folded into the
//    column thread's scalar (one DMUL per column instead of KL per step).
//  * rows enter the window KL+1 steps before they are pivot candidates: idle
//    "loader" lanes cp.async the next rows' pattern entries (values in the
//    handle's CSR or ELL layout, b) into a zeroed SMEM row ring D steps ahead.
//  * U (row j: 1/u_jj then u_j,j+1..u_j,j+W-1) and y go to a per-CTA global
//    workspace (HBM/L2) and are streamed back for the back substitution,
//    which keeps one accumulator per thread for the rows j-W+1..j.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bband {

struct BandParams {
  const double *values;   // [batch][sys_stride] in the handle's CSR or ELL layout
  const double *b;        // [batch][n]
  const int32_t *bnd;     // [E][n]: (value index << 8) | (col - row + 128), -1 = none
  double *x;              // [batch][n] out
  int32_t *info;          // [batch] out: 0, or j+1 if u_jj == 0 (LAPACK convention)
  int32_t *ipiv;          // [batch][n] out or nullptr: row swapped with row j (0-based)
  double *ws;             // per CTA: U [n][W] then y [n]
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
  static constexpr int NT = ((W + 2 + 31) / 32) * 32;  // + RHS thread + >= 1 loader
  static constexpr int D = R - 2 < 4 ? R - 2 : 4;      // row prefetch distance (steps)
  static constexpr int RB = W + 1;            // row ring stride (doubles)
  static constexpr int smem_bytes = R * RB * 8;
  static_assert(D >= 1, "KL must be >= 2");
};

// Loader lane e (< E: pattern entry e of the row; == E: b) issues the cp.async
// that brings row rr into ring slot `slot`: the entry of column c goes to
// position c mod W, b to position W.  pk = P.bnd[e][rr], loaded a step ahead.
template <int KL, int KU>
__device__ __forceinline__ void load_entry(const BandParams &P, const double *val, const double *bb,
                                           double *ring, int slot, int rr, int e, int pk) {
  using G = Geo<KL, KU>;
  if (rr >= P.n || e > P.E) return;
  double *row = ring + slot * G::RB;
  if (e == P.E) {
    cp_async8(row + G::W, bb + rr);
  } else if (pk >= 0) {
    const int col = rr + (pk & 255) - 128;
    cp_async8(row + col % G::W, val + (pk >> 8));
  }
}
__device__ __forceinline__ int load_pk(const BandParams &P, int rr, int e) {
  return (rr < P.n && e < P.E) ? __ldg(P.bnd + (size_t)e * P.n + rr) : -1;
}

template <int KL, int KU, int MINB>
__global__ void __launch_bounds__(Geo<KL, KU>::NT, MINB) banded_lu_kernel(const BandParams P) {
  using G = Geo<KL, KU>;
  constexpr int R = G::R, W = G::W, NT = G::NT, D = G::D, RB = G::RB;
  extern __shared__ __align__(16) double ring[];  // [R][RB]
  constexpr int RP = (R + 1) & ~1;
  __shared__ __align__(16) double colbuf[2][RP];  // pivot column rows 1..KL (index k-1)
  __shared__ double s_rp[2];
  __shared__ int s_p[2];
  __shared__ double s_xb[2];
  __shared__ int s_info;

  const int t = threadIdx.x;
  const bool owns = t <= W;        // column thread (t < W) or RHS thread (t == W)
  const bool loader = t > W;
  const int lidx = t - W - 1;  // loader lane = pattern entry (needs NT - W - 1 > E)
  const int n = P.n;
  const int nsteps = ((n + R - 1) / R) * R;
  double *U = P.ws + (size_t)blockIdx.x * ((size_t)n * W + n);
  double *Y = U + (size_t)n * W;

  for (int i = t; i < R * RB; i += NT) ring[i] = 0.0;
  __syncthreads();

  for (long long sys = blockIdx.x; sys < P.batch; sys += gridDim.x) {
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
    __syncthreads();
    double v[R];
#pragma unroll
    for (int r = 0; r < R; ++r) {
      v[r] = owns ? ring[r * RB + t] : 0.0;
      if (owns) ring[r * RB + t] = 0.0;
    }
    __syncthreads();
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
    int jm = 0;  // j mod W
    // ---- factorisation + forward substitution (dgbtf2 / dgbtrs L part) -----
#pragma unroll 1
    for (int j0 = 0; j0 < nsteps; j0 += R) {
#pragma unroll
      for (int u = 0; u < R; ++u) {
        const int j = j0 + u;
        const int jb = j & 1;
        int pos = t - jm;
        if (pos < 0) pos += W;
        if (t == W) pos = W;
        if (t < W && pos == 0) {
          // pivot: first index of max |a_kj|, k = 0..KL (tree keeps the left
          // operand unless the right one is strictly larger)
          double bv[R];
          int bi[R];
#pragma unroll
          for (int k = 0; k < R; ++k) {
            bv[k] = v[(u + k) % R];
            bi[k] = k;
          }
#pragma unroll
          for (int s = 1; s < R; s *= 2)
#pragma unroll
            for (int k = 0; k + s < R; k += 2 * s)
              if (fabs(bv[k + s]) > fabs(bv[k])) {
                bv[k] = bv[k + s];
                bi[k] = bi[k + s];
              }
          const int p = bi[0];
          const double pv = bv[0];
          const double rp = pv != 0.0 ? __drcp_rn(pv) : 0.0;
#pragma unroll
          for (int k = 1; k < R; ++k) colbuf[jb][k - 1] = v[(u + k) % R];
          if (p != 0) colbuf[jb][p - 1] = v[u];
          s_p[jb] = p;
          s_rp[jb] = rp;
          if (j < n) {
            U[(size_t)j * W] = rp;
            if (P.ipiv) P.ipiv[sys * n + j] = j + p;
            if (pv == 0.0 && s_info == 0) s_info = j + 1;
          }
#pragma unroll
          for (int k = 0; k < R; ++k) v[k] = 0.0;  // the thread takes column j + W next
        }
        if (loader) {
          load_entry<KL, KU>(P, val, bb, ring, (u + KL + 1 + D) % R, j + KL + 1 + D, lidx, pk);
          pk = load_pk(P, j + KL + 2 + D, lidx);
          cp_commit();
          cp_wait<D>();
        }
        __syncthreads();
        if (owns) {
          const int p = s_p[jb];
          const double rp = s_rp[jb];
          if (p != 0) {  // row swap j <-> j+p (uniform branch)
            const double a = v[u];
            double bsel = a;
#pragma unroll
            for (int k = 1; k < R; ++k) bsel = (p == k) ? v[(u + k) % R] : bsel;
#pragma unroll
            for (int k = 1; k < R; ++k) v[(u + k) % R] = (p == k) ? a : v[(u + k) % R];
            v[u] = bsel;
          }
          const double uc = v[u];
          if (j < n) {
            if (pos == W) Y[j] = uc;
            else if (pos != 0) U[(size_t)j * W + pos] = uc;
          }
          const double w = uc * rp;
          const double2 *cb = reinterpret_cast<const double2 *>(colbuf[jb]);
#pragma unroll
          for (int k = 1; k < R; k += 2) {
            const double2 m = cb[(k - 1) / 2];
            v[(u + k) % R] = fma(-m.x, w, v[(u + k) % R]);
            if (k + 1 < R) v[(u + k + 1) % R] = fma(-m.y, w, v[(u + k + 1) % R]);
          }
          // row j leaves; row j+KL+1 enters slot u
          v[u] = ring[u * RB + t];
          ring[u * RB + t] = 0.0;
        }
        jm = (jm + 1 == W) ? 0 : jm + 1;
      }
    }
    if (loader) cp_wait<0>();
    __syncthreads();  // U, y (global) and s_info visible to the whole CTA
    // ---- back substitution (dgbtrs U part, column order) --------------------
    // thread t < W holds the accumulator of row i = the largest i <= j with
    // i = t (mod W); at step j its U entry is U[i][j - i] (U[j][0] = 1/u_jj).
    {
      const bool act = t < W;
      int d = (n - 1 - t) % W;  // j - i at j = n-1 (n-1-t may be < 0)
      if (d < 0) d += W;
      int i = act ? n - 1 - d : -1;
      double acc = i >= 0 ? Y[i] : 0.0;
      double ynext = i - W >= 0 ? Y[i - W] : 0.0;
      // software pipeline: the U entries of the next PF steps are loaded ahead
      constexpr int PF = 8;
      double q[PF];
      int dq = d, iq = i;
#pragma unroll
      for (int s = 0; s < PF; ++s) {
        const int jj = n - 1 - s;
        q[s] = (iq >= 0 && jj >= 0) ? U[(size_t)iq * W + (jj - iq)] : 0.0;
        if (dq == 0) { dq = W - 1; iq -= W; } else { --dq; }
      }
#pragma unroll 1
      for (int jb0 = n - 1; jb0 >= 0; jb0 -= PF) {
#pragma unroll
        for (int s = 0; s < PF; ++s) {
          const int j = jb0 - s;
          const double uij = q[s];
          {  // refill: step j - PF
            const int jj = j - PF;
            q[s] = (iq >= 0 && jj >= 0) ? U[(size_t)iq * W + (jj - iq)] : 0.0;
            if (dq == 0) { dq = W - 1; iq -= W; } else { --dq; }
          }
          if (act && j >= 0 && d == 0) {
            const double xj = acc * uij;  // x_j = y_j / u_jj
            P.x[sys * n + j] = xj;
            s_xb[j & 1] = xj;
          }
          __syncthreads();
          if (act && j >= 0) {
            if (d == 0) {
              i -= W;
              d = W - 1;
              acc = ynext;
              ynext = i - W >= 0 ? Y[i - W] : 0.0;
            } else {
              if (i >= 0) acc = fma(-uij, s_xb[j & 1], acc);  // y_i -= u_ij x_j
              --d;
            }
          }
        }
      }
    }
    if (t == 0) P.info[sys] = s_info;
    __syncthreads();
  }
}

}  // namespace bband
