// line_kernel.cuh -- TMEM plan with LINE-TILED row ownership for 2D 9-point
// stencils (DESIGN.md "Kernels" 10).
//
// The 992-row XGC systems are a 9-point stencil on an NX-wide velocity grid
// (PAPER.md:519-530).  In the strided plans thread t owns rows t + 128 j, so
// each of the 8 off-diagonal entries of each row needs its own gathered
// operand: 64 shared-memory loads per thread per SpMV.  Here thread t owns the
// R = 8 CONSECUTIVE rows 8t .. 8t+7 of the grid.  The operands of all 8 rows
// then come from three short runs of the published vector:
//   line above : rows 8t - NX - 1 .. 8t - NX + 8   (10 loads)
//   own line   : rows 8t - 1 and 8t + 8            (2 loads; rows 8t..8t+7
//                                                   are the thread's own
//                                                   registers)
//   line below : rows 8t + NX - 1 .. 8t + NX + 8   (10 loads)
// = 22 loads instead of 64, i.e. 2.9x fewer shared-memory wavefronts for the
// gathers (the stores of the published vector are unchanged).
//
// Shared-memory layout of the published vector ("planes"): row r lives at
//   sg[(r mod 8) * S + GQ + floor(r / 8)]
// so for any fixed offset o the 32 lanes of a warp (t consecutive) read
// row 8t + o at consecutive addresses (plane o mod 8, column t + floor(o/8)):
// every load and every store is bank-conflict free whatever NX is.  GQ zero
// columns before and S - GQ - NT after the body absorb the stencil reach at
// the grid edges (their operands are multiplied by the 0.0 ELL padding).
//
// Matrix values: no SMEM staging at all.  Each thread reads its 8 rows x 9
// slots straight from HBM into registers (16-byte loads, fully used sectors)
// and moves the 8 off-diagonal values of each row into its own TMEM lane
// (tcgen05.st, 16 columns per row, in the canonical stencil order below);
// the diagonal stays in a register.  Every SpMV reads them back with
// tcgen05.ld, software-pipelined one row group ahead of the FMAs.
#pragma once
#include "gmres.cuh"
#include "kernels.cuh"

#ifndef BSOLVE_SPMV_SPLIT
#define BSOLVE_SPMV_SPLIT 0  // 1: two FMA chains per row (measured 8.01 vs 8.14 M sys/s)
#endif

namespace bsolve {

// Canonical order of the 8 off-diagonal stencil offsets (column - row):
//   0: -NX-1  1: -NX  2: -NX+1  3: -1  4: +1  5: NX-1  6: NX  7: NX+1
// SolveParams::c2s[c] = ELL slot holding canonical offset c (-1: absent).
// R rows per thread (R planes), NT threads per CTA, R * NT = 1024 rows.
template <int NX, int NT, int R>
struct LineGeom {
  __host__ __device__ static constexpr int floordivR(int o) {
    return o >= 0 ? o / R : -((-o + R - 1) / R);
  }
  static constexpr int GQ = (NX + 1 + R - 1) / R + 1;  // zero columns before the body
  // doubles per plane, even: every plane (and the GQ-column halo segment of
  // the cluster kernels' bulk copies) starts 16-byte aligned
  static constexpr int S = (NT + 2 * GQ + 1 + 1) & ~1;
  // element offset of row R t + o relative to sg + GQ + t
  __host__ __device__ static constexpr int idx(int o) {
    return (o - R * floordivR(o)) * S + floordivR(o);
  }
  static_assert(GQ >= (NX + 1 + R - 1) / R && S - GQ - NT >= floordivR(NX + R) + 1,
                "guards must cover the stencil reach");
};

template <int NX, int NT, int R>
struct LineComm {
  using L = LineGeom<NX, NT, R>;
  double *gq;    // sg + GQ + threadIdx.x
  double *sred;  // reduction scratch
  int buf;
  const bool (&act)[R];
  __device__ __forceinline__ LineComm(double *sg, double *sred_, const bool (&act_)[R])
      : gq(sg + L::GQ + threadIdx.x), sred(sred_), buf(0), act(act_) {}
  __device__ __forceinline__ int grow(int j) const { return R * threadIdx.x + j; }
  __device__ __forceinline__ bool leader() const { return threadIdx.x == 0; }
  // every thread writes all R of its entries, so the body [GQ, GQ + NT) of
  // every plane is fully rewritten by each publish.  Rows >= n need no select:
  // their diagonal and values are 0 and their b, x0 are 0, so every vector
  // entry of theirs stays 0 (unless a scalar is already non-finite, i.e. the
  // system breaks down anyway).
  __device__ __forceinline__ void publish(int j, double v) { gq[j * L::S] = v; }
  __device__ __forceinline__ void sync() { __syncthreads(); }
  __device__ __forceinline__ void barrier() { __syncthreads(); }  // CTA only, no halo
  template <int K>
  __device__ __forceinline__ void sum(double (&v)[K]) {
    block_sum<K, NT / 32>(v, sred, buf, threadIdx.x & 31, threadIdx.x >> 5);
  }
  // (cluster halo-state interface of line3_solve; nothing to exchange here)
  static constexpr bool kHalo2 = false;
  template <int K>
  __device__ __forceinline__ void sum_x(double (&v)[K], const double (&)[R], int,
                                        const double (&)[R]) {
    sum<K>(v);
  }
  __device__ __forceinline__ void halo_p(double, double) {}
  __device__ __forceinline__ void halo_s(double) {}
  __device__ __forceinline__ void halo_r(double) {}
  __device__ __forceinline__ void halo_restart() {}
  __device__ __forceinline__ void sync_local() { __syncthreads(); }
};

__device__ __forceinline__ double tmem_f64(const uint32_t (&w)[16], int c) {
  return __hiloint2double(static_cast<int>(w[2 * c + 1]), static_cast<int>(w[2 * c]));
}

// y = A g for rows Rt .. Rt+R-1.  gq = sg + GQ + t; own[j] = g[Rt + j].
// G rows per tcgen05.ld group; group k+1 is in flight while group k's FMAs run.
// NXG > NX: generic width (NX = width mod 8, A = width / 8 at run time, the
// plane geometry of width NXG; line3_kernel.cuh line3_spmv explains the shift)
template <int NX, int NT, int R, int G, int NXG = NX>
__device__ __forceinline__ void line_spmv(uint32_t tlane, const double *gq, const double (&a0)[R],
                                          const double (&own)[R], double (&y)[R], int A = 0) {
  using L = LineGeom<NXG, NT, R>;
  constexpr int NG = R / G;
  static_assert(R % G == 0, "G must divide R");
  uint32_t w[2][G][16];
#pragma unroll
  for (int g = 0; g < G; ++g) tmem_ld16(tlane + 16 * g, w[0][g]);
  double gm[R + 2], gp[R + 2];
#pragma unroll
  for (int e = 0; e < R + 2; ++e) {
    gm[e] = gq[L::idx(-NX + e - 1) - A];
    gp[e] = gq[L::idx(NX + e - 1) + A];
  }
  const double gl = gq[L::idx(-1)], gr = gq[L::idx(R)];
  tmem_wait_ld();
#pragma unroll
  for (int g = 0; g < G; ++g) tmem_regs_ready(w[0][g]);
#pragma unroll
  for (int k = 0; k < NG; ++k) {
    if (k + 1 < NG) {
#pragma unroll
      for (int g = 0; g < G; ++g) tmem_ld16(tlane + 16 * ((k + 1) * G + g), w[(k + 1) & 1][g]);
    }
#pragma unroll
    for (int g = 0; g < G; ++g) {
      const int j = k * G + g;
      const uint32_t(&v)[16] = w[k & 1][g];
#if BSOLVE_SPMV_SPLIT
      // two independent FMA chains per row (the line above + the left
      // neighbour | the diagonal, the right neighbour + the line below):
      // half the dependent-FMA latency per row
      double acc = tmem_f64(v, 0) * gm[j];
      double acc2 = a0[j] * own[j];
      acc = fma(tmem_f64(v, 1), gm[j + 1], acc);
      acc2 = fma(tmem_f64(v, 4), j == R - 1 ? gr : own[j == R - 1 ? j : j + 1], acc2);
      acc = fma(tmem_f64(v, 2), gm[j + 2], acc);
      acc2 = fma(tmem_f64(v, 5), gp[j], acc2);
      acc = fma(tmem_f64(v, 3), j == 0 ? gl : own[j == 0 ? 0 : j - 1], acc);
      acc2 = fma(tmem_f64(v, 6), gp[j + 1], acc2);
      acc2 = fma(tmem_f64(v, 7), gp[j + 2], acc2);
      y[j] = acc + acc2;  // rows >= n: a0 = 0 and zero values -> 0 (finite operands)
#else
      double acc = a0[j] * own[j];
      acc = fma(tmem_f64(v, 0), gm[j], acc);
      acc = fma(tmem_f64(v, 1), gm[j + 1], acc);
      acc = fma(tmem_f64(v, 2), gm[j + 2], acc);
      acc = fma(tmem_f64(v, 3), j == 0 ? gl : own[j == 0 ? 0 : j - 1], acc);
      acc = fma(tmem_f64(v, 4), j == R - 1 ? gr : own[j == R - 1 ? j : j + 1], acc);
      acc = fma(tmem_f64(v, 5), gp[j], acc);
      acc = fma(tmem_f64(v, 6), gp[j + 1], acc);
      acc = fma(tmem_f64(v, 7), gp[j + 2], acc);
      y[j] = acc;  // rows >= n: a0 = 0 and zero values -> acc = 0 (finite operands)
#endif
    }
    if (k + 1 < NG) {
      tmem_wait_ld();
#pragma unroll
      for (int g = 0; g < G; ++g) tmem_regs_ready(w[(k + 1) & 1][g]);
    }
  }
}

// One CTA of NT = 1024 / R threads per system (n <= 1024), 2 CTAs per SM.
// TMEM: 16 columns per row; with 256 threads warps w and w + 4 share lane
// quarter w % 4 and use consecutive column ranges (128 columns per CTA).
//   SMEM: [gather planes: R * S] [reduction scratch: 16 * NWARP] [TMEM base: 16 B]
//         GMRES only: [Krylov basis: kMaxRestart * R * NT] [R factor: kMaxRestart^2]
// SOLVER: SOLVER_BICGSTAB (Algorithm 1) or SOLVER_GMRES (gmres.cuh).
template <int NX, int R, int G, int SOLVER = SOLVER_BICGSTAB, int MINB = 2, int ROUNDS = 3,
          int NXG = NX>
__global__ void __launch_bounds__(1024 / R, MINB) bicgstab_tmem_line_kernel(const SolveParams P) {
  constexpr int NT = 1024 / R, NWARP = NT / 32;
  static_assert(R == 4 || R == 8, "4 or 8 rows per thread");
  using L = LineGeom<NXG, NT, R>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sg = reinterpret_cast<double *>(smem_raw);
  double *sred = sg + R * L::S;
  uint32_t *tbase_s = reinterpret_cast<uint32_t *>(sred + 16 * NWARP);

  const int tid = threadIdx.x, warp = tid >> 5;
  const int n = P.n;
  const long long sys = blockIdx.x;
  const int row0 = R * tid;
  const double *gval = P.values + sys * P.sys_stride;

  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s)),
                 "n"(128));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  // zero guard columns of every plane (the body is rewritten by each publish)
  for (int i = tid; i < R * (L::S - NT); i += NT) {
    const int pl = i / (L::S - NT), q = i % (L::S - NT);
    sg[pl * L::S + (q < L::GQ ? q : q + NT)] = 0.0;
  }
  // L2 prefetch (TMA bulk prefetch) of a system that starts later
  if (tid == 0 && P.pf_ahead > 0 && sys + P.pf_ahead < P.batch) {
    const long long ns = sys + P.pf_ahead;
    const uint32_t vb = static_cast<uint32_t>(P.sys_stride * 8) & ~15u;
    const void *va = P.values + ns * P.sys_stride;
    const void *ba = P.b + ns * n;
    if (((reinterpret_cast<uintptr_t>(va) | reinterpret_cast<uintptr_t>(ba)) & 15u) == 0) {
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(va), "r"(vb) : "memory");
      asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(ba),
                   "r"(static_cast<uint32_t>(n * 8) & ~15u)
                   : "memory");
      const void *xa = P.x0 ? P.x0 + ns * n : nullptr;  // warm start (Picard) guess
      if (xa && (reinterpret_cast<uintptr_t>(xa) & 15u) == 0)
        asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(xa),
                     "r"(static_cast<uint32_t>(n * 8) & ~15u)
                     : "memory");
    }
  }

  // ---- this thread's rows: b, x0, diagonal and the 8 off-diagonal values ----
  bool act[R];
  double x[R], r[R], d[R], a0[R];
  double val[R][8];
  const bool vec = !P.vidx && ((n & 1) == 0) && ((reinterpret_cast<uintptr_t>(gval) & 15u) == 0) &&
                   row0 + R <= n;
#pragma unroll
  for (int j = 0; j < R; ++j) act[j] = row0 + j < n;
  if (vec) {
#pragma unroll
    for (int j = 0; j < R; j += 2) {
      const double2 dg = __ldg(reinterpret_cast<const double2 *>(gval + row0 + j));
      a0[j] = dg.x;
      a0[j + 1] = dg.y;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const int k = P.c2s[c];
        double2 v = make_double2(0.0, 0.0);
        if (k >= 0) v = __ldg(reinterpret_cast<const double2 *>(gval + (long long)k * n + row0 + j));
        val[j][c] = v.x;
        val[j + 1][c] = v.y;
      }
    }
  } else if (P.vidx) {  // CSR values: the handle's (row, canonical slot) -> CSR index table
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const int e0 = act[j] ? __ldg(P.vidx + 8 * n + row0 + j) : -1;
      a0[j] = e0 >= 0 ? __ldg(gval + e0) : 0.0;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const int e = act[j] ? __ldg(P.vidx + c * n + row0 + j) : -1;
        val[j][c] = e >= 0 ? __ldg(gval + e) : 0.0;
      }
    }
  } else {
#pragma unroll
    for (int j = 0; j < R; ++j) {
      a0[j] = act[j] ? __ldg(gval + row0 + j) : 0.0;
#pragma unroll
      for (int c = 0; c < 8; ++c) {
        const int k = P.c2s[c];
        val[j][c] = (act[j] && k >= 0) ? __ldg(gval + (long long)k * n + row0 + j) : 0.0;
      }
    }
  }
  const double *bsys = P.b + sys * n;
#pragma unroll
  for (int j = 0; j < R; ++j) {
    d[j] = jacobi_inv(P.precond, a0[j]);
    r[j] = act[j] ? __ldg(bsys + row0 + j) : 0.0;
    x[j] = (act[j] && P.x0) ? __ldg(P.x0 + sys * n + row0 + j) : 0.0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tlane = *tbase_s + (static_cast<uint32_t>(32 * (warp & 3)) << 16) +
                         static_cast<uint32_t>((warp >> 2) * 16 * R);
#pragma unroll
  for (int j = 0; j < R; ++j) {
    uint32_t w[16];
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      w[2 * c] = static_cast<uint32_t>(__double2loint(val[j][c]));
      w[2 * c + 1] = static_cast<uint32_t>(__double2hiint(val[j][c]));
    }
    tmem_st16(tlane + 16 * j, w);
  }
  tmem_wait_st();

  LineComm<NXG, NT, R> comm(sg, sred, act);
  const int A = NXG == NX ? 0 : P.line_a;
  auto spmv = [&](const double(&own)[R], double(&y)[R]) {
    line_spmv<NX, NT, R, G, NXG>(tlane, comm.gq, a0, own, y, A);
  };
  if constexpr (SOLVER == SOLVER_GMRES) {
    double *sV = sred + 16 * NWARP + 2;
    gmres_core<R, NT, kMaxRestart>(P, sys, x, r, d, act, sV, sV + kMaxRestart * R * NT, comm,
                                   spmv);
  } else {
    bicgstab_core<R, NT, false, ROUNDS>(P, sys, x, r, d, act, r, comm, spmv);
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(*tbase_s), "n"(128));
}

}  // namespace bsolve
