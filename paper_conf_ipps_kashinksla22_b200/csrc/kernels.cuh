// kernels.cuh -- sm_100a device code of the batched Jacobi-BiCGSTAB solver.
//
// One CTA solves one system end to end: the whole
// Algorithm 1 loop runs inside a single kernel launch
// and each system stops on its own.
//
// B200 design:
//  * the system's matrix values (71,424 B for the 992-row 9-point ELL case)
//    are staged ONCE into shared memory with a TMA bulk copy
//    (cp.async.bulk + mbarrier complete_tx) while the threads load b, x0 and
//    the shared pattern; every SpMV then reads values and the gathered vector
//    from SMEM (PLACE_SMEM).  PLACE_STREAM re-reads values from global
//    memory (L2/L1) instead, for systems whose values do not fit.
//  * every BiCGSTAB vector lives in REGISTERS: thread t owns rows t + j*NT,
//    j < R.  Only the vector being multiplied (p^ or s^) is published to a
//    shared "gather" buffer for the SpMV.
//  * the shared-memory data pipe (LDS wavefronts + SHFL) is the bound, so the
//    kernel minimises wavefronts: conflict-free ELL slot map, diagonal in
//    slot 0 (its value and its gather operand stay in registers), offset
//    ("DIA") addressing for stencil patterns (no column registers, no index
//    arithmetic), and reductions that spend as few shuffles as possible.
#pragma once
#include <cstdint>
#include <cooperative_groups.h>
#include <cuda_runtime.h>

namespace bsolve {

// Kernel-level storage modes.  CSR and ELL are the paper's BatchCsr and
// BatchEll.  DIA is BatchEll values whose slot k holds,
// in every row r, the entry of column r + d_k (the host detects this for
// stencil patterns): the gather address is row + d_k with d_k uniform.
enum { FMT_CSR = 1, FMT_ELL = 2, FMT_DIA = 3 };
enum { PLACE_SMEM = 1, PLACE_STREAM = 2, PLACE_REGS = 3, PLACE_CLUSTER = 4, PLACE_TMEM = 5 };
enum { STOP_REL_B = 0, STOP_ABS = 1 };
enum { SYS_CONVERGED = 0, SYS_MAXITER = 1, SYS_BREAKDOWN = 2 };
enum { PREC_JACOBI = 0, PREC_NONE = 1,       // PRECOND(y) = d .* y
       PREC_BLOCK_JACOBI = 2 };               // 8-row blocks, line3 kernel only (R30)
enum { SOLVER_BICGSTAB = 0, SOLVER_GMRES = 1 };
constexpr int kMaxW = 16;
constexpr int kMaxRestart = 7;  // GMRES: CGS2 pass 2 reduces kMaxRestart + 1 <= 8 values at once

struct SolveParams {
  const double *values;     // [batch][sys_stride]
  const double *b;          // [batch][n]
  const double *x0;         // [batch][n] or nullptr
  double *x;                // [batch][n]
  int32_t *iters;           // [batch]
  double *resnorm;          // [batch]
  int8_t *status;           // [batch] or nullptr
  const int32_t *ell_col;   // [W][n] column table, column-major
  const int32_t *row_ptr;   // [n+1]
  const int32_t *diag_slot; // [n] CSR position of the diagonal in its row
  long long sys_stride;     // doubles per system in `values`
  double tol;
  int n, W, batch, maxiter, stop, trc;
  int smem_vals;            // doubles of SMEM reserved for values (even)
  int n_pad;                // doubles of the gather buffer body (even)
  int guard;                // zero doubles before and after the gather body (DIA)
  int doff[kMaxW];          // DIA: byte offset d_k * 8 of slot k
  int c2s[8];               // line-tiled stencil plan: ELL slot of canonical offset c, -1 none
  const int32_t *vidx;      // line plan with CSR values: [9][n] index of canonical slot c
                            // (8 = diagonal) of row r in a system's CSR block, -1 none;
                            // nullptr: ELL values (slot c2s[c] of the ELL block)
  int precond;              // PREC_JACOBI (d = 1 / a_ii) or PREC_NONE (d = 1)
  int restart;              // GMRES: Krylov steps per restart cycle (1 .. kMaxRestart)
  int pf_ahead;             // line plan: prefetch system sys + pf_ahead into L2 (0: off)
  int line_a;               // generic-width line kernels: grid width / 8 (0: compile-time width)
};

// Jacobi entry d_i for diagonal a (R11: zero diagonal -> 1); 1 without preconditioner.
__device__ __forceinline__ double jacobi_inv(int precond, double a) {
  return (precond == PREC_JACOBI && a != 0.0) ? 1.0 / a : 1.0;
}

// ------------------------------------------------------------ PTX helpers --
__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count)
               : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)),
               "r"(bytes)
               : "memory");
}
// TMA bulk copy global -> shared, completion counted on `bar` in bytes.
__device__ __forceinline__ void tma_bulk_g2s(void *dst, const void *src, uint32_t bytes,
                                             uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAIT_%=;\n}" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}

// Distributed shared memory helpers (thread-block clusters).
__device__ __forceinline__ uint32_t mapa_u32(uint32_t saddr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
// 8-byte store into a (possibly remote) CTA's SMEM that completes 8 bytes
// of transaction count on that CTA's mbarrier.
__device__ __forceinline__ void st_async_f64(uint32_t raddr, double v, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(
                   raddr),
               "l"(__double_as_longlong(v)), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void mbar_wait_parity_cluster(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P;\n"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P, [%0], %1;\n\t"
      "@!P bra WAITC_%=;\n}" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ bool bad(double v) { return v == 0.0 || !isfinite(v); }

// Sum over this thread's R rows of f(j) with two interleaved accumulators
// (even / odd rows): half the dependent-add latency of one chain at the
// register cost of two.  Fixed order.
template <int R, class F>
__device__ __forceinline__ double rows_sum(F &&f) {
  double e = 0.0, o = 0.0;
#pragma unroll
  for (int j = 0; j < R; j += 2) {
    e += f(j);
    if (j + 1 < R) o += f(j + 1);
  }
  return e + o;
}

// Pairwise (tree) sum of N doubles, fixed order: latency log2(N) adds.
template <int N>
__device__ __forceinline__ double tree_sum(const double *a) {
  if constexpr (N == 1) {
    return a[0];
  } else {
    return tree_sum<N / 2>(a) + tree_sum<N - N / 2>(a + N / 2);
  }
}

// Block-wide sum of K <= 8 doubles with ONE barrier.  On B200 every SHFL.32
// costs one shared-memory data-pipe wavefront (like an LDS) and ~20+ cycles
// of latency, so:
//  * inside a warp, recursive halving: with K > 1 the first steps exchange
//    only the half of the values a lane is NOT responsible for (lane bit 4,
//    then bit 3, select the value), the remaining steps are an xor butterfly
//    on one value; K values cost about the shuffles of one;
//  * lane 8q publishes the warp partial of value q (K = 1: lane 0);
//  * after the barrier every thread loads the NWARP partials of each value
//    (broadcast 16-byte loads, all values in flight together) and adds them
//    as a pairwise tree.
// After the butterfly all lanes that hold a value hold the same bits (each
// step adds the same two operands in both partner lanes; fp addition is
// commutative), and the tree has a fixed order, so every thread obtains
// bitwise-identical sums: uniform control flow, results independent of the
// batch slicing.  `buf` alternates between two scratch halves so the next
// reduction never overwrites partials that a slow warp is still reading.
template <int K, int NWARP>
__device__ __forceinline__ void block_sum(double (&v)[K], double *sred, int &buf, int lane,
                                          int warp) {
  static_assert(K >= 1 && K <= 8, "block_sum supports 1..8 values");
  static_assert(NWARP % 2 == 0 && NWARP <= 32, "NWARP must be even");
  constexpr int KP = K <= 1 ? 1 : K <= 2 ? 2 : K <= 4 ? 4 : 8;  // padded value count
  constexpr int SPAN = 32 / KP;  // lanes sharing one value after the halving steps
  double a[KP];
#pragma unroll
  for (int i = 0; i < KP; ++i) a[i] = i < K ? v[i] : 0.0;
  // recursive halving: at offset o a lane keeps the upper half of its values
  // if lane bit o is set, the lower half otherwise, and adds its partner's copy
#pragma unroll
  for (int cnt = KP, o = 16; cnt > 1; cnt >>= 1, o >>= 1) {
    const bool hi = lane & o;
#pragma unroll
    for (int i = 0; i < cnt / 2; ++i) {
      const double send = hi ? a[i] : a[i + cnt / 2];
      const double keep = hi ? a[i + cnt / 2] : a[i];
      a[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
    }
  }
  // xor butterfly over the SPAN lanes that hold the same value
#pragma unroll
  for (int o = SPAN / 2; o > 0; o >>= 1) a[0] += __shfl_xor_sync(0xffffffffu, a[0], o);
  double *S = sred + buf * (8 * NWARP);
  const int q = lane / SPAN;  // value index held by this lane
  if ((lane % SPAN) == 0 && q < K) S[q * NWARP + warp] = a[0];
  __syncthreads();
  double part[K][NWARP];
#pragma unroll
  for (int k = 0; k < K; ++k) {
    const double2 *S2 = reinterpret_cast<const double2 *>(S + k * NWARP);
#pragma unroll
    for (int w = 0; w < NWARP / 2; ++w) {
      const double2 qq = S2[w];
      part[k][2 * w] = qq.x;
      part[k][2 * w + 1] = qq.y;
    }
  }
#pragma unroll
  for (int k = 0; k < K; ++k) v[k] = tree_sum<NWARP>(part[k]);
  buf ^= 1;
}

// Extract the 16-bit field at bit `POS` of `pk`.  volatile keeps the unpack
// inside the SpMV loop instead of letting the compiler hoist twice as many
// unpacked offsets into registers (which spills at R = 4).
template <int POS>
__device__ __forceinline__ uint32_t field16(uint32_t pk) {
  uint32_t v;
  asm volatile("bfe.u32 %0, %1, %2, 16;" : "=r"(v) : "r"(pk), "n"(POS));
  return v;
}

// Per-thread view of its rows of the shared pattern.
template <int FMT, int WB, int R, int KREG = 0>
struct RowMeta {
  uint32_t cpk[R][(WB + 1) / 2]; // CSR/ELL: packed 16-bit byte offsets (col*8) into the gather body
  int vbase[R];                  // ELL/DIA: row (clamped for idle lanes); CSR: row_ptr[row]
  int vlen[R];                   // CSR row length
  double a0[R];                  // ELL/DIA: the diagonal value (slot 0)
  double vreg[R][KREG > 0 ? KREG : 1];  // ELL/DIA: values of slots 1..KREG in registers
  bool act[R];                   // row < n
};

// y = A * g for this thread's rows (one thread per row,
// W sequential slots, no intra-row reduction).  `gb` points at the gather
// body (byte address), `own[j]` is this thread's own gather entry g[row]
// (ELL/DIA: slot 0 is the diagonal, so its operand never leaves registers).
// Values come from V (shared or global).  EXACT: W == WB at compile time.
// Row blocks: a warp whose row block j lies entirely at or beyond n skips it.
// The common cases -- all R blocks of the warp active, or all but the last --
// run branch-free so the compiler interleaves the loads and FMA chains of
// all rows (per-row branches serialised them: DFMA latency was exposed).
// Idle lanes of a partial warp run on a clamped row and zero their result.
template <int FMT, int PLACE, int WB, bool EXACT, int R, int KREG, int NB>
__device__ __forceinline__ void spmv_block(const double *__restrict__ V,
                                           const unsigned char *gb, const SolveParams &P,
                                           const RowMeta<FMT, WB, R, KREG> &m,
                                           const double (&own)[R], double (&y)[R],
                                           int vstride) {
  double acc[R];
#pragma unroll
  for (int j = 0; j < NB; ++j) acc[j] = (FMT == FMT_CSR) ? 0.0 : m.a0[j] * own[j];  // slot 0
#pragma unroll
  for (int k = (FMT == FMT_CSR) ? 0 : 1; k < WB; ++k) {
#pragma unroll
    for (int j = 0; j < NB; ++j) {
      if (FMT == FMT_CSR) {
        if ((EXACT || k < P.W) && k < m.vlen[j]) {
          const uint32_t off =
              (k & 1) ? field16<16>(m.cpk[j][k >> 1]) : field16<0>(m.cpk[j][k >> 1]);
          const double g = *reinterpret_cast<const double *>(gb + off);
          const double *a_p = V + m.vbase[j] + k;
          acc[j] = fma((PLACE == PLACE_STREAM) ? __ldg(a_p) : *a_p, g, acc[j]);
        }
      } else if (EXACT || k < P.W) {
        double g;
        if (FMT == FMT_DIA) {
          g = *reinterpret_cast<const double *>(gb + m.vbase[j] * 8 + P.doff[k]);
        } else {
          const uint32_t off =
              (k & 1) ? field16<16>(m.cpk[j][k >> 1]) : field16<0>(m.cpk[j][k >> 1]);
          g = *reinterpret_cast<const double *>(gb + off);
        }
        double a;
        if (k <= KREG) {
          a = m.vreg[j][k - 1 < 0 ? 0 : k - 1];  // slots 1..KREG: registers
        } else {
          const double *a_p = V + m.vbase[j] + k * vstride;
          a = (PLACE == PLACE_STREAM) ? __ldg(a_p) : *a_p;
        }
        acc[j] = fma(a, g, acc[j]);
      }
    }
  }
#pragma unroll
  for (int j = 0; j < R; ++j) y[j] = (j < NB && m.act[j]) ? acc[j] : 0.0;
}

template <int FMT, int PLACE, int WB, bool EXACT, int R, int NT, int KREG>
__device__ __forceinline__ void spmv_rows(const double *__restrict__ V,
                                          const unsigned char *gb, const SolveParams &P,
                                          const RowMeta<FMT, WB, R, KREG> &m,
                                          const double (&own)[R], double (&y)[R], int nrows,
                                          int vstride) {
  // nrows: rows owned by this CTA (= n unless a cluster splits the system);
  // vstride: doubles between two ELL slots of the staged values
  const int wrow0 = threadIdx.x & ~31;
  const int n = nrows;
  if (wrow0 + (R - 1) * NT < n) {
    spmv_block<FMT, PLACE, WB, EXACT, R, KREG, R>(V, gb, P, m, own, y, vstride);
  } else if (R > 1 && wrow0 + (R - 2) * NT < n) {
    spmv_block<FMT, PLACE, WB, EXACT, R, KREG, (R > 1 ? R - 1 : 1)>(V, gb, P, m, own, y,
                                                                     vstride);
  } else {
    // generic tail (small n: several idle row blocks): one block at a time
#pragma unroll
    for (int j = 0; j < R; ++j) {
      double acc = 0.0;
      if (wrow0 + j * NT < n) {
        if (FMT != FMT_CSR) acc = m.a0[j] * own[j];  // slot 0, same order as spmv_block
#pragma unroll
        for (int k = (FMT == FMT_CSR) ? 0 : 1; k < WB; ++k) {
          if (FMT == FMT_CSR) {
            if ((EXACT || k < P.W) && k < m.vlen[j]) {
              const uint32_t off =
                  (k & 1) ? field16<16>(m.cpk[j][k >> 1]) : field16<0>(m.cpk[j][k >> 1]);
              const double *a_p = V + m.vbase[j] + k;
              acc = fma((PLACE == PLACE_STREAM) ? __ldg(a_p) : *a_p,
                        *reinterpret_cast<const double *>(gb + off), acc);
            }
          } else if (EXACT || k < P.W) {
            double g;
            if (FMT == FMT_DIA) {
              g = *reinterpret_cast<const double *>(gb + m.vbase[j] * 8 + P.doff[k]);
            } else {
              const uint32_t off =
                  (k & 1) ? field16<16>(m.cpk[j][k >> 1]) : field16<0>(m.cpk[j][k >> 1]);
              g = *reinterpret_cast<const double *>(gb + off);
            }
            double a;
            if (k <= KREG) {
              a = m.vreg[j][k - 1 < 0 ? 0 : k - 1];
            } else {
              const double *a_p = V + m.vbase[j] + k * vstride;
              a = (PLACE == PLACE_STREAM) ? __ldg(a_p) : *a_p;
            }
            acc = fma(a, g, acc);
          }
        }
      }
      y[j] = m.act[j] ? acc : 0.0;
    }
  }
}

// ------------------------------------------------------------ the solver --
// Communication policy of the single-CTA kernels: the gather buffer and the
// reductions are CTA-local.
template <int R, int NT>
struct CtaComm {
  double *sg;    // gather body
  double *sred;  // reduction scratch
  int buf;
  const bool (&act)[R];
  __device__ __forceinline__ CtaComm(double *sg_, double *sred_, const bool (&act_)[R])
      : sg(sg_), sred(sred_), buf(0), act(act_) {}
  __device__ __forceinline__ int grow(int j) const { return threadIdx.x + j * NT; }
  __device__ __forceinline__ bool leader() const { return threadIdx.x == 0; }
  __device__ __forceinline__ void publish(int j, double v) {
    if (act[j]) sg[threadIdx.x + j * NT] = v;
  }
  __device__ __forceinline__ void sync() { __syncthreads(); }
  __device__ __forceinline__ void barrier() { __syncthreads(); }  // CTA only, no halo
  template <int K>
  __device__ __forceinline__ void sum(double (&v)[K]) {
    block_sum<K, NT / 32>(v, sred, buf, threadIdx.x & 31, threadIdx.x >> 5);
  }
};

// Algorithm 1 for ONE system, shared by both kernels.
//   on entry: x = x0 (or 0), r = b, d = Jacobi diagonal, act = row < n;
//   spmv(own, y): y = A g for this thread's rows, where g was published to
//                 the gather body sg (and a barrier passed); own[j] = g[row].
//   bv: b in registers (B_IN_REGS) for the true residual, else re-read bsys.
// Writes x, iters, resnorm, status of system `sys`.  Every path executes at
// least one block_sum (one barrier) after entry.
template <int R, int NT, bool B_IN_REGS, int ROUNDS, class Comm, class SpMV>
__device__ __forceinline__ void bicgstab_core(const SolveParams &P, long long sys, double (&x)[R],
                                              double (&r)[R], const double (&d)[R],
                                              const bool (&act)[R], const double (&bv)[R],
                                              Comm &comm, SpMV &&spmv) {
  const int n = P.n;
  const double *bsys = P.b + sys * n;
  double rh[R], p[R], v[R];

  // ---- a3: r = b - A x0 ; r^ = r ; ||b|| --------------------------------
  double red3[2] = {0.0, 0.0};
#pragma unroll
  for (int j = 0; j < R; ++j) red3[0] += r[j] * r[j];  // b.b
  if (P.x0) {
#pragma unroll
    for (int j = 0; j < R; ++j)
      comm.publish(j, x[j]);
    comm.sync();
    double q[R];
    spmv(x, q);
#pragma unroll
    for (int j = 0; j < R; ++j) r[j] = r[j] - q[j];
  }
#pragma unroll
  for (int j = 0; j < R; ++j) {
    rh[j] = r[j];
    p[j] = 0.0;
    v[j] = 0.0;
    red3[1] += r[j] * r[j];
  }
  comm.template sum<2>(red3);
  const double bnorm = sqrt(red3[0]);
  const double tau = (P.stop == STOP_ABS) ? P.tol : P.tol * bnorm;
  // stop tests compare squared norms (no sqrt on the critical path) whenever
  // tau^2 neither underflows nor overflows; sqrt(a) < tau <=> a < tau^2 for
  // a >= 0 up to the rounding of tau^2 (R7)
  const double tau2 = tau * tau;
  const bool sq = tau2 > 1e-300 && tau2 < 1e300;
  auto below = [&](double nrm2) { return sq ? nrm2 < tau2 : sqrt(nrm2) < tau; };
  double rnorm = sqrt(red3[1]);
  double rnorm2 = red3[1];  // ||r||^2 of the current r (3-round schedule)
  double rho = red3[1];  // r^ . r with r^ = r

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

  auto true_residual = [&](double (&q)[R]) -> double {
    // publish x, q = b - A x, returns ||q||_2 (one more barrier)
#pragma unroll
    for (int j = 0; j < R; ++j)
      comm.publish(j, x[j]);
    comm.sync();
    double tr[1] = {0.0};
    spmv(x, q);
#pragma unroll
    for (int j = 0; j < R; ++j) {
      const double bj = B_IN_REGS ? bv[j] : (act[j] ? __ldg(bsys + comm.grow(j)) : 0.0);
      q[j] = act[j] ? bj - q[j] : 0.0;
      tr[0] += q[j] * q[j];
    }
    comm.template sum<1>(tr);
    return tr[0];
  };

  // Iteration schedules (DESIGN.md "Kernels" 5).  ROUNDS == 3 (register-
  // limited 2-CTA/SM kernels): r^.v | t.s, t.t, ||s|| | ||r||, r^.r -- ||s||
  // for stop test 2 is reduced with t.s and t.t after the second SpMV, which
  // is discarded (speculative) when the test fires.  ROUNDS == 2 (latency-
  // limited persistent kernel): two reduction rounds per iteration.
  //  * ||s|| (stop test 2) is reduced together with t.s and t.t after the
  //    second SpMV; when it fires, that SpMV was speculative and t is
  //    discarded;
  //  * rho_{i+1} = r^.r_{i+1} = r^.s - omega r^.t (exact algebra for
  //    r_{i+1} = s - omega t) comes from the same round;
  //  * ||r_{i+1}|| (stop test 1) is reduced together with r^.v after the next
  //    first SpMV; when it fires, that SpMV was speculative and the exit is
  //    reported at loop index i+1 with x untouched, as in Alg. 1.
  // x, the iteration count and the exit test are those of Alg. 1; only the
  // rounding of rho differs (fp sums in another order).
  int it = 0, st = -1, exit_kind = 0;
  double rho_old = 1.0, alpha = 1.0, omega = 1.0;
  double beta_c = 1.0;  // alpha / (rho_old * omega): beta = rho * beta_c (R2)
  double final_res = -1.0;
  bool have_rnorm = true;  // rnorm holds ||r|| of the current r
  for (;;) {
    exit_kind = 0;
    if constexpr (ROUNDS == 3) {
    while (true) {
      if (below(rnorm2)) { exit_kind = 1; break; }        // stop test 1
      if (it >= P.maxiter) break;
      if (bad(rho)) { st = SYS_BREAKDOWN; break; }
      // R2: beta = (rho / rho') (alpha / omega); the division alpha / (rho'
      // omega) was done before the last reduction, off the critical path
      const double beta = rho * beta_c;
      // a5: p = r + beta (p - omega v); publish p^ = d p for the gather
      double ph[R];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        p[j] = r[j] + beta * (p[j] - omega * v[j]);
        ph[j] = d[j] * p[j];
        comm.publish(j, ph[j]);
      }
      comm.sync();
      // a6: v = A p^
      spmv(ph, v);
      ++it;
      // a7: alpha = rho / (r^ . v)
      double rv[1];
      rv[0] = rows_sum<R>([&](int j) { return rh[j] * v[j]; });
      comm.template sum<1>(rv);
      if (bad(rv[0])) { st = SYS_BREAKDOWN; break; }
      alpha = rho / rv[0];                                 // R3
      // s = r - alpha v ; publish s^ = d s (all SpMV-1 reads finished: the
      // barrier in the reduction above separates them)
      double s[R], sh[R];
      double ts[3];  // t.s, t.t, s.s
#pragma unroll
      for (int j = 0; j < R; ++j) {
        s[j] = r[j] - alpha * v[j];
        sh[j] = d[j] * s[j];
        comm.publish(j, sh[j]);
      }
      comm.sync();  // publish s^
      ts[2] = rows_sum<R>([&](int j) { return s[j] * s[j]; });
      // a9: t = A s^ (speculative when stop test 2 fires)
      double t[R];
      spmv(sh, t);
      ts[0] = rows_sum<R>([&](int j) { return t[j] * s[j]; });
      ts[1] = rows_sum<R>([&](int j) { return t[j] * t[j]; });
      comm.template sum<3>(ts);
      if (below(ts[2])) {                                  // stop test 2
#pragma unroll
        for (int j = 0; j < R; ++j) x[j] = x[j] + alpha * (d[j] * p[j]);
        exit_kind = 2;
        break;
      }
      if (bad(ts[1])) { st = SYS_BREAKDOWN; break; }
      omega = ts[0] / ts[1];
      if (bad(omega)) { st = SYS_BREAKDOWN; break; }
      beta_c = alpha / (rho * omega);  // rho becomes rho' below
      double rr[2];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        x[j] = x[j] + alpha * (d[j] * p[j]) + omega * (d[j] * s[j]);
        r[j] = s[j] - omega * t[j];
      }
      rr[0] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
      rr[1] = rows_sum<R>([&](int j) { return rh[j] * r[j]; });
      rho_old = rho;
      // next iteration's ||r|| and rho = r^ . r in the same single barrier
      comm.template sum<2>(rr);
      rnorm2 = rr[0];
      rho = rr[1];
    }
    } else {
    while (true) {
      if (have_rnorm && rnorm < tau) { exit_kind = 1; break; }  // stop test 1
      if (it >= P.maxiter) break;
      if (bad(rho)) {
        if (!have_rnorm) {  // rare: settle stop test 1 before declaring breakdown
          double rr[1];
          rr[0] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
          comm.template sum<1>(rr);
          rnorm = sqrt(rr[0]);
          have_rnorm = true;
          continue;
        }
        st = SYS_BREAKDOWN;
        break;
      }
      const double beta = (rho * alpha) / (rho_old * omega);  // R2, one division
      // a5: p = r + beta (p - omega v); publish p^ = d p for the gather
      double ph[R];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        p[j] = r[j] + beta * (p[j] - omega * v[j]);
        ph[j] = d[j] * p[j];
        comm.publish(j, ph[j]);
      }
      comm.sync();
      // a6: v = A p^
      spmv(ph, v);
      // a7: r^.v, and ||r|| of the current r for the deferred stop test 1
      double red[2];
      red[0] = rows_sum<R>([&](int j) { return rh[j] * v[j]; });
      red[1] = rows_sum<R>([&](int j) { return r[j] * r[j]; });
      comm.template sum<2>(red);
      if (!have_rnorm) {
        rnorm = sqrt(red[1]);
        if (rnorm < tau) { exit_kind = 1; break; }         // stop test 1, deferred
      }
      have_rnorm = false;
      ++it;
      if (bad(red[0])) { st = SYS_BREAKDOWN; break; }
      alpha = rho / red[0];                                // R3
      // s = r - alpha v ; publish s^ = d s (all SpMV-1 reads finished: the
      // barrier in the reduction above separates them)
      double s[R], sh[R];
#pragma unroll
      for (int j = 0; j < R; ++j) {
        s[j] = r[j] - alpha * v[j];
        sh[j] = d[j] * s[j];
        comm.publish(j, sh[j]);
      }
      comm.sync();  // publish s^
      // a9: t = A s^ (speculative when stop test 2 fires)
      double t[R];
      spmv(sh, t);
      double ts[5];  // t.s, t.t, s.s, r^.s, r^.t
      ts[0] = rows_sum<R>([&](int j) { return t[j] * s[j]; });
      ts[1] = rows_sum<R>([&](int j) { return t[j] * t[j]; });
      ts[2] = rows_sum<R>([&](int j) { return s[j] * s[j]; });
      ts[3] = rows_sum<R>([&](int j) { return rh[j] * s[j]; });
      ts[4] = rows_sum<R>([&](int j) { return rh[j] * t[j]; });
      comm.template sum<5>(ts);
      if (sqrt(ts[2]) < tau) {                             // stop test 2
#pragma unroll
        for (int j = 0; j < R; ++j) x[j] = x[j] + alpha * (d[j] * p[j]);
        exit_kind = 2;
        break;
      }
      if (bad(ts[1])) { st = SYS_BREAKDOWN; break; }
      omega = ts[0] / ts[1];
      if (bad(omega)) { st = SYS_BREAKDOWN; break; }
#pragma unroll
      for (int j = 0; j < R; ++j) {
        x[j] = x[j] + alpha * (d[j] * p[j]) + omega * (d[j] * s[j]);
        r[j] = s[j] - omega * t[j];
      }
      rho_old = rho;
      rho = ts[3] - omega * ts[4];  // r^ . (s - omega t)
    }
    }
    if (st == SYS_BREAKDOWN || exit_kind == 0 || !P.trc) break;
    // ---- a11: true-residual guard (DESIGN R4) -----------------------------
    // (gather buffer is free: its last readers passed a barrier already)
    double q[R];
    const double tr2 = true_residual(q);
    final_res = sqrt(tr2);
    if (final_res < tau || it >= P.maxiter) break;
    // restart from the true residual, keep counting iterations
#pragma unroll
    for (int j = 0; j < R; ++j) {
      r[j] = q[j];
      rh[j] = q[j];
      p[j] = 0.0;
      v[j] = 0.0;
    }
    rho_old = alpha = omega = beta_c = 1.0;
    rnorm = final_res;
    rnorm2 = tr2;
    have_rnorm = true;
    rho = tr2;
    final_res = -1.0;
  }

  if (final_res < 0.0) {
    // final TRUE residual ||b - A x|| (always reported, R4)
    // previous gather readers of this CTA done before the publish overwrites
    // (a CTA barrier: no halo is in flight -- for the cluster plans the last
    // reduction already ordered every CTA's previous SpMV before this point)
    comm.barrier();
    double q[R];
    final_res = sqrt(true_residual(q));
  }
  if (st != SYS_BREAKDOWN) {
    if (P.trc) st = final_res < tau ? SYS_CONVERGED : SYS_MAXITER;
    else st = exit_kind != 0 ? SYS_CONVERGED : SYS_MAXITER;
  }
#pragma unroll
  for (int j = 0; j < R; ++j)
    if (act[j]) xout[comm.grow(j)] = x[j];
  if (comm.leader()) {
    P.iters[sys] = it;
    P.resnorm[sys] = final_res;
    if (P.status) P.status[sys] = static_cast<int8_t>(st);
  }
}

// Grid: one CTA per system (blockIdx.x = system).  Dynamic SMEM layout:
//   [values: smem_vals doubles (PLACE_SMEM only)]
//   [gather: guard | n_pad body | guard doubles]
//   [reduction scratch: 2 * 8 * NWARP doubles] [mbarrier: 8 B]
template <int FMT, int PLACE, int WB, bool EXACT, int R, int NT, int MINB, int KREG = 0>
__global__ void __launch_bounds__(NT, MINB) bicgstab_kernel(const SolveParams P) {
  constexpr int NWARP = NT / 32;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sval = reinterpret_cast<double *>(smem_raw);
  double *sgf = sval + (PLACE == PLACE_SMEM ? P.smem_vals : 0);  // gather incl. guards
  double *sg = sgf + P.guard;                                     // gather body
  double *sred = sgf + P.n_pad + 2 * P.guard;
  uint64_t *mbar = reinterpret_cast<uint64_t *>(sred + 16 * NWARP);
  const unsigned char *gb = reinterpret_cast<const unsigned char *>(sg);

  const int tid = threadIdx.x;
  const int n = P.n;
  const long long sys = blockIdx.x;
  const double *gval = P.values + sys * P.sys_stride;

  // ---- a1: stage this system's values into SMEM (TMA bulk copy) ----------
  bool use_tma = false;
  if (PLACE == PLACE_SMEM) {
    const uint32_t bytes = static_cast<uint32_t>(P.sys_stride * 8);
    use_tma = (bytes % 16u == 0) && ((reinterpret_cast<uintptr_t>(gval) & 15u) == 0);
    if (use_tma) {
      if (tid == 0) {
        mbar_init(mbar, 1);
        fence_mbar_init();
      }
      __syncthreads();
      if (tid == 0) {
        mbar_arrive_expect_tx(mbar, bytes);
        constexpr uint32_t CH = 32768;
        for (uint32_t off = 0; off < bytes; off += CH)
          tma_bulk_g2s(reinterpret_cast<unsigned char *>(sval) + off,
                       reinterpret_cast<const unsigned char *>(gval) + off,
                       bytes - off < CH ? bytes - off : CH, mbar);
      }
    } else {
      // unaligned system block (odd nnz in CSR): plain cooperative copy
      for (long long i = tid; i < P.sys_stride; i += NT) sval[i] = __ldg(gval + i);
    }
  }
  const double *V = (PLACE == PLACE_SMEM) ? sval : gval;
  // zero the gather guards (read, times a zero value, by DIA padding slots);
  // the first gather happens after at least one __syncthreads
  for (int i = tid; i < P.guard; i += NT) {
    sgf[i] = 0.0;
    sg[P.n_pad + i] = 0.0;
  }

  // ---- pattern + right-hand side + initial guess into registers ----------
  RowMeta<FMT, WB, R, KREG> m;
  double x[R], r[R], d[R];
  const double *bsys = P.b + sys * n;
  int dsl[R];
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int row = tid + j * NT;
    m.act[j] = row < n;
#pragma unroll
    for (int k = 0; k < (WB + 1) / 2; ++k) m.cpk[j][k] = 0u;
    m.vbase[j] = (FMT == FMT_CSR) ? 0 : (row < n ? row : n - 1);
    m.vlen[j] = 0;
    m.a0[j] = 0.0;
    dsl[j] = 0;
    r[j] = 0.0;
    x[j] = 0.0;
    if (m.act[j]) {
      if (FMT != FMT_DIA) {
#pragma unroll
        for (int k = 0; k < WB; ++k) {
          if (EXACT || k < P.W) {
            const uint32_t off =
                static_cast<uint32_t>(__ldg(P.ell_col + (size_t)k * n + row)) * 8u;
            m.cpk[j][k >> 1] |= (k & 1) ? (off << 16) : off;
          }
        }
      }
      if (FMT == FMT_CSR) {
        m.vbase[j] = __ldg(P.row_ptr + row);
        m.vlen[j] = __ldg(P.row_ptr + row + 1) - m.vbase[j];
        dsl[j] = __ldg(P.diag_slot + row);
      }
      r[j] = __ldg(bsys + row);  // r holds b until the initial residual is formed
      if (P.x0) x[j] = __ldg(P.x0 + sys * n + row);
    }
  }
  if (PLACE == PLACE_SMEM) {
    if (use_tma) mbar_wait_parity(mbar, 0);
    else __syncthreads();
  }

  // ---- a2: scalar Jacobi d = 1/a_rr (zero diagonal -> 1, DESIGN R11) -----
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int pos = (FMT == FMT_CSR) ? m.vbase[j] + dsl[j] : m.vbase[j];  // ELL/DIA: slot 0
    const double a = m.act[j] ? ((PLACE == PLACE_STREAM) ? __ldg(V + pos) : V[pos]) : 0.0;
    if (FMT != FMT_CSR) m.a0[j] = a;
#pragma unroll
    for (int k = 0; k < (KREG > 0 ? KREG : 0); ++k)  // hybrid: slots 1..KREG -> registers
      m.vreg[j][k] = (PLACE == PLACE_STREAM) ? __ldg(V + m.vbase[j] + (k + 1) * n)
                                             : V[m.vbase[j] + (k + 1) * n];
    d[j] = jacobi_inv(P.precond, a);
  }

  CtaComm<R, NT> comm(sg, sred, m.act);
  bicgstab_core<R, NT, false, 3>(
      P, sys, x, r, d, m.act, r, comm, [&](const double(&own)[R], double(&y)[R]) {
        spmv_rows<FMT, PLACE, WB, EXACT, R, NT, KREG>(V, gb, P, m, own, y, P.n, P.n);
      });
}

// ------------------------------------- persistent, register-resident values --
// PLACE_REGS (DESIGN.md "Kernels" 7): one CTA per SM (up to 255 registers per
// thread) loops over systems claimed from a device work counter.  The
// system's values, b and x0 arrive in SMEM by TMA; each thread moves ITS rows'
// values (all W slots) and b into registers, then thread 0 immediately
// claims the next system and re-arms the same SMEM buffers with TMA, so the
// HBM load of system k+1 overlaps the iterations of system k.  Every SpMV
// then reads only the gathered operands from SMEM: the matrix never touches
// the shared-memory data pipe again.
//   SMEM: [values: smem_vals][b: n_pad][x0: n_pad][gather: guard|n_pad|guard]
//         [reduction scratch: 16*NWARP][mbarrier][next-system slot]
// The counter (ctr[0]) and the finished-CTA count (ctr[1]) reset themselves
// when the last CTA leaves, so consecutive launches on one stream need no
// host-side reset.
template <int FMT, int WB, bool EXACT, int R, int NT>
__global__ void __launch_bounds__(NT, 1) bicgstab_persist_kernel(const SolveParams P,
                                                                 unsigned long long *ctr) {
  static_assert(FMT == FMT_ELL || FMT == FMT_DIA, "register-resident values need ELL/DIA");
  constexpr int NWARP = NT / 32;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sval = reinterpret_cast<double *>(smem_raw);
  double *sb = sval + P.smem_vals;
  double *sx0 = sb + P.n_pad;
  double *sgf = sx0 + P.n_pad;
  double *sg = sgf + P.guard;
  double *sred = sgf + P.n_pad + 2 * P.guard;
  uint64_t *mbar = reinterpret_cast<uint64_t *>(sred + 16 * NWARP);
  volatile long long *s_next = reinterpret_cast<volatile long long *>(mbar + 1);
  const unsigned char *gb = reinterpret_cast<const unsigned char *>(sg);

  const int tid = threadIdx.x;
  const int n = P.n;
  const long long batch = P.batch;
  const uint32_t vbytes = static_cast<uint32_t>(P.sys_stride * 8);
  const uint32_t nbytes = static_cast<uint32_t>(n * 8);

  auto issue = [&](long long s) {  // thread 0: TMA of system s into the staging buffers
    mbar_arrive_expect_tx(mbar, vbytes + nbytes + (P.x0 ? nbytes : 0u));
    const unsigned char *src = reinterpret_cast<const unsigned char *>(P.values + s * P.sys_stride);
    constexpr uint32_t CH = 32768;
    for (uint32_t off = 0; off < vbytes; off += CH)
      tma_bulk_g2s(reinterpret_cast<unsigned char *>(sval) + off, src + off,
                   vbytes - off < CH ? vbytes - off : CH, mbar);
    tma_bulk_g2s(sb, P.b + s * n, nbytes, mbar);
    if (P.x0) tma_bulk_g2s(sx0, P.x0 + s * n, nbytes, mbar);
  };

  // pattern registers (once per CTA) and gather guards.  All W - 1 off-
  // diagonal slots are "register slots" (KREG = WB - 1), so the shared SpMV
  // never dereferences the values buffer.
  RowMeta<FMT, WB, R, WB - 1> m;
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int row = tid + j * NT;
    m.act[j] = row < n;
    m.vbase[j] = row < n ? row : n - 1;
    m.vlen[j] = 0;
    m.a0[j] = 0.0;
#pragma unroll
    for (int k = 0; k < (WB + 1) / 2; ++k) m.cpk[j][k] = 0u;
    if (FMT == FMT_ELL && m.act[j]) {
#pragma unroll
      for (int k = 0; k < WB; ++k) {
        if (EXACT || k < P.W) {
          const uint32_t off = static_cast<uint32_t>(__ldg(P.ell_col + (size_t)k * n + row)) * 8u;
          m.cpk[j][k >> 1] |= (k & 1) ? (off << 16) : off;
        }
      }
    }
  }
  for (int i = tid; i < P.guard; i += NT) {
    sgf[i] = 0.0;
    sg[P.n_pad + i] = 0.0;
  }
  if (tid == 0) {
    mbar_init(mbar, 1);
    fence_mbar_init();
    const long long first = static_cast<long long>(atomicAdd(ctr, 1ull));
    *s_next = first;
    if (first < batch) issue(first);
  }
  __syncthreads();
  long long cur = *s_next;
  uint32_t phase = 0;
  CtaComm<R, NT> comm(sg, sred, m.act);
  while (cur < batch) {
    mbar_wait_parity(mbar, phase);
    phase ^= 1u;
    // ---- registers <- staging buffers -------------------------------------
    double x[R], r[R], d[R], bv[R];
#pragma unroll
    for (int j = 0; j < R; ++j) {
      m.a0[j] = sval[m.vbase[j]];  // slot 0 = diagonal
#pragma unroll
      for (int k = 1; k < WB; ++k)
        m.vreg[j][k - 1] = (EXACT || k < P.W) ? sval[k * n + m.vbase[j]] : 0.0;
      const double a = m.act[j] ? m.a0[j] : 0.0;
      d[j] = jacobi_inv(P.precond, a);
      bv[j] = m.act[j] ? sb[m.vbase[j]] : 0.0;
      r[j] = bv[j];
      x[j] = (P.x0 && m.act[j]) ? sx0[m.vbase[j]] : 0.0;
    }
    __syncthreads();  // every thread is done with the staging buffers
    if (tid == 0) {
      const long long nxt = static_cast<long long>(atomicAdd(ctr, 1ull));
      *s_next = nxt;
      if (nxt < batch) {
        fence_proxy_async_smem();  // generic reads above before the async-proxy writes
        issue(nxt);
      }
    }
    bicgstab_core<R, NT, true, 2>(
        P, cur, x, r, d, m.act, bv, comm,
        [&](const double(&own)[R], double(&y)[R]) {
          spmv_rows<FMT, PLACE_SMEM, WB, EXACT, R, NT, WB - 1>(sval, gb, P, m, own, y, P.n, P.n);
        });
    cur = *s_next;  // written before the core's first barrier
  }
  // ---- self-resetting work counter ------------------------------------------
  __syncthreads();
  if (tid == 0) {
    __threadfence();
    const unsigned long long done = atomicAdd(ctr + 1, 1ull);
    if (done == gridDim.x - 1) {
      atomicExch(ctr, 0ull);
      atomicExch(ctr + 1, 0ull);
    }
  }
}

// ----------------------------------------------- TMEM-resident matrix values --
// PLACE_TMEM (DESIGN.md "Kernels" 9): the register-limited hybrid keeps only
// ELL slots 1..4 in registers and reads slots 5..8 from SMEM.  Tensor memory
// (256 KB per SM, a separate read path measured at ~280 B/clk/SM with 8
// warps -- more than twice the shared-memory data pipe) holds ALL
// off-diagonal values instead: each thread owns its TMEM lane (warp w ->
// lanes 32*(w%4)..+31) and stores its R rows x 8 slots there once per system
// (16 32-bit columns per row; 128 columns per CTA, 2 CTAs per SM).  Every
// SpMV then reads values with tcgen05.ld while the gathered operands come
// from SMEM: the shared-memory pipe carries only gathers, the two publishes
// and the reductions.
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,"
      "%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,"
      "%14,%15,%16};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]),
      "r"(r[8]), "r"(r[9]), "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;");
}
// After tcgen05.wait::ld: make every later use of the loaded registers depend
// on an (empty) volatile asm that is ordered after the wait, so the compiler
// cannot schedule a use before the asynchronous TMEM load completed.  (No
// "memory" clobber on the wait: SMEM loads may be hoisted across it.)
__device__ __forceinline__ void tmem_regs_ready(uint32_t (&r)[16]) {
  asm volatile(""
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]),
                 "+r"(r[6]), "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]),
                 "+r"(r[12]), "+r"(r[13]), "+r"(r[14]), "+r"(r[15]));
}
__device__ __forceinline__ void tmem_wait_st() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}

// Move this thread's rows of the staged values into its TMEM lane: slot 0
// (diagonal) -> a0 register (and d = 1/a0), slots 1..8 -> 16 columns per row.
// `stride` = doubles between two ELL slots in the staging buffer.
template <int R, int WB>
__device__ __forceinline__ void tmem_fill(uint32_t tlane, const double *sval, int stride,
                                          const int (&vrow)[R], const bool (&act)[R],
                                          double (&a0)[R], double (&d)[R], int precond) {
#pragma unroll
  for (int j = 0; j < R; ++j) {
    a0[j] = act[j] ? sval[vrow[j]] : 0.0;
    d[j] = jacobi_inv(precond, a0[j]);
    uint32_t w[16];
#pragma unroll
    for (int k = 1; k < WB; ++k) {
      const double v = act[j] ? sval[k * stride + vrow[j]] : 0.0;
      w[2 * (k - 1)] = static_cast<uint32_t>(__double2loint(v));
      w[2 * (k - 1) + 1] = static_cast<uint32_t>(__double2hiint(v));
    }
    tmem_st16(tlane + 16 * j, w);
  }
  tmem_wait_st();
}

// y = A g with values from TMEM (G rows per tcgen05.ld group, their SMEM
// gathers issued before the wait so both latencies overlap) and DIA gathers.
template <int R, int G, int WB>
__device__ __forceinline__ void tmem_spmv(uint32_t tlane, const unsigned char *gb,
                                          const int (&vrow)[R], const double (&a0)[R],
                                          const bool (&act)[R], const int *doff,
                                          const double (&own)[R], double (&y)[R]) {
#pragma unroll
  for (int j0 = 0; j0 < R; j0 += G) {
    uint32_t w[G][16];
    double gat[G][WB - 1];
#pragma unroll
    for (int g = 0; g < G; ++g) tmem_ld16(tlane + 16 * (j0 + g), w[g]);
#pragma unroll
    for (int g = 0; g < G; ++g)
#pragma unroll
      for (int k = 1; k < WB; ++k)
        gat[g][k - 1] = *reinterpret_cast<const double *>(gb + vrow[j0 + g] * 8 + doff[k]);
    tmem_wait_ld();
#pragma unroll
    for (int g = 0; g < G; ++g) tmem_regs_ready(w[g]);
#pragma unroll
    for (int g = 0; g < G; ++g) {
      const int j = j0 + g;
      double acc = a0[j] * own[j];
#pragma unroll
      for (int k = 1; k < WB; ++k)
        acc = fma(__hiloint2double(static_cast<int>(w[g][2 * k - 1]),
                                   static_cast<int>(w[g][2 * k - 2])),
                  gat[g][k - 1], acc);
      y[j] = act[j] ? acc : 0.0;
    }
  }
}

// One CTA per system; 9-point DIA values (W = 9, slot 0 = diagonal kept in a
// register); NT = 128 threads x R = 8 rows; G rows per TMEM load group.
//   SMEM: [values staging: smem_vals] [gather: guard | n_pad | guard]
//         [reduction scratch: 16*NWARP] [mbarrier] [TMEM base address]
template <int R, int NT, int G, int ROUNDS = 3>
__global__ void __launch_bounds__(NT, 2) bicgstab_tmem_kernel(const SolveParams P) {
  constexpr int NWARP = NT / 32;
  constexpr int WB = 9;
  // 32-bit TMEM columns: 16 per row per thread; warps w and w+4 share lane
  // quarter w%4 and use consecutive column ranges
  constexpr int TCOLS_T = 16 * R;
  constexpr int TCOLS_USED = (NT / 128) * TCOLS_T;
  constexpr int TCOLS = TCOLS_USED <= 32 ? 32 : TCOLS_USED <= 64 ? 64 : TCOLS_USED <= 128 ? 128 : 256;
  static_assert((NT == 128 || NT == 256) && TCOLS_USED <= 256, "TMEM plan: 128 or 256 threads");
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sval = reinterpret_cast<double *>(smem_raw);
  double *sgf = sval + P.smem_vals;
  double *sg = sgf + P.guard;
  double *sred = sgf + P.n_pad + 2 * P.guard;
  uint64_t *mbar = reinterpret_cast<uint64_t *>(sred + 16 * NWARP);
  uint32_t *tbase_s = reinterpret_cast<uint32_t *>(mbar + 1);
  const unsigned char *gb = reinterpret_cast<const unsigned char *>(sg);

  const int tid = threadIdx.x, warp = tid >> 5;
  const int n = P.n;
  const long long sys = blockIdx.x;
  const double *gval = P.values + sys * P.sys_stride;

  // ---- TMEM allocation (warp 0) + TMA staging of the values (thread 0) -----
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s)),
                 "n"(TCOLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 32) {
    mbar_init(mbar, 1);
    fence_mbar_init();
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tlane = *tbase_s + (static_cast<uint32_t>(32 * (warp & 3)) << 16) +
                         static_cast<uint32_t>((warp >> 2) * TCOLS_T);
  const uint32_t vbytes = static_cast<uint32_t>(P.sys_stride * 8);
  const bool use_tma = (vbytes % 16u == 0) && ((reinterpret_cast<uintptr_t>(gval) & 15u) == 0);
  if (use_tma && tid == 0) {
    mbar_arrive_expect_tx(mbar, vbytes);
    constexpr uint32_t CH = 32768;
    for (uint32_t off = 0; off < vbytes; off += CH)
      tma_bulk_g2s(reinterpret_cast<unsigned char *>(sval) + off,
                   reinterpret_cast<const unsigned char *>(gval) + off,
                   vbytes - off < CH ? vbytes - off : CH, mbar);
  }
  if (!use_tma)  // unaligned system block: plain cooperative copy
    for (long long i = tid; i < P.sys_stride; i += NT) sval[i] = __ldg(gval + i);
  for (int i = tid; i < P.guard; i += NT) {
    sgf[i] = 0.0;
    sg[P.n_pad + i] = 0.0;
  }
  bool act[R];
  int vrow[R];
  double x[R], r[R], d[R], a0[R];
  const double *bsys = P.b + sys * n;
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int row = tid + j * NT;
    act[j] = row < n;
    vrow[j] = row < n ? row : n - 1;
    r[j] = act[j] ? __ldg(bsys + row) : 0.0;
    x[j] = (act[j] && P.x0) ? __ldg(P.x0 + sys * n + row) : 0.0;
  }
  if (use_tma) mbar_wait_parity(mbar, 0);
  else __syncthreads();
  // ---- values: diagonal -> register, slots 1..8 -> this thread's TMEM lane --
  tmem_fill<R, WB>(tlane, sval, n, vrow, act, a0, d, P.precond);

  CtaComm<R, NT> comm(sg, sred, act);
  bicgstab_core<R, NT, false, ROUNDS>(
      P, sys, x, r, d, act, r, comm, [&](const double(&own)[R], double(&y)[R]) {
        tmem_spmv<R, G, WB>(tlane, gb, vrow, a0, act, P.doff, own, y);
      });
  // ---- release TMEM -------------------------------------------------------
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(*tbase_s),
                 "n"(TCOLS < 32 ? 32 : TCOLS));
}

// ------------------------------------------ thread-block cluster per system --
// Systems too large for one CTA (n > 1024 rows, e.g. the 63x64 velocity
// grid, n = 4032) are split over a cluster of C CTAs
// (one per 1024 rows, C <= 8), all on one GPC, which exchange through
// distributed shared memory (DSMEM):
//  * each CTA TMA-stages the values of ITS rows (one bulk copy per ELL slot)
//    and keeps them in SMEM / registers as the single-CTA hybrid does;
//  * publishing p^ / s^ writes each row locally and, for the first / last G
//    rows of the CTA (G = max |stencil offset|), also into the halo of the
//    left / right neighbour's gather buffer with st.async, which completes
//    transaction bytes on the neighbour's halo mbarrier: point-to-point
//    synchronisation, no cluster barrier; every SpMV reads only local SMEM;
//  * a reduction st.async's each warp partial into every CTA's scratch and
//    waits on its own mbarrier for the C x NWARP partials, then every
//    thread adds them in the same fixed order (bitwise-identical scalars in
//    the whole cluster, uniform control flow).  cluster.sync() is used only
//    at kernel entry and exit.
template <int R, int NT, int C>
struct ClusterComm {
  static constexpr int NWARP = NT / 32;
  static constexpr int RPC = R * NT;  // rows per CTA
  double *sg;            // local gather body (local row 0)
  double *sred;          // scratch [2][8][C * NWARP]
  uint64_t *hbar;        // halo mbarrier (complete_tx from the neighbours' st.async)
  uint64_t *rbar;        // reduction mbarriers [2]
  uint32_t left_sg, right_sg, left_hbar, right_hbar;  // neighbours (shared::cluster)
  uint32_t sred_s, rbar_s;                             // own shared::cta addresses
  uint32_t hphase = 0, rphase = 0;                     // phase parity bits
  int buf = 0, rank, nloc, G, halo_bytes;
  const bool (&act)[R];
  __device__ __forceinline__ ClusterComm(double *sg_, double *sred_, uint64_t *bars, int rank_,
                                         int n, int G_, const bool (&act_)[R])
      : sg(sg_), sred(sred_), hbar(bars), rbar(bars + 1), rank(rank_),
        nloc(min(RPC, n - rank_ * RPC)), G(G_), act(act_) {
    const uint32_t sg_s = smem_addr(sg), hb_s = smem_addr(hbar);
    left_sg = rank > 0 ? mapa_u32(sg_s, rank - 1) : 0u;
    left_hbar = rank > 0 ? mapa_u32(hb_s, rank - 1) : 0u;
    right_sg = rank < C - 1 ? mapa_u32(sg_s, rank + 1) : 0u;
    right_hbar = rank < C - 1 ? mapa_u32(hb_s, rank + 1) : 0u;
    sred_s = smem_addr(sred);
    rbar_s = smem_addr(rbar);
    // halo rows this CTA receives: the left neighbour's last G rows and the
    // right neighbour's first min(G, its rows) rows
    const int nright = rank < C - 1 ? min(RPC, n - (rank + 1) * RPC) : 0;
    halo_bytes = 8 * ((rank > 0 ? G : 0) + min(G, nright));
  }
  __device__ __forceinline__ int grow(int j) const { return rank * RPC + threadIdx.x + j * NT; }
  __device__ __forceinline__ bool leader() const { return rank == 0 && threadIdx.x == 0; }
  __device__ __forceinline__ void publish(int j, double v) {
    const int i = threadIdx.x + j * NT;
    if (act[j]) {
      sg[i] = v;
      if (i < G && rank > 0)  // my first rows -> left neighbour's right halo
        st_async_f64(left_sg + 8u * static_cast<uint32_t>(RPC + i), v, left_hbar);
      if (i >= nloc - G && rank < C - 1)  // my last rows -> right neighbour's left halo
        st_async_f64(right_sg + 8u * static_cast<uint32_t>(i - nloc), v, right_hbar);
    }
  }
  // local writes: CTA barrier; neighbours' halo rows: their st.async bytes
  // complete this CTA's halo mbarrier.  (Two consecutive publishes are always
  // separated by a reduction that depends on every CTA's SpMV, so a halo is
  // never overwritten while it is still being gathered.)
  // CTA barrier without a halo exchange (no publish preceded it)
  __device__ __forceinline__ void barrier() { __syncthreads(); }
  __device__ __forceinline__ void sync() {
    if (threadIdx.x == 0) mbar_arrive_expect_tx(hbar, static_cast<uint32_t>(halo_bytes));
    __syncthreads();
    mbar_wait_parity_cluster(hbar, hphase);
    hphase ^= 1u;
  }
  template <int K>
  __device__ __forceinline__ void sum(double (&v)[K]) {
    static_assert(K >= 1 && K <= 8, "cluster sum supports 1..8 values");
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    constexpr int KP = K <= 1 ? 1 : K <= 2 ? 2 : K <= 4 ? 4 : 8;
    constexpr int SPAN = 32 / KP;
    double a[KP];
#pragma unroll
    for (int i = 0; i < KP; ++i) a[i] = i < K ? v[i] : 0.0;
#pragma unroll
    for (int cnt = KP, o = 16; cnt > 1; cnt >>= 1, o >>= 1) {
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
    constexpr int P_ = C * NWARP;  // partials per value
    const uint32_t bit = 1u << buf;
    if (threadIdx.x == 0) mbar_arrive_expect_tx(rbar + buf, K * P_ * 8);
    const int q = lane / SPAN;
    if ((lane % SPAN) == 0 && q < K) {
      // every CTA receives every warp partial (one 8-byte st.async each);
      // a round can only start after the previous one completed everywhere
      // (each depends on the last result), so double buffering is enough
      const uint32_t off = static_cast<uint32_t>((buf * 8 * P_ + q * P_ + rank * NWARP + warp) * 8);
#pragma unroll
      for (int r = 0; r < C; ++r)
        st_async_f64(mapa_u32(sred_s + off, r), a[0], mapa_u32(rbar_s + 8u * buf, r));
    }
    mbar_wait_parity_cluster(rbar + buf, (rphase & bit) ? 1u : 0u);
    rphase ^= bit;
    const double *S = sred + buf * (8 * P_);
    double part[K][P_];
#pragma unroll
    for (int k = 0; k < K; ++k) {
      const double2 *S2 = reinterpret_cast<const double2 *>(S + k * P_);
#pragma unroll
      for (int w = 0; w < P_ / 2; ++w) {
        const double2 qq = S2[w];
        part[k][2 * w] = qq.x;
        part[k][2 * w + 1] = qq.y;
      }
    }
#pragma unroll
    for (int k = 0; k < K; ++k) v[k] = tree_sum<P_>(part[k]);
    buf ^= 1;
  }
};

// One system per cluster of C CTAs; DIA (stencil) values, W = 9.
//   SMEM per CTA: [values: W x RPC doubles, slot-major] [gather: G | RPC | G]
//                 [scratch: 2 x 8 x C x NWARP] [mbarrier]
template <int FMT, int WB, bool EXACT, int R, int NT, int KREG, int C, int ROUNDS = 3>
__global__ void __launch_bounds__(NT, 2) bicgstab_cluster_kernel(const SolveParams P) {
  static_assert(FMT == FMT_DIA, "cluster kernel: DIA addressing only");
  constexpr int NWARP = NT / 32;
  constexpr int RPC = R * NT;
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  const int rank = static_cast<int>(cl.block_rank());
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sval = reinterpret_cast<double *>(smem_raw);
  double *sgf = sval + WB * RPC;
  double *sg = sgf + P.guard;
  double *sred = sgf + RPC + 2 * P.guard;
  uint64_t *mbar = reinterpret_cast<uint64_t *>(sred + 16 * C * NWARP);
  const unsigned char *gb = reinterpret_cast<const unsigned char *>(sg);

  const int tid = threadIdx.x;
  const int n = P.n;
  const long long sys = blockIdx.x / C;
  const int row0 = rank * RPC;
  const int nloc = min(RPC, n - row0);  // host guarantees nloc >= 1, even
  // ---- stage this CTA's rows of every ELL slot (TMA, one copy per slot) ----
  // mbar[0]: TMA, mbar[1]: halo rows, mbar[2..3]: reduction buffers
  if (tid == 0) {
    for (int i = 0; i < 4; ++i) mbar_init(mbar + i, 1);
    fence_mbar_init();
  }
  __syncthreads();
  if (tid == 0) {
    const uint32_t bytes = static_cast<uint32_t>(nloc) * 8u;
    mbar_arrive_expect_tx(mbar, bytes * (EXACT ? WB : P.W));
    const double *gsys = P.values + sys * P.sys_stride + row0;
    for (int k = 0; k < (EXACT ? WB : P.W); ++k)
      tma_bulk_g2s(sval + k * RPC, gsys + (long long)k * n, bytes, mbar);
  }
  // zero guards: global boundary halos and the unused tail of the last CTA
  for (int i = tid; i < P.guard; i += NT) {
    if (rank == 0) sgf[i] = 0.0;
    if (rank == C - 1) sg[RPC + i] = 0.0;
  }
  for (int i = nloc + tid; i < RPC; i += NT) sg[i] = 0.0;
  if (rank < C - 1) {  // right-halo entries of rows >= n (next CTA shorter than the reach)
    const int nnext = min(RPC, n - (rank + 1) * RPC);
    for (int i = nnext + tid; i < P.guard; i += NT) sg[RPC + i] = 0.0;
  }

  RowMeta<FMT, WB, R, KREG> m;
  double x[R], r[R], d[R];
  const double *bsys = P.b + sys * n;
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int li = tid + j * NT;
    m.act[j] = li < nloc;
    m.vbase[j] = li < nloc ? li : nloc - 1;
    m.vlen[j] = 0;
    m.a0[j] = 0.0;
    r[j] = m.act[j] ? __ldg(bsys + row0 + li) : 0.0;
    x[j] = (m.act[j] && P.x0) ? __ldg(P.x0 + sys * n + row0 + li) : 0.0;
  }
  cl.sync();  // every CTA of the cluster runs (DSMEM and its mbarriers are live)
  mbar_wait_parity(mbar, 0);
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const double a = m.act[j] ? sval[m.vbase[j]] : 0.0;  // slot 0 = diagonal
    m.a0[j] = a;
    d[j] = jacobi_inv(P.precond, a);
#pragma unroll
    for (int k = 0; k < (KREG > 0 ? KREG : 0); ++k) m.vreg[j][k] = sval[m.vbase[j] + (k + 1) * RPC];
  }
  ClusterComm<R, NT, C> comm(sg, sred, mbar + 1, rank, n, P.guard, m.act);
  bicgstab_core<R, NT, false, ROUNDS>(
      P, sys, x, r, d, m.act, r, comm, [&](const double(&own)[R], double(&y)[R]) {
        spmv_rows<FMT, PLACE_SMEM, WB, EXACT, R, NT, KREG>(sval, gb, P, m, own, y, nloc, RPC);
      });
  cl.sync();  // peers may write into this CTA's SMEM until they are done
}

// Cluster plan with TMEM-resident values (the default for 1024 < n <= 8192
// 9-point stencils): the cluster exchange of bicgstab_cluster_kernel plus the
// TMEM value path of bicgstab_tmem_kernel.
//   SMEM per CTA: [values staging: 9 x RPC] [gather: G | RPC | G]
//                 [scratch: 2 x 8 x C x NWARP] [4 mbarriers] [TMEM base]
template <int R, int NT, int C>
__global__ void __launch_bounds__(NT, 2) bicgstab_cluster_tmem_kernel(const SolveParams P) {
  constexpr int NWARP = NT / 32;
  constexpr int RPC = R * NT;
  constexpr int WB = 9;
  constexpr int TCOLS = 16 * R;
  static_assert(NT == 128 && TCOLS <= 256, "one warp per TMEM lane quarter");
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  const int rank = static_cast<int>(cl.block_rank());
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double *sval = reinterpret_cast<double *>(smem_raw);
  double *sgf = sval + WB * RPC;
  double *sg = sgf + P.guard;
  double *sred = sgf + RPC + 2 * P.guard;
  uint64_t *mbar = reinterpret_cast<uint64_t *>(sred + 16 * C * NWARP);
  uint32_t *tbase_s = reinterpret_cast<uint32_t *>(mbar + 4);
  const unsigned char *gb = reinterpret_cast<const unsigned char *>(sg);

  const int tid = threadIdx.x, warp = tid >> 5;
  const int n = P.n;
  const long long sys = blockIdx.x / C;
  const int row0 = rank * RPC;
  const int nloc = min(RPC, n - row0);
  // mbar[0]: TMA, mbar[1]: halo rows, mbar[2..3]: reduction buffers
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_addr(tbase_s)),
                 "n"(TCOLS));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 32) {
    for (int i = 0; i < 4; ++i) mbar_init(mbar + i, 1);
    fence_mbar_init();
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tlane = *tbase_s + (static_cast<uint32_t>(32 * (warp & 3)) << 16);
  if (tid == 0) {
    const uint32_t bytes = static_cast<uint32_t>(nloc) * 8u;
    mbar_arrive_expect_tx(mbar, bytes * WB);
    const double *gsys = P.values + sys * P.sys_stride + row0;
    for (int k = 0; k < WB; ++k) tma_bulk_g2s(sval + k * RPC, gsys + (long long)k * n, bytes, mbar);
  }
  for (int i = tid; i < P.guard; i += NT) {
    if (rank == 0) sgf[i] = 0.0;
    if (rank == C - 1) sg[RPC + i] = 0.0;
  }
  for (int i = nloc + tid; i < RPC; i += NT) sg[i] = 0.0;
  if (rank < C - 1) {
    const int nnext = min(RPC, n - (rank + 1) * RPC);
    for (int i = nnext + tid; i < P.guard; i += NT) sg[RPC + i] = 0.0;
  }
  bool act[R];
  int vrow[R];
  double x[R], r[R], d[R], a0[R];
  const double *bsys = P.b + sys * n;
#pragma unroll
  for (int j = 0; j < R; ++j) {
    const int li = tid + j * NT;
    act[j] = li < nloc;
    vrow[j] = li < nloc ? li : nloc - 1;
    r[j] = act[j] ? __ldg(bsys + row0 + li) : 0.0;
    x[j] = (act[j] && P.x0) ? __ldg(P.x0 + sys * n + row0 + li) : 0.0;
  }
  cl.sync();  // every CTA of the cluster runs (DSMEM and its mbarriers are live)
  mbar_wait_parity(mbar, 0);
  tmem_fill<R, WB>(tlane, sval, RPC, vrow, act, a0, d, P.precond);
  ClusterComm<R, NT, C> comm(sg, sred, mbar + 1, rank, n, P.guard, act);
  bicgstab_core<R, NT, false, 3>(
      P, sys, x, r, d, act, r, comm, [&](const double(&own)[R], double(&y)[R]) {
        tmem_spmv<R, 4, WB>(tlane, gb, vrow, a0, act, P.doff, own, y);
      });
  asm volatile("tcgen05.fence::before_thread_sync;");
  cl.sync();  // peers may write into this CTA's SMEM until they are done
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(*tbase_s),
                 "n"(TCOLS));
}

// -------------------------------------------------- standalone batched SpMV --
// y_i = A_i x_i (Fig. 7).  One CTA per system; x_i is
// staged into SMEM for the gather, values stream from global (coalesced for
// ELL: consecutive rows of one slot are contiguous).  `cols` is the column
// table of the handle's format ([W][n]; CSR: k-th entry of the row).
template <int FMT, int NT>
__global__ void __launch_bounds__(NT) spmv_kernel(const double *__restrict__ values,
                                                  const double *__restrict__ xin,
                                                  double *__restrict__ y,
                                                  const int32_t *__restrict__ cols,
                                                  const int32_t *__restrict__ row_ptr, int n,
                                                  int W, long long sys_stride) {
  extern __shared__ __align__(16) double sx[];
  const long long sys = blockIdx.x;
  const double *V = values + sys * sys_stride;
  for (int i = threadIdx.x; i < n; i += NT) sx[i] = __ldg(xin + sys * n + i);
  __syncthreads();
  for (int row = threadIdx.x; row < n; row += NT) {
    double acc = 0.0;
    if (FMT == FMT_CSR) {
      const int a = __ldg(row_ptr + row), e = __ldg(row_ptr + row + 1);
      for (int q = a; q < e; ++q)
        acc = fma(__ldg(V + q), sx[__ldg(cols + (size_t)(q - a) * n + row)], acc);
    } else {
      for (int k = 0; k < W; ++k)
        acc = fma(__ldg(V + (size_t)k * n + row), sx[__ldg(cols + (size_t)k * n + row)], acc);
    }
    y[sys * n + row] = acc;
  }
}

// ------------------------------------------------------- CSR -> ELL values --
static __global__ void csr_to_ell_kernel(const double *__restrict__ csr, double *__restrict__ ell,
                                  const int32_t *__restrict__ src, long long slots, int nnz,
                                  long long total) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const long long sys = i / slots, pos = i - sys * slots;
    const int e = __ldg(src + pos);
    ell[i] = e >= 0 ? __ldg(csr + sys * nnz + e) : 0.0;
  }
}

// -------------------------------------------------- SMEM bandwidth probe --
// Every thread streams conflict-free 32-byte shared loads; the sum is kept
// live through a conditional store.  bytes = grid * NT * iters * 4 * 32.
template <int NT>
__global__ void __launch_bounds__(NT) smem_probe_kernel(int iters, double *sink,
                                                        long long *cycles) {
  __shared__ __align__(32) double4 buf[1024];
  for (int i = threadIdx.x; i < 1024; i += NT)
    buf[i] = make_double4(i, i + 1, i + 2, i + 3);
  __syncthreads();
  const long long c0 = clock64();
  double a0 = 0, a1 = 0, a2 = 0, a3 = 0;
  int idx = threadIdx.x;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const double4 q = buf[(idx + u * NT) & 1023];
      a0 += q.x;
      a1 += q.y;
      a2 += q.z;
      a3 += q.w;
    }
    idx = (idx + 32) & 1023;
  }
  const long long c1 = clock64();
  const double s = a0 + a1 + a2 + a3;
  if (s == -1.0) sink[blockIdx.x] = s;
  if (threadIdx.x == 0) cycles[blockIdx.x] = c1 - c0;
}

// Measured FP64 roofline denominator ("measure it with a DFMA
// loop"): every thread runs 8 independent DFMA chains (enough in flight to
// cover the pipe latency), `iters` x 8 DFMA = 16 x iters flop per thread.
template <int NT>
__global__ void __launch_bounds__(NT) fp64_probe_kernel(int iters, double seed, double *sink,
                                                        long long *cycles) {
  double a[8];
#pragma unroll
  for (int k = 0; k < 8; ++k) a[k] = seed * (threadIdx.x + k);
  const double m = 1.0 - 1e-16 * seed, c = 1e-20 * seed;
  const long long c0 = clock64();
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int k = 0; k < 8; ++k) a[k] = fma(a[k], m, c);
  }
  const long long c1 = clock64();
  double s = 0.0;
#pragma unroll
  for (int k = 0; k < 8; ++k) s += a[k];
  if (s == -1.0) sink[blockIdx.x] = s;
  if (threadIdx.x == 0) cycles[blockIdx.x] = c1 - c0;
}

}  // namespace bsolve
