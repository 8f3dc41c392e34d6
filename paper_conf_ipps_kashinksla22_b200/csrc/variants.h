// variants.h -- kernel variant tables shared by the host plan (bsolve.cu) and
// the translation units that instantiate the kernels (k_*.cu).  Splitting the
// instantiations over several .cu files lets the build compile them in
// parallel; the tables hold host-side kernel stubs, launched from bsolve.cu.
#pragma once
#include <cstdint>

namespace bsolve {
struct SolveParams;
}
namespace bband {
struct BandParams;
}

typedef void (*solve_fn)(const bsolve::SolveParams);
typedef void (*banded_fn)(const bband::BandParams);
typedef void (*persist_fn)(const bsolve::SolveParams, unsigned long long *);

// per-system-CTA kernels (bicgstab_kernel), k_generic.cu
struct Variant {
  int fmt, place, wb;
  bool exact;
  int r, nt;
  int kreg;  // off-diagonal ELL slots held in registers (hybrid variants)
  solve_fn fn;
};
// persistent register-resident kernels (PLACE_REGS), k_special.cu
struct PVariant {
  int fmt, r;
  persist_fn fn;
};
// one system per thread-block cluster (PLACE_CLUSTER), k_special.cu
struct CVariant {
  int c, kreg, rounds;
  solve_fn fn;
};
// TMEM-resident values (PLACE_TMEM), k_special.cu
struct TVariant {
  int nt, r, g, rounds;
  solve_fn fn;
};
// TMEM + line-tiled 9-point stencil (PLACE_TMEM, kernel_mode 4), k_line.cu
struct LVariant {
  int nx, r, g;  // grid width, rows per thread (CTA = 1024 / r threads), TMEM load group
  int solver;    // SOLVER_BICGSTAB or SOLVER_GMRES
  int smem_bytes;  // dynamic SMEM of one CTA (gather planes + scratch + TMEM slot)
  int rounds;      // BiCGSTAB reduction rounds per iteration (3, or 2: algebraic rho)
  solve_fn fn;
  int ctas;        // resident CTAs per SM the kernel is built for (launch bounds)
  int pre;         // 0: scalar preconditioner (Jacobi / none), 1: block-Jacobi (8 rows)
  int nxmax;       // 0: grid width nx; > 0: any width = nx (mod 8) up to nxmax (generic)
};

// batched banded LU (dgbsv analogue), k_banded.cu
struct BVariant {
  int kb;          // padded bandwidth: serves patterns with kl, ku <= kb
  int nt;          // threads per CTA
  int max_entries; // loader lanes: rows with at most this many entries - 1
  int smem_bytes;  // dynamic SMEM (row ring)
  banded_fn fn;    // factor + back-substitution warps in one kernel
  int nt_split;    // split mode: factor-only CTA size
  banded_fn fn_split;    // split mode: factorisation (U, y to a per-system workspace)
  banded_fn fn_backsub;  // split mode: one warp per system back substitution
  banded_fn fn_warp;     // split mode: one warp per system factorisation (nullptr: none)
  int smem_warp;         // its dynamic SMEM
};

const Variant *variants_generic(int *count);
const PVariant *variants_persist(int *count);
const CVariant *variants_cluster(int *count);
const CVariant *variants_cluster_tmem(int *count);
// 3-CTA line-tiled plan on a cluster (line3_kernel.cuh), kreg = grid width NX
const CVariant *variants_cluster_line3(int *count, int *smem_bytes);
// the same with block-Jacobi (PRE = 1, halo exchange)
const CVariant *variants_cluster_line3_bj(int *count, int *smem_bytes);
const TVariant *variants_tmem(int *count);
const LVariant *variants_line(int *count);
// generic-width 3-CTA line kernels (nxmax > 0), k_line_generic.cu
const LVariant *variants_line_generic(int *count);
const BVariant *variants_banded(int *count);
