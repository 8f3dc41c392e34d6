// k_line.cu -- instantiations of the line-tiled TMEM kernel for 2D 9-point
// stencils (line_kernel.cuh): grid widths NX with 8 | rows per thread, G rows
// per TMEM load group.  NX = 32 is the paper's 32 x 31 velocity grid
// (PAPER.md:519-530); NX = 31 its transpose (tests).  Launched from bsolve.cu.
#include "line3_kernel.cuh"
#include "line_kernel.cuh"
#include "variants.h"

using namespace bsolve;

#define LSMEM_(NX, R) ((R * LineGeom<NX, 1024 / R, R>::S + 16 * (1024 / R / 32)) * 8 + 16)
#define LV_(NX, R, G) {NX, R, G, SOLVER_BICGSTAB, LSMEM_(NX, R), 3, \
                       (solve_fn)bicgstab_tmem_line_kernel<NX, R, G, SOLVER_BICGSTAB>, 2}
// 3 CTAs per SM (line3_kernel.cuh, the default plan): r^, a_ii in TMEM, x in
// SMEM, <= 168 registers, 3 partial sums per SpMV row.  RD = 2: rho and ||r||
// from the omega round (R29, default); RD = 3: the literal 3-round
// schedule of bicgstab_core.  (Measured and removed: double-buffered TMEM rows,
// one FMA chain per row, a shallower one-value reduction, gathers one row
// ahead -- DESIGN.md perf log.)
#define LV3_(NX, RD) {NX, 8, 3, SOLVER_BICGSTAB, Line3Geom<NX>::SMEM_BYTES, RD, \
                      (solve_fn)bicgstab_line3_kernel<NX, RD>, 3, 0}
// block-Jacobi preconditioner, one 8-row tridiagonal block per thread (f3, R30)
#define LV3B_(NX) {NX, 8, 3, SOLVER_BICGSTAB, Line3Geom<NX, 1>::SMEM_BYTES, 2, \
                   (solve_fn)bicgstab_line3_kernel<NX, 2, 1>, 3, 1}
// two reduction rounds per iteration (deferred stop test 1, algebraic rho)
#define LV2_(NX, R, G) {NX, R, G, SOLVER_BICGSTAB, LSMEM_(NX, R), 2, \
                        (solve_fn)bicgstab_tmem_line_kernel<NX, R, G, SOLVER_BICGSTAB, 2, 2>, 2}
// GMRES: + the Krylov basis and the triangular factor in SMEM
#define LVG_(NX, R, G) {NX, R, G, SOLVER_GMRES,                                          \
                        LSMEM_(NX, R) + (kMaxRestart * 1024 + kMaxRestart * kMaxRestart) * 8, 0, \
                        (solve_fn)bicgstab_tmem_line_kernel<NX, R, G, SOLVER_GMRES>, 2}
static const LVariant kLVariants[] = {LV_(32, 8, 2),  LV_(32, 8, 4),  LV_(32, 4, 2),
                                      LV_(32, 4, 4),  LV_(31, 8, 4),  LV_(31, 4, 2),
                                      LVG_(32, 8, 2), LVG_(31, 8, 2), LV2_(32, 8, 4),
                                      LV2_(31, 8, 4), LV3_(32, 2),    LV3_(31, 2),
                                      LV3_(32, 3),    LV3_(31, 3),    LV3B_(32),
                                      LV3B_(31)};

const LVariant *variants_line(int *count) {
  *count = (int)(sizeof(kLVariants) / sizeof(kLVariants[0]));
  return kLVariants;
}

// persistent line-tiled kernel (TMA prefetch of the next system), 8 rows x 128 threads
persist_fn variant_line_persist(int nx, int *smem_bytes, int smem_vals, int n_pad) {
  if (nx == 32) {
    *smem_bytes = line_persist_smem<32, 8, 4>(smem_vals, n_pad);
    return (persist_fn)bicgstab_tmem_line_persist_kernel<32, 8, 4>;
  }
  if (nx == 31) {
    *smem_bytes = line_persist_smem<31, 8, 4>(smem_vals, n_pad);
    return (persist_fn)bicgstab_tmem_line_persist_kernel<31, 8, 4>;
  }
  return nullptr;
}

// line-tiled TMEM plan on a cluster of C CTAs (n > 1024), NX = 64 (63 x 64 grid)
#define LCV_(NX, C) {C, NX, 3, (solve_fn)bicgstab_tmem_line_cluster_kernel<NX, C>}
static const CVariant kLCVariants[] = {LCV_(64, 2), LCV_(64, 3), LCV_(64, 4), LCV_(64, 5),
                                       LCV_(64, 6), LCV_(64, 7), LCV_(64, 8)};
const CVariant *variants_cluster_line(int *count, int *smem_bytes) {
  *count = (int)(sizeof(kLCVariants) / sizeof(kLCVariants[0]));
  *smem_bytes = line_cluster_smem<64, 8>();
  return kLCVariants;
}

// 3-CTA line-tiled plan on a cluster of C CTAs (line3_kernel.cuh), NX = 64
// rounds field: 2 = halo state kept per CTA, 2 exchanges per iteration (default);
// 1 = halo by bulk copies, 4 exchanges; 0 = cluster barriers (reference)
#define L3CV_(NX, C, M) {C, NX, M, (solve_fn)bicgstab_line3_cluster_kernel<NX, C, M >= 1, M == 2>}
static const CVariant kL3CVariants[] = {
    L3CV_(64, 2, 2), L3CV_(64, 3, 2), L3CV_(64, 4, 2), L3CV_(64, 5, 2), L3CV_(64, 6, 2),
    L3CV_(64, 7, 2), L3CV_(64, 8, 2), L3CV_(64, 2, 1), L3CV_(64, 3, 1), L3CV_(64, 4, 1),
    L3CV_(64, 5, 1), L3CV_(64, 6, 1), L3CV_(64, 7, 1), L3CV_(64, 8, 1), L3CV_(64, 2, 0),
    L3CV_(64, 3, 0), L3CV_(64, 4, 0), L3CV_(64, 5, 0), L3CV_(64, 6, 0), L3CV_(64, 7, 0),
    L3CV_(64, 8, 0)};
const CVariant *variants_cluster_line3(int *count, int *smem_bytes) {
  *count = (int)(sizeof(kL3CVariants) / sizeof(kL3CVariants[0]));
  *smem_bytes = Line3ClusterGeom<64, 8>::SMEM_BYTES;
  return kL3CVariants;
}
