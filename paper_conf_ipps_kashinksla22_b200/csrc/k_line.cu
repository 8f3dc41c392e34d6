// k_line.cu -- instantiations of the line-tiled TMEM kernels for 2D 9-point
// stencils: the 3-CTA kernel (line3_kernel.cuh; default, block-Jacobi, and on
// a cluster for n > 1024) and the 2-CTA kernel (line_kernel.cuh; GMRES, and
// BiCGSTAB via BSOLVE_LINE_CTAS=2).  NX = 32 is the paper's 32 x 31 velocity
// grid, NX = 31 its transpose, NX = 64 the 63 x 64 grid of
// BASELINE configs[4].  Launched from bsolve.cu.
#include "line3_kernel.cuh"
#include "line_kernel.cuh"
#include "variants.h"

using namespace bsolve;

#define LSMEM_(NX, R) ((R * LineGeom<NX, 1024 / R, R>::S + 16 * (1024 / R / 32)) * 8 + 16)
#define LV_(NX, R, G) {NX, R, G, SOLVER_BICGSTAB, LSMEM_(NX, R), 3, \
                       (solve_fn)bicgstab_tmem_line_kernel<NX, R, G, SOLVER_BICGSTAB>, 2, 0, 0}
// 3 CTAs per SM (line3_kernel.cuh, the default plan): r^, a_ii in TMEM, x in
// SMEM, <= 168 registers, 3 partial sums per SpMV row.  RD = 2: rho and ||r||
// from the omega round (R29, default); RD = 3: the literal 3-round
// schedule of bicgstab_core.  (Measured and removed: double-buffered TMEM rows,
// one FMA chain per row, a shallower one-value reduction, gathers one row
// ahead -- DESIGN.md perf log.)
#define LV3_(NX, RD) {NX, 8, 3, SOLVER_BICGSTAB, Line3Geom<NX>::SMEM_BYTES, RD, \
                      (solve_fn)bicgstab_line3_kernel<NX, RD>, 3, 0, 0}
// block-Jacobi preconditioner, one 8-row tridiagonal block per thread (f3, R30)
#define LV3B_(NX) {NX, 8, 3, SOLVER_BICGSTAB, Line3Geom<NX, 1>::SMEM_BYTES, 2, \
                   (solve_fn)bicgstab_line3_kernel<NX, 2, 1>, 3, 1, 0}
// GMRES: + the Krylov basis and the triangular factor in SMEM
#define LVG_(NX, R, G) {NX, R, G, SOLVER_GMRES,                                          \
                        LSMEM_(NX, R) + (kMaxRestart * 1024 + kMaxRestart * kMaxRestart) * 8, 0, \
                        (solve_fn)bicgstab_tmem_line_kernel<NX, R, G, SOLVER_GMRES>, 2, 0, 0}
static const LVariant kLVariants[] = {LV_(32, 8, 4),  LV_(31, 8, 4),  LVG_(32, 8, 2),
                                      LVG_(31, 8, 2), LV3_(32, 2),    LV3_(31, 2),
                                      LV3_(32, 3),    LV3_(31, 3),    LV3B_(32),
                                      LV3B_(31)};

const LVariant *variants_line(int *count) {
  *count = (int)(sizeof(kLVariants) / sizeof(kLVariants[0]));
  return kLVariants;
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
// block-Jacobi (PRE = 1) on the cluster plan: halo exchange (rounds field 1)
#define L3CVB_(NX, C) {C, NX, 1, (solve_fn)bicgstab_line3_cluster_kernel<NX, C, 1, 0, 2, 1>}
static const CVariant kL3CBVariants[] = {L3CVB_(64, 2), L3CVB_(64, 3), L3CVB_(64, 4),
                                         L3CVB_(64, 5), L3CVB_(64, 6), L3CVB_(64, 7),
                                         L3CVB_(64, 8)};
const CVariant *variants_cluster_line3_bj(int *count, int *smem_bytes) {
  *count = (int)(sizeof(kL3CBVariants) / sizeof(kL3CBVariants[0]));
  *smem_bytes = Line3ClusterGeom<64, 8, 1>::SMEM_BYTES;
  return kL3CBVariants;
}
const CVariant *variants_cluster_line3(int *count, int *smem_bytes) {
  *count = (int)(sizeof(kL3CVariants) / sizeof(kL3CVariants[0]));
  *smem_bytes = Line3ClusterGeom<64, 8>::SMEM_BYTES;
  return kL3CVariants;
}
