// k_line_generic.cu -- generic-width instances of the 3-CTA line-tiled kernel
// (line3_kernel.cuh): any 2D 9-point (or 5-point) stencil grid of width
// NX <= kLineNXG with n <= 1024 runs the line plan.  One instance per
// B = NX mod 8 (the plane pattern of the neighbour lines); A = NX / 8 is a
// run-time column shift (SolveParams::line_a).  The compile-time widths of
// the paper's grid (k_line.cu: NX = 32, 31) stay the preferred instances.
// Launched from bsolve.cu.
#include "line3_kernel.cuh"
#include "line_kernel.cuh"
#include "variants.h"

using namespace bsolve;

static constexpr int kLineNXG = 120;  // widest grid: guards of 17 columns per plane side
#define LVX_(B) {B, 8, 3, SOLVER_BICGSTAB, Line3Geom<kLineNXG>::SMEM_BYTES, 2, \
                 (solve_fn)bicgstab_line3_kernel<B, 2, 0, kLineNXG>, 3, 0, kLineNXG}
// block-Jacobi (R30): the 8-row blocks are tridiagonal for widths >= 9
#define LVXB_(B) {B, 8, 3, SOLVER_BICGSTAB, Line3Geom<kLineNXG, 1>::SMEM_BYTES, 2, \
                  (solve_fn)bicgstab_line3_kernel<B, 2, 1, kLineNXG>, 3, 1, kLineNXG}
// GMRES(m) on the 2-CTA line kernel (+ the Krylov basis and R factor in SMEM)
#define LVXG_(B) {B, 8, 2, SOLVER_GMRES,                                                     \
                  ((8 * LineGeom<kLineNXG, 128, 8>::S + 16 * 4) * 8 + 16) +                   \
                      (kMaxRestart * 1024 + kMaxRestart * kMaxRestart) * 8, 0,               \
                  (solve_fn)bicgstab_tmem_line_kernel<B, 8, 2, SOLVER_GMRES, 2, 3, kLineNXG>, \
                  2, 0, kLineNXG}
static const LVariant kLXVariants[] = {
    LVX_(0),  LVX_(1),  LVX_(2),  LVX_(3),  LVX_(4),  LVX_(5),  LVX_(6),  LVX_(7),
    LVXB_(0), LVXB_(1), LVXB_(2), LVXB_(3), LVXB_(4), LVXB_(5), LVXB_(6), LVXB_(7),
    LVXG_(0), LVXG_(1), LVXG_(2), LVXG_(3), LVXG_(4), LVXG_(5), LVXG_(6), LVXG_(7)};

const LVariant *variants_line_generic(int *count) {
  *count = (int)(sizeof(kLXVariants) / sizeof(kLXVariants[0]));
  return kLXVariants;
}
