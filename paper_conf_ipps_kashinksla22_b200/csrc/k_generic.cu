// k_generic.cu -- instantiations of the per-system-CTA kernel bicgstab_kernel
// (formats CSR / ELL / DIA x placements SMEM / STREAM x rows per thread x CTA
// size, and the 128-thread register hybrid).  Launched from bsolve.cu.
#include "kernels.cuh"
#include "variants.h"

using namespace bsolve;

#define V_(F, PL, WB, EX, R, NT, MB) \
  {F, PL, WB, EX, R, NT, 0, (solve_fn)bicgstab_kernel<F, PL, WB, EX, R, NT, MB>}
#define VK_(F, R, NT, MB, KR) \
  {F, PLACE_SMEM, 9, true, R, NT, KR, (solve_fn)bicgstab_kernel<F, PLACE_SMEM, 9, true, R, NT, MB, KR>}
#define V_FP(WB, EX, R, NT, MB)                                                         \
  V_(FMT_ELL, PLACE_SMEM, WB, EX, R, NT, MB), V_(FMT_ELL, PLACE_STREAM, WB, EX, R, NT, MB), \
      V_(FMT_DIA, PLACE_SMEM, WB, EX, R, NT, MB), V_(FMT_DIA, PLACE_STREAM, WB, EX, R, NT, MB), \
      V_(FMT_CSR, PLACE_SMEM, WB, EX, R, NT, MB), V_(FMT_CSR, PLACE_STREAM, WB, EX, R, NT, MB)

// W = 9 (the paper's 9-point stencil) gets exact-width variants; any other
// width <= 16 runs the generic WB = 16 variants with a per-slot test.
static const Variant kVariants[] = {
    V_FP(9, true, 1, 256, 2),   V_FP(9, true, 2, 256, 2),   V_FP(9, true, 4, 256, 2),
    V_FP(9, true, 4, 512, 1),   V_FP(16, false, 1, 256, 2), V_FP(16, false, 2, 256, 2),
    V_FP(16, false, 4, 256, 2), V_FP(16, false, 4, 512, 1),
    // hybrid: 128 threads x 8 rows, 2 CTAs/SM, slots 1..KREG in registers
    VK_(FMT_DIA, 8, 128, 2, 0), VK_(FMT_DIA, 8, 128, 2, 2), VK_(FMT_DIA, 8, 128, 2, 4),
    VK_(FMT_DIA, 8, 128, 2, 6), VK_(FMT_DIA, 8, 128, 2, 8),
};

const Variant *variants_generic(int *count) {
  *count = (int)(sizeof(kVariants) / sizeof(kVariants[0]));
  return kVariants;
}
