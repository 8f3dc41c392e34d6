// k_special.cu -- instantiations of the persistent register-resident kernel
// (PLACE_REGS), the thread-block-cluster kernels (PLACE_CLUSTER) and the
// TMEM-resident kernels with strided row ownership (PLACE_TMEM).  Launched
// from bsolve.cu.
#include "kernels.cuh"
#include "variants.h"

using namespace bsolve;

#define PV_(F, R) {F, R, (persist_fn)bicgstab_persist_kernel<F, 9, true, R, 256>}
static const PVariant kPVariants[] = {PV_(FMT_DIA, 1), PV_(FMT_DIA, 2), PV_(FMT_DIA, 4),
                                      PV_(FMT_ELL, 1), PV_(FMT_ELL, 2), PV_(FMT_ELL, 4)};

#define CV_(C, KR, RD) \
  {C, KR, RD, (solve_fn)bicgstab_cluster_kernel<FMT_DIA, 9, true, 8, 128, KR, C, RD>}
#define CV_ALLC(KR, RD) \
  CV_(2, KR, RD), CV_(3, KR, RD), CV_(4, KR, RD), CV_(5, KR, RD), CV_(6, KR, RD), \
      CV_(7, KR, RD), CV_(8, KR, RD)
// (a 2-round schedule spills at 255 registers and measured slower at n = 4032)
static const CVariant kCVariants[] = {CV_ALLC(4, 3), CV_ALLC(2, 3)};
// cluster plan with TMEM-resident values (kreg field unused: -1)
#define CVT_(C) {C, -1, 3, (solve_fn)bicgstab_cluster_tmem_kernel<8, 128, C>}
static const CVariant kCTVariants[] = {CVT_(2), CVT_(3), CVT_(4), CVT_(5),
                                       CVT_(6), CVT_(7), CVT_(8)};

// TMEM-resident values: 128 threads x 8 rows (or 256 x 4), G rows per load group
// (row groups 1, 2 and 256 x 4 geometries measured slower: removed in round 2)
static const TVariant kTVariants[] = {{128, 8, 4, 3, (solve_fn)bicgstab_tmem_kernel<8, 128, 4>}};

#define COUNT_(T) (int)(sizeof(T) / sizeof(T[0]))
const PVariant *variants_persist(int *count) {
  *count = COUNT_(kPVariants);
  return kPVariants;
}
const CVariant *variants_cluster(int *count) {
  *count = COUNT_(kCVariants);
  return kCVariants;
}
const CVariant *variants_cluster_tmem(int *count) {
  *count = COUNT_(kCTVariants);
  return kCTVariants;
}
const TVariant *variants_tmem(int *count) {
  *count = COUNT_(kTVariants);
  return kTVariants;
}
