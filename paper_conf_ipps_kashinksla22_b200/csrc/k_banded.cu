// k_banded.cu -- instantiations of the batched banded LU kernel (banded.cuh,
// SURVEY.md 8(f) f4), one per padded bandwidth KL = KU.  A pattern with
// kl, ku <= K runs on the K instance: the extra window rows/columns hold
// exact zeros, which never win the pivot search (ties keep the first index)
// and add exact zeros in the updates, so the result is that of the exact-
// bandwidth algorithm (R25).  Launched from bsolve.cu.
#include "banded.cuh"
#include "variants.h"

using namespace bband;

#define BV_(K, MINB, MINB_SPLIT, WARP)                                            \
  {K, Geo<K, K>::NT, Geo<K, K>::NTF - Geo<K, K>::W - 1, Geo<K, K>::smem_bytes,    \
   (banded_fn)banded_lu_kernel<K, K, MINB>, Geo<K, K>::NTF,                       \
   (banded_fn)banded_lu_kernel<K, K, MINB_SPLIT, true>,                          \
   (banded_fn)banded_backsub_kernel<K, K>, WARP}
#define BW_(K) (banded_fn) banded_lu_warp_kernel<K, K, 8>, WGeo<K, K>::smem_bytes
#define BW_NONE nullptr, 0
static const BVariant kBVariants[] = {BV_(4, 8, 8, BW_(4)), BV_(8, 8, 8, BW_(8)),
                                      BV_(16, 5, 8, BW_(16)), BV_(33, 5, 8, BW_(33)),
                                      BV_(65, 1, 1, BW_NONE)};

const BVariant *variants_banded(int *count) {
  *count = (int)(sizeof(kBVariants) / sizeof(kBVariants[0]));
  return kBVariants;
}
