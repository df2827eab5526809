// magis_eval2_am.cu -- instantiations of the variant-2 kernel with the
// first-argmax output (AM = true), every plan (two teams only on tier 0)
#include "magis_eval2_kernel.cuh"

namespace magis {
const void* eval2_kernel_am(const Plan2& pl, int mode) {
    switch (mode) {
        case 0: return pl.teams == 2 ? kernel_mode<0, 2, true>(pl) : kernel_mode<0, 1, true>(pl);
        case 1: return kernel_mode<1, 1, true>(pl);
        case 2: return kernel_mode<2, 1, true>(pl);
        default: return kernel_mode<3, 1, true>(pl);
    }
}
}  // namespace magis
