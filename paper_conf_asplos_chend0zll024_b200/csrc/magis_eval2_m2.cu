// magis_eval2_m2.cu -- instantiations of the variant-2 kernel for MODE 2, TEAMS 1
#include "magis_eval2_kernel.cuh"

namespace magis {
const void* eval2_kernel_m2(const Plan2& pl) { return kernel_mode<2, 1>(pl); }
}  // namespace magis
