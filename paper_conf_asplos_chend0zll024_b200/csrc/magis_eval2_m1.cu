// magis_eval2_m1.cu -- instantiations of the variant-2 kernel for MODE 1, TEAMS 1
#include "magis_eval2_kernel.cuh"

namespace magis {
const void* eval2_kernel_m1(const Plan2& pl) { return kernel_mode<1, 1>(pl); }
}  // namespace magis
