// magis_eval2_m0t1.cu -- instantiations of the variant-2 kernel for MODE 0, TEAMS 1
#include "magis_eval2_kernel.cuh"

namespace magis {
const void* eval2_kernel_m0t1(const Plan2& pl) { return kernel_mode<0, 1>(pl); }
}  // namespace magis
