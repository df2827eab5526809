// magis_eval2_m3.cu -- instantiations of the variant-2 kernel for MODE 3, TEAMS 1
#include "magis_eval2_kernel.cuh"

namespace magis {
const void* eval2_kernel_m3(const Plan2& pl) { return kernel_mode<3, 1>(pl); }
}  // namespace magis
