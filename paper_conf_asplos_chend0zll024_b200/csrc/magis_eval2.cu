// magis_eval2.cu -- host side of the variant-2 evaluation kernel: kernel
// selection by plan (mode, packing, chunk length, teams), occupancy and
// launch.  The kernel itself is magis_eval2_kernel.cuh, instantiated per mode
// in magis_eval2_m*.cu.
#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "magis_internal.h"

namespace magis {
const void* eval2_kernel_m0t1(const Plan2& pl);
const void* eval2_kernel_m0t2(const Plan2& pl);
const void* eval2_kernel_m1(const Plan2& pl);
const void* eval2_kernel_m2(const Plan2& pl);
const void* eval2_kernel_m3(const Plan2& pl);
// with the first-argmax output (magis_eval2_am.cu)
const void* eval2_kernel_am(const Plan2& pl, int mode);

static const void* kernel_for(const Plan2& pl, bool am = false) {
    const int mode = pl.gmem_af ? 2 : pl.delta_slots ? 3 : (pl.gmem_static ? 1 : 0);
    if (am) return eval2_kernel_am(pl, mode);
    if (mode == 0) return pl.teams == 2 ? eval2_kernel_m0t2(pl) : eval2_kernel_m0t1(pl);
    return mode == 1 ? eval2_kernel_m1(pl) : mode == 3 ? eval2_kernel_m3(pl) : eval2_kernel_m2(pl);
}

int eval2_block(const Plan2& pl) { return kMainThreads2 + pl.teams * 32 * pl.P; }

cudaError_t eval2_occupancy(const Plan2& pl, int* blocks) {
    if (pl.L > 64 || (!pl.gmem_static && pl.L > 32)) { *blocks = 0; return cudaSuccess; }
    if (pl.teams == 2 && pl.gmem_static) { *blocks = 0; return cudaSuccess; }   // teams only with smem tables
    const void* fn = kernel_for(pl);
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem_total);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
    if (e != cudaSuccess) return e;
    if (std::getenv("MAGIS_DEBUG")) {
        cudaFuncAttributes fa;
        cudaFuncGetAttributes(&fa, fn);
        std::fprintf(stderr, "[magis] eval2 P=%d teams=%d regs=%d static_smem=%zu local=%zu\n", pl.P, pl.teams,
                     fa.numRegs, fa.sharedSizeBytes, fa.localSizeBytes);
    }
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks, fn, eval2_block(pl), pl.smem_total);
}

cudaError_t eval2_launch(const DevGraph& g, const Plan2& pl, const void* blob, void* ovf, void* afg, int grid,
                         int64_t K, const int32_t* perm, const uint8_t* dec, uint8_t* status,
                         int64_t* peak, double* lat, cudaStream_t stream, int32_t* argmax) {
    if (K <= 0) return cudaSuccess;
    const void* fn = kernel_for(pl, argmax != nullptr);
    if (!fn) return cudaErrorNotSupported;
    if (argmax) {
        cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)pl.smem_total);
        if (e == cudaSuccess)
            e = cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, (int)cudaSharedmemCarveoutMaxShared);
        if (e != cudaSuccess) return e;
    }
    const int64_t ngroups = (K + pl.P - 1) / pl.P;
    const int gr = (int)std::min<int64_t>(grid, (ngroups + pl.teams - 1) / pl.teams);
    void* args[] = {(void*)&g, (void*)&pl, (void*)&blob, (void*)&K, (void*)&perm, (void*)&dec,
                    (void*)&status, (void*)&peak, (void*)&lat, (void*)&ovf, (void*)&afg, (void*)&argmax};
    if (pl.gmem_static && pl.l2win_bytes > 0) {
        // tiers reading the graph image from global memory: an L2 persisting
        // access window over it for this launch (the streamed candidate rows
        // must not evict the rows every group re-reads); no stream state changes
        cudaLaunchConfig_t cfg{};
        cfg.gridDim = dim3(gr);
        cfg.blockDim = dim3(eval2_block(pl));
        cfg.dynamicSmemBytes = pl.smem_total;
        cfg.stream = stream;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeAccessPolicyWindow;
        at[0].val.accessPolicyWindow.base_ptr = const_cast<void*>(blob);
        at[0].val.accessPolicyWindow.num_bytes = pl.l2win_bytes;
        at[0].val.accessPolicyWindow.hitRatio = 1.0f;
        at[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        at[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        return cudaLaunchKernelExC(&cfg, fn, args);
    }
    return cudaLaunchKernel(fn, dim3(gr), dim3(eval2_block(pl)), args, pl.smem_total, stream);
}

}  // namespace magis
