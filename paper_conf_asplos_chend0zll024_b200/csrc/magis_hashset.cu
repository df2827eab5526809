// magis_hashset.cu -- the seen-graph set X of Alg. 3 (lines 10-12,
// P:1703-1705) on the device: batched duplicate filter over graph hashes
// (SURVEY §8(f) NEXT-2).  Open addressing with linear probing over 64-bit
// keys; the owner word of a slot holds (filter epoch << 40 | smallest
// candidate id of this batch), so one atomicMin per candidate decides both
// "already in X" (an older epoch) and "first occurrence in the batch".
#include <algorithm>
#include <cstdint>
#include <new>
#include <string>

#include "magis_internal.h"

struct magis_hashset {
    int device = 0;
    uint64_t cap = 0;                  // power of two
    unsigned long long* keys = nullptr;     // [cap] 0 = empty
    unsigned long long* owner = nullptr;    // [cap + 1] (epoch << 40 | first id); [cap] = key 0
    unsigned long long* stats = nullptr;    // [2] occupied slots, overflowed inserts
    uint32_t epoch = 0;
};

namespace magis {
namespace {

__host__ __device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// hash set: open addressing, linear probing, 64-bit keys (0 = empty; the
// key 0 has its own owner word at [cap])
__device__ __forceinline__ uint64_t probe_start(uint64_t h, uint64_t mask) { return mix64(h) & mask; }

__global__ void hs_insert_kernel(magis_hashset s, int64_t K, const uint64_t* __restrict__ hash,
                                 const uint8_t* __restrict__ status) {
    const uint64_t mask = s.cap - 1;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        if (status && status[k]) continue;
        const unsigned long long h = hash[k];
        const unsigned long long me = ((unsigned long long)s.epoch << 40) | (unsigned long long)k;
        if (h == 0) { atomicMin(s.owner + s.cap, me); continue; }
        uint64_t i = probe_start(h, mask);
        bool done = false;
        for (uint64_t p = 0; p < s.cap; p++) {
            const unsigned long long prev = atomicCAS(s.keys + i, 0ull, h);
            if (prev == 0ull || prev == h) {
                if (prev == 0ull) atomicAdd(s.stats, 1ull);
                atomicMin(s.owner + i, me);
                done = true;
                break;
            }
            i = (i + 1) & mask;
        }
        if (!done) atomicAdd(s.stats + 1, 1ull);
    }
}

__global__ void hs_mark_kernel(magis_hashset s, int64_t K, const uint64_t* __restrict__ hash,
                               const uint8_t* __restrict__ status, uint8_t* __restrict__ is_new) {
    const uint64_t mask = s.cap - 1;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < K; k += (int64_t)gridDim.x * blockDim.x) {
        if (status && status[k]) { is_new[k] = 0; continue; }
        const unsigned long long h = hash[k];
        const unsigned long long me = ((unsigned long long)s.epoch << 40) | (unsigned long long)k;
        uint8_t r = 1;                           // not found (table full): kept as new
        if (h == 0) {
            r = s.owner[s.cap] == me;
        } else {
            uint64_t i = probe_start(h, mask);
            for (uint64_t p = 0; p < s.cap; p++) {
                const unsigned long long key = s.keys[i];
                if (key == h) { r = s.owner[i] == me; break; }
                if (key == 0ull) break;
                i = (i + 1) & mask;
            }
        }
        is_new[k] = r;
    }
}


struct DeviceGuard {
    int prev = -1;
    explicit DeviceGuard(int d) { cudaGetDevice(&prev); cudaSetDevice(d); }
    ~DeviceGuard() { if (prev >= 0) cudaSetDevice(prev); }
};

#define GCK(call)                                                                             \
    do {                                                                                      \
        cudaError_t _e = (call);                                                              \
        if (_e != cudaSuccess) {                                                              \
            cudaGetLastError();                                                               \
            return set_error(MAGIS_E_CUDA, std::string(#call ": ") + cudaGetErrorString(_e)); \
        }                                                                                     \
    } while (0)


}  // namespace
}  // namespace magis

using namespace magis;

extern "C" int magis_hashset_create(int device, int64_t capacity, magis_hashset** out) {
    clear_error();
    if (!out) return set_error(MAGIS_E_INVAL, "out is NULL");
    *out = nullptr;
    if (capacity < 1 || capacity > (1ll << 40)) return set_error(MAGIS_E_INVAL, "capacity out of range");
    if (!magis_device_supported(device))
        return set_error(MAGIS_E_UNSUPPORTED, "device " + std::to_string(device) +
                         " is not an sm_100 (B200) GPU; there is no CPU fallback");
    DeviceGuard guard(device);
    magis_hashset* s = new (std::nothrow) magis_hashset();
    if (!s) return set_error(MAGIS_E_NOMEM, "host allocation failed");
    uint64_t cap = 1;
    while (cap < (uint64_t)capacity) cap <<= 1;
    s->device = device;
    s->cap = cap;
    if (cudaMalloc(&s->keys, cap * 8) != cudaSuccess || cudaMalloc(&s->owner, (cap + 1) * 8) != cudaSuccess ||
        cudaMalloc(&s->stats, 16) != cudaSuccess) {
        cudaGetLastError();
        if (s->keys) cudaFree(s->keys);
        if (s->owner) cudaFree(s->owner);
        delete s;
        return set_error(MAGIS_E_NOMEM, "cudaMalloc hash set failed");
    }
    const int rc = magis_hashset_clear(s, nullptr);
    if (rc != MAGIS_SUCCESS || cudaDeviceSynchronize() != cudaSuccess) {
        cudaGetLastError();
        cudaFree(s->keys);
        cudaFree(s->owner);
        cudaFree(s->stats);
        delete s;
        return set_error(MAGIS_E_CUDA, "hash set initialisation failed");
    }
    *out = s;
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_clear(magis_hashset* s, void* cuda_stream) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    DeviceGuard guard(s->device);
    cudaStream_t st = (cudaStream_t)cuda_stream;
    GCK(cudaMemsetAsync(s->keys, 0, s->cap * 8, st));
    GCK(cudaMemsetAsync(s->owner, 0xFF, (s->cap + 1) * 8, st));
    GCK(cudaMemsetAsync(s->stats, 0, 16, st));
    s->epoch = 0;   // the owners were reset to all-ones on the same stream
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_free(magis_hashset* s) {
    clear_error();
    if (!s) return MAGIS_SUCCESS;
    DeviceGuard guard(s->device);
    cudaDeviceSynchronize();
    cudaFree(s->keys);
    cudaFree(s->owner);
    cudaFree(s->stats);
    cudaGetLastError();
    delete s;
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_filter(magis_hashset* s, int64_t K, const uint64_t* d_hash, const uint8_t* d_status,
                                    uint8_t* d_new, void* cuda_stream) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    if (K < 0 || K >= (1ll << 40)) return set_error(MAGIS_E_INVAL, "K out of range");
    if (K == 0) return MAGIS_SUCCESS;
    if (!d_hash || !d_new) return set_error(MAGIS_E_INVAL, "null device pointer");
    if (s->epoch + 1 >= (1u << 24)) return set_error(MAGIS_E_CAPACITY, "hash set epoch exhausted: clear it");
    DeviceGuard guard(s->device);
    s->epoch++;
    cudaStream_t st = (cudaStream_t)cuda_stream;
    const int grid = (int)std::min<int64_t>((K + 255) / 256, 148 * 16);
    hs_insert_kernel<<<grid, 256, 0, st>>>(*s, K, d_hash, d_status);
    GCK(cudaGetLastError());
    hs_mark_kernel<<<grid, 256, 0, st>>>(*s, K, d_hash, d_status, d_new);
    GCK(cudaGetLastError());
    return MAGIS_SUCCESS;
}

extern "C" int magis_hashset_stats(const magis_hashset* s, int64_t* n_keys, int64_t* n_overflow) {
    clear_error();
    if (!s) return set_error(MAGIS_E_INVAL, "hash set is NULL");
    DeviceGuard guard(s->device);
    unsigned long long h[2] = {0, 0};
    GCK(cudaMemcpy(h, s->stats, 16, cudaMemcpyDeviceToHost));
    unsigned long long z = 0;
    GCK(cudaMemcpy(&z, s->owner + s->cap, 8, cudaMemcpyDeviceToHost));
    if (n_keys) *n_keys = (int64_t)h[0] + (z != ~0ull ? 1 : 0);
    if (n_overflow) *n_overflow = (int64_t)h[1];
    return MAGIS_SUCCESS;
}

