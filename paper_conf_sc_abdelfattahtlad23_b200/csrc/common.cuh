// common.cuh -- batch addressing and small PTX helpers shared by the sm_100a
// band LU / solve kernels.  (No arithmetic of the method lives here.)
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bandlu {

// Batch addressing: strided (base + i*stride) or pointer array.
template <class T>
struct Strided {
    T *base;
    int64_t stride;
    __device__ __forceinline__ T *get(int64_t i) const { return base + i * stride; }
};
template <class T>
struct PtrArray {
    T *const *ptrs;
    __device__ __forceinline__ T *get(int64_t i) const { return ptrs[i]; }
};

__device__ __forceinline__ unsigned lane_id() { return threadIdx.x & 31u; }

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// cp.async (LDGSTS) 8-byte copy global -> shared, L1-allocating; when
// src_bytes == 0 the destination is zero-filled and global memory is not read.
__device__ __forceinline__ void cp_async8(uint32_t dst, const void *src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async4(uint32_t dst, const void *src, uint32_t src_bytes) {
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes)
                 : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// |x| as an ordered integer key: for non-negative doubles the IEEE bit
// pattern orders like the value (used for the exact pivot search).
__device__ __forceinline__ uint64_t abs_key(double x) {
    return static_cast<uint64_t>(__double_as_longlong(x)) & 0x7fffffffffffffffull;
}

__host__ __device__ constexpr int pow2_ceil(int x) {
    int p = 1;
    while (p < x) p *= 2;
    return p;
}

}  // namespace bandlu
