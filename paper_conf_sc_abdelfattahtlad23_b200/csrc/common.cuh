// common.cuh -- batch addressing and small PTX helpers shared by the sm_100a
// band LU / solve kernels.  (No arithmetic of the method lives here.)
#pragma once
#ifdef __CUDACC_RTC__
// run-time compilation (jit.cuh, NVRTC): no host headers; the few types used here
typedef unsigned int uint32_t;
typedef unsigned long long uint64_t;
typedef long long int64_t;
typedef unsigned long long uintptr_t;
typedef unsigned long size_t;
namespace std {
template <class T, T v>
struct integral_constant {
    static constexpr T value = v;
};
}  // namespace std
#else
#include <cstdint>
#include <cuda_runtime.h>
#endif

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

// valid global address for zero-filling cp.async (src-size 0 reads nothing)
__device__ double g_dummy[2];

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
// 16-byte copy, L2 only (streamed data); src_bytes == 0 zero-fills
__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }

// Predicated shared-memory moves (no branch / reconvergence; a predicated-off
// load leaves its destination register unchanged).
__device__ __forceinline__ void st_shared_f64_if(bool p, uint32_t addr, double v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %0, 0;\n\t@q st.shared.f64 [%1], %2;\n\t}\n" ::"r"((int)p),
                 "r"(addr), "d"(v)
                 : "memory");
}
__device__ __forceinline__ void st_shared_s32_if(bool p, uint32_t addr, int v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %0, 0;\n\t@q st.shared.s32 [%1], %2;\n\t}\n" ::"r"((int)p),
                 "r"(addr), "r"(v)
                 : "memory");
}
__device__ __forceinline__ void ld_shared_f64_if(bool p, uint32_t addr, double &v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %1, 0;\n\t@q ld.shared.f64 %0, [%2];\n\t}\n"
                 : "+d"(v)
                 : "r"((int)p), "r"(addr)
                 : "memory");
}

// Four predicated 8-byte shared loads / stores under ONE predicate (one asm
// block so ptxas keeps them predicated instead of branching around each).
__device__ __forceinline__ void ld4_shared_if(bool p, uint32_t a, double &x0, double &x1, double &x2, double &x3) {
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %4, 0;\n\t"
        "@q ld.shared.f64 %0, [%5+%6];\n\t@q ld.shared.f64 %1, [%5+%7];\n\t"
        "@q ld.shared.f64 %2, [%5+%8];\n\t@q ld.shared.f64 %3, [%5+%9];\n\t}\n"
        : "+d"(x0), "+d"(x1), "+d"(x2), "+d"(x3)
        : "r"((int)p), "r"(a), "n"(0), "n"(8), "n"(16), "n"(24)
        : "memory");
}
__device__ __forceinline__ void st4_shared_if(bool p, uint32_t a, double x0, double x1, double x2, double x3) {
    asm volatile(
        "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %0, 0;\n\t"
        "@q st.shared.f64 [%1+%6], %2;\n\t@q st.shared.f64 [%1+%7], %3;\n\t"
        "@q st.shared.f64 [%1+%8], %4;\n\t@q st.shared.f64 [%1+%9], %5;\n\t}\n" ::"r"((int)p),
        "r"(a), "d"(x0), "d"(x1), "d"(x2), "d"(x3), "n"(0), "n"(8), "n"(16), "n"(24)
        : "memory");
}

__device__ __forceinline__ void st_shared_v2_if(bool p, uint32_t a, double2 v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %0, 0;\n\t@q st.shared.v2.f64 [%1], {%2, %3};\n\t}\n" ::"r"(
                     (int)p),
                 "r"(a), "d"(v.x), "d"(v.y)
                 : "memory");
}
__device__ __forceinline__ double2 ld_shared_v2(uint32_t a) {
    double2 v;
    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];\n" : "=d"(v.x), "=d"(v.y) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ void ld_shared_v2_if(bool p, uint32_t a, double2 &v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q ld.shared.v2.f64 {%0, %1}, [%3];\n\t}\n"
                 : "+d"(v.x), "+d"(v.y)
                 : "r"((int)p), "r"(a)
                 : "memory");
}
__device__ __forceinline__ int ld_shared_s32(uint32_t a) {
    int v;
    asm volatile("ld.shared.s32 %0, [%1];\n" : "=r"(v) : "r"(a) : "memory");
    return v;
}
__device__ __forceinline__ double ld_shared_f64(uint32_t a) {
    double v;
    asm volatile("ld.shared.f64 %0, [%1];\n" : "=d"(v) : "r"(a) : "memory");
    return v;
}

// volatile: ptxas may not merge neighbouring loads into one 128-bit access
// (a 64-bit broadcast read costs one wavefront for all groups of a warp)
__device__ __forceinline__ double ld_volatile_shared_f64(uint32_t a) {
    double v;
    asm volatile("ld.volatile.shared.f64 %0, [%1];\n" : "=d"(v) : "r"(a) : "memory");
    return v;
}

// Predicated global accesses (one instruction under a predicate, no branch).
__device__ __forceinline__ void st_global_f64_if(bool p, double *a, double v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %0, 0;\n\t@q st.global.f64 [%1], %2;\n\t}\n" ::"r"((int)p),
                 "l"(a), "d"(v)
                 : "memory");
}
__device__ __forceinline__ void ld_global_f64_if(bool p, const double *a, double &v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %1, 0;\n\t@q ld.global.f64 %0, [%2];\n\t}\n"
                 : "+d"(v)
                 : "r"((int)p), "l"(a)
                 : "memory");
}

// y = fma(a, b, y) (round to nearest) on lanes where p holds: one predicated DFMA
// instead of an FMA and a 64-bit select.
__device__ __forceinline__ void fma_rn_if(bool p, double a, double b, double &y) {
    asm("{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %1, 0;\n\t@q fma.rn.f64 %0, %2, %3, %0;\n\t}\n"
        : "+d"(y)
        : "r"((int)p), "d"(a), "d"(b));
}

// ---- mbarrier + bulk (TMA 1D) copies
__device__ __forceinline__ void mbar_init(uint32_t bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra WAIT_%=;\n\t}\n" ::"r"(bar),
        "r"(parity)
        : "memory");
}
// global -> shared bulk copy (16 B aligned src/dst, size multiple of 16), completes on `bar`
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(dst),
                 "l"(src), "r"(bytes), "r"(bar)
                 : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory"); }

// |x| as an ordered integer key: for non-negative doubles the IEEE bit
// pattern orders like the value (used for the exact pivot search).
__device__ __forceinline__ uint64_t abs_key(double x) {
    return static_cast<uint64_t>(__double_as_longlong(x)) & 0x7fffffffffffffffull;
}

// RN(a / b) on lanes where p holds, else a.  The compiler if-converts a
// guarded division and runs it on every lane; lanes with !p divide 1 by 1 so
// that none of them leaves the inline fast path for the slow-path CALL (0 / 0
// would), and a CALL waits for every outstanding load of the warp.
// The operands pass through an opaque move: otherwise the compiler sees that
// q is only used where p holds and divides a by b on every lane again.
__device__ __forceinline__ double ddiv_rn_if(bool p, double a, double b) {
    double na, nb;
    asm("mov.b64 %0, %1;" : "=d"(na) : "d"(p ? a : 1.0));
    asm("mov.b64 %0, %1;" : "=d"(nb) : "d"(p ? b : 1.0));
    const double q = __ddiv_rn(na, nb);
    return p ? q : a;
}

// RN(1/x) for x != 0 and 0 for x == 0, without ever entering the slow path for
// x == 0 (the operand passes an opaque move, as in ddiv_rn_if).  A zero result
// marks a zero pivot (a finite nonzero x never has a zero reciprocal).
__device__ __forceinline__ double drcp_rn_nz(double x) {
    double xg;
    asm("mov.b64 %0, %1;" : "=d"(xg) : "d"(x != 0.0 ? x : 1.0));
    const double r = __drcp_rn(xg);
    return x != 0.0 ? r : 0.0;
}

__host__ __device__ constexpr int pow2_ceil(int x) {
    int p = 1;
    while (p < x) p *= 2;
    return p;
}

}  // namespace bandlu
