// Clean throughput probe: LDS.64 (2 addresses/warp), STS.64 (2 active lanes), SHFL.32,
// and LDS+SHFL interleaved.  asm volatile keeps one instruction per op.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ double lds(unsigned a) { double v; asm volatile("ld.shared.f64 %0, [%1];" : "=d"(v) : "r"(a)); return v; }
__device__ __forceinline__ unsigned shfl(unsigned v, int src) { unsigned r; asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, 0xffffffff;" : "=r"(r) : "r"(v), "r"(src)); return r; }
__device__ __forceinline__ void sts_if(bool p, unsigned a, double v) { asm volatile("{.reg .pred q; setp.ne.b32 q, %0, 0; @q st.shared.f64 [%1], %2;}" :: "r"((int)p), "r"(a), "d"(v)); }
template <int MODE>
__global__ void k(double* out, int iters) {
    __shared__ double s[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
    __syncthreads();
    unsigned base = (unsigned)__cvta_generic_to_shared(s) + ((threadIdx.x >> 4) & 1) * 512 + (threadIdx.x >> 5) * 2048;
    double acc[8] = {0, 0, 0, 0, 0, 0, 0, 0}; unsigned u[8] = {1, 2, 3, 4, 5, 6, 7, 8};
    int lane = threadIdx.x & 31;
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            if (MODE == 0) acc[r] += lds(base + r * 8);
            if (MODE == 1) u[r] = shfl(u[r], (lane & 16) + r);
            if (MODE == 2) { acc[r] += lds(base + r * 8); u[r] = shfl(u[r], (lane & 16) + r); }
            if (MODE == 3) sts_if(lane == r || lane == 16 + r, base + r * 8, acc[r]);
        }
    }
    double t = 0; for (int r = 0; r < 8; ++r) t += acc[r] + u[r];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
int main() {
    double* d; cudaMalloc(&d, 1 << 24);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
    int iters = 2048, warps = 16;
    void (*ks[4])(double*, int) = {k<0>, k<1>, k<2>, k<3>};
    const char* names[4] = {"LDS.64 (2 addr)", "SHFL.32", "LDS.64 + SHFL pair", "STS.64 (2 lanes)"};
    for (int i = 0; i < 4; ++i) {
        ks[i]<<<148, 32 * warps>>>(d, 8); cudaDeviceSynchronize();
        cudaEventRecord(e0); ks[i]<<<148, 32 * warps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        double n = (double)warps * iters * 8;
        printf("%-20s: %.3f ms, %.2f cycles per op(pair) per SM\n", names[i], ms, ms * 1e-3 * 1.965e9 / n);
    }
    return 0;
}
