// Shared-memory instruction cost on B200: cycles per warp instruction per SM, by
// width (32/64/128-bit), active lanes and address pattern.  asm volatile + memory
// clobber keeps every op in the loop.
#include <cstdio>
#include <cuda_runtime.h>
#define LD(W, T, C)                                                                                         \
    __device__ __forceinline__ void ld##W(bool p, unsigned a, T &x) {                                        \
        asm volatile("{.reg .pred q; setp.ne.b32 q, %1, 0; @q ld.volatile.shared." #W " %0, [%2];}" : "+" C(x) : "r"((int)p), "r"(a) : "memory"); \
    }
LD(f64, double, "d")
LD(f32, float, "f")
__device__ __forceinline__ void ld128(bool p, unsigned a, double &x, double &y) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %2, 0; @q ld.volatile.shared.v2.f64 {%0,%1}, [%3];}" : "+d"(x), "+d"(y) : "r"((int)p), "r"(a) : "memory");
}
__device__ __forceinline__ void st128(bool p, unsigned a, double x, double y) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %0, 0; @q st.shared.v2.f64 [%1], {%2,%3};}" :: "r"((int)p), "r"(a), "d"(x), "d"(y) : "memory");
}
__device__ __forceinline__ void st64(bool p, unsigned a, double x) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %0, 0; @q st.shared.f64 [%1], %2;}" :: "r"((int)p), "r"(a), "d"(x) : "memory");
}
__device__ __forceinline__ void st32(bool p, unsigned a, float x) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %0, 0; @q st.shared.f32 [%1], %2;}" :: "r"((int)p), "r"(a), "f"(x) : "memory");
}
__device__ __forceinline__ unsigned shfl(unsigned v, int src) { unsigned r; asm volatile("shfl.sync.idx.b32 %0, %1, %2, 0x1f, 0xffffffff;" : "=r"(r) : "r"(v), "r"(src) : "memory"); return r; }

// OP: 0 ld128, 1 st128, 2 ld64, 3 st64, 4 ld32, 5 st32, 6 shfl32
// PAT: 0 one lane, 1 two lanes (0,16), 2 all lanes broadcast one addr, 3 all lanes distinct conflict-free, 4 two addrs halves (bcast)
template <int OP, int PAT>
__global__ void k(double *out, int iters) {
    __shared__ __align__(16) double s[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned sb = (unsigned)__cvta_generic_to_shared(s) + (w & 7) * 4096;
    const int width = (OP <= 1) ? 16 : (OP <= 3) ? 8 : 4;
    bool act = true; unsigned addr = sb;
    if (PAT == 0) act = lane == 0;
    if (PAT == 1) { act = lane == 0 || lane == 16; addr = sb + (lane == 16 ? 64 : 0); }
    if (PAT == 3) addr = sb + lane * width;
    if (PAT == 4) addr = sb + (lane >= 16 ? 64 : 0);
    if (PAT == 5) { act = lane == 0 || lane == 1; addr = sb + (lane == 1 ? 64 : 0); }
    if (PAT == 6) { act = lane == 0 || lane == 8; addr = sb + (lane == 8 ? 64 : 0); }
    if (PAT == 7) addr = sb + (lane >= 16 ? 64 : 0) + (lane == 5 || lane == 20 ? 32 : 0);
    double ax[8] = {0}, ay[8] = {0}; float af[8] = {0}; unsigned u[8] = {1, 2, 3, 4, 5, 6, 7, 8};
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const unsigned a = addr + (r & 3) * 512;
            if (OP == 0) ld128(act, a, ax[r], ay[r]);
            if (OP == 1) st128(act, a, ax[r], ay[r]);
            if (OP == 2) ldf64(act, a, ax[r]);
            if (OP == 3) st64(act, a, ax[r]);
            if (OP == 4) ldf32(act, a, af[r]);
            if (OP == 5) st32(act, a, af[r]);
            if (OP == 6) u[r] = shfl(u[r], (lane + r) & 31);
        }
    }
    double t = 0;
    for (int r = 0; r < 8; ++r) t += ax[r] + ay[r] + af[r] + u[r];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
template <int OP, int PAT>
void run(const char *name, double *d) {
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
    const int iters = 4096, warps = 16;
    k<OP, PAT><<<148, 32 * warps>>>(d, 8); cudaDeviceSynchronize();
    cudaEventRecord(e0); k<OP, PAT><<<148, 32 * warps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("%-40s: %.3f cycles per warp op per SM\n", name, ms * 1e-3 * 1.965e9 / ((double)warps * iters * 8));
}
int main() {
    double *d; cudaMalloc(&d, 1 << 24);
    run<0, 0>("LDS.128 1 lane", d); run<0, 1>("LDS.128 2 lanes (0,16)", d); run<0, 2>("LDS.128 bcast 1 addr", d);
    run<0, 4>("LDS.128 bcast 2 addr (halves)", d); run<0, 3>("LDS.128 32 distinct", d);
    run<1, 0>("STS.128 1 lane", d); run<1, 1>("STS.128 2 lanes (0,16)", d); run<1, 3>("STS.128 32 distinct", d);
    run<2, 0>("LDS.64 1 lane", d); run<2, 2>("LDS.64 bcast", d); run<2, 4>("LDS.64 bcast 2 addr", d); run<2, 3>("LDS.64 32 distinct", d);
    run<3, 0>("STS.64 1 lane", d); run<3, 1>("STS.64 2 lanes", d); run<3, 3>("STS.64 32 distinct", d);
    run<4, 0>("LDS.32 1 lane", d); run<4, 3>("LDS.32 32 distinct", d);
    run<5, 0>("STS.32 1 lane", d); run<5, 3>("STS.32 32 distinct", d);
    run<6, 3>("SHFL.32", d);
    run<1, 5>("STS.128 2 lanes (0,1)", d); run<1, 6>("STS.128 2 lanes (0,8)", d);
    run<0, 5>("LDS.128 2 lanes (0,1)", d); run<0, 6>("LDS.128 2 lanes (0,8)", d);
    run<0, 7>("LDS.128 bcast halves + 1 odd lane each", d);
    run<3, 5>("STS.64 2 lanes (0,1)", d); run<2, 1>("LDS.64 2 lanes (0,16)", d); run<2, 5>("LDS.64 2 lanes (0,1)", d);
    return 0;
}
