// 128-bit shared access cost vs active-lane / address pattern (cycles per warp op per SM).
#include <cstdio>
#include <cuda_runtime.h>
struct d2 { double x, y; };
__device__ __forceinline__ void lds_if(bool p, unsigned a, double &x, double &y) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %2, 0; @q ld.shared.v2.f64 {%0,%1}, [%3];}" : "+d"(x), "+d"(y) : "r"((int)p), "r"(a));
}
__device__ __forceinline__ void sts_if(bool p, unsigned a, double x, double y) {
    asm volatile("{.reg .pred q; setp.ne.b32 q, %0, 0; @q st.shared.v2.f64 [%1], {%2,%3};}" :: "r"((int)p), "r"(a), "d"(x), "d"(y));
}
template <int MODE>
__global__ void k(double *out, int iters) {
    __shared__ __align__(16) double s[4096];
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) s[i] = i;
    __syncthreads();
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    const unsigned sb = (unsigned)__cvta_generic_to_shared(s) + w * 2048;  // 256 doubles per warp
    double ax[8] = {0}, ay[8] = {0};
    bool act = true; unsigned addr = sb;
    // address offsets in bytes; "A" at 0, "B" at 64 (banks 16..19), "C" at 32, "D" at 96
    switch (MODE) {
    case 0: act = (lane == 0 || lane == 16); addr = sb + (lane == 16 ? 64 : 0); break;   // STS 2 lanes, halves
    case 1: act = (lane == 0 || lane == 8); addr = sb + (lane == 8 ? 64 : 0); break;     // STS 2 lanes, quarters 0/1
    case 2: act = (lane == 0 || lane == 1); addr = sb + (lane == 1 ? 64 : 0); break;     // STS 2 lanes, same quarter
    case 3: act = (lane == 0); break;                                                     // STS 1 lane
    case 4: act = true; addr = sb + (lane >= 16 ? 64 : 0); break;                         // LDS bcast 2 addr, halves
    case 5: act = true; addr = sb; break;                                                 // LDS bcast 1 addr
    case 6: act = true; addr = sb + ((lane & 1) ? 64 : 0); break;                         // LDS bcast 2 addr interleaved
    case 7: act = true; addr = sb + (lane >= 16 ? 64 : 0) + (lane == 5 ? 32 : 0) + (lane == 20 ? 32 : 0); break;  // bcast + 1 odd lane per half
    case 8: act = (lane == 0); break;                                                     // LDS 1 lane
    case 9: act = (lane == 0 || lane == 16); addr = sb + (lane == 16 ? 64 : 0); break;   // LDS 2 lanes, halves
    case 10: act = (lane == 0 || lane == 1); addr = sb + (lane == 1 ? 64 : 0); break;    // LDS 2 lanes same quarter
    case 11: act = (lane == 0 || lane == 4); addr = sb + (lane == 4 ? 64 : 0); break;    // LDS 2 lanes same quarter (0,4)
    case 12: act = (lane == 0 || lane == 8); addr = sb + (lane == 8 ? 64 : 0); break;    // LDS 2 lanes quarters 0/1
    }
    for (int it = 0; it < iters; ++it) {
#pragma unroll
        for (int r = 0; r < 8; ++r) {
            const unsigned a = addr + r * 128 * 2;
            if (MODE <= 3) sts_if(act, a, ax[r] + 1.0, ay[r]);
            else lds_if(act, a, ax[r], ay[r]);
        }
    }
    double t = 0;
    for (int r = 0; r < 8; ++r) t += ax[r] + ay[r];
    out[blockIdx.x * blockDim.x + threadIdx.x] = t;
}
int main() {
    double *d; cudaMalloc(&d, 1 << 24);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1); float ms;
    const int iters = 4096, warps = 16;
    void (*ks[13])(double *, int) = {k<0>, k<1>, k<2>, k<3>, k<4>, k<5>, k<6>, k<7>, k<8>, k<9>, k<10>, k<11>, k<12>};
    const char *names[13] = {"STS.128 2 lanes (0,16)", "STS.128 2 lanes (0,8)", "STS.128 2 lanes (0,1)", "STS.128 1 lane",
                             "LDS.128 bcast 2 addr halves", "LDS.128 bcast 1 addr", "LDS.128 bcast 2 addr even/odd",
                             "LDS.128 bcast halves + 1 odd/half", "LDS.128 1 lane", "LDS.128 2 lanes (0,16)",
                             "LDS.128 2 lanes (0,1)", "LDS.128 2 lanes (0,4)", "LDS.128 2 lanes (0,8)"};
    for (int i = 0; i < 13; ++i) {
        ks[i]<<<148, 32 * warps>>>(d, 8); cudaDeviceSynchronize();
        cudaEventRecord(e0); ks[i]<<<148, 32 * warps>>>(d, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
        cudaEventElapsedTime(&ms, e0, e1);
        double n = (double)warps * iters * 8;
        printf("%-36s: %.3f cycles per warp op per SM\n", names[i], ms * 1e-3 * 1.965e9 / n);
    }
    return 0;
}
