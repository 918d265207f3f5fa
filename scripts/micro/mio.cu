// MIO / pipe throughput per SM for the primitives a GETRF step is built from
// (16 warps per SM, 148 CTAs of 512 threads).  Not part of the library.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 scripts/micro/mio.cu -o scripts/micro/mio
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 512
template <int OP>
__global__ void __launch_bounds__(512) k(double *out, long long *cyc, int salt) {
    __shared__ __align__(16) double sh[16 * 34 * 8];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 16 * 34 * 8; i += blockDim.x) sh[i] = i;
    __syncthreads();
    double a0 = lane, a1 = 1, a2 = 2, a3 = 3;
    double *ws = sh + w * 34 * 8;
    const int p = (salt + w) & 31;
    long long t0 = clock64();
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if constexpr (OP == 0) {  // STS.128, one lane active
                if (lane == p) *reinterpret_cast<double2 *>(ws + 2 * q) = make_double2(a0, a1);
            }
            if constexpr (OP == 1) {  // STS.128, 4 lanes active (distinct 16-B slots)
                if ((lane & 7) == 0) *reinterpret_cast<double2 *>(ws + 2 * (lane >> 3) + 8 * q) = make_double2(a0, a1);
            }
            if constexpr (OP == 2) {  // STS.128, 8 lanes active (distinct, one 128-B wavefront)
                if ((lane & 3) == 0) *reinterpret_cast<double2 *>(ws + 2 * (lane >> 2) + 16 * (q & 3)) = make_double2(a0, a1);
            }
            if constexpr (OP == 3) {  // STS.128 all lanes, 34-double row stride (lane = row)
                *reinterpret_cast<double2 *>(sh + (lane * 34 + 2 * (q & 7)) + (w & 1)) = make_double2(a0, a1);
            }
            if constexpr (OP == 4) {  // LDS.128 broadcast
                const double2 v = *reinterpret_cast<const double2 *>(ws + 2 * q);
                a0 += v.x; a1 += v.y;
            }
            if constexpr (OP == 5) {  // LDS.64 broadcast
                a0 += ws[q];
            }
            if constexpr (OP == 6) {  // SHFL double, warp-uniform runtime source
                a0 = __shfl_sync(0xffffffffu, a0, p) + 1e-300;
            }
            if constexpr (OP == 7) {  // DFMA x4 independent
                a0 = __fma_rn(a0, 1.0000001, 1e-300); a1 = __fma_rn(a1, 1.0000001, 1e-300);
                a2 = __fma_rn(a2, 1.0000001, 1e-300); a3 = __fma_rn(a3, 1.0000001, 1e-300);
            }
            if constexpr (OP == 8) {  // STS.64 one lane
                if (lane == p) ws[q] = a0;
            }
            if constexpr (OP == 9) {  // STS.128 one lane via predicated asm (no branch)
                asm volatile("{.reg .pred pp; setp.eq.s32 pp, %0, %1; @pp st.shared.v2.f64 [%2], {%3, %4};}"
                             :: "r"(lane), "r"(p), "r"((unsigned)__cvta_generic_to_shared(ws + 2 * q)), "d"(a0), "d"(a1) : "memory");
            }
            if constexpr (OP == 10) {  // LDS.64 per-lane column (lane = column, same row), conflict-free
                a0 += sh[(q * 34) + lane + (w & 1)];
            }
            if constexpr (OP == 11) {  // REDUX.MAX
                a0 += (double)__reduce_max_sync(0xffffffffu, (unsigned)lane + q + it);
            }
        }
        a0 += 1.0;
    }
    long long t1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = a0 + a1 + a2 + a3 + sh[(threadIdx.x * 7) & 2047];
}
template <int OP>
void run(const char *name, double per = 1.0) {
    double *o; long long *c;
    cudaMalloc(&o, 148 * 512 * 8); cudaMallocManaged(&c, 148 * 8);
    k<OP><<<148, 512>>>(o, c, 1); cudaDeviceSynchronize();
    k<OP><<<148, 512>>>(o, c, 2); cudaDeviceSynchronize();
    double mx = 0; for (int i = 0; i < 148; ++i) mx = mx > c[i] ? mx : c[i];
    const double warp_instr = 16.0 * ITERS * 8 * per;
    printf("%-46s %6.2f SM-clk per warp-instr  (%s)\n", name, mx / warp_instr, cudaGetErrorString(cudaGetLastError()));
}
int main() {
    run<0>("STS.128 1 lane (branch)");
    run<9>("STS.128 1 lane (predicated asm)");
    run<8>("STS.64 1 lane");
    run<1>("STS.128 4 lanes");
    run<2>("STS.128 8 lanes");
    run<3>("STS.128 32 lanes (rows, stride 34)");
    run<4>("LDS.128 broadcast");
    run<5>("LDS.64 broadcast");
    run<10>("LDS.64 per-lane column");
    run<6>("SHFL.IDX x2 (double) uniform src");
    run<11>("REDUX.MAX");
    run<7>("DFMA (per instr)", 4.0);
    return 0;
}
