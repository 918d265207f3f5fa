// Broadcast-primitive throughput: 16 warps/SM.
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 1024
template <int OP>
__global__ void __launch_bounds__(512) k(double *out, double *g, long long *cyc, int salt) {
    __shared__ __align__(16) double sh[2048];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 2048; i += blockDim.x) sh[i] = i;
    __syncthreads();
    double acc0 = lane, acc1 = 1;
    unsigned u0 = lane + salt, u1 = lane + 1;
    double *gw = g + (blockIdx.x * 16 + w) * 64;
    long long t0 = clock64();
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int o = (((it * 8 + q) * 2) & 63) + w * 128;
            if constexpr (OP == 0) { // REDUX.OR broadcast of a double (2 redux)
                const unsigned m = (lane == ((it + q) & 31)) ? 0xffffffffu : 0u;
                unsigned hi = __reduce_or_sync(0xffffffffu, (unsigned)__double2hiint(acc0) & m);
                unsigned lo = __reduce_or_sync(0xffffffffu, (unsigned)__double2loint(acc0) & m);
                acc1 = __fma_rn(acc1, __hiloint2double(hi, lo), 1e-300);
            }
            if constexpr (OP == 1) { // LDS.128 + REDUX interleaved
                double2 v = *reinterpret_cast<double2 *>(sh + o); acc0 += v.x; acc1 += v.y;
                u0 += __reduce_max_sync(0xffffffffu, u1 + q + it);
            }
            if constexpr (OP == 2) { // STG.256 one lane
                if (lane == ((it + q) & 31)) {
                    asm volatile("st.global.v4.f64 [%0], {%1,%2,%3,%4};" :: "l"(gw + ((q * 4) & 63)), "d"(acc0), "d"(acc1), "d"(acc0 + 1), "d"(acc1 + 1) : "memory");
                }
            }
            if constexpr (OP == 3) { // LDG.128 broadcast (L1 hit)
                double vx, vy; asm volatile("ld.global.v2.f64 {%0,%1}, [%2];" : "=d"(vx), "=d"(vy) : "l"(gw + ((q * 2 + it * 2) & 63))); acc0 += vx; acc1 += vy;
            }
            if constexpr (OP == 4) { // STS.64 one lane
                if (lane == ((it + q) & 31)) sh[o] = acc0 + q;
            }
            if constexpr (OP == 5) { // LDS.128 + DFMA x2 (GER-like)
                double2 v = *reinterpret_cast<double2 *>(sh + o); acc0 = __fma_rn(-acc1, v.x, acc0); acc1 = __fma_rn(-acc0, v.y, acc1);
            }
            if constexpr (OP == 6) { // SHFL of a double (2x SHFL.IDX), warp-uniform source
                acc0 = __shfl_sync(0xffffffffu, acc0, (it + q) & 31) + 1e-300;
            }
            if constexpr (OP == 7) { // SHFL double, width 16, constant index
                acc0 = __shfl_sync(0xffffffffu, acc0, q & 15, 16) + 1e-300;
            }
            if constexpr (OP == 8) { // SHFL double, 2 distinct sources (per half warp)
                acc0 = __shfl_sync(0xffffffffu, acc0, ((it + q) & 15) + (lane & 16)) + 1e-300;
            }
            if constexpr (OP == 9) { // SHFL double, per-lane different source
                acc0 = __shfl_sync(0xffffffffu, acc0, (lane + it + q) & 31) + 1e-300;
            }
            if constexpr (OP == 10) { // SHFL double, source from a ballot (runtime-uniform)
                const int src = __ffs(__ballot_sync(0xffffffffu, ((unsigned)(acc1 * 0) + lane) == ((it + q) & 31))) - 1;
                acc0 = __shfl_sync(0xffffffffu, acc0, src) + 1e-300;
            }
        }
    }
    long long t1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc0 + acc1 + u0 + u1 + sh[(threadIdx.x * 7) & 2047];
}
template <int OP>
void run(const char *name) {
    double *o, *g; long long *c;
    cudaMalloc(&o, 148 * 512 * 8); cudaMalloc(&g, 148 * 16 * 64 * 8); cudaMemset(g, 0, 148 * 16 * 64 * 8); cudaMallocManaged(&c, 148 * 8);
    k<OP><<<148, 512>>>(o, g, c, 1); cudaDeviceSynchronize();
    k<OP><<<148, 512>>>(o, g, c, 2); cudaDeviceSynchronize();
    double mx = 0; for (int i = 0; i < 148; ++i) mx = mx > c[i] ? mx : c[i];
    const double warp_instr = 16.0 * ITERS * 8;
    printf("%-40s %6.2f clk per item per SM\n", name, mx / warp_instr);
}
int main() {
    run<0>("REDUX.OR x2 broadcast of a double");
    run<1>("LDS.128 bcast + REDUX.MAX (pair)");
    run<2>("STG.256 one lane");
    run<3>("LDG.128 broadcast (L1)");
    run<4>("STS.64 one lane");
    run<5>("LDS.128 bcast + 2 DFMA");
    run<6>("SHFL double (2x SHFL.IDX) uniform src");
    run<7>("SHFL double width16 const idx");
    run<8>("SHFL double 2 srcs (half-warps)");
    run<9>("SHFL double per-lane src");
    run<10>("SHFL double src=ffs(ballot) (+vote)");
    return 0;
}
