// MIO / pipe throughput microbenchmarks: 16 warps per SM, independent ops.
#include <cstdio>
#include <cuda_runtime.h>
#define ITERS 1024
template <int OP>
__global__ void __launch_bounds__(512) k(double *out, long long *cyc, int salt) {
    __shared__ __align__(16) double sh[2048];
    const int lane = threadIdx.x & 31;
    const int w = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < 2048; i += blockDim.x) sh[i] = i;
    __syncthreads();
    double acc0 = lane, acc1 = 1;
    unsigned u0 = lane + salt, u1 = lane + 1;
    long long t0 = clock64();
#pragma unroll 1
    for (int it = 0; it < ITERS; ++it) {
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            const int o = (((it * 8 + q) * 2) & 63) + w * 128;   // 16-B aligned, warp-private
            if constexpr (OP == 0) { double2 v = *reinterpret_cast<double2 *>(sh + o); acc0 += v.x; acc1 += v.y; }
            if constexpr (OP == 1) { double2 v = *reinterpret_cast<double2 *>(sh + o + (lane >> 4) * 64); acc0 += v.x; acc1 += v.y; }
            if constexpr (OP == 2) { acc0 += sh[o]; }
            if constexpr (OP == 3) { if (lane == ((it + q) & 31)) *reinterpret_cast<double2 *>(sh + o) = make_double2(acc0 + q, acc1); }
            if constexpr (OP == 4) { if ((lane & 15) == ((it + q) & 15)) *reinterpret_cast<double2 *>(sh + o + (lane >> 4) * 64) = make_double2(acc0 + q, acc1); }
            if constexpr (OP == 5) { u0 = __shfl_sync(0xffffffffu, u0 + q, (lane + it + q) & 31); }
            if constexpr (OP == 6) { u0 += __reduce_max_sync(0xffffffffu, u1 + q + it); }
            if constexpr (OP == 7) { u0 += __ballot_sync(0xffffffffu, ((u1 + it) >> q) & 1); }
            if constexpr (OP == 8) { *reinterpret_cast<double2 *>(sh + ((w * 128 + lane * 4 + q * 2) & 2047)) = make_double2(acc0 + q, acc1); }
            if constexpr (OP == 9) { u0 = max(u0, __shfl_xor_sync(0xffffffffu, u0 + q, 1 << (q & 3))); }
        }
    }
    long long t1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    out[blockIdx.x * blockDim.x + threadIdx.x] = acc0 + acc1 + u0 + u1 + sh[(threadIdx.x * 7) & 2047];
}
template <int OP>
void run(const char *name) {
    double *o; long long *c;
    cudaMalloc(&o, 148 * 512 * 8); cudaMallocManaged(&c, 148 * 8);
    k<OP><<<148, 512>>>(o, c, 1); cudaDeviceSynchronize();
    k<OP><<<148, 512>>>(o, c, 2); cudaDeviceSynchronize();
    double mx = 0; for (int i = 0; i < 148; ++i) mx = mx > c[i] ? mx : c[i];
    const double warp_instr = 16.0 * ITERS * 8;
    printf("%-36s %6.3f warp-instr/clk/SM  (%.2f clk each)\n", name, warp_instr / mx, mx / warp_instr);
}
int main() {
    run<0>("LDS.128 broadcast (1 addr)");
    run<1>("LDS.128 2 addrs (2 half-warps)");
    run<2>("LDS.64 broadcast");
    run<3>("STS.128 one lane");
    run<4>("STS.128 two lanes");
    run<5>("SHFL.IDX 32b");
    run<6>("REDUX.MAX");
    run<7>("VOTE.ANY");
    run<8>("STS.128 all lanes (512 B)");
    run<9>("SHFL.BFLY 32b + IMNMX");
    return 0;
}
