// Latency microbenchmarks (one warp, dependent chains) for the B200 design
// decisions of the GETRF/GETRS kernels.  Build: nvcc -arch=sm_100a -O3.
#include <cstdio>
#include <cuda_runtime.h>
#define N 512
__global__ void k(double *out, long long *cyc, double seed) {
    __shared__ double sh[64];
    const int lane = threadIdx.x;
    double x = seed + lane * 1e-3, y = 1.0000001;
    unsigned u = lane;
    long long t0, t1;
    int c = 0;
#define TIME(NAME, BODY) { __syncwarp(); t0 = clock64(); _Pragma("unroll 1") for (int i = 0; i < N / 16; ++i) { _Pragma("unroll") for (int q = 0; q < 16; ++q) { BODY; } } __syncwarp(); t1 = clock64(); if (lane == 0) cyc[c] = (t1 - t0); c++; }
    TIME("dfma", x = __fma_rn(x, y, 1e-9));
    TIME("dmul", x = __dmul_rn(x, y));
    TIME("ffma", { float f = (float)x; f = __fmaf_rn(f, 1.0001f, 1e-9f); x = f; });
    TIME("mufu_rcp64h", { double r; asm volatile("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x)); x = r + 1e-300; });
    TIME("ddiv", x = __ddiv_rn(x, y));
    TIME("shfl32", { u = __shfl_sync(0xffffffffu, u, (lane + 1) & 31) + 1; });
    TIME("shfl64", { x = __shfl_sync(0xffffffffu, x, (lane + 1) & 31) + 1e-9; });
    TIME("redux", { u = __reduce_max_sync(0xffffffffu, u) + lane; });
    TIME("ballot", { u = __ballot_sync(0xffffffffu, (u & 1)) + lane; });
    TIME("sts_lds", { sh[lane] = x; __syncwarp(); x = sh[(lane + 1) & 31] + 1e-9; });
    TIME("lds_bcast", { sh[0] = x; x = sh[((int)x) & 0] + 1e-9; });
    TIME("lds_dep", { x = sh[((unsigned)(x * 0)) & 31] + 1e-9; });
    TIME("imad", { u = u * 3 + 1; });
    out[lane] = x + u;
}
int main() {
    double *o; long long *c;
    cudaMalloc(&o, 32 * 8); cudaMallocManaged(&c, 64 * 8);
    k<<<1, 32>>>(o, c, 1.0); cudaDeviceSynchronize();
    k<<<1, 32>>>(o, c, 1.0); cudaDeviceSynchronize();
    const char *names[] = {"dfma", "dmul", "ffma(+cvt)", "mufu.rcp64h(+dadd)", "ddiv_rn", "shfl32(+iadd)", "shfl64(+dadd)",
                           "redux.max(+iadd)", "ballot(+iadd)", "sts->syncwarp->lds(+dadd)", "sts+lds bcast(+dadd)", "lds dep(+dadd)", "imad"};
    for (int i = 0; i < 13; ++i) printf("%-28s %7.1f cycles/iter\n", names[i], (double)c[i] / N);
    return 0;
}
