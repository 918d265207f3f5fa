// Throughput / latency micro benchmark of the warp primitives the GETRF step
// is built from (B200, sm_100a).  Not part of the library.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 scripts/micro/prims.cu -o prims
//
// Throughput: W warps per SM, each issuing N instructions of one kind in 8
// independent chains; reported as SM-wide warp-instructions per cycle.
// Latency: one warp, one dependent chain; cycles per instruction.
#include <cstdio>
#include <cuda_runtime.h>

#define ITERS 256
enum Op {
    STS128_1, STS64_1, STS32_1, STS128_ALL, STS64_ALL, LDS128_B, LDS64_B, LDS32_B, LDS128_ROW,
    SHFL_U, SHFL_V, REDUX, DFMA, DMUL, BALLOT, FFMA, IADD, VOTEANY, NOPS
};
static const char *names[] = {"sts.128 1 lane", "sts.64 1 lane", "sts.32 1 lane", "sts.128 all lanes",
                              "sts.64 all lanes", "lds.128 bcast", "lds.64 bcast", "lds.32 bcast",
                              "lds.128 per-lane row", "shfl.idx uniform src", "shfl.idx var src",
                              "redux.max", "dfma", "dmul", "ballot", "ffma", "iadd3", "vote.any"};

template <int OP>
__global__ void __launch_bounds__(1024) k_tput(unsigned long long *cyc, double *sink, int reps) {
    __shared__ __align__(16) double sh[4096];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    double d[8];
    unsigned u[8];
    for (int c = 0; c < 8; ++c) { d[c] = 1.0 + lane * 1e-3 + c; u[c] = lane * 7 + c; }
    for (int i = threadIdx.x; i < 4096; i += blockDim.x) sh[i] = i;
    __syncthreads();
    const unsigned base = (unsigned)__cvta_generic_to_shared(sh) + (w * 128) * 8;
    unsigned long long t0 = clock64();
    for (int r = 0; r < reps; ++r) {
#pragma unroll 4
        for (int i = 0; i < ITERS; ++i) {
#pragma unroll
            for (int c = 0; c < 8; ++c) {
                const unsigned a = base + ((i * 8 + c) & 15) * 16;
                if constexpr (OP == STS128_1) {
                    asm volatile("{.reg .pred p; setp.eq.u32 p, %0, %3; @p st.shared.v2.f64 [%1], {%2, %2};}"
                                 ::"r"(lane), "r"(a), "d"(d[c]), "r"(c));
                } else if constexpr (OP == STS64_1) {
                    asm volatile("{.reg .pred p; setp.eq.u32 p, %0, %3; @p st.shared.f64 [%1], %2;}"
                                 ::"r"(lane), "r"(a), "d"(d[c]), "r"(c));
                } else if constexpr (OP == STS32_1) {
                    asm volatile("{.reg .pred p; setp.eq.u32 p, %0, %3; @p st.shared.u32 [%1], %2;}"
                                 ::"r"(lane), "r"(a), "r"(u[c]), "r"(c));
                } else if constexpr (OP == STS128_ALL) {
                    const unsigned b = (unsigned)__cvta_generic_to_shared(sh) + ((w * 32 + lane) & 255) * 16;
                    asm volatile("st.shared.v2.f64 [%0], {%1, %1};" ::"r"(b), "d"(d[c]));
                } else if constexpr (OP == STS64_ALL) {
                    const unsigned b = (unsigned)__cvta_generic_to_shared(sh) + ((w * 32 + lane) & 511) * 8;
                    asm volatile("st.shared.f64 [%0], %1;" ::"r"(b), "d"(d[c]));
                } else if constexpr (OP == LDS128_B) {
                    double x, y;
                    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(x), "=d"(y) : "r"(a));
                    d[c] += x; d[c] += y;
                } else if constexpr (OP == LDS64_B) {
                    double x;
                    asm volatile("ld.shared.f64 %0, [%1];" : "=d"(x) : "r"(a));
                    d[c] += x;
                } else if constexpr (OP == LDS32_B) {
                    unsigned x;
                    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(x) : "r"(a));
                    u[c] += x;
                } else if constexpr (OP == LDS128_ROW) {
                    const unsigned b = (unsigned)__cvta_generic_to_shared(sh) + ((w * 32 + lane) & 255) * 16;
                    double x, y;
                    asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(x), "=d"(y) : "r"(b));
                    d[c] += x; d[c] += y;
                } else if constexpr (OP == SHFL_U) {
                    u[c] = __shfl_sync(0xffffffffu, u[c], (i + c) & 31);
                } else if constexpr (OP == SHFL_V) {
                    u[c] = __shfl_sync(0xffffffffu, u[c], (lane + i + c) & 31);
                } else if constexpr (OP == REDUX) {
                    u[c] = __reduce_max_sync(0xffffffffu, u[c] ^ lane);
                } else if constexpr (OP == DFMA) {
                    d[c] = __fma_rn(d[c], 1.0000001, 1e-9);
                } else if constexpr (OP == DMUL) {
                    d[c] = __dmul_rn(d[c], 1.0000001);
                } else if constexpr (OP == BALLOT) {
                    u[c] = __ballot_sync(0xffffffffu, (u[c] >> (lane & 7)) & 1) ^ lane;
                } else if constexpr (OP == FFMA) {
                    float f = __uint_as_float(u[c]);
                    f = __fmaf_rn(f, 1.0001f, 1e-9f);
                    u[c] = __float_as_uint(f);
                } else if constexpr (OP == IADD) {
                    u[c] = u[c] + (unsigned)i + 3u;
                } else if constexpr (OP == VOTEANY) {
                    u[c] = __any_sync(0xffffffffu, (u[c] & (1u << (lane & 3))) != 0) ^ (u[c] + 1);
                }
            }
        }
    }
    __syncwarp();
    unsigned long long t1 = clock64();
    double s = 0;
    for (int c = 0; c < 8; ++c) s += d[c] + u[c];
    sink[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}

// latency: one dependent chain
template <int OP>
__global__ void k_lat(unsigned long long *cyc, double *sink) {
    __shared__ __align__(16) double sh[64];
    const int lane = threadIdx.x & 31;
    double d = 1.0 + lane * 1e-3;
    unsigned u = lane;
    sh[lane] = lane;
    sh[lane + 32] = lane;
    __syncwarp();
    unsigned long long t0 = clock64();
#pragma unroll 16
    for (int i = 0; i < 1024; ++i) {
        if constexpr (OP == DFMA) d = __fma_rn(d, 1.0000001, 1e-9);
        else if constexpr (OP == DMUL) d = __dmul_rn(d, 1.0000001);
        else if constexpr (OP == FFMA) { float f = __uint_as_float(u); f = __fmaf_rn(f, 1.0001f, 1e-9f); u = __float_as_uint(f); }
        else if constexpr (OP == SHFL_U) u = __shfl_sync(0xffffffffu, u, 3) + lane;
        else if constexpr (OP == SHFL_V) u = __shfl_sync(0xffffffffu, u, (lane + 1) & 31);
        else if constexpr (OP == REDUX) u = __reduce_max_sync(0xffffffffu, u) ^ lane;
        else if constexpr (OP == BALLOT) u = __ballot_sync(0xffffffffu, u & 1) ^ lane;
        else if constexpr (OP == LDS64_B) { d = sh[((unsigned)__double2loint(d)) & 0]; }
        else if constexpr (OP == STS64_1) {   // store -> load round trip through smem
            if (lane == (int)(u & 31)) sh[u & 31] = d;
            __syncwarp();
            d = sh[u & 31] + 1.0;
            u = (unsigned)__double2loint(d) & 0;
        }
        else if constexpr (OP == IADD) u = u + 3u;
        else if constexpr (OP == VOTEANY) u = __any_sync(0xffffffffu, (u & 1) != 0) + u;
    }
    unsigned long long t1 = clock64();
    sink[threadIdx.x] = d + u;
    if (threadIdx.x == 0) cyc[0] = t1 - t0;
}

template <int OP>
void tput(int warps_per_sm, int nsm) {
    unsigned long long *cyc;
    double *sink;
    const int threads = warps_per_sm * 32 > 1024 ? 1024 : warps_per_sm * 32;
    const int ctas_per_sm = warps_per_sm * 32 / threads;
    const int grid = nsm * ctas_per_sm;
    cudaMalloc(&cyc, grid * 8);
    cudaMalloc(&sink, (size_t)grid * threads * 8);
    const int reps = 4;
    k_tput<OP><<<grid, threads>>>(cyc, sink, 1);
    k_tput<OP><<<grid, threads>>>(cyc, sink, reps);
    cudaDeviceSynchronize();
    unsigned long long h[2048];
    cudaMemcpy(h, cyc, grid * 8, cudaMemcpyDeviceToHost);
    double mx = 0;
    for (int i = 0; i < grid; ++i) mx = h[i] > mx ? h[i] : mx;
    const double instr_per_sm = (double)warps_per_sm * reps * ITERS * 8;
    printf("  %-22s warps/SM=%2d  %7.3f warp-instr/cycle/SM  (%6.2f cycles per instr per SM)  %s\n", names[OP],
           warps_per_sm, instr_per_sm / mx, mx / instr_per_sm, cudaGetErrorString(cudaGetLastError()));
    cudaFree(cyc);
    cudaFree(sink);
}

template <int OP>
void lat() {
    unsigned long long *cyc;
    double *sink;
    cudaMalloc(&cyc, 8);
    cudaMalloc(&sink, 32 * 8);
    k_lat<OP><<<1, 32>>>(cyc, sink);
    k_lat<OP><<<1, 32>>>(cyc, sink);
    unsigned long long h;
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("  %-22s latency %6.1f cycles/iter  %s\n", names[OP], h / 1024.0, cudaGetErrorString(cudaGetLastError()));
    cudaFree(cyc);
    cudaFree(sink);
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    printf("SMs %d\n== latency (one warp, dependent chain; includes the chain's glue op)\n", nsm);
    lat<DFMA>(); lat<DMUL>(); lat<FFMA>(); lat<SHFL_U>(); lat<SHFL_V>(); lat<REDUX>(); lat<BALLOT>();
    lat<LDS64_B>(); lat<STS64_1>(); lat<IADD>(); lat<VOTEANY>();
    printf("== throughput\n");
    for (int w : {8, 16, 32}) {
        tput<STS128_1>(w, nsm); tput<STS64_1>(w, nsm); tput<STS32_1>(w, nsm); tput<STS128_ALL>(w, nsm);
        tput<STS64_ALL>(w, nsm); tput<LDS128_B>(w, nsm); tput<LDS64_B>(w, nsm); tput<LDS32_B>(w, nsm);
        tput<LDS128_ROW>(w, nsm); tput<SHFL_U>(w, nsm); tput<SHFL_V>(w, nsm); tput<REDUX>(w, nsm);
        tput<DFMA>(w, nsm); tput<DMUL>(w, nsm); tput<BALLOT>(w, nsm); tput<FFMA>(w, nsm); tput<IADD>(w, nsm);
        tput<VOTEANY>(w, nsm);
    }
    return 0;
}
