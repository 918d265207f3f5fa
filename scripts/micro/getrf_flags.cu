// Per-order GETRF flag sweep (micro benchmark; not part of the library).\n// nvcc ... -DFV=<flags> -DMSTART=<first order>\n// Micro benchmark of the library's GETRF kernel variants (getrf_fast.cuh,
// compile-time flag F) on fixed batches; not part of the library.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        -I paper_conf_icpp_anztdfq17_b200/csrc scripts/micro/getrf_var.cu -o scripts/micro/bin/getrf_var
#include <algorithm>
#include <cstdio>
#include <vector>
#include "getrf_fast.cuh"

namespace bj {
void count_launch(int) {}
int sm_count() { int n; cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, 0); return n; }
}
using namespace bj;

__global__ void fill(double *a, int64_t n, unsigned long long seed) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long z = (i + 1) * 0x9E3779B97F4A7C15ull + seed;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
        a[i] = (double)(z >> 11) * 0x1p-53 * 2.0 - 1.0;
    }
}

__global__ void to_float(const double *a, float *f, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        f[i] = (float)a[i];
}

struct Batch {
    int64_t nb;
    std::vector<int> m_of;
    double *A, *A0;
    float *Af, *Af0;
    int64_t *dvo, *dve, *dbs;
    int32_t *dord, *piv, *info, *safe;
    unsigned *cnt;
    double bytes;
};

static Batch make(int64_t nb, int lo, int hi) {
    Batch b;
    b.nb = nb;
    b.m_of.resize(nb);
    std::vector<int64_t> vo(nb + 1), ve(nb + 1), cntb(kBins + 1, 0), bs(kBins + 1, 0);
    std::vector<int32_t> ord(nb);
    for (int64_t i = 0; i < nb; ++i) b.m_of[i] = lo + (int)((i * (hi - lo + 1)) / nb);
    vo[0] = ve[0] = 0;
    b.bytes = 0;
    for (int64_t i = 0; i < nb; ++i) {
        int m = b.m_of[i];
        vo[i + 1] = vo[i] + (m * m + 3) / 4 * 4; ve[i + 1] = ve[i] + m; ord[i] = (int32_t)i; cntb[m]++;
        b.bytes += 2.0 * 8 * m * m + 4 * m + 20;
    }
    int64_t acc = 0;
    for (int k = 0; k < kBins; ++k) { bs[k] = acc; acc += cntb[k]; }
    bs[kBins] = acc;
    cudaMalloc(&b.A, vo[nb] * 8); cudaMalloc(&b.A0, vo[nb] * 8);
    cudaMalloc(&b.dvo, (nb + 1) * 8); cudaMalloc(&b.dve, (nb + 1) * 8); cudaMalloc(&b.dbs, (kBins + 1) * 8);
    cudaMalloc(&b.dord, nb * 4); cudaMalloc(&b.piv, ve[nb] * 4); cudaMalloc(&b.info, nb * 4);
    cudaMalloc(&b.safe, nb * 4); cudaMalloc(&b.cnt, 4);
    cudaMemcpy(b.dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(b.dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(b.dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(b.dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(b.A0, vo[nb], 12345);
    b.cnt = b.cnt;
    static int64_t tot;
    tot = vo[nb];
    cudaMemcpy(b.A, b.A0, tot * 8, cudaMemcpyDeviceToDevice);
    cudaMalloc(&b.Af, tot * 4); cudaMalloc(&b.Af0, tot * 4);
    to_float<<<1024, 256>>>(b.A0, b.Af0, tot);
    return b;
}


#ifdef FLOAT
using RT = float;
#else
using RT = double;
#endif
template <int M, int F>
void run_order(int64_t nb) {
    Batch b = make(nb, M, M);
    int64_t tot = 0;
    for (int64_t i = 0; i < nb; ++i) tot += (int64_t)(M * M + 3) / 4 * 4;
    auto kern = k_getrf_fast<RT, M, M, F>;
    RT *A = sizeof(RT) == 8 ? (RT *)b.A : (RT *)b.Af;
    const RT *A0 = sizeof(RT) == 8 ? (const RT *)b.A0 : (const RT *)b.Af0;
    int per_sm = 0;
    cudaFuncSetAttribute(kern, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kFastThreads, 0);
    const int grid = per_sm * sm_count();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    for (int rep = 0; rep < 8; ++rep) {
        cudaMemcpy(A, A0, tot * sizeof(RT), cudaMemcpyDeviceToDevice);
        cudaMemset(b.cnt, 0, 4);
        cudaEventRecord(e0);
        kern<<<grid, kFastThreads>>>(A, b.dvo, b.dve, b.piv, b.info, b.dord, b.dbs, b.safe, b.cnt, nullptr, nullptr);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep > 1) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    printf("%s M=%2d F=%3d occ=%2d warps/SM med %8.1f us min %8.1f us err=%s\n", sizeof(RT) == 8 ? "f64" : "f32", M, F,
           per_sm * 4, ts[ts.size() / 2] * 1e3, ts[0] * 1e3, cudaGetErrorString(cudaGetLastError()));
    cudaFree(b.A); cudaFree(b.A0); cudaFree(b.Af); cudaFree(b.Af0);
}
template <int M>
void run_all() {
    run_order<M, FV>(34500);
#ifndef MEND
#define MEND 32
#endif
    if constexpr (M < MEND) run_all<M + 1>();
}
int main() {
    setvbuf(stdout, NULL, _IONBF, 0);
    run_all<MSTART>();
    return 0;
}
