// Micro benchmark of GETRF kernel variants on fixed-order batches (one size
// class kernel restricted to a single order).  Not part of the library.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 \
//        -I include -I paper_conf_icpp_anztdfq17_b200/csrc scripts/micro/getrf_bench.cu
#include <cstdio>
#include <vector>
#include <algorithm>
#include "getrf_kernels.cuh"
#include "getrf_r2_experiment.cuh"

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

// Mixed-order batch of class [LO, HI] (orders cycling LO..HI), like C3.
template <int LO, int HI, int V>
void run_mix(int64_t nb, const char *name) {
    std::vector<int64_t> vo(nb + 1), ve(nb + 1);
    std::vector<int32_t> ord(nb);
    std::vector<int64_t> cnt(kBins + 1, 0);
    // blocks sorted by order already (as the plan would): order m for a contiguous range
    std::vector<int> m_of(nb);
    for (int64_t i = 0; i < nb; ++i) m_of[i] = LO + (int)((i * (HI - LO + 1)) / nb);
    vo[0] = 0; ve[0] = 0;
    for (int64_t i = 0; i < nb; ++i) { int m = m_of[i]; vo[i + 1] = vo[i] + (m * m + 1) / 2 * 2; ve[i + 1] = ve[i] + m; ord[i] = (int32_t)i; cnt[m]++; }
    std::vector<int64_t> bs(kBins + 1, 0);
    int64_t acc = 0;
    for (int b = 0; b < kBins; ++b) { bs[b] = acc; acc += cnt[b]; }
    bs[kBins] = acc;
    double *A, *A0; int64_t *dvo, *dve, *dbs; int32_t *dord, *piv, *info;
    const int64_t tot = vo[nb];
    cudaMalloc(&A, tot * 8); cudaMalloc(&A0, tot * 8);
    cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&piv, ve[nb] * 4); cudaMalloc(&info, nb * 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(A0, tot, 12345);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_class<double, LO, HI, V>, kGetrfThreads, 0);
    const int grid = per_sm * sm_count();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    for (int rep = 0; rep < 5; ++rep) {
        cudaMemcpy(A, A0, tot * 8, cudaMemcpyDeviceToDevice);
        cudaEventRecord(e0);
        k_getrf_class<double, LO, HI, V><<<grid, kGetrfThreads>>>(A, dvo, dve, piv, info, dord, dbs);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    double bytes = 0;
    for (int64_t i = 0; i < nb; ++i) bytes += 2.0 * 8 * m_of[i] * m_of[i] + 4 * m_of[i] + 20;
    printf("%-26s M=%2d..%2d V=%2d occ=%d/SM  %8.1f us  %7.1f GB/s  %6.1f Mblk/s  err=%s\n", name, LO, HI, V, per_sm * 4,
           ts[0] * 1e3, bytes / (ts[0] * 1e-3) / 1e9, nb / (ts[0] * 1e-3) / 1e6, cudaGetErrorString(cudaGetLastError()));
    cudaFree(A); cudaFree(A0); cudaFree(dvo); cudaFree(dve); cudaFree(dbs); cudaFree(dord); cudaFree(piv); cudaFree(info);
}

template <int LO, int HI, int F>
void run_mix_fast(int64_t nb, const char *name) {
    std::vector<int64_t> vo(nb + 1), ve(nb + 1);
    std::vector<int32_t> ord(nb), sz(nb);
    std::vector<int64_t> cnt(kBins + 1, 0);
    std::vector<int> m_of(nb);
    for (int64_t i = 0; i < nb; ++i) m_of[i] = LO + (int)((i * (HI - LO + 1)) / nb);
    vo[0] = 0; ve[0] = 0;
    for (int64_t i = 0; i < nb; ++i) { int m = m_of[i]; sz[i] = m; vo[i + 1] = vo[i] + (m * m + 1) / 2 * 2; ve[i + 1] = ve[i] + m; ord[i] = (int32_t)i; cnt[m]++; }
    std::vector<int64_t> bs(kBins + 1, 0);
    int64_t acc = 0;
    for (int b = 0; b < kBins; ++b) { bs[b] = acc; acc += cnt[b]; }
    bs[kBins] = acc;
    double *A, *A0; int64_t *dvo, *dve, *dbs; int32_t *dord, *piv, *info, *list, *dsz; unsigned *count;
    const int64_t tot = vo[nb];
    cudaMalloc(&A, tot * 8); cudaMalloc(&A0, tot * 8);
    cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&piv, ve[nb] * 4); cudaMalloc(&info, nb * 4); cudaMalloc(&list, nb * 4);
    cudaMalloc(&count, 4); cudaMalloc(&dsz, nb * 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dsz, sz.data(), nb * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(A0, tot, 12345);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_fast<double, LO, HI, F>, kFastThreads, 0);
    const int grid = per_sm * sm_count();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    unsigned hc = 0;
    for (int rep = 0; rep < 5; ++rep) {
        cudaMemcpy(A, A0, tot * 8, cudaMemcpyDeviceToDevice);
        cudaMemset(count, 0, 4);
        cudaEventRecord(e0);
        k_getrf_fast<double, LO, HI, F><<<grid, kFastThreads>>>(A, dvo, dve, piv, info, dord, dbs, list, count);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) ts.push_back(ms);
        cudaMemcpy(&hc, count, 4, cudaMemcpyDeviceToHost);
    }
    std::sort(ts.begin(), ts.end());
    double bytes = 0;
    for (int64_t i = 0; i < nb; ++i) bytes += 2.0 * 8 * m_of[i] * m_of[i] + 4 * m_of[i] + 20;
    printf("%-26s M=%2d..%2d  occ=%d/SM  %8.1f us  %7.1f GB/s  %6.1f Mblk/s  deferred=%u err=%s\n", name, LO, HI, per_sm * 4,
           ts[0] * 1e3, bytes / (ts[0] * 1e-3) / 1e9, nb / (ts[0] * 1e-3) / 1e6, hc, cudaGetErrorString(cudaGetLastError()));
    cudaFree(A); cudaFree(A0); cudaFree(dvo); cudaFree(dve); cudaFree(dbs); cudaFree(dord); cudaFree(piv); cudaFree(info);
    cudaFree(list); cudaFree(count); cudaFree(dsz);
}

template <int M>
void run_fast1(int64_t nb, const char *name) {
    const int64_t per = (M * M + 1) / 2 * 2;
    std::vector<int64_t> vo(nb + 1), ve(nb + 1); std::vector<int32_t> ord(nb);
    for (int64_t i = 0; i <= nb; ++i) { vo[i] = i * per; ve[i] = i * M; }
    for (int64_t i = 0; i < nb; ++i) ord[i] = (int32_t)i;
    std::vector<int64_t> bs(kBins + 1); for (int b = 0; b <= kBins; ++b) bs[b] = b <= M ? 0 : nb;
    double *A; int64_t *dvo, *dve, *dbs; int32_t *dord, *piv, *info, *list; unsigned *count;
    cudaMalloc(&A, per * nb * 8); cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&piv, nb * M * 4); cudaMalloc(&info, nb * 4); cudaMalloc(&list, nb * 4); cudaMalloc(&count, 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice); cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice); cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(A, per * nb, 777); cudaMemset(count, 0, 4);
    k_getrf_fast<double, M, M, 0><<<sm_count(), 32>>>(A, dvo, dve, piv, info, dord, dbs, list, count);
    cudaDeviceSynchronize();
#ifdef BJ_TRACE
    long long t[64]; cudaMemcpyFromSymbol(t, g_ftrace, sizeof(t));
#else
    long long t[64] = {0};
#endif
    printf("%s M=%d per-step cycles:", name, M);
    for (int k = 0; k + 1 < M; ++k) printf(" %lld", t[k + 1] - t[k]);
    printf("\n");
}

template <int M, int V>
void run(int64_t nb, const char *name, int force_warps_per_sm = 0) {
    const int64_t per = (M * M + 1) / 2 * 2;
    std::vector<int64_t> vo(nb + 1), ve(nb + 1);
    std::vector<int32_t> ord(nb);
    for (int64_t i = 0; i <= nb; ++i) { vo[i] = i * per; ve[i] = i * M; }
    for (int64_t i = 0; i < nb; ++i) ord[i] = (int32_t)i;
    std::vector<int64_t> bs(kBins + 1);
    for (int b = 0; b <= kBins; ++b) bs[b] = b <= M ? 0 : nb;
    double *A, *A0; int64_t *dvo, *dve, *dbs; int32_t *dord, *piv, *info;
    cudaMalloc(&A, per * nb * 8); cudaMalloc(&A0, per * nb * 8);
    cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&piv, nb * M * 4); cudaMalloc(&info, nb * 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(A0, per * nb, 12345);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_class<double, M, M, V>, kGetrfThreads, 0);
    int grid = per_sm * sm_count();
    int threads = kGetrfThreads;
    if (force_warps_per_sm) { grid = sm_count() * force_warps_per_sm; threads = 32; }
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    for (int rep = 0; rep < 6; ++rep) {
        cudaMemcpy(A, A0, per * nb * 8, cudaMemcpyDeviceToDevice);
        cudaEventRecord(e0);
        k_getrf_class<double, M, M, V><<<grid, threads>>>(A, dvo, dve, piv, info, dord, dbs);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    const double bytes = (double)nb * (2.0 * 8 * M * M + 4 * M + 20);
    const double blocks_per_warp = (double)nb / (grid * threads / 32);
    printf("%-22s M=%2d V=%d warps/SM=%2d  %8.1f us  %7.1f GB/s  %6.1f Mblk/s  cycles/block/warp=%8.0f err=%s\n", name, M, V,
           grid * threads / 32 / sm_count(), ts[0] * 1e3, bytes / (ts[0] * 1e-3) / 1e9, nb / (ts[0] * 1e-3) / 1e6,
           ts[0] * 1e-3 * 1.965e9 / blocks_per_warp, cudaGetErrorString(cudaGetLastError()));
    cudaFree(A); cudaFree(A0); cudaFree(dvo); cudaFree(dve); cudaFree(dbs); cudaFree(dord); cudaFree(piv); cudaFree(info);
}

template <typename R, bool R2 = true>
void run_r2(int64_t nb, int LO, int HI, const char *name) {
    std::vector<int64_t> vo(nb + 1), ve(nb + 1);
    std::vector<int32_t> ord(nb);
    std::vector<int64_t> cnt(kBins + 1, 0);
    std::vector<int> m_of(nb);
    const int el = 16 / (int)sizeof(R);
    for (int64_t i = 0; i < nb; ++i) m_of[i] = LO + (int)((i * (HI - LO + 1)) / nb);
    vo[0] = 0; ve[0] = 0;
    for (int64_t i = 0; i < nb; ++i) { int m = m_of[i]; vo[i + 1] = vo[i] + (m * m + el - 1) / el * el; ve[i + 1] = ve[i] + m; ord[i] = (int32_t)i; cnt[m]++; }
    std::vector<int64_t> bs(kBins + 1, 0);
    int64_t acc = 0;
    for (int b = 0; b < kBins; ++b) { bs[b] = acc; acc += cnt[b]; }
    bs[kBins] = acc;
    R *A, *A0; int64_t *dvo, *dve, *dbs; int32_t *dord, *piv, *info, *list; unsigned *count;
    const int64_t tot = vo[nb];
    cudaMalloc(&A, tot * sizeof(R)); cudaMalloc(&A0, tot * sizeof(R));
    cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&piv, ve[nb] * 4); cudaMalloc(&info, nb * 4); cudaMalloc(&list, nb * 4);
    cudaMalloc(&count, 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    {
        std::vector<R> h(tot);
        unsigned long long z = 88172645463325252ull;
        for (int64_t i = 0; i < tot; ++i) { z ^= z << 13; z ^= z >> 7; z ^= z << 17; h[i] = (R)((double)(z >> 11) * 0x1p-52 - 1.0); }
        cudaMemcpy(A0, h.data(), tot * sizeof(R), cudaMemcpyHostToDevice);
    }
    PlanView pv; pv.nblocks = nb; pv.order = dord; pv.bin_start = dbs;
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    unsigned hc = 0;
    for (int rep = 0; rep < 6; ++rep) {
        cudaMemcpy(A, A0, tot * sizeof(R), cudaMemcpyDeviceToDevice);
        cudaMemset(count, 0, 4);
        cudaEventRecord(e0);
        if constexpr (R2) launch_getrf_r2<R>(A, dvo, dve, piv, info, pv, list, count, 0);
        else launch_getrf_fast<R, 17, 32>(A, dvo, dve, piv, info, pv, list, count, 0);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) ts.push_back(ms);
        cudaMemcpy(&hc, count, 4, cudaMemcpyDeviceToHost);
    }
    std::sort(ts.begin(), ts.end());
    double bytes = 0;
    for (int64_t i = 0; i < nb; ++i) bytes += 2.0 * sizeof(R) * m_of[i] * m_of[i] + 4 * m_of[i] + 20;
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrf_r2<R>, kR2Threads, r2_dyn_smem(sizeof(R)));
    printf("%s sel=%d minb=%d %-22s occ=%d warps/SM  %8.1f us  %7.1f GB/s  %6.1f Mblk/s  deferred=%u err=%s\n",
           R2 ? "R2" : "F0", BJ_R2_SELECT, BJ_R2_MINB, name, per_sm * 4, ts[ts.size() / 2] * 1e3, bytes / (ts[ts.size() / 2] * 1e-3) / 1e9,
           nb / (ts[ts.size() / 2] * 1e-3) / 1e6, hc, cudaGetErrorString(cudaGetLastError()));
    cudaFree(A); cudaFree(A0); cudaFree(dvo); cudaFree(dve); cudaFree(dbs); cudaFree(dord); cudaFree(piv); cudaFree(info);
    cudaFree(list); cudaFree(count);
}

int main(int argc, char **argv) {
#ifdef BJ_TRACE
    run_fast1<32>(148, "FAST 1 warp");
#else
    if (argc > 2) {
        run_r2<float, false>(552000, 17, 32, "mix 17..32 f32 F0");
        run_r2<float, true>(552000, 17, 32, "mix 17..32 f32 R2");
        run_r2<double, false>(552000, 17, 32, "mix 17..32 f64 F0");
        run_r2<double, true>(552000, 17, 32, "mix 17..32 f64 R2");
        return 0;
    }
    if (argc > 1) {
        run_r2<double>(40000, 32, 32, "m=32 f64");
        run_r2<double>(552000, 17, 32, "mix 17..32 f64");
        run_r2<float>(552000, 17, 32, "mix 17..32 f32");
        return 0;
    }
    run_mix_fast<32, 32, 0>(40000, "m=32 F0");
    run_mix_fast<32, 32, 16>(40000, "m=32 X no publish");
    run_mix_fast<32, 32, 32>(40000, "m=32 X no division");
    run_mix_fast<32, 32, 64>(40000, "m=32 X no search");
    run_mix_fast<32, 32, 128>(40000, "m=32 X all lanes store");
    run_mix_fast<32, 32, 256>(40000, "m=32 X one pair only");
    run_mix_fast<17, 32, 0>(552000, "mix 17..32 F0");
#endif
    return 0;
}
