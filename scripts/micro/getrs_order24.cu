// GETRS single-order kernel vs class kernel on the C5 apply (micro; not part of the library).
// (derived from getrs_bench.cu) Micro benchmark of the GETRS size-class kernel (ring depth BJ_RS_DEPTH,
// occupancy BJ_RS_MINB) on a fixed-order and a mixed-order batch.  Not part
// of the library.  Build (per variant):
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -DBJ_RS_DEPTH=8 -DBJ_RS_MINB=4 \
//        -I include -I paper_conf_icpp_anztdfq17_b200/csrc scripts/micro/getrs_bench.cu -o /tmp/rsb
#include <cstdio>
#include <vector>
#include <algorithm>
#include "getrs_kernels.cuh"

namespace bj {
void count_launch(int) {}
int sm_count() { int n; cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, 0); return n; }
}
using namespace bj;

__global__ void fill(double *a, int64_t n, unsigned long long seed) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long z = (i + 1) * 0x9E3779B97F4A7C15ull + seed;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
        a[i] = (double)(z >> 11) * 0x1p-53 + 1.0;   // [1, 2): no slow-path quotients
    }
}

template <int LO, int HI>
void run(int64_t nb, int mlo, int mhi, const char *name) {
    std::vector<int> m_of(nb);
    for (int64_t i = 0; i < nb; ++i) m_of[i] = mlo + (int)((i * 7919) % (mhi - mlo + 1));   // interleaved orders
    std::vector<int64_t> vo(nb + 1), ve(nb + 1), cnt(kBins + 1, 0);
    for (int64_t i = 0; i < nb; ++i) { int m = m_of[i]; vo[i + 1] = vo[i] + (m * m + 1) / 2 * 2; ve[i + 1] = ve[i] + m; cnt[m]++; }
    std::vector<int64_t> bs(kBins + 1, 0);
    int64_t acc = 0;
    for (int b = 0; b < kBins; ++b) { bs[b] = acc; acc += cnt[b]; }
    bs[kBins] = acc;
    std::vector<int32_t> ord(nb), pos(kBins, 0);
    for (int b = 0; b < kBins; ++b) pos[b] = (int)bs[b];
    for (int64_t i = 0; i < nb; ++i) ord[pos[m_of[i]]++] = (int32_t)i;
    std::vector<int32_t> piv(ve[nb]);
    for (int64_t i = 0; i < nb; ++i) for (int r = 0; r < m_of[i]; ++r) piv[ve[i] + r] = (r * 5 + 3) % m_of[i];
    double *A, *bv, *xv; int64_t *dvo, *dve, *dbs; int32_t *dord, *dpiv;
    cudaMalloc(&A, vo[nb] * 8); cudaMalloc(&bv, ve[nb] * 8); cudaMalloc(&xv, ve[nb] * 8);
    cudaMalloc(&dvo, (nb + 1) * 8); cudaMalloc(&dve, (nb + 1) * 8); cudaMalloc(&dbs, (kBins + 1) * 8);
    cudaMalloc(&dord, nb * 4); cudaMalloc(&dpiv, ve[nb] * 4);
    cudaMemcpy(dvo, vo.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dve, ve.data(), (nb + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dbs, bs.data(), (kBins + 1) * 8, cudaMemcpyHostToDevice);
    cudaMemcpy(dord, ord.data(), nb * 4, cudaMemcpyHostToDevice);
    cudaMemcpy(dpiv, piv.data(), ve[nb] * 4, cudaMemcpyHostToDevice);
    fill<<<1024, 256>>>(A, vo[nb], 12345);
    fill<<<1024, 256>>>(bv, ve[nb], 999);
    // L2 flush buffer
    char *flush; const size_t fl = 256u << 20; cudaMalloc(&flush, fl);
    int per_sm = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_getrs_class<double, LO, HI>, kGetrsThreads, 0);
    const int grid = per_sm * sm_count();
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    std::vector<float> ts;
    for (int rep = 0; rep < 8; ++rep) {
        cudaMemsetAsync(flush, rep, fl);
        cudaEventRecord(e0);
        k_getrs_class<double, LO, HI><<<grid, kGetrsThreads>>>(A, dvo, dve, dpiv, bv, xv, dord, dbs);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (rep) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    double bytes = 0;
    for (int64_t i = 0; i < nb; ++i) { double m = m_of[i]; bytes += 8 * m * m + 4 * m + 16 * m + 16; }
    const double med = ts[ts.size() / 2];
    printf("D=%2d MINB=%d %-20s occ=%2d warps/SM  med %8.1f us  %7.1f GB/s  %7.1f Mblk/s  err=%s\n", BJ_RS_DEPTH,
           BJ_RS_MINB, name, per_sm * 4, med * 1e3, bytes / (med * 1e-3) / 1e9, nb / (med * 1e-3) / 1e6,
           cudaGetErrorString(cudaGetLastError()));
    cudaFree(A); cudaFree(bv); cudaFree(xv); cudaFree(dvo); cudaFree(dve); cudaFree(dbs); cudaFree(dord);
    cudaFree(dpiv); cudaFree(flush);
}

int main() {
    run<24, 24>(83259, 24, 24, "C5 83k x 24 (order-24 kernel)");
    run<17, 32>(83259, 24, 24, "C5 83k x 24 (class kernel)");
    return 0;
}
