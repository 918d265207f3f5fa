// selftest.cu -- device self-test of the split IEEE divisions of common.cuh
// (Num<R>::div_pre, div_pre_flag, div_nz_flag), which the GETRF / GETRS /
// GETRI kernels use for every quotient (R3).  Each variant's quotient, where
// it claims validity, must be bit-identical to the CUDA intrinsic __ddiv_rn /
// __fdiv_rn (the correctly rounded IEEE quotient).  Test hook, not part of the
// hot path (tests/test_gpu_div.py).
#include "common.cuh"

namespace bj {

__device__ inline unsigned long long st_mix(unsigned long long z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

// Operand i of the test stream: every exponent (incl. 0 = zero/subnormal and
// all-ones = Inf/NaN) equally likely, random sign and mantissa; 1/16 of the
// operands are exact specials (+-0, +-Inf, NaN, +-1, +-min normal, +-max).
__device__ inline double st_operand_d(unsigned long long h) {
    const unsigned sel = (unsigned)(h & 15ull);
    const unsigned long long sign = (h >> 4) & 1ull;
    if (sel == 0) {
        const double sp[8] = {0.0, __longlong_as_double(0x7ff0000000000000ll), __longlong_as_double(0x7ff8000000000000ll),
                              1.0, 2.2250738585072014e-308, 1.7976931348623157e308, 4.9406564584124654e-324,
                              0.5};
        const double v = sp[(h >> 5) & 7ull];
        return sign ? -v : v;
    }
    const unsigned long long e = ((h >> 5) % 2048ull) << 52;
    const unsigned long long mant = (h >> 16) & 0xFFFFFFFFFFFFFull;
    return __longlong_as_double((long long)((sign << 63) | e | mant));
}
__device__ inline float st_operand_s(unsigned long long h) {
    const unsigned sel = (unsigned)(h & 15ull);
    const unsigned sign = (unsigned)((h >> 4) & 1ull);
    if (sel == 0) {
        const float sp[8] = {0.0f, __int_as_float(0x7f800000), __int_as_float(0x7fc00000), 1.0f, 1.17549435e-38f,
                             3.40282347e38f, 1.4e-45f, 0.5f};
        const float v = sp[(h >> 5) & 7ull];
        return sign ? -v : v;
    }
    const unsigned e = (unsigned)((h >> 5) % 256ull) << 23;
    const unsigned mant = (unsigned)((h >> 16) & 0x7FFFFFull);
    return __uint_as_float((sign << 31) | e | mant);
}

__device__ inline bool same_d(double x, double y) {
    return (x != x && y != y) || __double_as_longlong(x) == __double_as_longlong(y);
}
__device__ inline bool same_s(float x, float y) { return (x != x && y != y) || __float_as_uint(x) == __float_as_uint(y); }
__device__ inline bool normal_in_range_d(double b) {
    const unsigned e = ((unsigned)__double2hiint(b) >> 20) & 0x7ffu;
    return e != 0u && e != 0x7ffu;
}

// counts[0]: div_pre mismatches; [1]: div_pre_flag unflagged mismatches;
// [2]: div_pre_flag flagged count; [3]: div_nz_flag unflagged mismatches
// (b normal); [4]: div_nz_flag flagged; [5]: pairs tested.
template <typename R>
__global__ void k_selftest_div(int64_t n, unsigned long long seed, unsigned long long *counts, R *sample, int64_t ns) {
    unsigned long long c[6] = {0, 0, 0, 0, 0, 0};
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const unsigned long long ha = st_mix(seed ^ (2ull * (unsigned long long)i)),
                                 hb = st_mix(seed ^ (2ull * (unsigned long long)i + 1ull));
        R a, b, ref;
        bool nb;
        if constexpr (sizeof(R) == 8) {
            a = st_operand_d(ha);
            b = st_operand_d(hb);
            ref = __ddiv_rn(a, b);
            nb = normal_in_range_d(b);
        } else {
            a = st_operand_s(ha);
            b = st_operand_s(hb);
            ref = __fdiv_rn(a, b);
            nb = Num<float>::in_range(b);
        }
        auto same = [](R x, R y) {
            if constexpr (sizeof(R) == 8) return same_d(x, y);
            else return same_s(x, y);
        };
        const R y = Num<R>::rcp_refine(b);
        if (!same(Num<R>::div_pre(a, b, y), ref)) ++c[0];
        bool bad = false;
        const R q = Num<R>::div_pre_flag(a, b, y, bad);
        if (bad) ++c[2];
        else if (!same(q, ref)) ++c[1];
        // div_nz_flag's domain (GETRF fast path): b normal (fp32: in range),
        // a finite and not -0
        const bool a_ok = (a == a) && (fabs(a) <= Num<R>::big()) && !(a == R(0) && signbit(a));
        if (nb && a_ok) {
            bool bad2 = false;
            const R q2 = Num<R>::div_nz_flag(a, b, y, bad2);
            if (bad2) ++c[4];
            else if (!same(q2, ref)) ++c[3];
        }
        ++c[5];
        if (i < ns) {
            sample[3 * i] = a;
            sample[3 * i + 1] = b;
            sample[3 * i + 2] = Num<R>::div_pre(a, b, y);
        }
    }
    for (int k = 0; k < 6; ++k) atomicAdd(counts + k, c[k]);
}

}  // namespace bj

using namespace bj;

extern "C" bj_status bj_selftest_div(bj_dtype dtype, int64_t n, uint64_t seed, uint64_t *counts_h, void *sample_h,
                                     int64_t nsample) {
    if (n < 0 || !counts_h || nsample < 0 || nsample > n || (nsample > 0 && !sample_h)) return BJ_ERR_ARG;
    const size_t es = dtype == BJ_F64 ? 8 : 4;
    if (dtype != BJ_F64 && dtype != BJ_F32) return BJ_ERR_ARG;
    unsigned long long *counts = nullptr;
    void *sample = nullptr;
    BJ_CUDA_TRY(cudaMalloc((void **)&counts, 6 * sizeof(unsigned long long)));
    if (cudaMalloc(&sample, 3 * es * (size_t)(nsample > 0 ? nsample : 1)) != cudaSuccess) {
        cudaFree(counts);
        return BJ_ERR_NOMEM;
    }
    cudaMemset(counts, 0, 6 * sizeof(unsigned long long));
    const int grid = 8 * sm_count();
    if (dtype == BJ_F64)
        k_selftest_div<double><<<grid, 256>>>(n, seed, counts, (double *)sample, nsample);
    else
        k_selftest_div<float><<<grid, 256>>>(n, seed, counts, (float *)sample, nsample);
    cudaError_t e = cudaGetLastError();
    if (e == cudaSuccess) e = cudaMemcpy(counts_h, counts, 6 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    if (e == cudaSuccess && nsample > 0) e = cudaMemcpy(sample_h, sample, 3 * es * nsample, cudaMemcpyDeviceToHost);
    cudaFree(counts);
    cudaFree(sample);
    return e == cudaSuccess ? BJ_OK : BJ_ERR_CUDA;
}
