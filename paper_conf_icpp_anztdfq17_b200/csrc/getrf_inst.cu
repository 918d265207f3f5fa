// getrf_inst.cu -- one (dtype, order range) instantiation of the GETRF kernels
// (plain and with the fused solve); compiled once per -DBJ_R=<double|float>
// -DBJ_LO=<m> -DBJ_HI=<m> so they compile in parallel.
#include "getrf_fast.cuh"
#include "setup_fused.cuh"

namespace bj {
template bj_status launch_getrf_fast<BJ_R, BJ_LO, BJ_HI, false>(BJ_R *, const int64_t *, const int64_t *, int32_t *,
                                                                int32_t *, const PlanView &, int32_t *, unsigned *,
                                                                const BJ_R *, BJ_R *, cudaStream_t);
template bj_status launch_getrf_fast<BJ_R, BJ_LO, BJ_HI, true>(BJ_R *, const int64_t *, const int64_t *, int32_t *,
                                                               int32_t *, const PlanView &, int32_t *, unsigned *,
                                                               const BJ_R *, BJ_R *, cudaStream_t);
#if BJ_LO == BJ_HI && BJ_LO >= 17
template bj_status launch_setup_fused<BJ_R, BJ_LO>(const bj_csr &, const int32_t *, BJ_R *, const int64_t *,
                                                   const int64_t *, int32_t *, int32_t *, const PlanView &,
                                                   int32_t *, unsigned *, cudaStream_t);
#endif
}  // namespace bj
