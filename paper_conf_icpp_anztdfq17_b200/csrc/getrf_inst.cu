// getrf_inst.cu -- one (dtype, size class) instantiation of the GETRF kernels;
// compiled once per -DBJ_R=<double|float> -DBJ_LO=<m> -DBJ_HI=<m>.
#include "getrf_fast.cuh"

namespace bj {
template bj_status launch_getrf_fast<BJ_R, BJ_LO, BJ_HI>(BJ_R *, const int64_t *, const int64_t *, int32_t *,
                                                         int32_t *, const PlanView &, int32_t *, unsigned *,
                                                         cudaStream_t);
}  // namespace bj
