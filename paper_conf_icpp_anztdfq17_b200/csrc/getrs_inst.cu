// getrs_inst.cu -- one (dtype, size class) instantiation of the GETRS kernels;
// compiled once per -DBJ_R=<double|float> -DBJ_LO=<m> -DBJ_HI=<m>.
#include "getrs_kernels.cuh"

namespace bj {
template bj_status launch_getrs_class<BJ_R, BJ_LO, BJ_HI>(const BJ_R *, const int64_t *, const int64_t *,
                                                          const int32_t *, const BJ_R *, BJ_R *, const PlanView &,
                                                          cudaStream_t);
}  // namespace bj
