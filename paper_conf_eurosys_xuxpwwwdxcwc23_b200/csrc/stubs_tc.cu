// placeholder, replaced by tc_conv.cu / dwconv.cu / tune.cpp
#include "ops.h"
namespace alt {
alt_status dw_conv(const ConvProblem &, cudaStream_t, alt_kernel_cfg *) { return ALT_E_UNSUPPORTED; }
}
extern "C" alt_status alt_tune(alt_op_kind, const void *, alt_dtype, const alt_tune_space *, alt_stream_t, alt_tune_result *, float *) { return ALT_E_UNSUPPORTED; }
