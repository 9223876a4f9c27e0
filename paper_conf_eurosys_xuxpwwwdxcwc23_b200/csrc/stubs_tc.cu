// placeholder until tune.cpp lands
#include "ops.h"
extern "C" alt_status alt_tune(alt_op_kind, const void *, alt_dtype, const alt_tune_space *, alt_stream_t, alt_tune_result *, float *) { return ALT_E_UNSUPPORTED; }
