// ops.h — internal operator descriptions passed from the C-ABI layer
// (capi.cpp) to the kernel launchers.
#pragma once
#include <cuda_runtime.h>

#include "layout.h"

namespace alt {

struct OpEpilogue {
  const float *scale = nullptr;
  const float *bias = nullptr;
  const void *residual = nullptr;
  Layout *residual_l = nullptr;
  int32_t act = 0;
  // store_at-attached bias (alt_matmul_store_at): see EpiParams::batt
  const void *bias_att = nullptr;
  const int64_t *bias_att_rd = nullptr;
  int64_t bias_att_base = 0;
  int32_t bias_att_bf16 = 0;
  int32_t pads_zero = 0;  // ALT_EPI_PADS_ZERO: y's pad positions already hold 0
};

struct ConvProblem {
  int64_t N, C, H, W, K, R, S, Ho, Wo;
  int32_t Vh, Vw, ph, pw, groups;
  int32_t dh = 1, dw = 1;  // dilation (SIMT path)
  // 3-D convolution (C3D): depth extent / taps / output depth and its
  // stride, padding, dilation; D = T = Do = 1 for conv2d (logical rank 4)
  int64_t D = 1, T = 1, Do = 1;
  int32_t Vd = 1, pd = 0, dd = 1;
  bool c3d = false;
  Layout *xl, *wl, *yl;
  const void *x, *w;
  void *y;
  alt_dtype dtype;
  OpEpilogue epi;
};

struct GemmProblem {
  int64_t M, N, K;
  Layout *al, *bl, *cl;
  const void *a, *b;
  void *c;
  alt_dtype dtype;
  OpEpilogue epi;
};

alt_status relayout_launch(Layout *S, const void *src, Layout *D, void *dst, int wb,
                           cudaStream_t stream);
alt_status simt_conv(const ConvProblem &P, cudaStream_t stream);
alt_status simt_conv3d(const ConvProblem &P, cudaStream_t stream);
alt_status simt_gemm(const GemmProblem &P, cudaStream_t stream);
// tensor-core path; returns ALT_E_UNSUPPORTED (without launching) when the
// layouts / shapes cannot be served, filling *why
alt_status tc_conv(const ConvProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream,
                   alt_kernel_cfg *used);
alt_status tc_gemm(const GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream,
                   alt_kernel_cfg *used);
alt_status dw_conv(const ConvProblem &P, cudaStream_t stream, alt_kernel_cfg *used);
alt_status pool2d(const ConvProblem &P, int kind, cudaStream_t stream);
// store_at.cu (reading A26)
alt_status store_at_launch(Layout *A, const void *a, const void *b, int32_t dim, Layout *Z, void *z, int wb,
                           cudaStream_t stream);
alt_status decouple_at_launch(Layout *Z, const void *z, int32_t dim, Layout *A, void *a, void *b, int wb,
                              cudaStream_t stream);
alt_status attached_row_f32(Layout *Z, const void *z, int32_t dim, int wb, float *out, cudaStream_t stream);
// separable layout whose channel dim (logical 1) runs in 16-byte-aligned
// groups of 8 contiguous elements (pads allowed when allow_pad: owner offsets)
bool chan_vec8(const Layout &L, bool allow_pad);
// device-resident ones / zeros (>= K floats, 16-byte aligned, process lifetime)
alt_status identity_vectors(int64_t K, const float **ones, const float **zeros);

}  // namespace alt
