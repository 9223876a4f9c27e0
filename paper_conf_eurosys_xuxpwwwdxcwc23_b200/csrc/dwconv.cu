// dwconv.cu — depthwise conv2d (groups == C == K) on channel-tiled layouts.
//
// DEP is memory-bound: 9 MACs per output for 3x3.  The
// layout-native formulation: with NCHW[x]c-family layouts (x >= 8 channels
// contiguous per pixel) one thread owns one output pixel x 8 channels,
// reads each 3x3 window as 16-byte vectors (coalesced across the warp:
// consecutive threads = consecutive pixels) and writes one 16-byte vector
// through the output layout.  HBM traffic ~ input once + output once; the
// window overlap is served by L1/L2.  Other layouts run the generic path.
#include <cuda_runtime.h>

#include <algorithm>

#include "epilogue.cuh"
#include "ops.h"

namespace alt {

alt_status make_reader(Layout *L, Reader *r);
alt_status make_writer(Layout *L, Writer *w);
alt_status make_epi(const OpEpilogue &e, EpiParams *p);

struct DwArgs {
  int32_t N, C, H, W, Ho, Wo, R, S, Vh, Vw, ph, pw;
  const int64_t *xrd[4];  // x tables (n, c, h, w)
  Reader wr;              // weights (k, 0, r, s)
  const int64_t *yrd[4];  // y tables when vec_out
  int32_t vec_out;
  Writer yw;
  EpiParams epi;
};

__device__ __forceinline__ void unpack8(const uint4 &u, float *f) {
  f[0] = __uint_as_float(u.x << 16); f[1] = __uint_as_float(u.x & 0xffff0000u);
  f[2] = __uint_as_float(u.y << 16); f[3] = __uint_as_float(u.y & 0xffff0000u);
  f[4] = __uint_as_float(u.z << 16); f[5] = __uint_as_float(u.z & 0xffff0000u);
  f[6] = __uint_as_float(u.w << 16); f[7] = __uint_as_float(u.w & 0xffff0000u);
}

// one thread = one output pixel x 8 channels; bf16 in / out, fp32 math
template <int RS>
__global__ void __launch_bounds__(256) k_dw_vec8(DwArgs a, const uint16_t *__restrict__ x,
                                                 const uint16_t *__restrict__ w, uint16_t *__restrict__ y) {
  const int64_t cg = a.C / 8;
  const int64_t total = (int64_t)a.N * cg * a.Ho * a.Wo;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    // pixel fastest (coalesced for NCHW[x]c), then h, channel group, image
    const int q = (int)(idx % a.Wo);
    int64_t t = idx / a.Wo;
    const int p = (int)(t % a.Ho);
    t /= a.Ho;
    const int c0 = (int)(t % cg) * 8;
    const int n = (int)(t / cg);
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = 0.f;
    const int64_t base = __ldg(a.xrd[0] + n) + __ldg(a.xrd[1] + c0);
#pragma unroll
    for (int rs = 0; rs < RS; rs++) {
      const int r = rs / a.S, s = rs % a.S;
      const int ih = p * a.Vh - a.ph + r, iw = q * a.Vw - a.pw + s;
      if (ih < 0 || ih >= a.H || iw < 0 || iw >= a.W) continue;
      const uint4 u = __ldg(reinterpret_cast<const uint4 *>(x + base + __ldg(a.xrd[2] + ih) + __ldg(a.xrd[3] + iw)));
      float f[8];
      unpack8(u, f);
#pragma unroll
      for (int j = 0; j < 8; j++) {
        const int64_t wo = a.wr.off4(c0 + j, 0, r, s);
        acc[j] = fmaf(f[j], bf16_to_f32(__ldg(w + wo)), acc[j]);
      }
    }
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) {
      float t2 = acc[j];
      if (a.epi.scale) t2 *= __ldg(a.epi.scale + c0 + j);
      if (a.epi.bias) t2 += __ldg(a.epi.bias + c0 + j);
      if (a.epi.residual) {
        const int64_t o = a.epi.res.off4(n, c0 + j, p, q);
        if (o >= 0) t2 += bf16_to_f32(__ldg(static_cast<const uint16_t *>(a.epi.residual) + o));
      }
      v[j] = apply_act(t2, a.epi.act);
    }
    if (a.vec_out) {
      uint4 u;
      u.x = (uint32_t)f32_to_bf16_rne(v[0]) | ((uint32_t)f32_to_bf16_rne(v[1]) << 16);
      u.y = (uint32_t)f32_to_bf16_rne(v[2]) | ((uint32_t)f32_to_bf16_rne(v[3]) << 16);
      u.z = (uint32_t)f32_to_bf16_rne(v[4]) | ((uint32_t)f32_to_bf16_rne(v[5]) << 16);
      u.w = (uint32_t)f32_to_bf16_rne(v[6]) | ((uint32_t)f32_to_bf16_rne(v[7]) << 16);
      const int64_t o = __ldg(a.yrd[0] + n) + __ldg(a.yrd[1] + c0) + __ldg(a.yrd[2] + p) + __ldg(a.yrd[3] + q);
      *reinterpret_cast<uint4 *>(y + o) = u;
    } else {
#pragma unroll
      for (int j = 0; j < 8; j++) write4<uint16_t>(a.yw, y, n, c0 + j, p, q, f32_to_bf16_rne(v[j]));
    }
  }
}

// channel runs of 8 contiguous, 16-byte aligned vectors, one copy per element
static bool chan_vec8(const Layout &L, bool allow_pad) {
  if (!L.separable) return false;
  if (!allow_pad && (L.flags & (ALT_HAS_PAD | ALT_HAS_UNFOLD))) return false;
  for (int d = 0; d < L.lrank; d++)
    if (L.max_copies[d] != 1 && !allow_pad) return false;
  const auto &rc = L.rd[1];
  if (rc.size() % 8) return false;
  for (size_t c = 0; c < rc.size(); c += 8) {
    if (rc[c] < 0 || rc[c] % 8) return false;
    for (int j = 1; j < 8; j++)
      if (rc[c + j] != rc[c] + j) return false;
  }
  for (int d = 0; d < L.lrank; d++) {
    if (d == 1) continue;
    for (int64_t o : L.rd[d])
      if (o < 0 || o % 8) return false;
  }
  return true;
}

alt_status dw_conv(const ConvProblem &P, cudaStream_t stream, alt_kernel_cfg *used) {
  if (P.dtype != ALT_BF16 || P.groups != P.C || P.K != P.C) { set_error("dw: bf16 depthwise only"); return ALT_E_UNSUPPORTED; }
  if (P.C % 8) { set_error("dw: C %% 8 != 0"); return ALT_E_UNSUPPORTED; }
  // x: channel runs of 8 (pads allowed: they are only read as real zeros)
  if (!chan_vec8(*P.xl, true)) { set_error("dw: x layout has no 8-channel vectors"); return ALT_E_UNSUPPORTED; }
  const int RS = (int)(P.R * P.S);
  if (RS != 9 && RS != 1 && RS != 25) { set_error("dw: window %lld unsupported", (long long)RS); return ALT_E_UNSUPPORTED; }
  DwArgs a{};
  a.N = (int32_t)P.N; a.C = (int32_t)P.C; a.H = (int32_t)P.H; a.W = (int32_t)P.W;
  a.Ho = (int32_t)P.Ho; a.Wo = (int32_t)P.Wo; a.R = (int32_t)P.R; a.S = (int32_t)P.S;
  a.Vh = P.Vh; a.Vw = P.Vw; a.ph = P.ph; a.pw = P.pw;
  SepDev sx{};
  alt_status st;
  if ((st = device_tables(P.xl, &sx, nullptr)) != ALT_OK) return st;
  for (int d = 0; d < 4; d++) a.xrd[d] = sx.rd[d];
  if ((st = make_reader(P.wl, &a.wr)) != ALT_OK) return st;
  if ((st = make_writer(P.yl, &a.yw)) != ALT_OK) return st;
  if ((st = make_epi(P.epi, &a.epi)) != ALT_OK) return st;
  a.vec_out = chan_vec8(*P.yl, false) ? 1 : 0;
  if (a.vec_out) {
    SepDev sy{};
    if ((st = device_tables(P.yl, &sy, nullptr)) != ALT_OK) return st;
    for (int d = 0; d < 4; d++) a.yrd[d] = sy.rd[d];
  }
  const int64_t total = P.N * (P.C / 8) * P.Ho * P.Wo;
  int dev = 0, nsm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, (int64_t)nsm * 16));
  const auto *x = static_cast<const uint16_t *>(P.x);
  const auto *w = static_cast<const uint16_t *>(P.w);
  auto *y = static_cast<uint16_t *>(P.y);
  if (RS == 9) k_dw_vec8<9><<<grid, 256, 0, stream>>>(a, x, w, y);
  else if (RS == 1) k_dw_vec8<1><<<grid, 256, 0, stream>>>(a, x, w, y);
  else k_dw_vec8<25><<<grid, 256, 0, stream>>>(a, x, w, y);
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("dw launch failed"); return ALT_E_CUDA; }
  alt_kernel_cfg u{};
  u.path = ALT_PATH_DW;
  if (used) *used = u;
  return ALT_OK;
}

// ------------------------------------------------------------------ pooling
// Support op of the ResNet chains (not one of the paper's operators, SURVEY
// K10): max / average over an R x S window; padded taps are skipped (max) or
// excluded from the count (avg, count_include_pad = false).
struct PoolArgs {
  int32_t N, C, H, W, Ho, Wo, R, S, Vh, Vw, ph, pw, kind;
  Reader xr;
  Writer yw;
};

template <typename T>
__global__ void __launch_bounds__(256) k_pool(PoolArgs a, const T *__restrict__ x, T *__restrict__ y) {
  const int64_t total = (int64_t)a.N * a.C * a.Ho * a.Wo;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    // channel fastest: neighbouring threads read neighbouring channels
    const int c = (int)(idx % a.C);
    int64_t t = idx / a.C;
    const int q = (int)(t % a.Wo);
    t /= a.Wo;
    const int p = (int)(t % a.Ho);
    const int n = (int)(t / a.Ho);
    float acc = a.kind == 0 ? -INFINITY : 0.f;
    int cnt = 0;
    for (int r = 0; r < a.R; r++) {
      const int ih = p * a.Vh - a.ph + r;
      if (ih < 0 || ih >= a.H) continue;
      for (int s = 0; s < a.S; s++) {
        const int iw = q * a.Vw - a.pw + s;
        if (iw < 0 || iw >= a.W) continue;
        const int64_t o = a.xr.off4(n, c, ih, iw);
        if (o < 0) continue;
        const float v = load_as_f32<T>(x, o);
        acc = a.kind == 0 ? fmaxf(acc, v) : acc + v;
        cnt++;
      }
    }
    if (a.kind == 1) acc = cnt ? acc / (float)cnt : 0.f;
    write4<T>(a.yw, y, n, c, p, q, from_f32<T>(acc));
  }
}

alt_status pool2d(const ConvProblem &P, int kind, cudaStream_t stream) {
  PoolArgs a{};
  a.N = (int32_t)P.N; a.C = (int32_t)P.C; a.H = (int32_t)P.H; a.W = (int32_t)P.W;
  a.Ho = (int32_t)P.Ho; a.Wo = (int32_t)P.Wo; a.R = (int32_t)P.R; a.S = (int32_t)P.S;
  a.Vh = P.Vh; a.Vw = P.Vw; a.ph = P.ph; a.pw = P.pw; a.kind = kind;
  alt_status st;
  if ((st = make_reader(P.xl, &a.xr)) != ALT_OK) return st;
  if ((st = make_writer(P.yl, &a.yw)) != ALT_OK) return st;
  const int64_t total = P.N * P.C * P.Ho * P.Wo;
  if (total == 0) return ALT_OK;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, 148 * 32));
  if (P.dtype == ALT_BF16)
    k_pool<uint16_t><<<grid, 256, 0, stream>>>(a, static_cast<const uint16_t *>(P.x), static_cast<uint16_t *>(P.y));
  else
    k_pool<float><<<grid, 256, 0, stream>>>(a, static_cast<const float *>(P.x), static_cast<float *>(P.y));
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("pool launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

}  // namespace alt
