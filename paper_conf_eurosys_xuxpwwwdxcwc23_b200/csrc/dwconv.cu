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
  // work item = one output pixel x 8 channels, decoded (fastest first) as
  // channel group inside a contiguous channel run (cvec groups), q, p,
  // channel run, n: neighbouring threads touch neighbouring 16-byte vectors
  // for any NCHW[x]c (x >= 8) layout
  int32_t cvec, nrun;
  uint32_t total;
  FastDiv f_cvec, f_wo, f_ho, f_nrun;
  const int64_t *xrd[4];  // x tables (n, c, h, w)
  const int64_t *wrd[4];  // weight tables (k, 0, r, s) when w_vec
  int32_t w_vec;          // weights: 8 consecutive k contiguous per tap
  Reader wr;              // weights, any layout (slow path)
  const int64_t *yrd[4];  // y tables when vec_out
  int32_t vec_out;
  int32_t res_vec;        // residual read as 8-channel vectors (epi.res tables)
  int32_t sb_vec;         // scale / bias 16-byte aligned (float4 loads)
  Writer yw;
  EpiParams epi;
};

__device__ __forceinline__ void unpack8(const uint4 &u, float *f) {
  f[0] = __uint_as_float(u.x << 16); f[1] = __uint_as_float(u.x & 0xffff0000u);
  f[2] = __uint_as_float(u.y << 16); f[3] = __uint_as_float(u.y & 0xffff0000u);
  f[4] = __uint_as_float(u.z << 16); f[5] = __uint_as_float(u.z & 0xffff0000u);
  f[6] = __uint_as_float(u.w << 16); f[7] = __uint_as_float(u.w & 0xffff0000u);
}

struct DwItem { int n, c0, p, q; };
__device__ __forceinline__ DwItem dw_item(const DwArgs &a, uint32_t idx) {
  DwItem it;
  uint32_t t = a.f_cvec.div(idx);
  const int gi = (int)(idx - t * (uint32_t)a.cvec);
  uint32_t t2 = a.f_wo.div(t);
  it.q = (int)(t - t2 * (uint32_t)a.Wo);
  t = a.f_ho.div(t2);
  it.p = (int)(t2 - t * (uint32_t)a.Ho);
  t2 = a.f_nrun.div(t);
  const int go = (int)(t - t2 * (uint32_t)a.nrun);
  it.n = (int)t2;
  it.c0 = (go * a.cvec + gi) * 8;
  return it;
}

// one thread = one output pixel x 8 channels; bf16 in / out, fp32 math
// (taps accumulate in (r, s) order, as the oracle's O3)
template <int R, int S>
__global__ void __launch_bounds__(256, 2) k_dw_vec8(DwArgs a, const uint16_t *__restrict__ x,
                                                 const uint16_t *__restrict__ w, uint16_t *__restrict__ y) {
  pdl_wait();
  for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < a.total; idx += gridDim.x * blockDim.x) {
    const DwItem it = dw_item(a, idx);
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = 0.f;
    const int64_t base = __ldg(a.xrd[0] + it.n) + __ldg(a.xrd[1] + it.c0);
    int64_t ro[R], co[S];
#pragma unroll
    for (int r = 0; r < R; r++) {
      const int ih = it.p * a.Vh - a.ph + r;
      ro[r] = (ih < 0 || ih >= a.H) ? -1 : __ldg(a.xrd[2] + ih);
    }
#pragma unroll
    for (int s2 = 0; s2 < S; s2++) {
      const int iw = it.q * a.Vw - a.pw + s2;
      co[s2] = (iw < 0 || iw >= a.W) ? -1 : __ldg(a.xrd[3] + iw);
    }
    const int64_t wk = a.w_vec ? __ldg(a.wrd[0] + it.c0) : 0;
#pragma unroll
    for (int r = 0; r < R; r++) {
      const int64_t wr = a.w_vec ? wk + __ldg(a.wrd[2] + r) : 0;
#pragma unroll
      for (int s2 = 0; s2 < S; s2++) {
        if (ro[r] < 0 || co[s2] < 0) continue;
        const uint4 u = __ldg(reinterpret_cast<const uint4 *>(x + base + ro[r] + co[s2]));
        float f[8], g[8];
        unpack8(u, f);
        if (a.w_vec) {
          unpack8(__ldg(reinterpret_cast<const uint4 *>(w + wr + __ldg(a.wrd[3] + s2))), g);
        } else {
#pragma unroll
          for (int j = 0; j < 8; j++) g[j] = bf16_to_f32(__ldg(w + a.wr.off4(it.c0 + j, 0, r, s2)));
        }
#pragma unroll
        for (int j = 0; j < 8; j++) acc[j] = fmaf(f[j], g[j], acc[j]);
      }
    }
    float res[8];
#pragma unroll
    for (int j = 0; j < 8; j++) res[j] = 0.f;
    if (a.epi.residual) {
      const uint16_t *rp = static_cast<const uint16_t *>(a.epi.residual);
      if (a.res_vec) {
        const int64_t o = __ldg(a.epi.res.rd[0] + it.n) + __ldg(a.epi.res.rd[1] + it.c0) +
                          __ldg(a.epi.res.rd[2] + it.p) + __ldg(a.epi.res.rd[3] + it.q);
        unpack8(__ldg(reinterpret_cast<const uint4 *>(rp + o)), res);
      } else {
#pragma unroll
        for (int j = 0; j < 8; j++) {
          const int64_t o = a.epi.res.off4(it.n, it.c0 + j, it.p, it.q);
          if (o >= 0) res[j] = bf16_to_f32(__ldg(rp + o));
        }
      }
    }
    float v[8];
    {
      float ss[8], bb[8];
      if (a.sb_vec) {
        const float4 *sc = reinterpret_cast<const float4 *>(a.epi.scale + it.c0);
        const float4 *bi = reinterpret_cast<const float4 *>(a.epi.bias + it.c0);
        const float4 s0 = __ldg(sc), s1 = __ldg(sc + 1), b0 = __ldg(bi), b1 = __ldg(bi + 1);
        ss[0] = s0.x; ss[1] = s0.y; ss[2] = s0.z; ss[3] = s0.w; ss[4] = s1.x; ss[5] = s1.y; ss[6] = s1.z; ss[7] = s1.w;
        bb[0] = b0.x; bb[1] = b0.y; bb[2] = b0.z; bb[3] = b0.w; bb[4] = b1.x; bb[5] = b1.y; bb[6] = b1.z; bb[7] = b1.w;
      } else {
#pragma unroll
        for (int j = 0; j < 8; j++) { ss[j] = __ldg(a.epi.scale + it.c0 + j); bb[j] = __ldg(a.epi.bias + it.c0 + j); }
      }
#pragma unroll
      for (int j = 0; j < 8; j++) v[j] = apply_act(fmaf(acc[j], ss[j], bb[j]) + res[j], a.epi.act);
    }
    if (a.vec_out) {
      uint4 u;
      u.x = (uint32_t)f32_to_bf16_rne(v[0]) | ((uint32_t)f32_to_bf16_rne(v[1]) << 16);
      u.y = (uint32_t)f32_to_bf16_rne(v[2]) | ((uint32_t)f32_to_bf16_rne(v[3]) << 16);
      u.z = (uint32_t)f32_to_bf16_rne(v[4]) | ((uint32_t)f32_to_bf16_rne(v[5]) << 16);
      u.w = (uint32_t)f32_to_bf16_rne(v[6]) | ((uint32_t)f32_to_bf16_rne(v[7]) << 16);
      const int64_t o = __ldg(a.yrd[0] + it.n) + __ldg(a.yrd[1] + it.c0) + __ldg(a.yrd[2] + it.p) +
                        __ldg(a.yrd[3] + it.q);
      *reinterpret_cast<uint4 *>(y + o) = u;
    } else {
#pragma unroll
      for (int j = 0; j < 8; j++) write4<uint16_t>(a.yw, y, it.n, it.c0 + j, it.p, it.q, f32_to_bf16_rne(v[j]));
    }
  }
}

#ifndef ALT_DW_MINB
// resident CTAs per SM the fast form's register budget targets: measured on
// the MV2 b16 chain 2 -> 0.666 ms, 3 -> 0.760 (spills), 4 -> 0.654 (64 registers)
#define ALT_DW_MINB 4
#endif
// Fast 3x3 form (vector weights, vector output, aligned scale / bias,
// vector or no residual): every tap's x and w vectors are requested before
// any arithmetic (18 independent 16-byte loads in flight per thread; the
// padded taps load a valid address and are zeroed), so the kernel is not
// bound by one load latency per tap.  Same (r, s) accumulation order.
__global__ void __launch_bounds__(256, ALT_DW_MINB) k_dw3x3_fast(DwArgs a, const uint16_t *__restrict__ x,
                                                       const uint16_t *__restrict__ w, uint16_t *__restrict__ y) {
  pdl_wait();
  for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < a.total; idx += gridDim.x * blockDim.x) {
    const DwItem it = dw_item(a, idx);
    const int64_t base = __ldg(a.xrd[0] + it.n) + __ldg(a.xrd[1] + it.c0);
    int64_t ro[3], co[3];
    bool vr[3], vc[3];
#pragma unroll
    for (int r = 0; r < 3; r++) {
      const int ih = it.p * a.Vh - a.ph + r;
      vr[r] = ih >= 0 && ih < a.H;
      ro[r] = __ldg(a.xrd[2] + (vr[r] ? ih : 0));
    }
#pragma unroll
    for (int s2 = 0; s2 < 3; s2++) {
      const int iw = it.q * a.Vw - a.pw + s2;
      vc[s2] = iw >= 0 && iw < a.W;
      co[s2] = __ldg(a.xrd[3] + (vc[s2] ? iw : 0));
    }
    const int64_t wk = __ldg(a.wrd[0] + it.c0);
    int64_t wro[3], wco[3];
#pragma unroll
    for (int r = 0; r < 3; r++) { wro[r] = __ldg(a.wrd[2] + r); wco[r] = __ldg(a.wrd[3] + r); }
    uint4 xv[9], wv[9];
#pragma unroll
    for (int r = 0; r < 3; r++)
#pragma unroll
      for (int s2 = 0; s2 < 3; s2++) {
        xv[r * 3 + s2] = __ldg(reinterpret_cast<const uint4 *>(x + base + ro[r] + co[s2]));
        wv[r * 3 + s2] = __ldg(reinterpret_cast<const uint4 *>(w + wk + wro[r] + wco[s2]));
      }
    uint4 rv = make_uint4(0u, 0u, 0u, 0u);
    if (a.res_vec) {
      const int64_t o = __ldg(a.epi.res.rd[0] + it.n) + __ldg(a.epi.res.rd[1] + it.c0) +
                        __ldg(a.epi.res.rd[2] + it.p) + __ldg(a.epi.res.rd[3] + it.q);
      rv = __ldg(reinterpret_cast<const uint4 *>(static_cast<const uint16_t *>(a.epi.residual) + o));
    }
    const float4 *scp = reinterpret_cast<const float4 *>(a.epi.scale + it.c0);
    const float4 *bip = reinterpret_cast<const float4 *>(a.epi.bias + it.c0);
    const float4 s0 = __ldg(scp), s1 = __ldg(scp + 1), b0 = __ldg(bip), b1 = __ldg(bip + 1);
    const int64_t yo = __ldg(a.yrd[0] + it.n) + __ldg(a.yrd[1] + it.c0) + __ldg(a.yrd[2] + it.p) +
                       __ldg(a.yrd[3] + it.q);
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = 0.f;
#pragma unroll
    for (int t = 0; t < 9; t++) {
      if (!(vr[t / 3] && vc[t % 3])) continue;
      float f[8], g[8];
      unpack8(xv[t], f);
      unpack8(wv[t], g);
#pragma unroll
      for (int j = 0; j < 8; j++) acc[j] = fmaf(f[j], g[j], acc[j]);
    }
    float res[8];
    unpack8(rv, res);
    const float ss[8] = {s0.x, s0.y, s0.z, s0.w, s1.x, s1.y, s1.z, s1.w};
    const float bb[8] = {b0.x, b0.y, b0.z, b0.w, b1.x, b1.y, b1.z, b1.w};
    float v[8];
#pragma unroll
    for (int j = 0; j < 8; j++) v[j] = apply_act(fmaf(acc[j], ss[j], bb[j]) + res[j], a.epi.act);
    uint4 u;
    u.x = (uint32_t)f32_to_bf16_rne(v[0]) | ((uint32_t)f32_to_bf16_rne(v[1]) << 16);
    u.y = (uint32_t)f32_to_bf16_rne(v[2]) | ((uint32_t)f32_to_bf16_rne(v[3]) << 16);
    u.z = (uint32_t)f32_to_bf16_rne(v[4]) | ((uint32_t)f32_to_bf16_rne(v[5]) << 16);
    u.w = (uint32_t)f32_to_bf16_rne(v[6]) | ((uint32_t)f32_to_bf16_rne(v[7]) << 16);
    *reinterpret_cast<uint4 *>(y + yo) = u;
  }
}

// channel runs of 8 contiguous, 16-byte aligned vectors, one copy per element
bool chan_vec8(const Layout &L, bool allow_pad) {
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
  const bool r3 = P.R == 3 && P.S == 3, r5 = P.R == 5 && P.S == 5, r1 = P.R == 1 && P.S == 1;
  if (!r3 && !r5 && !r1) { set_error("dw: window %lldx%lld unsupported", (long long)P.R, (long long)P.S); return ALT_E_UNSUPPORTED; }
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
  // weights [K, 1, R, S]: fast path when 8 consecutive k are contiguous
  // (e.g. reorder to R S K), read as one 16-byte vector per tap
  {
    const Layout &L = *P.wl;
    bool ok = L.separable && (reinterpret_cast<uintptr_t>(P.w) & 15) == 0;
    if (ok) {
      const auto &rk = L.rd[0];
      for (size_t k = 0; k < rk.size() && ok; k += 8) {
        if (rk[k] < 0 || rk[k] % 8) ok = false;
        for (int j = 1; j < 8 && ok; j++) if (rk[k + j] != rk[k] + j) ok = false;
      }
      for (int d = 1; d < 4 && ok; d++)
        for (int64_t o : L.rd[d]) if (o < 0 || o % 8) { ok = false; break; }
    }
    a.w_vec = ok ? 1 : 0;
    if (ok) {
      SepDev sw{};
      if ((st = device_tables(P.wl, &sw, nullptr)) != ALT_OK) return st;
      for (int d = 0; d < 4; d++) a.wrd[d] = sw.rd[d];
    }
  }
  a.res_vec = P.epi.residual && a.epi.res.sep && chan_vec8(*P.epi.residual_l, true) &&
              (reinterpret_cast<uintptr_t>(P.epi.residual) & 15) == 0 ? 1 : 0;
  // identity scale / bias are materialised so the kernel reads them as vectors
  if (!a.epi.scale || !a.epi.bias) {
    const float *ones = nullptr, *zeros = nullptr;
    if ((st = identity_vectors(P.K, &ones, &zeros)) != ALT_OK) return st;
    if (!a.epi.scale) a.epi.scale = ones;
    if (!a.epi.bias) a.epi.bias = zeros;
  }
  a.sb_vec = ((reinterpret_cast<uintptr_t>(a.epi.scale) | reinterpret_cast<uintptr_t>(a.epi.bias)) & 15) == 0;
  // contiguous 8-channel groups of x (and y): the fastest work-item digit
  {
    const auto &rc = P.xl->rd[1];
    int cvec = 1;
    const int ng = (int)(P.C / 8);
    while (cvec * 2 <= ng && ng % (cvec * 2) == 0) {
      bool ok = true;
      for (int g = 0; g < ng && ok; g += cvec * 2)
        for (int j = 0; j < cvec * 2 * 8; j++) if (rc[g * 8 + j] != rc[g * 8] + j) { ok = false; break; }
      if (!ok) break;
      cvec *= 2;
    }
    a.cvec = cvec;
    a.nrun = ng / cvec;
  }
  const int64_t total = P.N * (P.C / 8) * P.Ho * P.Wo;
  if (total == 0) return ALT_OK;
  if (total >= (1ll << 31)) { set_error("dw: too many outputs"); return ALT_E_UNSUPPORTED; }
  a.total = (uint32_t)total;
  a.f_cvec = FastDiv((uint32_t)a.cvec);
  a.f_wo = FastDiv((uint32_t)a.Wo);
  a.f_ho = FastDiv((uint32_t)a.Ho);
  a.f_nrun = FastDiv((uint32_t)a.nrun);
  int dev = 0, nsm = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((total + 255) / 256, (int64_t)nsm * 16));
  const auto *x = static_cast<const uint16_t *>(P.x);
  const auto *w = static_cast<const uint16_t *>(P.w);
  auto *y = static_cast<uint16_t *>(P.y);
  const bool fast = r3 && a.w_vec && a.vec_out && a.sb_vec && (!P.epi.residual || a.res_vec);
  if (fast) launch_pdl(k_dw3x3_fast, grid, 256, 0, stream, a, x, w, y);
  else if (r3) launch_pdl(k_dw_vec8<3, 3>, grid, 256, 0, stream, a, x, w, y);
  else if (r1) launch_pdl(k_dw_vec8<1, 1>, grid, 256, 0, stream, a, x, w, y);
  else launch_pdl(k_dw_vec8<5, 5>, grid, 256, 0, stream, a, x, w, y);
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
  // vector path (bf16, 8-channel runs in x and y): work-item order as DwArgs
  int32_t cvec, nrun;
  uint32_t total;
  FastDiv f_cvec, f_wo, f_ho, f_nrun;
  const int64_t *xrd[4], *yrd[4];
};

// one thread = one output pixel x 8 channels (bf16); max is exact, the
// average sums in (r, s) order in fp32 like the scalar kernel
__global__ void __launch_bounds__(256) k_pool_vec8(PoolArgs a, const uint16_t *__restrict__ x,
                                                   uint16_t *__restrict__ y) {
  pdl_wait();
  DwArgs d{};  // work-item decode shared with the depthwise kernel
  d.cvec = a.cvec; d.nrun = a.nrun; d.Wo = a.Wo; d.Ho = a.Ho;
  d.f_cvec = a.f_cvec; d.f_wo = a.f_wo; d.f_ho = a.f_ho; d.f_nrun = a.f_nrun;
  for (uint32_t idx = blockIdx.x * blockDim.x + threadIdx.x; idx < a.total; idx += gridDim.x * blockDim.x) {
    const DwItem it = dw_item(d, idx);
    const int64_t base = __ldg(a.xrd[0] + it.n) + __ldg(a.xrd[1] + it.c0);
    float acc[8];
#pragma unroll
    for (int j = 0; j < 8; j++) acc[j] = a.kind == 0 ? -INFINITY : 0.f;
    int cnt = 0;
    if (a.R == 3 && a.S == 3) {
      // all nine window vectors requested before any arithmetic (padded taps
      // load a valid address and are skipped), same (r, s) order
      int64_t ro[3], co[3];
      bool vr[3], vc[3];
#pragma unroll
      for (int r = 0; r < 3; r++) {
        const int ih = it.p * a.Vh - a.ph + r;
        vr[r] = ih >= 0 && ih < a.H;
        ro[r] = __ldg(a.xrd[2] + (vr[r] ? ih : 0));
        const int iw = it.q * a.Vw - a.pw + r;
        vc[r] = iw >= 0 && iw < a.W;
        co[r] = __ldg(a.xrd[3] + (vc[r] ? iw : 0));
      }
      uint4 xv[9];
#pragma unroll
      for (int t = 0; t < 9; t++) xv[t] = __ldg(reinterpret_cast<const uint4 *>(x + base + ro[t / 3] + co[t % 3]));
#pragma unroll
      for (int t = 0; t < 9; t++) {
        if (!(vr[t / 3] && vc[t % 3])) continue;
        float f[8];
        unpack8(xv[t], f);
#pragma unroll
        for (int j = 0; j < 8; j++) acc[j] = a.kind == 0 ? fmaxf(acc[j], f[j]) : acc[j] + f[j];
        cnt++;
      }
    } else
    for (int r = 0; r < a.R; r++) {
      const int ih = it.p * a.Vh - a.ph + r;
      if (ih < 0 || ih >= a.H) continue;
      const int64_t ro = base + __ldg(a.xrd[2] + ih);
      for (int s2 = 0; s2 < a.S; s2++) {
        const int iw = it.q * a.Vw - a.pw + s2;
        if (iw < 0 || iw >= a.W) continue;
        float f[8];
        unpack8(__ldg(reinterpret_cast<const uint4 *>(x + ro + __ldg(a.xrd[3] + iw))), f);
#pragma unroll
        for (int j = 0; j < 8; j++) acc[j] = a.kind == 0 ? fmaxf(acc[j], f[j]) : acc[j] + f[j];
        cnt++;
      }
    }
    if (a.kind == 1) {
#pragma unroll
      for (int j = 0; j < 8; j++) acc[j] = cnt ? acc[j] / (float)cnt : 0.f;
    }
    uint4 u;
    u.x = (uint32_t)f32_to_bf16_rne(acc[0]) | ((uint32_t)f32_to_bf16_rne(acc[1]) << 16);
    u.y = (uint32_t)f32_to_bf16_rne(acc[2]) | ((uint32_t)f32_to_bf16_rne(acc[3]) << 16);
    u.z = (uint32_t)f32_to_bf16_rne(acc[4]) | ((uint32_t)f32_to_bf16_rne(acc[5]) << 16);
    u.w = (uint32_t)f32_to_bf16_rne(acc[6]) | ((uint32_t)f32_to_bf16_rne(acc[7]) << 16);
    const int64_t o = __ldg(a.yrd[0] + it.n) + __ldg(a.yrd[1] + it.c0) + __ldg(a.yrd[2] + it.p) +
                      __ldg(a.yrd[3] + it.q);
    *reinterpret_cast<uint4 *>(y + o) = u;
  }
}


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
  if (P.dtype == ALT_BF16 && P.C % 8 == 0 && chan_vec8(*P.xl, true) && chan_vec8(*P.yl, false) &&
      total / 8 < (1ll << 31)) {
    SepDev sx{}, sy{};
    if ((st = device_tables(P.xl, &sx, nullptr)) != ALT_OK) return st;
    if ((st = device_tables(P.yl, &sy, nullptr)) != ALT_OK) return st;
    for (int d = 0; d < 4; d++) { a.xrd[d] = sx.rd[d]; a.yrd[d] = sy.rd[d]; }
    // contiguous 8-channel groups common to x and y
    const int ng = (int)(P.C / 8);
    int cvec = 1;
    while (cvec * 2 <= ng && ng % (cvec * 2) == 0) {
      bool ok = true;
      for (const Layout *L : {P.xl, P.yl}) {
        const auto &rc = L->rd[1];
        for (int g = 0; g < ng && ok; g += cvec * 2)
          for (int j = 0; j < cvec * 2 * 8; j++) if (rc[g * 8 + j] != rc[g * 8] + j) { ok = false; break; }
      }
      if (!ok) break;
      cvec *= 2;
    }
    a.cvec = cvec; a.nrun = ng / cvec;
    a.total = (uint32_t)(total / 8);
    a.f_cvec = FastDiv((uint32_t)a.cvec); a.f_wo = FastDiv((uint32_t)a.Wo);
    a.f_ho = FastDiv((uint32_t)a.Ho); a.f_nrun = FastDiv((uint32_t)a.nrun);
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((a.total + 255) / 256, 148 * 16));
    launch_pdl(k_pool_vec8, grid, 256, 0, stream, a, static_cast<const uint16_t *>(P.x), static_cast<uint16_t *>(P.y));
    count_launch();
    if (cudaGetLastError() != cudaSuccess) { set_error("pool launch failed"); return ALT_E_CUDA; }
    return ALT_OK;
  }
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
