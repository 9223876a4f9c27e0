// simt_conv.cu — the generic CUDA-core path: conv2d / GEMM whose operands are
// gathered through ANY compiled layout (separable tables or the primitive
// interpreter) and whose result is written through any separable layout.
//
// This is the "operators consume transformed layouts without
// re-implementation" property in its most general
// form; it is the correctness fallback and the fp32 path.  The tensor-core
// path (tc_conv.cu) covers the layouts a TMA box can be cut from.
//
//   conv : y[n,k,p,q] = sum_{c,r,s} x[n, g(k) C/G + c, pV-pad+r, qV-pad+s] w[k,c,r,s]
//          (P:498-514), implicit GEMM rows = (n,p,q), cols = k, red = (c,r,s)
//   gemm : C[m,n] = sum_k A[m,k] B[k,n]
#include <cuda_runtime.h>

#include <algorithm>

#include "epilogue.cuh"
#include "ops.h"

namespace alt {

struct SimtArgs {
  int32_t is_conv;
  int64_t M, Ncol, Kred;        // implicit GEMM sizes
  // conv geometry
  int64_t N, C, H, W, K, R, S, Ho, Wo;
  int32_t Vh, Vw, ph, pw;
  int32_t dh, dw;  // dilation
  Reader xr, wr;                // conv: x (n,c,h,w), w (k,c,r,s); gemm: A (m,k), B (k,n)
  Writer yw;
  EpiParams epi;
};

constexpr int BM = 64, BN = 64, BK = 16;

template <typename T>
__global__ void __launch_bounds__(256) k_simt_igemm(SimtArgs a, const T *__restrict__ x,
                                                    const T *__restrict__ w, T *__restrict__ y) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  __shared__ int64_t row_n[BM];
  __shared__ int32_t row_h[BM], row_w[BM];
  const int tid = threadIdx.x;
  const int64_t m0 = (int64_t)blockIdx.x * BM, n0 = (int64_t)blockIdx.y * BN;
  const int64_t RS = a.R * a.S;
  if (tid < BM) {
    int64_t m = m0 + tid;
    if (a.is_conv) {
      int64_t mm = m < a.M ? m : 0;
      int64_t q = mm % a.Wo, t2 = mm / a.Wo;
      int64_t p = t2 % a.Ho, n = t2 / a.Ho;
      row_n[tid] = m < a.M ? n : -1;
      row_h[tid] = (int32_t)(p * a.Vh - a.ph);
      row_w[tid] = (int32_t)(q * a.Vw - a.pw);
    } else {
      row_n[tid] = m < a.M ? m : -1;
    }
  }
  __syncthreads();
  const int tx = tid % 16, ty = tid / 16;
  float acc[4][4] = {};
  for (int64_t k0 = 0; k0 < a.Kred; k0 += BK) {
    // A tile: BM x BK, 4 per thread
#pragma unroll
    for (int e = 0; e < 4; e++) {
      const int idx = tid + e * 256;
      const int mm = idx % BM, kk = idx / BM;
      const int64_t k = k0 + kk;
      float v = 0.f;
      const int64_t rn = row_n[mm];
      if (rn >= 0 && k < a.Kred) {
        int64_t off;
        if (a.is_conv) {
          const int64_t c = k / RS, rs = k - c * RS;
          const int64_t r = rs / a.S, s = rs - r * a.S;
          const int64_t ih = row_h[mm] + r * a.dh, iw = row_w[mm] + s * a.dw;
          off = (ih >= 0 && ih < a.H && iw >= 0 && iw < a.W) ? a.xr.off4(rn, c, ih, iw) : -1;
        } else {
          off = a.xr.off2(rn, k);
        }
        if (off >= 0) v = load_as_f32<T>(x, off);
      }
      As[kk][mm] = v;
    }
    // B tile: BK x BN
#pragma unroll
    for (int e = 0; e < 4; e++) {
      const int idx = tid + e * 256;
      const int nn = idx % BN, kk = idx / BN;
      const int64_t k = k0 + kk, n = n0 + nn;
      float v = 0.f;
      if (k < a.Kred && n < a.Ncol) {
        int64_t off;
        if (a.is_conv) {
          const int64_t c = k / RS, rs = k - c * RS;
          const int64_t r = rs / a.S, s = rs - r * a.S;
          off = a.wr.off4(n, c, r, s);
        } else {
          off = a.wr.off2(k, n);
        }
        if (off >= 0) v = load_as_f32<T>(w, off);
      }
      Bs[kk][nn] = v;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; kk++) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; i++) av[i] = As[kk][ty * 4 + i];
#pragma unroll
      for (int j = 0; j < 4; j++) bv[j] = Bs[kk][tx * 4 + j];
#pragma unroll
      for (int i = 0; i < 4; i++)
#pragma unroll
        for (int j = 0; j < 4; j++) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    __syncthreads();
  }
  // fused epilogue, stored through the output layout
#pragma unroll
  for (int i = 0; i < 4; i++) {
    const int mm = ty * 4 + i;
    const int64_t rn = row_n[mm];
    if (rn < 0) continue;
    const int64_t m = m0 + mm;
#pragma unroll
    for (int j = 0; j < 4; j++) {
      const int64_t n = n0 + tx * 4 + j;
      if (n >= a.Ncol) continue;
      float v = acc[i][j];
      if (a.epi.scale) v *= __ldg(a.epi.scale + n);
      if (a.epi.bias || a.epi.batt) v += epi_bias(a.epi, n);
      if (a.is_conv) {
        const int64_t q = m % a.Wo, p = (m / a.Wo) % a.Ho;
        if (a.epi.residual) {
          int64_t o = a.epi.res.off4(rn, n, p, q);
          if (o >= 0) v += load_as_f32<T>(static_cast<const T *>(a.epi.residual), o);
        }
        v = apply_act(v, a.epi.act);
        write4<T>(a.yw, y, rn, n, p, q, from_f32<T>(v));
      } else {
        if (a.epi.residual) {
          int64_t o = a.epi.res.off2(m, n);
          if (o >= 0) v += load_as_f32<T>(static_cast<const T *>(a.epi.residual), o);
        }
        v = apply_act(v, a.epi.act);
        write2<T>(a.yw, y, m, n, from_f32<T>(v));
      }
    }
  }
}

// grouped / depthwise conv: one thread per output element, k fastest
template <typename T>
__global__ void __launch_bounds__(256) k_simt_grouped(SimtArgs a, int64_t G, const T *__restrict__ x,
                                                      const T *__restrict__ w, T *__restrict__ y) {
  const int64_t total = a.N * a.K * a.Ho * a.Wo;
  const int64_t Cg = a.C / G, Kg = a.K / G;
  for (int64_t idx = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; idx < total;
       idx += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = idx % a.K;
    int64_t t = idx / a.K;
    const int64_t q = t % a.Wo;
    t /= a.Wo;
    const int64_t p = t % a.Ho, n = t / a.Ho;
    const int64_t g = k / Kg;
    float acc = 0.f;
    for (int64_t c = 0; c < Cg; c++)
      for (int64_t r = 0; r < a.R; r++) {
        const int64_t ih = p * a.Vh - a.ph + r * a.dh;
        if (ih < 0 || ih >= a.H) continue;
        for (int64_t s = 0; s < a.S; s++) {
          const int64_t iw = q * a.Vw - a.pw + s * a.dw;
          if (iw < 0 || iw >= a.W) continue;
          const int64_t xo = a.xr.off4(n, g * Cg + c, ih, iw);
          const int64_t wo = a.wr.off4(k, c, r, s);
          if (xo < 0 || wo < 0) continue;
          acc = fmaf(load_as_f32<T>(x, xo), load_as_f32<T>(w, wo), acc);
        }
      }
    float v = acc;
    if (a.epi.scale) v *= __ldg(a.epi.scale + k);
    if (a.epi.bias) v += __ldg(a.epi.bias + k);
    if (a.epi.residual) {
      const int64_t o = a.epi.res.off4(n, k, p, q);
      if (o >= 0) v += load_as_f32<T>(static_cast<const T *>(a.epi.residual), o);
    }
    v = apply_act(v, a.epi.act);
    write4<T>(a.yw, y, n, k, p, q, from_f32<T>(v));
  }
}

// ------------------------------------------------------------------- host --
alt_status make_reader(Layout *L, Reader *r) {
  SepDev sd{};
  const LayoutDesc *desc = nullptr;
  alt_status st = device_tables(L, &sd, &desc);
  if (st != ALT_OK) return st;
  r->sep = L->separable ? 1 : 0;
  r->lrank = L->lrank;
  for (int d = 0; d < 4; d++) r->rd[d] = d < L->lrank ? sd.rd[d] : nullptr;
  r->desc = desc;
  return ALT_OK;
}

alt_status make_writer(Layout *L, Writer *w) {
  if (!L->separable) {
    set_error("output layouts must be separable (no fuse across logical dims); relayout instead");
    return ALT_E_UNSUPPORTED;
  }
  SepDev sd{};
  alt_status st = device_tables(L, &sd, nullptr);
  if (st != ALT_OK) return st;
  w->lrank = L->lrank;
  for (int d = 0; d < 4; d++) {
    w->wptr[d] = d < L->lrank ? sd.wptr[d] : nullptr;
    w->wlist[d] = d < L->lrank ? sd.wlist[d] : nullptr;
  }
  return ALT_OK;
}

alt_status make_epi(const OpEpilogue &e, EpiParams *p) {
  p->scale = e.scale;
  p->bias = e.bias;
  p->residual = e.residual;
  p->act = e.act;
  p->batt = e.bias_att;
  p->batt_rd = e.bias_att_rd;
  p->batt_base = e.bias_att_base;
  p->batt_bf16 = e.bias_att_bf16;
  p->res = Reader{};
  if (e.residual) return make_reader(e.residual_l, &p->res);
  return ALT_OK;
}

alt_status simt_conv(const ConvProblem &P, cudaStream_t stream) {
  SimtArgs a{};
  a.is_conv = 1;
  a.N = P.N; a.C = P.C; a.H = P.H; a.W = P.W; a.K = P.K; a.R = P.R; a.S = P.S;
  a.Ho = P.Ho; a.Wo = P.Wo;
  a.Vh = P.Vh; a.Vw = P.Vw; a.ph = P.ph; a.pw = P.pw;
  a.dh = P.dh; a.dw = P.dw;
  a.M = P.N * P.Ho * P.Wo;
  a.Ncol = P.K;
  a.Kred = (P.C / P.groups) * P.R * P.S;
  alt_status st;
  if ((st = make_reader(P.xl, &a.xr)) != ALT_OK) return st;
  if ((st = make_reader(P.wl, &a.wr)) != ALT_OK) return st;
  if ((st = make_writer(P.yl, &a.yw)) != ALT_OK) return st;
  if ((st = make_epi(P.epi, &a.epi)) != ALT_OK) return st;
  if (a.M == 0 || a.Ncol == 0) return ALT_OK;
  if (P.groups == 1) {
    dim3 grid((unsigned)((a.M + BM - 1) / BM), (unsigned)((a.Ncol + BN - 1) / BN));
    if (P.dtype == ALT_BF16)
      k_simt_igemm<uint16_t><<<grid, 256, 0, stream>>>(a, (const uint16_t *)P.x, (const uint16_t *)P.w, (uint16_t *)P.y);
    else
      k_simt_igemm<float><<<grid, 256, 0, stream>>>(a, (const float *)P.x, (const float *)P.w, (float *)P.y);
  } else {
    int64_t total = P.N * P.K * P.Ho * P.Wo;
    int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 32);
    if (P.dtype == ALT_BF16)
      k_simt_grouped<uint16_t><<<grid, 256, 0, stream>>>(a, P.groups, (const uint16_t *)P.x, (const uint16_t *)P.w, (uint16_t *)P.y);
    else
      k_simt_grouped<float><<<grid, 256, 0, stream>>>(a, P.groups, (const float *)P.x, (const float *)P.w, (float *)P.y);
  }
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("simt conv launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

alt_status simt_gemm(const GemmProblem &P, cudaStream_t stream) {
  SimtArgs a{};
  a.is_conv = 0;
  a.M = P.M;
  a.Ncol = P.N;
  a.Kred = P.K;
  alt_status st;
  if ((st = make_reader(P.al, &a.xr)) != ALT_OK) return st;
  if ((st = make_reader(P.bl, &a.wr)) != ALT_OK) return st;
  if ((st = make_writer(P.cl, &a.yw)) != ALT_OK) return st;
  if ((st = make_epi(P.epi, &a.epi)) != ALT_OK) return st;
  if (a.M == 0 || a.Ncol == 0) return ALT_OK;
  dim3 grid((unsigned)((a.M + BM - 1) / BM), (unsigned)((a.Ncol + BN - 1) / BN));
  if (P.dtype == ALT_BF16)
    k_simt_igemm<uint16_t><<<grid, 256, 0, stream>>>(a, (const uint16_t *)P.a, (const uint16_t *)P.b, (uint16_t *)P.c);
  else
    k_simt_igemm<float><<<grid, 256, 0, stream>>>(a, (const float *)P.a, (const float *)P.b, (float *)P.c);
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("simt gemm launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

}  // namespace alt

// ------------------------------------------------------------ C3D (SIMT) --
// The generic CUDA-core path of alt_conv3d: one thread per
// output element y[n,k,od,oh,ow], the (c, t, r, s) sum in fp32 with x / w
// gathered through any compiled rank-5 layout, the epilogue of O6, and the
// result written to every position y's layout holds it at (pad zeros
// included).  Correctness fallback; the tensor-core path (tc_conv.cu) serves
// the layouts a TMA box can be cut from.
namespace alt {

struct Simt3Args {
  int64_t N, C, D, H, W, K, T, R, S, Do, Ho, Wo;
  int32_t Vd, Vh, Vw, pd, ph, pw, dd, dh, dw, G;
  Reader5 xr, wr, rr;
  Writer5 yw;
  const float *scale, *bias;
  const void *residual;
  int32_t act;
};

template <typename T>
__global__ void __launch_bounds__(256) k_simt_conv3d(const Simt3Args a, const T *__restrict__ x,
                                                     const T *__restrict__ w, T *__restrict__ y) {
  const int64_t total = a.N * a.K * a.Do * a.Ho * a.Wo;
  const int64_t Cg = a.C / a.G;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t r_ = i;
    const int64_t ow = r_ % a.Wo; r_ /= a.Wo;
    const int64_t oh = r_ % a.Ho; r_ /= a.Ho;
    const int64_t od = r_ % a.Do; r_ /= a.Do;
    const int64_t k = r_ % a.K;
    const int64_t n = r_ / a.K;
    const int64_t g = k * a.G / a.K;
    float acc = 0.f;
    for (int64_t c = 0; c < Cg; c++)
      for (int64_t t = 0; t < a.T; t++) {
        const int64_t id = od * a.Vd - a.pd + a.dd * t;
        if (id < 0 || id >= a.D) continue;
        for (int64_t r = 0; r < a.R; r++) {
          const int64_t ih = oh * a.Vh - a.ph + a.dh * r;
          if (ih < 0 || ih >= a.H) continue;
          for (int64_t s = 0; s < a.S; s++) {
            const int64_t iw = ow * a.Vw - a.pw + a.dw * s;
            if (iw < 0 || iw >= a.W) continue;
            const int64_t xo = a.xr.off5(n, g * Cg + c, id, ih, iw), wo = a.wr.off5(k, c, t, r, s);
            if (xo < 0 || wo < 0) continue;
            acc = fmaf(load_as_f32<T>(x, xo), load_as_f32<T>(w, wo), acc);
          }
        }
      }
    float v = (a.scale ? __ldg(a.scale + k) : 1.f) * acc + (a.bias ? __ldg(a.bias + k) : 0.f);
    if (a.residual) {
      const int64_t ro = a.rr.off5(n, k, od, oh, ow);
      if (ro >= 0) v += load_as_f32<T>(static_cast<const T *>(a.residual), ro);
    }
    v = apply_act(v, a.act);
    const T out = from_f32<T>(v);
    // every position y's layout holds (n, k, od, oh, ow) at; owned pads get 0
    const int64_t idx[5] = {n, k, od, oh, ow};
    int32_t lo[5], hi[5];
#pragma unroll
    for (int d = 0; d < 5; d++) {
      lo[d] = __ldg(a.yw.wptr[d] + idx[d]);
      hi[d] = __ldg(a.yw.wptr[d] + idx[d] + 1);
    }
    for (int32_t i0 = lo[0]; i0 < hi[0]; i0++) {
      const int64_t c0 = __ldg(a.yw.wlist[0] + i0);
      for (int32_t i1 = lo[1]; i1 < hi[1]; i1++) {
        const int64_t c1 = __ldg(a.yw.wlist[1] + i1);
        for (int32_t i2 = lo[2]; i2 < hi[2]; i2++) {
          const int64_t c2 = __ldg(a.yw.wlist[2] + i2);
          for (int32_t i3 = lo[3]; i3 < hi[3]; i3++) {
            const int64_t c3 = __ldg(a.yw.wlist[3] + i3);
            for (int32_t i4 = lo[4]; i4 < hi[4]; i4++) {
              const int64_t c4 = __ldg(a.yw.wlist[4] + i4);
              const int64_t o = (c0 >> 1) + (c1 >> 1) + (c2 >> 1) + (c3 >> 1) + (c4 >> 1);
              y[o] = ((c0 | c1 | c2 | c3 | c4) & 1) ? T(0) : out;
            }
          }
        }
      }
    }
  }
}

static alt_status make_reader5(Layout *L, Reader5 *r) {
  SepDev sd{};
  const LayoutDesc *desc = nullptr;
  alt_status st = device_tables(L, &sd, &desc);
  if (st != ALT_OK) return st;
  r->sep = L->separable ? 1 : 0;
  for (int d = 0; d < 5; d++) r->rd[d] = sd.rd[d];
  r->desc = desc;
  return ALT_OK;
}

alt_status simt_conv3d(const ConvProblem &P, cudaStream_t stream) {
  if (!P.yl->separable) {
    set_error("output layouts must be separable (no fuse across logical dims); relayout instead");
    return ALT_E_UNSUPPORTED;
  }
  Simt3Args a{};
  a.N = P.N; a.C = P.C; a.D = P.D; a.H = P.H; a.W = P.W; a.K = P.K; a.T = P.T; a.R = P.R; a.S = P.S;
  a.Do = P.Do; a.Ho = P.Ho; a.Wo = P.Wo;
  a.Vd = P.Vd; a.Vh = P.Vh; a.Vw = P.Vw; a.pd = P.pd; a.ph = P.ph; a.pw = P.pw;
  a.dd = P.dd; a.dh = P.dh; a.dw = P.dw; a.G = P.groups;
  alt_status st;
  if ((st = make_reader5(P.xl, &a.xr)) != ALT_OK) return st;
  if ((st = make_reader5(P.wl, &a.wr)) != ALT_OK) return st;
  if (P.epi.residual && (st = make_reader5(P.epi.residual_l, &a.rr)) != ALT_OK) return st;
  SepDev sy{};
  if ((st = device_tables(P.yl, &sy, nullptr)) != ALT_OK) return st;
  for (int d = 0; d < 5; d++) { a.yw.wptr[d] = sy.wptr[d]; a.yw.wlist[d] = sy.wlist[d]; }
  a.scale = P.epi.scale;
  a.bias = P.epi.bias;
  a.residual = P.epi.residual;
  a.act = P.epi.act;
  const int64_t total = P.N * P.K * P.Do * P.Ho * P.Wo;
  if (total == 0) return ALT_OK;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 32);
  if (P.dtype == ALT_BF16)
    k_simt_conv3d<uint16_t><<<grid, 256, 0, stream>>>(a, (const uint16_t *)P.x, (const uint16_t *)P.w, (uint16_t *)P.y);
  else
    k_simt_conv3d<float><<<grid, 256, 0, stream>>>(a, (const float *)P.x, (const float *)P.w, (float *)P.y);
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("simt conv3d launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

}  // namespace alt
