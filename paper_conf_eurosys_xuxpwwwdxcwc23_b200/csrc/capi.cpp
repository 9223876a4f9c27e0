// capi.cpp — the C-ABI of libalt.so (include/alt.h): validation and dispatch.
#include <cuda_runtime.h>

#include <atomic>
#include <cstring>
#include <new>

#include "alt.h"
#include "layout.h"
#include "ops.h"

namespace alt {
const char *last_error();
static std::atomic<uint64_t> g_launches{0};
void count_launch(int n) { g_launches.fetch_add((uint64_t)n, std::memory_order_relaxed); }
static thread_local alt_kernel_cfg g_last_plan{};
void set_last_plan(const alt_kernel_cfg &c) { g_last_plan = c; }

// device (or managed) pointer?  Host pointers are rejected: no CPU fallback.
// Validated pointers are remembered (direct-mapped, per thread) so the hot
// path does not pay cudaPointerGetAttributes on every call.
static bool is_device_ptr(const void *p) {
  if (!p) return false;
  static thread_local const void *seen[512] = {};
  const size_t h = (reinterpret_cast<uintptr_t>(p) >> 8) & 511;
  if (seen[h] == p) return true;
  cudaPointerAttributes at{};
  if (cudaPointerGetAttributes(&at, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  const bool ok = at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
  if (ok) seen[h] = p;
  return ok;
}

static bool shape_is(const Layout *L, int r, const int64_t *s) {
  if (L->lrank != r) return false;
  for (int d = 0; d < r; d++)
    if (L->lshape[d] != s[d]) return false;
  return true;
}

static alt_status fill_epi(const alt_epilogue *e, const Layout *yl, OpEpilogue *o) {
  *o = OpEpilogue{};
  if (!e) return ALT_OK;
  if (e->act < 0 || e->act > 2) { set_error("epilogue: unknown activation %d", e->act); return ALT_E_INVALID; }
  o->scale = e->scale;
  o->bias = e->bias;
  o->act = e->act;
  o->pads_zero = (e->flags & ALT_EPI_PADS_ZERO) ? 1 : 0;
  if ((e->scale && !is_device_ptr(e->scale)) || (e->bias && !is_device_ptr(e->bias))) {
    set_error("epilogue: scale / bias must be device pointers");
    return ALT_E_INVALID;
  }
  if (e->residual) {
    if (!e->residual_l) { set_error("epilogue: residual without layout"); return ALT_E_INVALID; }
    if (!is_device_ptr(e->residual)) { set_error("epilogue: residual must be a device pointer"); return ALT_E_INVALID; }
    Layout *rl = &e->residual_l->impl;
    if (!shape_is(rl, yl->lrank, yl->lshape)) { set_error("epilogue: residual logical shape != output"); return ALT_E_SHAPE; }
    o->residual = e->residual;
    o->residual_l = rl;
  }
  return ALT_OK;
}
}  // namespace alt

using namespace alt;

extern "C" {

const char *alt_status_str(alt_status s) {
  switch (s) {
    case ALT_OK: return "ALT_OK";
    case ALT_E_INVALID: return "ALT_E_INVALID";
    case ALT_E_SHAPE: return "ALT_E_SHAPE";
    case ALT_E_NONDIVISIBLE: return "ALT_E_NONDIVISIBLE";
    case ALT_E_LOSSY: return "ALT_E_LOSSY";
    case ALT_E_UNSUPPORTED: return "ALT_E_UNSUPPORTED";
    case ALT_E_CUDA: return "ALT_E_CUDA";
    case ALT_E_NOMEM: return "ALT_E_NOMEM";
  }
  return "ALT_E_?";
}

const char *alt_last_error(void) { return alt::last_error(); }

alt_status alt_layout_create(int32_t logical_rank, const int64_t *logical_shape,
                             const alt_prim *prims, int32_t nprims, alt_layout *out) {
  if (!out) { set_error("alt_layout_create: out is NULL"); return ALT_E_INVALID; }
  *out = nullptr;
  alt_layout_s *h = new (std::nothrow) alt_layout_s();
  if (!h) return ALT_E_NOMEM;
  alt_status st = compile_layout(logical_rank, logical_shape, prims, nprims, &h->impl);
  if (st != ALT_OK) { delete h; return st; }
  *out = h;
  set_error("");
  return ALT_OK;
}

alt_status alt_layout_destroy(alt_layout l) {
  delete l;
  return ALT_OK;
}

alt_status alt_layout_query(alt_layout l, int32_t *phys_rank, int64_t *phys_shape,
                            int64_t *phys_numel, uint32_t *flags) {
  if (!l) { set_error("alt_layout_query: NULL layout"); return ALT_E_INVALID; }
  const Layout &L = l->impl;
  if (phys_rank) *phys_rank = L.prank;
  if (phys_shape) for (int d = 0; d < L.prank; d++) phys_shape[d] = L.pshape[d];
  if (phys_numel) *phys_numel = L.pnumel;
  if (flags) *flags = L.flags;
  return ALT_OK;
}

alt_status alt_layout_logical(alt_layout l, int32_t *logical_rank, int64_t *logical_shape) {
  if (!l) { set_error("alt_layout_logical: NULL layout"); return ALT_E_INVALID; }
  if (logical_rank) *logical_rank = l->impl.lrank;
  if (logical_shape) for (int d = 0; d < l->impl.lrank; d++) logical_shape[d] = l->impl.lshape[d];
  return ALT_OK;
}

alt_status alt_layout_phys_to_logical(alt_layout l, int64_t j, int64_t *logical_coords, int32_t *valid) {
  if (!l || !logical_coords || !valid) { set_error("phys_to_logical: NULL argument"); return ALT_E_INVALID; }
  const Layout &L = l->impl;
  if (j < 0 || j >= L.pnumel) { set_error("phys_to_logical: index out of range"); return ALT_E_INVALID; }
  int64_t c[kMaxP];
  for (int d = L.prank - 1; d >= 0; d--) { c[d] = j % L.pshape[d]; j /= L.pshape[d]; }
  *valid = host_G(L.desc, c, logical_coords) ? 1 : 0;
  return ALT_OK;
}

alt_status alt_layout_logical_to_phys(alt_layout l, const int64_t *logical_coords, int64_t *j) {
  if (!l || !logical_coords || !j) { set_error("logical_to_phys: NULL argument"); return ALT_E_INVALID; }
  const Layout &L = l->impl;
  for (int d = 0; d < L.lrank; d++)
    if (logical_coords[d] < 0 || logical_coords[d] >= L.lshape[d]) { set_error("logical_to_phys: out of range"); return ALT_E_INVALID; }
  int64_t c[kMaxP];
  if (!host_F(L.desc, logical_coords, c)) { set_error("element has no copy"); return ALT_E_LOSSY; }
  int64_t o = 0;
  for (int d = 0; d < L.prank; d++) o += c[d] * L.pstride[d];
  *j = o;
  return ALT_OK;
}

alt_status alt_relayout(alt_layout src_l, const void *src, alt_layout dst_l, void *dst,
                        alt_dtype dtype, alt_stream_t stream) {
  if (!src_l || !dst_l) { set_error("alt_relayout: NULL layout"); return ALT_E_INVALID; }
  if (dtype != ALT_F32 && dtype != ALT_BF16) { set_error("alt_relayout: bad dtype"); return ALT_E_INVALID; }
  if (!is_device_ptr(src) || !is_device_ptr(dst)) { set_error("alt_relayout: src/dst must be device pointers"); return ALT_E_INVALID; }
  return relayout_launch(&src_l->impl, src, &dst_l->impl, dst, dtype == ALT_BF16 ? 2 : 4,
                         reinterpret_cast<cudaStream_t>(stream));
}

alt_status alt_conv2d(const alt_conv2d_params *p, alt_layout x_l, const void *x, alt_layout w_l,
                      const void *w, alt_layout y_l, void *y, alt_dtype dtype,
                      const alt_epilogue *epi, const alt_kernel_cfg *cfg, alt_stream_t stream) {
  if (!p || !x_l || !w_l || !y_l) { set_error("alt_conv2d: NULL argument"); return ALT_E_INVALID; }
  if (dtype != ALT_F32 && dtype != ALT_BF16) { set_error("alt_conv2d: bad dtype"); return ALT_E_INVALID; }
  if (p->N < 0 || p->C < 1 || p->H < 1 || p->W < 1 || p->K < 1 || p->R < 1 || p->S < 1 ||
      p->stride_h < 1 || p->stride_w < 1 || p->pad_h < 0 || p->pad_w < 0) {
    set_error("alt_conv2d: bad geometry");
    return ALT_E_INVALID;
  }
  const int32_t dh = p->dil_h < 1 ? 1 : p->dil_h, dw = p->dil_w < 1 ? 1 : p->dil_w;
  const int32_t G = p->groups < 1 ? 1 : p->groups;
  if (p->C % G || p->K % G) { set_error("alt_conv2d: groups must divide C and K"); return ALT_E_INVALID; }
  const int64_t Ho = (p->H + 2 * p->pad_h - (int64_t)dh * (p->R - 1) - 1) / p->stride_h + 1;
  const int64_t Wo = (p->W + 2 * p->pad_w - (int64_t)dw * (p->S - 1) - 1) / p->stride_w + 1;
  if (p->H + 2 * p->pad_h < (int64_t)dh * (p->R - 1) + 1 || p->W + 2 * p->pad_w < (int64_t)dw * (p->S - 1) + 1 ||
      Ho < 1 || Wo < 1) { set_error("alt_conv2d: empty output"); return ALT_E_INVALID; }
  const int64_t xs[4] = {p->N, p->C, p->H, p->W}, ws[4] = {p->K, p->C / G, p->R, p->S},
                ys[4] = {p->N, p->K, Ho, Wo};
  if (p->N > 0 && (!shape_is(&x_l->impl, 4, xs) || !shape_is(&w_l->impl, 4, ws) || !shape_is(&y_l->impl, 4, ys))) {
    set_error("alt_conv2d: layout logical shapes do not match x[N,C,H,W] / w[K,C/g,R,S] / y[N,K,Ho,Wo]");
    return ALT_E_SHAPE;
  }
  if (p->N == 0) return ALT_OK;
  if (!is_device_ptr(x) || !is_device_ptr(w) || !is_device_ptr(y)) { set_error("alt_conv2d: x/w/y must be device pointers"); return ALT_E_INVALID; }
  ConvProblem P{};
  P.N = p->N; P.C = p->C; P.H = p->H; P.W = p->W; P.K = p->K; P.R = p->R; P.S = p->S;
  P.Ho = Ho; P.Wo = Wo;
  P.Vh = p->stride_h; P.Vw = p->stride_w; P.ph = p->pad_h; P.pw = p->pad_w; P.groups = G;
  P.dh = dh; P.dw = dw;
  P.xl = &x_l->impl; P.wl = &w_l->impl; P.yl = &y_l->impl;
  P.x = x; P.w = w; P.y = y; P.dtype = dtype;
  alt_status st = fill_epi(epi, P.yl, &P.epi);
  if (st != ALT_OK) return st;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int32_t path = cfg ? cfg->path : ALT_PATH_AUTO;
  alt_kernel_cfg used{};
  // dilation: tensor-core path (tap offsets d r in the TMA box rule) or the
  // generic path; the depthwise kernel cuts undilated windows
  const bool dil = dh > 1 || dw > 1;
  if (dil && path == ALT_PATH_DW) {
    set_error("alt_conv2d: dilation > 1 has no depthwise kernel (SIMT or tensor-core path)");
    return ALT_E_UNSUPPORTED;
  }
  const bool grp_tc = G > 1 && G < p->C && (p->C / G) % 8 == 0 && (p->K / G) % 8 == 0;
  if (path == ALT_PATH_TC || (path == ALT_PATH_AUTO && (G == 1 || grp_tc))) {
    st = tc_conv(P, cfg, s, &used);
    if (st != ALT_E_UNSUPPORTED || path == ALT_PATH_TC) {
      if (st == ALT_OK) set_last_plan(used);
      return st;
    }
  }
  if (!dil && (path == ALT_PATH_DW || (path == ALT_PATH_AUTO && G == p->C && G == p->K))) {
    st = dw_conv(P, s, &used);
    if (st != ALT_E_UNSUPPORTED || path == ALT_PATH_DW) {
      if (st == ALT_OK) set_last_plan(used);
      return st;
    }
  }
  st = simt_conv(P, s);
  if (st == ALT_OK) {
    used = alt_kernel_cfg{};
    used.path = ALT_PATH_SIMT;
    set_last_plan(used);
  }
  return st;
}

alt_status alt_conv3d(const alt_conv3d_params *p, alt_layout x_l, const void *x, alt_layout w_l,
                      const void *w, alt_layout y_l, void *y, alt_dtype dtype,
                      const alt_epilogue *epi, const alt_kernel_cfg *cfg, alt_stream_t stream) {
  if (!p || !x_l || !w_l || !y_l) { set_error("alt_conv3d: NULL argument"); return ALT_E_INVALID; }
  if (dtype != ALT_F32 && dtype != ALT_BF16) { set_error("alt_conv3d: bad dtype"); return ALT_E_INVALID; }
  if (p->N < 0 || p->C < 1 || p->D < 1 || p->H < 1 || p->W < 1 || p->K < 1 || p->T < 1 || p->R < 1 || p->S < 1 ||
      p->stride_d < 1 || p->stride_h < 1 || p->stride_w < 1 || p->pad_d < 0 || p->pad_h < 0 || p->pad_w < 0) {
    set_error("alt_conv3d: bad geometry");
    return ALT_E_INVALID;
  }
  const int32_t dd = p->dil_d < 1 ? 1 : p->dil_d, dh = p->dil_h < 1 ? 1 : p->dil_h, dw = p->dil_w < 1 ? 1 : p->dil_w;
  const int32_t G = p->groups < 1 ? 1 : p->groups;
  if (p->C % G || p->K % G) { set_error("alt_conv3d: groups must divide C and K"); return ALT_E_INVALID; }
  const int64_t Do = (p->D + 2 * p->pad_d - (int64_t)dd * (p->T - 1) - 1) / p->stride_d + 1;
  const int64_t Ho = (p->H + 2 * p->pad_h - (int64_t)dh * (p->R - 1) - 1) / p->stride_h + 1;
  const int64_t Wo = (p->W + 2 * p->pad_w - (int64_t)dw * (p->S - 1) - 1) / p->stride_w + 1;
  if (p->D + 2 * p->pad_d < (int64_t)dd * (p->T - 1) + 1 || p->H + 2 * p->pad_h < (int64_t)dh * (p->R - 1) + 1 ||
      p->W + 2 * p->pad_w < (int64_t)dw * (p->S - 1) + 1 || Do < 1 || Ho < 1 || Wo < 1) {
    set_error("alt_conv3d: empty output");
    return ALT_E_INVALID;
  }
  const int64_t xs[5] = {p->N, p->C, p->D, p->H, p->W}, wsh[5] = {p->K, p->C / G, p->T, p->R, p->S},
                ys[5] = {p->N, p->K, Do, Ho, Wo};
  if (p->N > 0 && (!shape_is(&x_l->impl, 5, xs) || !shape_is(&w_l->impl, 5, wsh) || !shape_is(&y_l->impl, 5, ys))) {
    set_error("alt_conv3d: layout logical shapes do not match x[N,C,D,H,W] / w[K,C/g,T,R,S] / y[N,K,Do,Ho,Wo]");
    return ALT_E_SHAPE;
  }
  if (p->N == 0) return ALT_OK;
  if (!is_device_ptr(x) || !is_device_ptr(w) || !is_device_ptr(y)) { set_error("alt_conv3d: x/w/y must be device pointers"); return ALT_E_INVALID; }
  ConvProblem P{};
  P.N = p->N; P.C = p->C; P.H = p->H; P.W = p->W; P.K = p->K; P.R = p->R; P.S = p->S;
  P.Ho = Ho; P.Wo = Wo;
  P.Vh = p->stride_h; P.Vw = p->stride_w; P.ph = p->pad_h; P.pw = p->pad_w; P.groups = G;
  P.dh = dh; P.dw = dw;
  P.D = p->D; P.T = p->T; P.Do = Do; P.Vd = p->stride_d; P.pd = p->pad_d; P.dd = dd; P.c3d = true;
  P.xl = &x_l->impl; P.wl = &w_l->impl; P.yl = &y_l->impl;
  P.x = x; P.w = w; P.y = y; P.dtype = dtype;
  alt_status st = fill_epi(epi, P.yl, &P.epi);
  if (st != ALT_OK) return st;
  if (P.epi.bias_att) { set_error("alt_conv3d: attached bias unsupported"); return ALT_E_INVALID; }
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  const int32_t path = cfg ? cfg->path : ALT_PATH_AUTO;
  alt_kernel_cfg used{};
  if (path == ALT_PATH_TC || (path == ALT_PATH_AUTO && G == 1)) {
    st = tc_conv(P, cfg, s, &used);
    if (st != ALT_E_UNSUPPORTED || path == ALT_PATH_TC) {
      if (st == ALT_OK) set_last_plan(used);
      return st;
    }
  }
  if (path == ALT_PATH_DW) { set_error("alt_conv3d: no depthwise kernel"); return ALT_E_UNSUPPORTED; }
  st = simt_conv3d(P, s);
  if (st == ALT_OK) {
    used = alt_kernel_cfg{};
    used.path = ALT_PATH_SIMT;
    set_last_plan(used);
  }
  return st;
}

static alt_status gemm_dispatch(GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t s);

alt_status alt_matmul(int64_t M, int64_t N, int64_t K, alt_layout a_l, const void *a,
                      alt_layout b_l, const void *b, alt_layout c_l, void *c, alt_dtype dtype,
                      const alt_epilogue *epi, const alt_kernel_cfg *cfg, alt_stream_t stream) {
  if (!a_l || !b_l || !c_l) { set_error("alt_matmul: NULL layout"); return ALT_E_INVALID; }
  if (dtype != ALT_F32 && dtype != ALT_BF16) { set_error("alt_matmul: bad dtype"); return ALT_E_INVALID; }
  if (M < 0 || N < 1 || K < 1) { set_error("alt_matmul: bad sizes"); return ALT_E_INVALID; }
  const int64_t as[2] = {M, K}, bs[2] = {K, N}, cs[2] = {M, N};
  if (M > 0 && (!shape_is(&a_l->impl, 2, as) || !shape_is(&b_l->impl, 2, bs) || !shape_is(&c_l->impl, 2, cs))) {
    set_error("alt_matmul: layout logical shapes do not match A[M,K] / B[K,N] / C[M,N]");
    return ALT_E_SHAPE;
  }
  if (M == 0) return ALT_OK;
  if (!is_device_ptr(a) || !is_device_ptr(b) || !is_device_ptr(c)) { set_error("alt_matmul: A/B/C must be device pointers"); return ALT_E_INVALID; }
  GemmProblem P{};
  P.M = M; P.N = N; P.K = K;
  P.al = &a_l->impl; P.bl = &b_l->impl; P.cl = &c_l->impl;
  P.a = a; P.b = b; P.c = c; P.dtype = dtype;
  alt_status st = fill_epi(epi, P.cl, &P.epi);
  if (st != ALT_OK) return st;
  return gemm_dispatch(P, cfg, reinterpret_cast<cudaStream_t>(stream));
}

static alt_status gemm_dispatch(GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t s) {
  alt_status st = ALT_OK;
  const int32_t path = cfg ? cfg->path : ALT_PATH_AUTO;
  alt_kernel_cfg used{};
  if (path == ALT_PATH_TC || path == ALT_PATH_AUTO) {
    st = tc_gemm(P, cfg, s, &used);
    if (st != ALT_E_UNSUPPORTED || path == ALT_PATH_TC) {
      if (st == ALT_OK) set_last_plan(used);
      return st;
    }
  }
  st = simt_gemm(P, s);
  if (st == ALT_OK) {
    used = alt_kernel_cfg{};
    used.path = ALT_PATH_SIMT;
    set_last_plan(used);
  }
  return st;
}

alt_status alt_pool2d(const alt_conv2d_params *p, alt_layout x_l, const void *x, alt_layout y_l, void *y,
                      alt_dtype dtype, int32_t kind, alt_stream_t stream) {
  if (!p || !x_l || !y_l) { set_error("alt_pool2d: NULL argument"); return ALT_E_INVALID; }
  if (dtype != ALT_F32 && dtype != ALT_BF16) { set_error("alt_pool2d: bad dtype"); return ALT_E_INVALID; }
  if (kind != ALT_POOL_MAX && kind != ALT_POOL_AVG) { set_error("alt_pool2d: bad kind"); return ALT_E_INVALID; }
  if (p->N < 0 || p->C < 1 || p->H < 1 || p->W < 1 || p->R < 1 || p->S < 1 || p->stride_h < 1 ||
      p->stride_w < 1 || p->pad_h < 0 || p->pad_w < 0) {
    set_error("alt_pool2d: bad geometry");
    return ALT_E_INVALID;
  }
  const int64_t Ho = (p->H + 2 * p->pad_h - p->R) / p->stride_h + 1;
  const int64_t Wo = (p->W + 2 * p->pad_w - p->S) / p->stride_w + 1;
  const int64_t xs[4] = {p->N, p->C, p->H, p->W}, ys[4] = {p->N, p->C, Ho, Wo};
  if (p->N > 0 && (!shape_is(&x_l->impl, 4, xs) || !shape_is(&y_l->impl, 4, ys))) {
    set_error("alt_pool2d: layout logical shapes do not match x[N,C,H,W] / y[N,C,Ho,Wo]");
    return ALT_E_SHAPE;
  }
  if (p->N == 0) return ALT_OK;
  if (!is_device_ptr(x) || !is_device_ptr(y)) { set_error("alt_pool2d: x/y must be device pointers"); return ALT_E_INVALID; }
  ConvProblem P{};
  P.N = p->N; P.C = p->C; P.H = p->H; P.W = p->W; P.K = p->C; P.R = p->R; P.S = p->S;
  P.Ho = Ho; P.Wo = Wo; P.Vh = p->stride_h; P.Vw = p->stride_w; P.ph = p->pad_h; P.pw = p->pad_w;
  P.groups = 1;
  P.xl = &x_l->impl; P.yl = &y_l->impl; P.wl = nullptr;
  P.x = x; P.y = y; P.dtype = dtype;
  return pool2d(P, kind, reinterpret_cast<cudaStream_t>(stream));
}

alt_status alt_last_plan(alt_kernel_cfg *cfg) {
  if (!cfg) return ALT_E_INVALID;
  *cfg = g_last_plan;
  return ALT_OK;
}

static int dtype_wb(alt_dtype d) { return d == ALT_BF16 ? 2 : d == ALT_F32 ? 4 : 0; }

// Z's logical shape must be A's with dim extended by one
static alt_status check_attach(const char *what, const Layout *A, const Layout *Z, int32_t dim) {
  if (dim < 0 || dim >= A->lrank) { set_error("%s: dim %d out of range", what, dim); return ALT_E_INVALID; }
  if (Z->lrank != A->lrank) { set_error("%s: logical ranks differ", what); return ALT_E_SHAPE; }
  for (int d = 0; d < A->lrank; d++)
    if (Z->lshape[d] != A->lshape[d] + (d == dim ? 1 : 0)) {
      set_error("%s: z logical shape must be a's with dim %d extended by one (dim %d)", what, dim, d);
      return ALT_E_SHAPE;
    }
  return ALT_OK;
}

alt_status alt_store_at(alt_layout a_l, const void *a, const void *b, int32_t dim, alt_layout z_l, void *z,
                        alt_dtype dtype, alt_stream_t stream) {
  if (!a_l || !z_l) { set_error("alt_store_at: NULL layout"); return ALT_E_INVALID; }
  const int wb = dtype_wb(dtype);
  if (!wb) { set_error("alt_store_at: bad dtype"); return ALT_E_INVALID; }
  alt_status st = check_attach("alt_store_at", &a_l->impl, &z_l->impl, dim);
  if (st != ALT_OK) return st;
  if (!(a_l->impl.flags & ALT_LOSSLESS)) { set_error("alt_store_at: a's layout is lossy"); return ALT_E_LOSSY; }
  if (z_l->impl.pnumel == 0) return ALT_OK;
  if (!is_device_ptr(z) || (a_l->impl.lnumel && !is_device_ptr(a)) ||
      (z_l->impl.lnumel / z_l->impl.lshape[dim] && !is_device_ptr(b))) {
    set_error("alt_store_at: a / b / z must be device pointers");
    return ALT_E_INVALID;
  }
  return store_at_launch(&a_l->impl, a, b, dim, &z_l->impl, z, wb, reinterpret_cast<cudaStream_t>(stream));
}

alt_status alt_decouple_at(alt_layout z_l, const void *z, int32_t dim, alt_layout a_l, void *a, void *b,
                           alt_dtype dtype, alt_stream_t stream) {
  if (!a_l || !z_l) { set_error("alt_decouple_at: NULL layout"); return ALT_E_INVALID; }
  const int wb = dtype_wb(dtype);
  if (!wb) { set_error("alt_decouple_at: bad dtype"); return ALT_E_INVALID; }
  alt_status st = check_attach("alt_decouple_at", &a_l->impl, &z_l->impl, dim);
  if (st != ALT_OK) return st;
  if (!(z_l->impl.flags & ALT_LOSSLESS)) { set_error("alt_decouple_at: z's layout is lossy"); return ALT_E_LOSSY; }
  if (z_l->impl.lnumel == 0) return ALT_OK;
  if (!is_device_ptr(z) || !is_device_ptr(a) || !is_device_ptr(b)) {
    set_error("alt_decouple_at: z / a / b must be device pointers");
    return ALT_E_INVALID;
  }
  return decouple_at_launch(&z_l->impl, z, dim, &a_l->impl, a, b, wb, reinterpret_cast<cudaStream_t>(stream));
}

alt_status alt_matmul_store_at(int64_t M, int64_t N, int64_t K, alt_layout a_l, const void *a, alt_layout z_l,
                               const void *z, alt_layout c_l, void *c, alt_dtype dtype, const alt_epilogue *epi,
                               const alt_kernel_cfg *cfg, alt_stream_t stream) {
  if (!a_l || !z_l || !c_l) { set_error("alt_matmul_store_at: NULL layout"); return ALT_E_INVALID; }
  const int wb = dtype_wb(dtype);
  if (!wb) { set_error("alt_matmul_store_at: bad dtype"); return ALT_E_INVALID; }
  if (M < 0 || N < 1 || K < 1) { set_error("alt_matmul_store_at: bad sizes"); return ALT_E_INVALID; }
  if (epi && epi->bias) { set_error("alt_matmul_store_at: the bias is the attached row of z; epi->bias must be NULL"); return ALT_E_INVALID; }
  const int64_t as[2] = {M, K}, zs[2] = {K + 1, N}, cs[2] = {M, N};
  if (M > 0 && (!shape_is(&a_l->impl, 2, as) || !shape_is(&z_l->impl, 2, zs) || !shape_is(&c_l->impl, 2, cs))) {
    set_error("alt_matmul_store_at: layout logical shapes do not match A[M,K] / Z[K+1,N] / C[M,N]");
    return ALT_E_SHAPE;
  }
  // every element of Z (B and the attached bias row) must have a stored copy:
  // a lossy Z (e.g. unfold with B < S) has owner offsets of -1 (reading A4)
  if (!(z_l->impl.flags & ALT_LOSSLESS)) { set_error("alt_matmul_store_at: z's layout is lossy"); return ALT_E_LOSSY; }
  if (M == 0) return ALT_OK;
  if (!is_device_ptr(a) || !is_device_ptr(z) || !is_device_ptr(c)) { set_error("alt_matmul_store_at: A/Z/C must be device pointers"); return ALT_E_INVALID; }
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  GemmProblem P{};
  P.M = M; P.N = N; P.K = K;
  P.al = &a_l->impl; P.bl = &z_l->impl; P.cl = &c_l->impl;  // rows k < K of Z are B
  P.a = a; P.b = z; P.c = c; P.dtype = dtype;
  alt_status st = fill_epi(epi, P.cl, &P.epi);
  if (st != ALT_OK) return st;
  Layout *Z = &z_l->impl;
  if (Z->separable) {
    // the epilogue reads bias[n] = Z[K, n] in place: offset rd0[K] + rd1[n]
    SepDev sz{};
    const LayoutDesc *dz = nullptr;
    if ((st = device_tables(Z, &sz, &dz)) != ALT_OK) return st;
    P.epi.bias_att = z;
    P.epi.bias_att_rd = sz.rd[1];
    P.epi.bias_att_base = Z->rd[0][K];
    P.epi.bias_att_bf16 = dtype == ALT_BF16;
    return gemm_dispatch(P, cfg, s);
  }
  // non-separable Z: gather the attached row into fp32 scratch first
  float *bias = nullptr;
  if (cudaMallocAsync(reinterpret_cast<void **>(&bias), (size_t)N * sizeof(float), s) != cudaSuccess) {
    cudaGetLastError();
    set_error("alt_matmul_store_at: scratch allocation failed");
    return ALT_E_NOMEM;
  }
  st = attached_row_f32(&z_l->impl, z, 0, wb, bias, s);
  if (st == ALT_OK) {
    P.epi.bias = bias;
    st = gemm_dispatch(P, cfg, s);
  }
  cudaFreeAsync(bias, s);
  return st;
}

uint64_t alt_launch_count(void) { return g_launches.load(); }

}  // extern "C"
