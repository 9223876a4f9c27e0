// tune.cpp — alt_tune: ALT's joint layout + loop tuning (§5)
// replaced by a bounded grid measured on the device.
//
// Conv template (GPU form): x = N C/it H W it (optionally with
// the conv zero padding materialised: pad(H), pad(W), reading A7),
// w = K/ot' C/it R S ot' it (c innermost: K-major B operand, reading A11),
// y = N K/ot Ho Wo ot; kernel ("loop") parameters: BLOCK_N and the
// (tile_n x tile_h x tile_w) output-pixel tile.  C is padded to a multiple of
// 8 first when needed (reading A2: non-divisible tiling = pad then split).
// GEMM template: A = M/mt K/kt mt kt, B = N/nt K/kt nt kt
// (K innermost), C = M/mt N/nt mt nt.
//
// Each point: compile the layouts, allocate operands in them (values do not
// affect timing), run `warmup` launches, then `reps` launches each preceded
// by an L2 flush (a 2x-L2 memset, not timed), timed with CUDA events on the
// caller's stream.  The fastest point is returned.  Parity of the tuner is
// unpinned by the paper (reading A19): the result is only required to be a
// valid layout pair whose kernels are oracle-exact.
#include <cuda_runtime.h>

#include <algorithm>
#include <cfloat>
#include <cstring>
#include <functional>
#include <vector>

#include "alt.h"
#include "layout.h"
#include "ops.h"

namespace alt {

namespace {

alt_prim P_split(int dim, std::initializer_list<int64_t> f) {
  alt_prim p{};
  p.kind = ALT_SPLIT;
  p.dim = dim;
  p.n = (int32_t)f.size();
  int i = 0;
  for (int64_t x : f) p.v[i++] = x;
  return p;
}
alt_prim P_reorder(std::initializer_list<int64_t> perm) {
  alt_prim p{};
  p.kind = ALT_REORDER;
  p.n = (int32_t)perm.size();
  int i = 0;
  for (int64_t x : perm) p.v[i++] = x;
  return p;
}
alt_prim P_pad(int dim, int64_t lo, int64_t hi) {
  alt_prim p{};
  p.kind = ALT_PAD;
  p.dim = dim;
  p.v[0] = lo;
  p.v[1] = hi;
  return p;
}

struct Seq {
  std::vector<alt_prim> p;
};

// N C/x H W x, with C padded to Cp and optional materialised conv padding
Seq act_layout(int64_t C, int64_t Cp, int64_t x, int64_t pad_hw) {
  Seq s;
  if (Cp != C) s.p.push_back(P_pad(1, 0, Cp - C));
  if (pad_hw) {
    s.p.push_back(P_pad(2, pad_hw, pad_hw));
    s.p.push_back(P_pad(3, pad_hw, pad_hw));
  }
  s.p.push_back(P_split(1, {Cp / x, x}));
  s.p.push_back(P_reorder({0, 1, 3, 4, 2}));
  return s;
}
// K/y C/x R S y x (c innermost), C padded to Cp
Seq wgt_layout(int64_t K, int64_t C, int64_t Cp, int64_t y, int64_t x) {
  Seq s;
  if (Cp != C) s.p.push_back(P_pad(1, 0, Cp - C));
  s.p.push_back(P_split(0, {K / y, y}));
  s.p.push_back(P_split(2, {Cp / x, x}));
  s.p.push_back(P_reorder({0, 2, 4, 5, 1, 3}));
  return s;
}
// The paper's C2D input template: N H/ht W/wt C/it
// (ht+KH-1)(wt+KW-1) it with the conv padding before the unfold; stride V
// uses B = V(ht-1)+R, S = V ht (reading A6).  ht or wt = 0 keeps that dim
// whole (no unfold).
Seq act_layout_tiled(int64_t C, int64_t Cp, int64_t x, int64_t pad, int64_t V, int64_t R, int64_t S, int64_t ht,
                     int64_t wt) {
  Seq s;
  if (Cp != C) s.p.push_back(P_pad(1, 0, Cp - C));
  s.p.push_back(P_pad(2, pad, pad));
  s.p.push_back(P_pad(3, pad, pad));
  // dim names after each step: N C H W -> N C [Ht Bh | H] [Wt Bw | W]
  int wdim = 3;
  if (ht) {
    alt_prim u{};
    u.kind = ALT_UNFOLD; u.dim = 2; u.v[0] = V * (ht - 1) + R; u.v[1] = V * ht;
    s.p.push_back(u);
    wdim = 4;
  }
  if (wt) {
    alt_prim u{};
    u.kind = ALT_UNFOLD; u.dim = wdim; u.v[0] = V * (wt - 1) + S; u.v[1] = V * wt;
    s.p.push_back(u);
  }
  s.p.push_back(P_split(1, {Cp / x, x}));
  // now N Cc it [Ht Bh | H] [Wt Bw | W]
  std::vector<int64_t> perm;
  const int hbase = 3, wbase = ht ? 5 : 4;
  perm.push_back(0);
  if (ht) perm.push_back(hbase);
  if (wt) perm.push_back(wbase);
  perm.push_back(1);
  perm.push_back(ht ? hbase + 1 : hbase);
  perm.push_back(wt ? wbase + 1 : wbase);
  perm.push_back(2);
  alt_prim r{};
  r.kind = ALT_REORDER;
  r.n = (int32_t)perm.size();
  for (size_t i = 0; i < perm.size(); i++) r.v[i] = perm[i];
  s.p.push_back(r);
  return s;
}
// Output template N Ho/ht Wo/wt K/ot ht wt ot; ht | Ho, wt | Wo
Seq out_layout_tiled(int64_t K, int64_t ot, int64_t Ho, int64_t Wo, int64_t ht, int64_t wt) {
  Seq s;
  int wdim = 3;
  if (ht) { s.p.push_back(P_split(2, {Ho / ht, ht})); wdim = 4; }
  if (wt) s.p.push_back(P_split(wdim, {Wo / wt, wt}));
  s.p.push_back(P_split(1, {K / ot, ot}));
  // N Kc ot [Ht ht | H] [Wt wt | W]
  std::vector<int64_t> perm;
  const int hbase = 3, wbase = ht ? 5 : 4;
  perm.push_back(0);
  if (ht) perm.push_back(hbase);
  if (wt) perm.push_back(wbase);
  perm.push_back(1);
  perm.push_back(ht ? hbase + 1 : hbase);
  perm.push_back(wt ? wbase + 1 : wbase);
  perm.push_back(2);
  alt_prim r{};
  r.kind = ALT_REORDER;
  r.n = (int32_t)perm.size();
  for (size_t i = 0; i < perm.size(); i++) r.v[i] = perm[i];
  s.p.push_back(r);
  return s;
}
// Two-level output template: N H/(h2 ht) W/(w2 wt) K/(o2 ot)
// h2 w2 o2 ht wt ot; h2 (w2) | Ho / ht (Wo / wt), o2 | K / ot
Seq out_layout_two_level(int64_t K, int64_t ot, int64_t o2, int64_t Ho, int64_t Wo, int64_t ht, int64_t wt,
                         int64_t h2, int64_t w2) {
  Seq s;
  s.p.push_back(P_split(2, {Ho / (h2 * ht), h2, ht}));                // N K Hoo h2 ht W
  s.p.push_back(P_split(5, {Wo / (w2 * wt), w2, wt}));                // N K Hoo h2 ht Woo w2 wt
  s.p.push_back(P_split(1, {K / (o2 * ot), o2, ot}));                 // N Koo o2 ot Hoo h2 ht Woo w2 wt
  // -> N Hoo Woo Koo h2 w2 o2 ht wt ot
  s.p.push_back(P_reorder({0, 4, 7, 1, 5, 8, 2, 6, 9, 3}));
  return s;
}
// the paper's weight order O/ot I/it KH KW it ot (o innermost)
Seq wgt_layout_paper(int64_t K, int64_t C, int64_t Cp, int64_t y, int64_t x) {
  Seq s;
  if (Cp != C) s.p.push_back(P_pad(1, 0, Cp - C));
  s.p.push_back(P_split(0, {K / y, y}));
  s.p.push_back(P_split(2, {Cp / x, x}));
  s.p.push_back(P_reorder({0, 2, 4, 5, 3, 1}));
  return s;
}
Seq tiled2(int64_t R0, int64_t R1, int64_t t0, int64_t t1, bool swap_inner) {
  // [R0/t0][R1/t1][t0][t1]  (swap_inner: [R1/t1][R0/t0][t1][t0])
  Seq s;
  s.p.push_back(P_split(0, {R0 / t0, t0}));
  s.p.push_back(P_split(2, {R1 / t1, t1}));
  if (swap_inner) s.p.push_back(P_reorder({2, 0, 3, 1}));
  else s.p.push_back(P_reorder({0, 2, 1, 3}));
  return s;
}

struct Scratch {
  std::vector<void *> bufs;
  void *get(size_t bytes, cudaStream_t s) {
    void *p = nullptr;
    if (cudaMallocAsync(&p, bytes, s) != cudaSuccess) return nullptr;
    cudaMemsetAsync(p, 0, bytes, s);
    bufs.push_back(p);
    return p;
  }
  void release(cudaStream_t s) {
    for (void *p : bufs) cudaFreeAsync(p, s);
    bufs.clear();
  }
};

struct LayoutHolder {
  alt_layout h = nullptr;
  ~LayoutHolder() { if (h) alt_layout_destroy(h); }
};

std::vector<int64_t> vals_or(const alt_tune_space *sp, int i, std::initializer_list<int64_t> def) {
  std::vector<int64_t> v;
  if (sp && sp->nvals[i] > 0) {
    for (int k = 0; k < sp->nvals[i] && k < ALT_TUNE_MAX_VALS; k++) v.push_back(sp->vals[i][k]);
  } else {
    v.assign(def.begin(), def.end());
  }
  return v;
}

// time one callable (launches on `s`) with an L2 flush before every rep
template <typename F>
float time_point(F &&launch, cudaStream_t s, void *flush, size_t flush_bytes, int warmup, int reps,
                 alt_status *st) {
  for (int i = 0; i < warmup; i++) {
    *st = launch();
    if (*st != ALT_OK) return FLT_MAX;
  }
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  std::vector<float> t;
  for (int i = 0; i < reps; i++) {
    if (flush) cudaMemsetAsync(flush, i & 0xff, flush_bytes, s);
    cudaEventRecord(e0, s);
    *st = launch();
    cudaEventRecord(e1, s);
    if (*st != ALT_OK) break;
    cudaEventSynchronize(e1);
    float ms = 0.f;
    cudaEventElapsedTime(&ms, e0, e1);
    t.push_back(ms);
  }
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  if (*st != ALT_OK || t.empty()) return FLT_MAX;
  std::sort(t.begin(), t.end());
  return t[t.size() / 2] * 1000.f;  // median, us
}

// one grid point: layouts (x / w / y or A / B / C) and the kernel config
struct Point {
  Seq seq[3];
  bool fixed_x = false;
  alt_kernel_cfg cfg{};
  float us = FLT_MAX;
  alt_kernel_cfg used{};
};

}  // namespace
}  // namespace alt

using namespace alt;

extern "C" alt_status alt_tune(alt_op_kind op, const void *op_params, alt_dtype dtype, const alt_tune_space *space,
                               alt_stream_t stream_, alt_tune_result *out, float *all_us) {
  if (!op_params || !out) { set_error("alt_tune: NULL argument"); return ALT_E_INVALID; }
  if (dtype != ALT_BF16 && dtype != ALT_F32) { set_error("alt_tune: bad dtype"); return ALT_E_INVALID; }
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream_);
  const int esize = dtype == ALT_BF16 ? 2 : 4;
  const int max_points = space && space->max_points > 0 ? std::min(space->max_points, 4096) : 64;
  const int warmup = space && space->warmup > 0 ? space->warmup : 2;
  const int reps = space && space->reps > 0 ? space->reps : 5;
  memset(out, 0, sizeof(*out));
  out->best_us = FLT_MAX;
  int dev = 0;
  cudaGetDevice(&dev);
  int l2 = 0;
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
  const size_t flush_bytes = (size_t)std::max(l2, 1 << 20) * 2;
  Scratch scratch;
  void *flush = scratch.get(flush_bytes, s);

  std::vector<Point> pts;
  // measure one point on the device (its layouts compiled for the call)
  std::function<float(Point &, int)> measure;

  if (op == ALT_OP_CONV2D) {
    const alt_conv2d_params &p = *static_cast<const alt_conv2d_params *>(op_params);
    if (p.groups > 1) { set_error("alt_tune: grouped conv has no template (NEXT)"); scratch.release(s); return ALT_E_UNSUPPORTED; }
    if (p.dil_h > 1 || p.dil_w > 1) { set_error("alt_tune: dilated conv has no template (NEXT)"); scratch.release(s); return ALT_E_UNSUPPORTED; }
    const int64_t Ho = (p.H + 2 * p.pad_h - p.R) / p.stride_h + 1, Wo = (p.W + 2 * p.pad_w - p.S) / p.stride_w + 1;
    const int64_t Cp = p.C % 8 ? (p.C + 7) / 8 * 8 : p.C;
    const int64_t xl[4] = {p.N, p.C, p.H, p.W}, wl[4] = {p.K, p.C, p.R, p.S}, yl[4] = {p.N, p.K, Ho, Wo};
    // x sized for the largest template (overlapped tiles duplicate rows)
    const size_t xbytes = (size_t)p.N * Cp * (2 * p.H + 2 * p.pad_h + p.R) * (2 * p.W + 2 * p.pad_w + p.S) * esize;
    void *x = scratch.get(xbytes, s);
    void *w = scratch.get((size_t)p.K * Cp * p.R * p.S * esize, s);
    void *y = scratch.get((size_t)p.N * p.K * Ho * Wo * esize, s);
    if (!x || !w || !y || !flush) { scratch.release(s); set_error("alt_tune: scratch allocation failed"); return ALT_E_NOMEM; }
    std::vector<int64_t> its = vals_or(space, 0, {64, 32, 16, 8, 128, 256});
    std::vector<int64_t> ots = vals_or(space, 1, {64, 32});
    std::vector<int64_t> bns = vals_or(space, 6, {256, 128, 64});
    std::vector<int64_t> pads = vals_or(space, 7, {0});
    std::vector<int64_t> ths = vals_or(space, 4, {0});  // 0 = kernel heuristic
    std::vector<int64_t> tws = vals_or(space, 5, {0});
    std::vector<int64_t> pairs = vals_or(space, 3, {0});  // cta_pair: 0 auto (pair when BN >= 128), 1 pair, 2 single
    std::vector<int64_t> sks = vals_or(space, 2, {1});    // split-K factor
    std::vector<int64_t> lhts = vals_or(space, 8, {0});   // layout spatial tiles (0 = none)
    std::vector<int64_t> lwts = vals_or(space, 9, {0});
    std::vector<int64_t> stgs = vals_or(space, 10, {0});
    std::vector<int64_t> words = vals_or(space, 11, {0});
    std::vector<int64_t> h2s = vals_or(space, 12, {0});   // two-level output factors (0 / 1 = one level)
    std::vector<int64_t> w2s = vals_or(space, 13, {0});
    std::vector<int64_t> o2s = vals_or(space, 14, {0});
    std::vector<int64_t> halos = vals_or(space, 15, {0});  // 1: halo mode (stride-1 3x3)
    for (int64_t it : its) {
      if (it > Cp || Cp % it || it % 8) continue;
      if (space && space->fix_x) { if (it != its[0]) continue; }
      for (int64_t ot : ots) {
        if (ot > p.K || p.K % ot) continue;
        for (int64_t bn : bns) {
          if (bn > 64 && bn > p.K) continue;
          const int64_t y_w = std::min<int64_t>(bn, p.K);
          if (p.K % y_w) continue;
          for (int64_t pad : pads)
          for (int64_t lht : lhts)
          for (int64_t lwt : lwts)
          for (int64_t wo : words)
          for (int64_t h2 : h2s)
          for (int64_t w2 : w2s)
          for (int64_t o2 : o2s)
          for (int64_t hl : halos)
          for (int64_t th : ths)
          for (int64_t tw : tws)
          for (int64_t pr : pairs)
          for (int64_t sk : sks)
          for (int64_t sg : stgs) {
            if ((int)pts.size() >= max_points) break;
            if (pr == 1 && bn < 128) continue;
            if ((lht || lwt) && pad) continue;  // the tiled template materialises its padding itself
            if (lht > Ho || lwt > Wo) continue;
            Point pt;
            pt.seq[0] = (lht || lwt) ? act_layout_tiled(p.C, Cp, it, p.pad_h, p.stride_h, p.R, p.S, lht, lwt)
                                     : act_layout(p.C, Cp, it, pad ? p.pad_h : 0);
            pt.seq[1] = wo ? wgt_layout_paper(p.K, p.C, Cp, y_w, it) : wgt_layout(p.K, p.C, Cp, y_w, it);
            const bool ytiled = (lht || lwt) && (!lht || Ho % lht == 0) && (!lwt || Wo % lwt == 0);
            const int64_t H2 = h2 > 1 ? h2 : 1, W2 = w2 > 1 ? w2 : 1, O2 = o2 > 1 ? o2 : 1;
            const bool two = (H2 > 1 || W2 > 1 || O2 > 1);
            if (two && !(lht && lwt && Ho % (H2 * lht) == 0 && Wo % (W2 * lwt) == 0 && p.K % (O2 * ot) == 0)) continue;
            pt.seq[2] = two ? out_layout_two_level(p.K, ot, O2, Ho, Wo, lht, lwt, H2, W2)
                            : ytiled ? out_layout_tiled(p.K, ot, Ho, Wo, lht, lwt) : act_layout(p.K, p.K, ot, 0);
            pt.fixed_x = space && space->fix_x && space->fixed_x;
            alt_kernel_cfg &cfg = pt.cfg;
            cfg.path = ALT_PATH_AUTO;
            cfg.block_n = (int32_t)bn;
            cfg.cta_pair = (int32_t)pr;
            cfg.split_k = (int32_t)(sk < 0 ? -sk : sk);  // negative: the cluster (DSMEM) form
            cfg.split_cluster = sk < 0 ? 1 : 0;
            cfg.stages = (int32_t)sg;
            cfg.block_k = hl ? 1 : 0;
            if (th && tw) {
              cfg.tile_h = (int32_t)th;
              cfg.tile_w = (int32_t)tw;
              cfg.tile_n = (int32_t)(128 / (th * tw));
              if (cfg.tile_n < 1) continue;
            }
            pts.push_back(pt);
          }
        }
      }
    }
    measure = [=](Point &pt, int r) -> float {  // by value: the branch locals end before the calls
      LayoutHolder Lx, Lw, Ly;
      if (!pt.fixed_x && alt_layout_create(4, xl, pt.seq[0].p.data(), (int32_t)pt.seq[0].p.size(), &Lx.h) != ALT_OK)
        return FLT_MAX;
      if (alt_layout_create(4, wl, pt.seq[1].p.data(), (int32_t)pt.seq[1].p.size(), &Lw.h) != ALT_OK) return FLT_MAX;
      if (alt_layout_create(4, yl, pt.seq[2].p.data(), (int32_t)pt.seq[2].p.size(), &Ly.h) != ALT_OK) return FLT_MAX;
      alt_layout xh = Lx.h ? Lx.h : space->fixed_x;
      int64_t xn = 0;
      alt_layout_query(xh, nullptr, nullptr, &xn, nullptr);
      if ((size_t)xn * esize > xbytes) return FLT_MAX;
      alt_status st = ALT_OK;
      const float us = time_point(
          [&]() { return alt_conv2d(&p, xh, x, Lw.h, w, Ly.h, y, dtype, nullptr, &pt.cfg, stream_); }, s, flush,
          flush_bytes, warmup, r, &st);
      if (st != ALT_OK) return FLT_MAX;
      alt_last_plan(&pt.used);
      return us;
    };
  } else if (op == ALT_OP_MATMUL) {
    const alt_matmul_params &g = *static_cast<const alt_matmul_params *>(op_params);
    void *a = scratch.get((size_t)g.M * g.K * esize, s);
    void *b = scratch.get((size_t)g.K * g.N * esize, s);
    void *c = scratch.get((size_t)g.M * g.N * esize, s);
    if (!a || !b || !c || !flush) { scratch.release(s); set_error("alt_tune: scratch allocation failed"); return ALT_E_NOMEM; }
    const int64_t al[2] = {g.M, g.K}, bl[2] = {g.K, g.N}, cl[2] = {g.M, g.N};
    std::vector<int64_t> mts = vals_or(space, 0, {128, 256, 64});
    std::vector<int64_t> kts = vals_or(space, 1, {64, 32});
    std::vector<int64_t> nts = vals_or(space, 2, {128, 256, 64});
    std::vector<int64_t> bns = vals_or(space, 6, {256, 128});
    std::vector<int64_t> stgs = vals_or(space, 10, {0});
    std::vector<int64_t> bords = vals_or(space, 11, {0});
    for (int64_t mt : mts) {
      if (g.M % mt) continue;
      for (int64_t kt : kts) {
        if (g.K % kt) continue;
        for (int64_t nt : nts) {
          if (g.N % nt) continue;
          for (int64_t bn : bns)
          for (int64_t bo : bords)
          for (int64_t sg : stgs) {
            if ((int)pts.size() >= max_points) break;
            if (bn > g.N) continue;
            Point pt;
            pt.seq[0] = tiled2(g.M, g.K, mt, kt, false);
            pt.seq[1] = tiled2(g.K, g.N, kt, nt, bo == 0);   // 0: N/nt K/kt nt kt; 1: K/kt N/nt kt nt
            pt.seq[2] = tiled2(g.M, g.N, mt, nt, false);
            pt.cfg.block_n = (int32_t)bn;
            pt.cfg.stages = (int32_t)sg;
            pts.push_back(pt);
          }
        }
      }
    }
    measure = [=](Point &pt, int r) -> float {
      LayoutHolder La, Lb, Lc;
      if (alt_layout_create(2, al, pt.seq[0].p.data(), (int32_t)pt.seq[0].p.size(), &La.h) != ALT_OK) return FLT_MAX;
      if (alt_layout_create(2, bl, pt.seq[1].p.data(), (int32_t)pt.seq[1].p.size(), &Lb.h) != ALT_OK) return FLT_MAX;
      if (alt_layout_create(2, cl, pt.seq[2].p.data(), (int32_t)pt.seq[2].p.size(), &Lc.h) != ALT_OK) return FLT_MAX;
      alt_status st = ALT_OK;
      const float us = time_point(
          [&]() { return alt_matmul(g.M, g.N, g.K, La.h, a, Lb.h, b, Lc.h, c, dtype, nullptr, &pt.cfg, stream_); },
          s, flush, flush_bytes, warmup, r, &st);
      if (st != ALT_OK) return FLT_MAX;
      alt_last_plan(&pt.used);
      return us;
    };
  } else {
    scratch.release(s);
    set_error("alt_tune: unknown op");
    return ALT_E_INVALID;
  }
  // every grid point once (median of reps), then the top-k finalists again
  // (median of 3 x reps); the best re-measured finalist wins
  int measured = 0;
  for (Point &pt : pts) {
    pt.us = measure(pt, reps);
    if (all_us && measured < max_points) all_us[measured] = pt.us;
    measured++;
  }
  std::vector<int> order;
  for (int i = 0; i < (int)pts.size(); i++)
    if (pts[i].us < FLT_MAX) order.push_back(i);
  std::sort(order.begin(), order.end(), [&](int i, int j) { return pts[i].us < pts[j].us; });
  const int topk = std::min<int>((int)order.size(), space && space->topk > 0 ? space->topk : 3);
  int best = -1;
  float best_us = FLT_MAX;
  for (int k = 0; k < topk; k++) {
    Point &pt = pts[order[k]];
    const float us = measure(pt, 3 * reps);
    if (us < best_us) { best_us = us; best = order[k]; }
  }
  if (best >= 0) {
    const Point &pt = pts[best];
    out->best_us = best_us;
    out->cfg = pt.used;
    for (int i = 0; i < 3; i++) {
      const bool skip = i == 0 && pt.fixed_x;
      out->nprims[i] = skip ? 0 : (int32_t)pt.seq[i].p.size();
      for (int k = 0; k < out->nprims[i]; k++) out->prims[i][k] = pt.seq[i].p[k];
    }
  }
  scratch.release(s);
  cudaStreamSynchronize(s);
  out->measured = measured;
  if (best < 0) { set_error("alt_tune: no valid grid point"); return ALT_E_UNSUPPORTED; }
  return ALT_OK;
}
