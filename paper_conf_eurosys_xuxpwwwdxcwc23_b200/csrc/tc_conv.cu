// tc_conv.cu — conv2d and GEMM on ALT layouts with tcgen05 tensor cores.
//
// Implicit GEMM (paper Fig. 3, computes the same sum):
//   rows  = output pixels (n, p, q)   — a (tile_n x tile_h x tile_w) = 128 block
//   cols  = output channels k         — BLOCK_N
//   red.  = (tap r,s) x (channel slab of `sw` channels)
// GEMM is the special case n = h = 1, rows = m, taps = 1.
//
// The B200-native idea: the layout chosen by ALT's template (NCHW[x]c,
// KCRS[y]k[x]c, overlapped (unfolded) tiles, tiled GEMM operands, padded
// copies) decides how a TMA box is cut out of memory.  The host builds, from
// the compiled layout's affine index map, a <=5-D tensor map over the
// PHYSICAL dims and an affine rule for box coordinates; the innermost
// physical dim (a channel tile of x elements) becomes the 16/32/64/128-byte
// K-major row of a UMMA canonical smem layout (swizzle = row bytes).  No data
// is converted to run on the tensor cores.
//
// Kernel: one CTA per 128 x BLOCK_N output tile, 6 warps:
//   warp 0     TMA producer (one elected thread), STAGES-deep smem ring
//   warp 1     TMEM allocator + single-thread tcgen05.mma issuer (M=128)
//   warps 2-5  epilogue: tcgen05.ld -> act(scale*acc + bias + residual) ->
//              stored through the output layout (propagation, Fig. 5b)
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstring>
#include <vector>

#include "epilogue.cuh"
#include "ops.h"
#include "sm100.cuh"

namespace alt {

void set_last_plan(const alt_kernel_cfg &c);

enum Var { V_N0 = 0, V_PT, V_PR, V_QT, V_QR, V_GT, V_GR, V_R, V_S, V_ONE, NVAR };

struct OperandMap {
  int32_t coef[5][NVAR];
  int32_t divp, divq, divg;
  int32_t slab_bytes;
  int32_t oob0;  // dim-0 coordinate that makes a box all zeros
  int32_t _pad;
};

struct TcArgs {
  OperandMap A, B;
  int32_t is_conv;
  int32_t N, K, Ho, Wo;  // output: conv y[N,K,Ho,Wo]; GEMM: N=1, Ho=1, Wo=M, K=cols
  int32_t tile_n, tile_h, tile_w;
  int32_t mt_h, mt_w;    // # tiles along h, w (n is the slowest)
  int32_t S, Gc;
  int32_t total_slabs, spi, num_iters;
  int32_t sw;
  int32_t vec_out;       // output fast path (single copy, contiguous channel runs)
  const int64_t *yrd[4];
  Writer yw;
  EpiParams epi;
};

constexpr int kThreads = 192;

template <int BN, int STAGES>
struct TcSmem {
  static constexpr int kA = 128 * 64 * 2;  // bytes per stage, A
  static constexpr int kB = BN * 64 * 2;   // bytes per stage, B
  static constexpr int kBytes = STAGES * (kA + kB) + 1024 /*barriers*/ + 1024 /*align slack*/;
};

__device__ __forceinline__ void coords(const OperandMap &m, const int32_t (&v)[NVAR], int32_t (&c)[5]) {
#pragma unroll
  for (int d = 0; d < 5; d++) {
    int32_t s = 0;
#pragma unroll
    for (int k = 0; k < NVAR; k++) s += m.coef[d][k] * v[k];
    c[d] = s;
  }
}

template <typename OutT>
__device__ __forceinline__ void store_vec(OutT *y, int64_t off, const float *v);
template <>
__device__ __forceinline__ void store_vec<uint16_t>(uint16_t *y, int64_t off, const float *v) {
  uint4 u;
  u.x = (uint32_t)f32_to_bf16_rne(v[0]) | ((uint32_t)f32_to_bf16_rne(v[1]) << 16);
  u.y = (uint32_t)f32_to_bf16_rne(v[2]) | ((uint32_t)f32_to_bf16_rne(v[3]) << 16);
  u.z = (uint32_t)f32_to_bf16_rne(v[4]) | ((uint32_t)f32_to_bf16_rne(v[5]) << 16);
  u.w = (uint32_t)f32_to_bf16_rne(v[6]) | ((uint32_t)f32_to_bf16_rne(v[7]) << 16);
  *reinterpret_cast<uint4 *>(y + off) = u;
}
template <>
__device__ __forceinline__ void store_vec<float>(float *y, int64_t off, const float *v) {
  *reinterpret_cast<float4 *>(y + off) = make_float4(v[0], v[1], v[2], v[3]);
  *reinterpret_cast<float4 *>(y + off + 4) = make_float4(v[4], v[5], v[6], v[7]);
}

template <int BN, int STAGES, typename OutT>
__global__ void __launch_bounds__(kThreads, 1)
    k_tc_igemm(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
               const __grid_constant__ TcArgs a, OutT *__restrict__ y) {
  using namespace sm100;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  // 1024-align the ring (swizzle atoms)
  unsigned char *smem = reinterpret_cast<unsigned char *>(
      (reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  constexpr int kA = TcSmem<BN, STAGES>::kA, kB = TcSmem<BN, STAGES>::kB;
  unsigned char *sA = smem;
  unsigned char *sB = smem + STAGES * kA;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + STAGES * (kA + kB));
  uint64_t *empty = full + STAGES;
  uint64_t *tmem_full = empty + STAGES;
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tmem_full + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  // M tile -> (n0, p0, q0); N tile -> k0
  const int mt = blockIdx.x;
  const int tw_i = mt % a.mt_w;
  const int th_i = (mt / a.mt_w) % a.mt_h;
  const int tn_i = mt / (a.mt_w * a.mt_h);
  const int n0 = tn_i * a.tile_n, p0 = th_i * a.tile_h, q0 = tw_i * a.tile_w;
  const int k0 = blockIdx.y * BN;

  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
    for (int s = 0; s < STAGES; s++) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    mbar_init(tmem_full, 1);
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<(BN < 32 ? 32 : BN)>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    if (lane == 0) {
      // ------------------------------------------------ TMA producer
      int32_t va[NVAR], vb[NVAR];
      va[V_N0] = n0;
      va[V_PT] = p0 / a.A.divp; va[V_PR] = p0 % a.A.divp;
      va[V_QT] = q0 / a.A.divq; va[V_QR] = q0 % a.A.divq;
      va[V_ONE] = 1;
      vb[V_N0] = 0; vb[V_PT] = 0; vb[V_PR] = 0;
      vb[V_QT] = k0 / a.B.divq; vb[V_QR] = k0 % a.B.divq;
      vb[V_ONE] = 1;
      const int RS_G = a.Gc;
      for (int it = 0; it < a.num_iters; it++) {
        const int stage = it % STAGES, round = it / STAGES;
        if (round > 0) mbar_wait(&empty[stage], (round - 1) & 1);
        mbar_expect_tx(&full[stage], kA + kB);
        for (int j = 0; j < a.spi; j++) {
          const int slab = it * a.spi + j;
          const bool valid = slab < a.total_slabs;
          const int sl = valid ? slab : 0;
          const int tap = sl / RS_G, g = sl % RS_G;
          const int r = tap / a.S, s = tap % a.S;
          va[V_GT] = g / a.A.divg; va[V_GR] = g % a.A.divg; va[V_R] = r; va[V_S] = s;
          vb[V_GT] = g / a.B.divg; vb[V_GR] = g % a.B.divg; vb[V_R] = r; vb[V_S] = s;
          int32_t ca[5], cb[5];
          coords(a.A, va, ca);
          coords(a.B, vb, cb);
          if (!valid) { ca[0] = a.A.oob0; cb[0] = a.B.oob0; }
          tma_load_5d(sA + stage * kA + j * a.A.slab_bytes, &tmA, &full[stage], ca[0], ca[1], ca[2], ca[3], ca[4]);
          tma_load_5d(sB + stage * kB + j * a.B.slab_bytes, &tmB, &full[stage], cb[0], cb[1], cb[2], cb[3], cb[4]);
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ------------------------------------------------ MMA issuer
      constexpr uint32_t idesc = idesc_f32acc(1 /*bf16*/, 128, BN);
      const int sw = a.sw;
      const uint32_t layout = sw == 8 ? 0u : (sw == 16 ? 6u : (sw == 32 ? 4u : 2u));
      const uint32_t sbo = sw == 8 ? 128u : (uint32_t)(8 * sw * 2);
      const uint32_t aS = (uint32_t)a.A.slab_bytes, bS = (uint32_t)a.B.slab_bytes;
      const uint32_t lboA = sw == 8 ? aS : 16u, lboB = sw == 8 ? bS : 16u;
      for (int it = 0; it < a.num_iters; it++) {
        const int stage = it % STAGES, round = it / STAGES;
        mbar_wait(&full[stage], round & 1);
        tc_fence_after();
        const uint32_t baseA = smem_u32(sA + stage * kA), baseB = smem_u32(sB + stage * kB);
#pragma unroll
        for (int kk = 0; kk < 4; kk++) {
          const int kc = kk * 16;
          const int slab = kc / sw;
          const uint32_t off = (uint32_t)((kc % sw) * 2);
          const uint64_t ad = smem_desc(baseA + slab * aS + off, lboA, sbo, layout);
          const uint64_t bd = smem_desc(baseB + slab * bS + off, lboB, sbo, layout);
          mma_bf16(tmem, ad, bd, idesc, (it | kk) != 0);
        }
        mma_commit(&empty[stage]);
      }
      mma_commit(tmem_full);
    }
  } else {
    // -------------------------------------------------- epilogue warps
    const int wq = warp & 3;
    const int row = wq * 32 + lane;
    const int tn = a.tile_h * a.tile_w;
    const int n = n0 + row / tn, p = p0 + (row / a.tile_w) % a.tile_h, q = q0 + row % a.tile_w;
    const bool vrow = n < a.N && p < a.Ho && q < a.Wo;
    mbar_wait(tmem_full, 0);
    tc_fence_after();
    int64_t base = 0;
    if (vrow && a.vec_out) {
      base = a.is_conv ? (__ldg(a.yrd[0] + n) + __ldg(a.yrd[2] + p) + __ldg(a.yrd[3] + q))
                       : __ldg(a.yrd[0] + q);
    }
#pragma unroll 1
    for (int c0 = 0; c0 < BN; c0 += 32) {
      uint32_t raw[32];
      tmem_ld_32x32b_x32(tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)c0, raw);
      tmem_ld_wait();
      if (!vrow) continue;
      float v[32];
#pragma unroll
      for (int j = 0; j < 32; j++) {
        const int k = k0 + c0 + j;
        float t = __uint_as_float(raw[j]);
        if (k < a.K) {
          if (a.epi.scale) t *= __ldg(a.epi.scale + k);
          if (a.epi.bias) t += __ldg(a.epi.bias + k);
        }
        v[j] = t;
      }
      if (a.epi.residual) {
        const OutT *res = static_cast<const OutT *>(a.epi.residual);
#pragma unroll 4
        for (int j = 0; j < 32; j++) {
          const int k = k0 + c0 + j;
          if (k >= a.K) break;
          const int64_t o = a.is_conv ? a.epi.res.off4(n, k, p, q) : a.epi.res.off2(q, k);
          if (o >= 0) v[j] += load_as_f32<OutT>(res, o);
        }
      }
#pragma unroll
      for (int j = 0; j < 32; j++) v[j] = apply_act(v[j], a.epi.act);
      if (a.vec_out && k0 + c0 + 32 <= a.K) {
        const int64_t *rk = a.is_conv ? a.yrd[1] : a.yrd[1];
#pragma unroll
        for (int j = 0; j < 32; j += 8) store_vec<OutT>(y, base + __ldg(rk + k0 + c0 + j), v + j);
      } else {
        for (int j = 0; j < 32; j++) {
          const int k = k0 + c0 + j;
          if (k >= a.K) break;
          if (a.is_conv) write4<OutT>(a.yw, y, n, k, p, q, from_f32<OutT>(v[j]));
          else write2<OutT>(a.yw, y, q, k, from_f32<OutT>(v[j]));
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc<(BN < 32 ? 32 : BN)>(tmem);
}

// =========================================================== host planner ==
enum Role { R_NONE = 0, R_N, R_H, R_W, R_C, R_TR, R_TS };

struct RoleInfo {
  int role = R_NONE;
  int tile = 1;  // rows of the M (or N) tile along this dim
  int V = 1;     // conv stride
  int pad = 0;   // conv padding
  int win = 1;   // window (R or S) for spatial dims
  int tap = 0;   // add the filter tap (r or s) to the coordinate (conv input)
};

struct VDim {
  int64_t extent, stride;  // elements
  int box, estride;
  int32_t coef[NVAR];
  int order;               // smem order key (lower = inner)
};

struct View {
  int rank = 0;
  VDim d[kMaxP];
  int divp = 1 << 30, divq = 1 << 30, divg = 1;
  int64_t xlo = 0;  // channel run (extent of the stride-1 channel dim)
};

static bool build_view(const Layout &L, const RoleInfo *roles, int sw, View *out, char *why) {
  auto fail = [&](const char *m) { snprintf(why, 160, "%s", m); return false; };
  if (!L.separable || !L.aff.ok) return fail("layout not separable-affine");
  View v;
  int nphys[kMaxL] = {};
  int plist[kMaxL][kMaxP];
  for (int p = 0; p < L.prank; p++) {
    if (L.pshape[p] == 1) continue;
    const int d = L.pdim_owner[p];
    plist[d][nphys[d]++] = p;
  }
  // channel: stride-1 innermost dim
  for (int d = 0; d < L.lrank; d++) {
    const RoleInfo &ri = roles[d];
    const int64_t off = L.aff.off[d];
    auto add = [&](int p, int box, int es, int order) -> VDim & {
      VDim &x = v.d[v.rank++];
      x.extent = L.pshape[p];
      x.stride = L.pstride[p];
      x.box = box;
      x.estride = es;
      memset(x.coef, 0, sizeof(x.coef));
      x.order = order;
      return x;
    };
    switch (ri.role) {
      case R_C: {
        if (nphys[d] == 0 || nphys[d] > 2) return fail("channel dim must have 1-2 physical dims");
        if (off != 0) return fail("channel pad-before offset unsupported");
        int plo = -1, phi = -1;
        for (int i = 0; i < nphys[d]; i++) {
          const int p = plist[d][i];
          if (L.aff.coef[p] == 1) plo = p; else phi = p;
        }
        if (plo < 0 || L.pstride[plo] != 1) return fail("channel tile is not the innermost (stride-1) dim");
        const int64_t xlo = L.pshape[plo];
        if (xlo % sw) return fail("slab width does not divide channel tile");
        if (phi >= 0 && L.aff.coef[phi] != xlo) return fail("channel digits not a plain split");
        v.xlo = xlo;
        v.divg = (int)(xlo / sw);
        VDim &lo = add(plo, sw, 1, 0);
        lo.coef[V_GR] = sw;
        if (phi >= 0) {
          VDim &hi = add(phi, 1, 1, 100);
          hi.coef[V_GT] = 1;
        }
        break;
      }
      case R_N: {
        if (nphys[d] == 0) { if (ri.tile != 1) return fail("tile_n > 1 on a size-1 dim"); break; }
        if (nphys[d] != 1 || L.aff.coef[plist[d][0]] != 1 || off != 0) return fail("batch dim must be plain");
        VDim &x = add(plist[d][0], ri.tile, 1, 50);
        x.coef[V_N0] = 1;
        break;
      }
      case R_TR:
      case R_TS: {
        if (nphys[d] == 0) break;
        if (nphys[d] != 1 || L.aff.coef[plist[d][0]] != 1 || off != 0) return fail("filter tap dim must be plain");
        VDim &x = add(plist[d][0], 1, 1, 100);
        x.coef[ri.role == R_TR ? V_R : V_S] = 1;
        break;
      }
      case R_H:
      case R_W: {
        const bool isH = ri.role == R_H;
        const int VT = isH ? V_PT : V_QT, VR = isH ? V_PR : V_QR, VTAP = isH ? V_R : V_S;
        const int base_order = isH ? 20 : 10;
        int &div = isH ? v.divp : v.divq;
        if (nphys[d] == 0) {
          if (ri.tile != 1 || ri.win != 1) return fail("tile > 1 on a size-1 spatial dim");
          break;
        }
        if (nphys[d] == 1) {
          const int p = plist[d][0];
          if (L.aff.coef[p] != 1) return fail("spatial dim coefficient != 1");
          const int box = ri.tile * ri.V;
          if (box > 256) return fail("box > 256");
          VDim &x = add(p, box, ri.V, base_order);
          x.coef[VR] = ri.V;
          x.coef[VTAP] = ri.tap;
          x.coef[V_ONE] = (int32_t)(-ri.pad - off);
          break;
        }
        if (nphys[d] != 2) return fail("spatial dim with >2 physical dims");
        int plo = -1, phi = -1;
        for (int i = 0; i < 2; i++) {
          const int p = plist[d][i];
          if (L.aff.coef[p] == 1 && plo < 0) plo = p; else phi = p;
        }
        if (plo < 0 || phi < 0) return fail("spatial digits without unit coefficient");
        const int64_t Elo = L.pshape[plo], ch = L.aff.coef[phi];
        if (ch == Elo) {
          // plain split (GEMM-like): no window, no stride, no padding
          if (ri.V != 1 || ri.win != 1 || ri.pad != 0 || off != 0) return fail("split spatial dim with window/stride");
          div = (int)Elo;
          if (ri.tile <= Elo) {
            if (Elo % ri.tile) return fail("tile does not divide spatial split");
            VDim &lo = add(plo, ri.tile, 1, base_order);
            lo.coef[VR] = 1;
            VDim &hi = add(phi, 1, 1, 100);
            hi.coef[VT] = 1;
          } else {
            if (ri.tile % Elo) return fail("spatial split does not divide tile");
            VDim &lo = add(plo, (int)Elo, 1, base_order);
            lo.coef[VR] = 1;
            VDim &hi = add(phi, (int)(ri.tile / Elo), 1, base_order + 1);
            hi.coef[VT] = 1;
          }
        } else {
          // unfold (overlapped tiles): tile must sit inside one
          // layout tile; Eq. (1) gives the in-tile offset
          if (ch % ri.V) return fail("unfold stride not a multiple of conv stride");
          const int64_t ht = ch / ri.V;  // windows per layout tile (Eq. 1's w)
          if (ht % ri.tile) return fail("M tile does not divide the unfold tile");
          const int64_t bmin = -ri.pad - off;
          const int64_t bmax = ri.V * (ht - 1) + ri.win - 1 - ri.pad - off;
          if (bmin < 0 || bmax >= Elo) return fail("unfold tile does not hold the conv window");
          div = (int)ht;
          const int box = ri.tile * ri.V;
          if (box > 256) return fail("box > 256");
          VDim &lo = add(plo, box, ri.V, base_order);
          lo.coef[VR] = ri.V;
          lo.coef[VTAP] = ri.tap;
          lo.coef[V_ONE] = (int32_t)(-ri.pad - off);
          VDim &hi = add(phi, 1, 1, 100);
          hi.coef[VT] = 1;
        }
        break;
      }
      default:
        if (nphys[d] != 0) return fail("unexpected dim");
    }
  }
  if (v.xlo == 0) return fail("no channel dim");
  // order: dim 0 = channel run, then box>1 dims inner->outer, then box-1
  std::stable_sort(v.d, v.d + v.rank, [](const VDim &x, const VDim &y) { return x.order < y.order; });
  // merge box-1 dims adjacent in memory until rank <= 5
  while (v.rank > 5) {
    bool merged = false;
    for (int i = 1; i < v.rank && !merged; i++) {
      for (int j = 1; j < v.rank && !merged; j++) {
        if (i == j || v.d[i].box != 1 || v.d[j].box != 1) continue;
        // i outer, j inner
        if (v.d[i].stride != v.d[j].stride * v.d[j].extent) continue;
        VDim m = v.d[j];
        m.extent = v.d[i].extent * v.d[j].extent;
        for (int k = 0; k < NVAR; k++) m.coef[k] = (int32_t)(v.d[i].coef[k] * v.d[j].extent + v.d[j].coef[k]);
        v.d[j] = m;
        for (int k = i; k < v.rank - 1; k++) v.d[k] = v.d[k + 1];
        v.rank--;
        merged = true;
      }
    }
    if (!merged) return fail("more than 5 TMA dims and no mergeable pair");
  }
  // TMA: strides (dims >= 1) must be 16-byte multiples
  *out = v;
  return true;
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    cudaDriverEntryPointQueryResult q;
    void *p = nullptr;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

static bool encode_view(const View &v, const void *base, int esize, int sw, CUtensorMap *tm, OperandMap *om,
                        char *why) {
  cuuint64_t dims[5], strides[4];
  cuuint32_t box[5], es[5];
  int64_t prev = 1;
  for (int i = 0; i < 5; i++) {
    if (i < v.rank) {
      dims[i] = (cuuint64_t)v.d[i].extent;
      box[i] = (cuuint32_t)v.d[i].box;
      es[i] = (cuuint32_t)v.d[i].estride;
      if (i > 0) strides[i - 1] = (cuuint64_t)(v.d[i].stride * esize);
      prev = v.d[i].stride * v.d[i].extent;
    } else {
      dims[i] = 1;
      box[i] = 1;
      es[i] = 1;
      strides[i - 1] = (cuuint64_t)(((prev * esize) + 15) & ~int64_t(15));
    }
  }
  if (v.d[0].stride != 1) { snprintf(why, 160, "dim0 not contiguous"); return false; }
  for (int i = 0; i < 4; i++)
    if (strides[i] % 16) { snprintf(why, 160, "TMA stride %llu not a multiple of 16 B", (unsigned long long)strides[i]); return false; }
  if ((reinterpret_cast<uintptr_t>(base) & 15)) { snprintf(why, 160, "base not 16-B aligned"); return false; }
  const int row_bytes = sw * esize;
  CUtensorMapSwizzle swz = row_bytes == 16 ? CU_TENSOR_MAP_SWIZZLE_NONE
                           : row_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                           : row_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                             : CU_TENSOR_MAP_SWIZZLE_128B;
  auto enc = get_encode();
  if (!enc) { snprintf(why, 160, "cuTensorMapEncodeTiled unavailable"); return false; }
  CUresult r = enc(tm, esize == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 5,
                   const_cast<void *>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                   CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { snprintf(why, 160, "cuTensorMapEncodeTiled failed (%d)", (int)r); return false; }
  memset(om, 0, sizeof(*om));
  for (int i = 0; i < 5; i++)
    for (int k = 0; k < NVAR; k++) om->coef[i][k] = i < v.rank ? v.d[i].coef[k] : 0;
  om->divp = v.divp;
  om->divq = v.divq;
  om->divg = v.divg;
  int64_t rows = 1;
  for (int i = 1; i < v.rank; i++) rows *= (int64_t)((v.d[i].box + v.d[i].estride - 1) / v.d[i].estride);
  om->slab_bytes = (int32_t)(rows * row_bytes);
  om->oob0 = (int32_t)v.d[0].extent;
  return true;
}

// output fast path: single copy per element, no pads, channel runs of 8
static bool out_vec_ok(const Layout &L, int chan_dim, int esize) {
  if (!L.separable || (L.flags & (ALT_HAS_PAD | ALT_HAS_UNFOLD))) return false;
  for (int d = 0; d < L.lrank; d++)
    if (L.max_copies[d] != 1) return false;
  const int V = 8;
  const auto &rk = L.rd[chan_dim];
  if (rk.size() % V) return false;
  for (size_t k = 0; k < rk.size(); k += V) {
    if (rk[k] < 0 || rk[k] % V) return false;
    for (int j = 1; j < V; j++)
      if (rk[k + j] != rk[k] + j) return false;
  }
  for (int d = 0; d < L.lrank; d++) {
    if (d == chan_dim) continue;
    for (int64_t o : L.rd[d])
      if (o < 0 || o % V) return false;
  }
  (void)esize;
  return true;
}

alt_status make_reader(Layout *L, Reader *r);
alt_status make_writer(Layout *L, Writer *w);
alt_status make_epi(const OpEpilogue &e, EpiParams *p);

static int pow2_floor(int64_t x) {
  int p = 1;
  while ((int64_t)p * 2 <= x) p *= 2;
  return p;
}

template <int BN, int STAGES, typename OutT>
static cudaError_t launch_tc(const CUtensorMap &ta, const CUtensorMap &tb, const TcArgs &a, OutT *y, dim3 grid,
                             cudaStream_t s) {
  auto kern = k_tc_igemm<BN, STAGES, OutT>;
  const int smem = TcSmem<BN, STAGES>::kBytes;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  kern<<<grid, kThreads, smem, s>>>(ta, tb, a, y);
  return cudaGetLastError();
}

// common driver for conv and GEMM (GEMM: N=1, H=W... expressed via roles)
struct TcProblem {
  bool is_conv;
  Layout *al, *bl, *yl;
  const void *a, *b;
  void *y;
  RoleInfo ra[kMaxL], rb[kMaxL];
  int64_t N, K, Ho, Wo;       // output geometry (GEMM: 1, cols, 1, M)
  int64_t R, S, C;            // taps and reduction channels
  int y_chan_dim;             // channel dim of y's logical shape
  OpEpilogue epi;
};

static alt_status tc_run(TcProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used,
                         int tile_n_fixed, int tile_h_fixed) {
  char why[160] = "";
  // slab width: largest power of two <= 64 dividing both channel runs
  // (determined after the views are built; try 64 down to 8)
  const int esize = 2;
  // M-tile candidates
  struct Cand { int tn, th, tw; };
  std::vector<Cand> cands;
  if (cfg && cfg->tile_n * cfg->tile_h * cfg->tile_w == 128) {
    cands.push_back({cfg->tile_n, cfg->tile_h, cfg->tile_w});
  } else if (!P.is_conv) {
    cands.push_back({1, 1, 128});
  } else {
    for (int tw = 1; tw <= 128; tw *= 2)
      for (int th = 1; th * tw <= 128; th *= 2) {
        const int tn = 128 / (tw * th);
        if (tile_n_fixed && tn != tile_n_fixed) continue;
        if (tile_h_fixed && th != tile_h_fixed) continue;
        if (tn > 1 && (tn > P.N)) continue;
        cands.push_back({tn, th, tw});
      }
    // prefer the least wasted rows: coverage = ceil(Ho/th)*th*ceil(Wo/tw)*tw*ceil(N/tn)*tn
    std::stable_sort(cands.begin(), cands.end(), [&](const Cand &x, const Cand &y) {
      auto cov = [&](const Cand &c) {
        return (double)((P.Ho + c.th - 1) / c.th * c.th) * ((P.Wo + c.tw - 1) / c.tw * c.tw) *
               ((P.N + c.tn - 1) / c.tn * c.tn);
      };
      double a = cov(x), b = cov(y);
      if (a != b) return a < b;
      return x.tw > y.tw;  // longer contiguous runs first
    });
  }
  int BN = cfg && cfg->block_n ? cfg->block_n : (P.K >= 256 && P.K % 256 == 0 ? 256 : (P.K >= 128 ? 128 : 64));
  if (BN != 64 && BN != 128 && BN != 256) { set_error("tc: block_n must be 64/128/256"); return ALT_E_UNSUPPORTED; }
  for (const Cand &c : cands) {
    RoleInfo ra[kMaxL], rb[kMaxL];
    memcpy(ra, P.ra, sizeof(ra));
    memcpy(rb, P.rb, sizeof(rb));
    for (int d = 0; d < kMaxL; d++) {
      if (ra[d].role == R_N) ra[d].tile = c.tn;
      if (ra[d].role == R_H) ra[d].tile = c.th;
      if (ra[d].role == R_W) ra[d].tile = c.tw;
      if (rb[d].role == R_W) rb[d].tile = BN;
    }
    for (int sw = 64; sw >= 8; sw /= 2) {
      View va, vb;
      if (!build_view(*P.al, ra, sw, &va, why)) continue;
      if (!build_view(*P.bl, rb, sw, &vb, why)) continue;
      // check TMA row count = 128 for A and BN for B
      int64_t rowsA = 1, rowsB = 1;
      for (int i = 1; i < va.rank; i++) rowsA *= (va.d[i].box + va.d[i].estride - 1) / va.d[i].estride;
      for (int i = 1; i < vb.rank; i++) rowsB *= (vb.d[i].box + vb.d[i].estride - 1) / vb.d[i].estride;
      if (rowsA != 128 || rowsB != BN) { snprintf(why, 160, "rows A %lld B %lld", (long long)rowsA, (long long)rowsB); continue; }
      CUtensorMap ta, tb;
      TcArgs a;
      memset(&a, 0, sizeof(a));
      if (!encode_view(va, P.a, esize, sw, &ta, &a.A, why)) continue;
      if (!encode_view(vb, P.b, esize, sw, &tb, &a.B, why)) continue;
      a.is_conv = P.is_conv;
      a.N = (int32_t)P.N; a.K = (int32_t)P.K; a.Ho = (int32_t)P.Ho; a.Wo = (int32_t)P.Wo;
      a.tile_n = c.tn; a.tile_h = c.th; a.tile_w = c.tw;
      a.mt_h = (int32_t)((P.Ho + c.th - 1) / c.th);
      a.mt_w = (int32_t)((P.Wo + c.tw - 1) / c.tw);
      const int64_t mt_n = (P.N + c.tn - 1) / c.tn;
      a.S = (int32_t)P.S;
      a.Gc = (int32_t)((P.C + sw - 1) / sw);
      a.total_slabs = (int32_t)(P.R * P.S * a.Gc);
      a.spi = 64 / sw;
      a.num_iters = (a.total_slabs + a.spi - 1) / a.spi;
      a.sw = sw;
      alt_status st;
      if ((st = make_epi(P.epi, &a.epi)) != ALT_OK) return st;
      if ((st = make_writer(P.yl, &a.yw)) != ALT_OK) return st;
      a.vec_out = out_vec_ok(*P.yl, P.y_chan_dim, esize) ? 1 : 0;
      if (a.vec_out) {
        SepDev sd{};
        if ((st = device_tables(P.yl, &sd, nullptr)) != ALT_OK) return st;
        if (P.is_conv) {
          a.yrd[0] = sd.rd[0]; a.yrd[1] = sd.rd[1]; a.yrd[2] = sd.rd[2]; a.yrd[3] = sd.rd[3];
        } else {
          a.yrd[0] = sd.rd[0]; a.yrd[1] = sd.rd[1];
        }
      }
      const int64_t mtiles = mt_n * a.mt_h * a.mt_w;
      const int64_t ntiles = (P.K + BN - 1) / BN;
      if (mtiles > 0x7fffffff || ntiles > 65535) { set_error("tc: grid too large"); return ALT_E_UNSUPPORTED; }
      dim3 grid((unsigned)mtiles, (unsigned)ntiles);
      cudaError_t e;
      uint16_t *y = static_cast<uint16_t *>(P.y);
      if (BN == 64) e = launch_tc<64, 6, uint16_t>(ta, tb, a, y, grid, stream);
      else if (BN == 128) e = launch_tc<128, 4, uint16_t>(ta, tb, a, y, grid, stream);
      else e = launch_tc<256, 4, uint16_t>(ta, tb, a, y, grid, stream);
      count_launch();
      if (e != cudaSuccess) { set_error("tc launch failed: %s", cudaGetErrorString(e)); return ALT_E_CUDA; }
      alt_kernel_cfg u{};
      u.path = ALT_PATH_TC;
      u.block_m = 128;
      u.block_n = BN;
      u.block_k = 64;
      u.stages = BN == 64 ? 6 : 4;
      u.tile_n = c.tn; u.tile_h = c.th; u.tile_w = c.tw;
      if (used) *used = u;
      return ALT_OK;
    }
  }
  set_error("tc path unavailable: %s", why);
  return ALT_E_UNSUPPORTED;
}

alt_status tc_conv(const ConvProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used) {
  if (P.dtype != ALT_BF16) { set_error("tc path: bf16 only"); return ALT_E_UNSUPPORTED; }
  if (P.groups != 1) { set_error("tc path: groups == 1 only"); return ALT_E_UNSUPPORTED; }
  TcProblem T{};
  T.is_conv = true;
  T.al = P.xl; T.bl = P.wl; T.yl = P.yl;
  T.a = P.x; T.b = P.w; T.y = P.y;
  // x logical (n, c, h, w); w logical (k, c, r, s)
  T.ra[0].role = R_N;
  T.ra[1].role = R_C;
  T.ra[2] = RoleInfo{R_H, 1, P.Vh, P.ph, (int)P.R, 1};
  T.ra[3] = RoleInfo{R_W, 1, P.Vw, P.pw, (int)P.S, 1};
  T.rb[0] = RoleInfo{R_W, 1, 1, 0, 1};
  T.rb[1].role = R_C;
  T.rb[2].role = R_TR;
  T.rb[3].role = R_TS;
  T.N = P.N; T.K = P.K; T.Ho = P.Ho; T.Wo = P.Wo;
  T.R = P.R; T.S = P.S; T.C = P.C;
  T.y_chan_dim = 1;
  T.epi = P.epi;
  if (P.N * P.Ho * P.Wo >= (1ll << 31)) { set_error("tc: too many output pixels"); return ALT_E_UNSUPPORTED; }
  return tc_run(T, cfg, stream, used, 0, 0);
}

alt_status tc_gemm(const GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used) {
  if (P.dtype != ALT_BF16) { set_error("tc path: bf16 only"); return ALT_E_UNSUPPORTED; }
  TcProblem T{};
  T.is_conv = false;
  T.al = P.al; T.bl = P.bl; T.yl = P.cl;
  T.a = P.a; T.b = P.b; T.y = P.c;
  // A logical (m, k): m = rows (W role), k = reduction; B logical (k, n)
  T.ra[0] = RoleInfo{R_W, 128, 1, 0, 1};
  T.ra[1].role = R_C;
  T.rb[0].role = R_C;
  T.rb[1] = RoleInfo{R_W, 1, 1, 0, 1};
  T.N = 1; T.K = P.N; T.Ho = 1; T.Wo = P.M;
  T.R = 1; T.S = 1; T.C = P.K;
  T.y_chan_dim = 1;
  T.epi = P.epi;
  return tc_run(T, cfg, stream, used, 1, 1);
}

}  // namespace alt
