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
// is converted to run on the tensor cores.  The output is written
// the same way in reverse (TMA store boxes cut from y's layout), so a layer
// writes its consumer's layout directly (propagation, Fig. 5b).
//
// Persistent kernel, one CTA per SM, 6 warps:
//   warp 0     TMA producer (one thread), STAGES-deep smem ring
//   warp 1     TMEM allocator + single-thread tcgen05.mma issuer (M = 128),
//              accumulator double-buffered in TMEM (2 x BLOCK_N columns)
//   warps 2-5  epilogue: tcgen05.ld -> act(scale*acc + bias + residual) ->
//              bf16 -> swizzled smem -> TMA store (or the generic writer for
//              layouts with pads / unfold copies); overlaps the next tile's MMA
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <unordered_map>
#include <type_traits>
#include <vector>

#include "epilogue.cuh"
#include "ops.h"
#include "sm100.cuh"

namespace alt {

// V_DO / V_T: output depth and depth tap of a 3-D conv (C3D), 0 for conv2d
enum Var { V_N0 = 0, V_PT, V_PR, V_QT, V_QR, V_GT, V_GR, V_R, V_S, V_ONE, V_DO, V_T, NVAR };

// box-coordinate rule for one tensor map: coord[d] = sum_k coef[d][k] * var[k]
struct OperandMap {
  int32_t coef[5][NVAR];
  int32_t divp, divq, divg;
  FastDiv fp, fq, fg;  // the same divisors as multiply-shift (no integer division on the device)
  int32_t slab_bytes;
  int32_t oob0;  // dim-0 coordinate that makes a box all zeros
  int32_t sw;    // slab width (channels)
  // MN-major operand (mnw > 0): the stride-1 physical dim is the M (or N)
  // dim, not the reduction; smem holds ng groups of mnw M-elements x 64
  // K rows (gbytes each, K rows mnw * 2 bytes apart), one TMA box per
  // (group, channel slab).  mnw = 0: K-major (channel run innermost).
  int32_t mnw, ng, gbytes;
};

struct TcArgs {
  OperandMap A, B, O;
  int32_t out_mode;      // 1: TMA-store epilogue, 2: direct 16-byte stores, 0: generic writer
  int32_t res_vec;       // residual read as 16-byte vectors of 8 channels (epi.res tables)
  // grouped conv: one launch per group; the group's input channel slabs start
  // at slab a_goff of x, its weight rows at b_koff, its outputs at channel y_koff
  int32_t a_goff, b_koff, y_koff;
  int32_t is_conv;
  int32_t N, K, Ho, Wo;  // output: conv y[N,K,Ho,Wo]; GEMM: N=1, Ho=1, Wo=M, K=cols
  int32_t tile_n, tile_h, tile_w;
  int32_t mt_h, mt_w;    // # tiles along h, w (n is the slowest)
  int32_t num_n_tiles, num_tiles;
  int32_t S, Gc;
  FastDiv f_nnt, f_mtw, f_mth, f_spl, f_Gc, f_S;  // num_n_tiles, mt_w, mt_h, splits, Gc, S
  int32_t total_slabs, spi, num_iters;
  // fp32 operands split into three bf16 planes (reading A27): pairs = 6
  // plane products per reduction step (0 = plain bf16); rsg = R * S * Gc
  // slabs per pair; out_f32: the output (and residual) are fp32
  int32_t pairs, rsg, out_f32;
  FastDiv f_rsg;
  int32_t nst;           // smem ring stages in use (<= the instantiation's STAGES; tuner knob)
  int32_t hboff;         // halo mode: set the descriptor base-offset field for row-shifted A starts
  int32_t a_bytes;       // bytes of one A stage's box(es) (expect_tx): 128 rows x 128 B, or the
                         // 2-D halo tile's (tile_h + R - 1) tile_w rows
  int32_t b_res;         // resident weights: every unit of this CTA has the same N tile and the
                         // reduction fits the ring (num_iters <= nst), so the B slabs loaded with
                         // the first tile stay in the ring's B slots (slot = k iteration) and later
                         // tiles stream A only (one B read per CTA instead of one per tile)
  // C3D: tile batch index b = n Do + od (tile_n = 1); taps (t, r, s), RS = R S
  int32_t Do3, RS3;
  FastDiv f_Do3, f_RS3;
  int32_t yvec;          // out_mode 0 with 8-channel runs: copies written as 16-byte vectors
  int32_t out_round;     // out_mode 1, round stores: the 8 epilogue warps stage a whole 128-row x
                         // 64-channel round in smem, one thread TMA-stores it (a.O views 128 rows)
  int32_t pads_zero;     // ALT_EPI_PADS_ZERO: skip y's pad (structural zero) positions
  int32_t sw;
  Writer yw;
  Reader yr;             // out_mode 2: owner offsets of y
  EpiParams epi;
  uint64_t *dbg;         // optional per-CTA timestamps (ALT_TC_DEBUG)
  int32_t epi_dbg;       // developer knob (ALT_TC_EPI_DBG): 1 skip output stores, 2 skip the whole drain,
                         // 3 also skip the MMAs (the TMA pipeline alone)
  // split-K: work unit = (output tile, reduction range); partial fp32 tiles
  // in ws[cta_tile][split][BN/32][128][32], arrivals counted in cnt[cta_tile]
  int32_t splits;
  int32_t full_units;    // units [0, full_units) run unsplit; later output tiles are split
                         // `splits` ways (0 = every tile split; tail mode: the last wave only)
  float *ws;
  int32_t *cnt;
  int32_t coop;          // split tiles reduced cooperatively: each of the splits CTAs
                         // finishes 1 / splits of the tile's rows (all pieces co-resident)
  int32_t *done;         // per split tile: CTAs finished (resets cnt / done for the next launch)
};

#ifndef ALT_EPI_WARPS
#define ALT_EPI_WARPS 8
#endif
// epilogue warps: 4 TMEM lane quarters x kParts column parts.  The drain is
// latency-bound (TMEM load -> FMA -> pack -> smem -> TMA store per 32-column
// chunk).  16 warps (ALT_EPI_WARPS=16) were measured slower: the 576-thread
// CTA is capped at 96 registers and the epilogue spills.
constexpr int kEpiWarps = ALT_EPI_WARPS;
constexpr int kParts = kEpiWarps / 4;
constexpr int kStep = 32 * kParts;     // columns per chunk round
constexpr int kEpiThreads = 32 * kEpiWarps;
constexpr int kThreads = 64 + kEpiThreads;  // producer, MMA, epilogue warps
constexpr int kStageBytesA = 128 * 64 * 2;
constexpr int kOutStage = 128 * 64 * 2;  // one 64-column bf16 chunk of the tile

// accumulator buffers in TMEM (512 columns): the MMA of tile i + NACC - 1
// may run while the epilogue drains tile i
template <int BN>
struct Nacc { static constexpr int value = BN >= 192 ? 2 : 4; };
// TMEM allocations are powers of two >= 32 columns
constexpr int tmem_cols(int c) { return c <= 32 ? 32 : (c <= 64 ? 64 : (c <= 128 ? 128 : (c <= 256 ? 256 : 512))); }

// Reduction-slab coordinate table: for every slab (filter tap x channel
// slab) of the reduction, the part of the A / B box coordinates that depends
// on the slab (5 ints each, A at [0..4], B at [8..12] of a 64-byte row).
// Built once per CTA in the prologue, so the producer's per-stage work is
// one shared load + 5 adds per box instead of the divisions and the 5 x 10
// coefficient products of coords() (the single producer thread's issue
// latency bounds the stage rate).
constexpr int kTabSlabs = kEpiWarps == 8 ? 288 : 240;
constexpr int kTabBytes = kTabSlabs * 64;

// HS > 0: halo mode for stride-1 filters of width HS (3x3): an A stage is
// loaded once per (filter row, channel slab) with 8 spare rows after the
// 128, and the HS taps along W read it at row offsets 0 .. HS-1; B holds the
// HS tap slabs of the stage
// HR > 0 (with HS): two-dimensional halo for stride-1 R x S filters with one
// 64-channel slab (C <= 64): an A stage holds the tile's (tile_h + R - 1)
// input rows of tile_w pixels (<= 256 rows, one TMA box per tile) and the
// R x S taps read it at row offsets r tile_w + s; the weights of all taps sit
// in one resident B slot after the A ring (loaded with the CTA's first tile)
template <int BN, int STAGES, int CG = 1, int HS = 0, int HR = 0>
struct TcSmem {
  static constexpr int kAst = HR ? 256 * 128 + 1024 : kStageBytesA + (HS ? 1024 : 0);  // A stage stride
  static constexpr int kB = (BN / CG) * 64 * 2 * (HS ? HS : 1) * (HR ? HR : 1);  // this CTA's share of the B tile(s)
  static constexpr int kRing = HR ? STAGES * kAst + kB : STAGES * (kAst + kB);
  static constexpr int kOut = kRing;                       // 2 staging buffers for TMA stores
  static constexpr int kSB = kOut + kEpiWarps * 4096;      // scale / bias of the tile (2 x BN floats)
  static constexpr int kBar = kSB + 2 * BN * 4;             // barriers
  static constexpr int kTab = kBar + 256;                   // slab coordinate table
  static constexpr int kBytes = kTab + kTabBytes + 1008 /*1024-B alignment slack*/;
};

__device__ __forceinline__ uint64_t gtimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#ifndef ALT_DBG_TILE
#define ALT_DBG_TILE 0  // which of a CTA's tiles the epilogue timestamps follow
#endif
#define DBG(slot) \
  if (a.dbg) a.dbg[(size_t)blockIdx.x * 40 + (slot)] = gtimer()

// reduction slab -> filter tap (r, s) and the channel slab of A and of B.
// Plain operands: slab = tap * Gc + g.  fp32 split operands (a.pairs = 6):
// slab = pair * (R S Gc) + tap * Gc + g, the pair selecting the bf16 planes
// (pa, pb) in {lh, hl, mm, mh, hm, hh} (every product of weight > 2^-24); a
// plane starts Gc channel slabs after the previous one.  Smallest products
// first: the tensor core's fp32 accumulation rounds each MMA step relative
// to the accumulator's magnitude, so the five small pairs are summed while
// the accumulator is still small and only the hh steps see the full value
// (measured 6x lower error than hh first).
// D3: C3D instantiation (depth taps / output depth); the conv2d / GEMM
// kernels compile the depth terms out (measured 11 us per R50 step)
template <bool D3>
__device__ __forceinline__ void slab_decode(const TcArgs &a, int sl, int &r, int &sx, int &t, int &gA, int &gB) {
  int rem = sl, pa = 0, pb = 0;
  if (a.pairs) {
    const int pr = (int)a.f_rsg.div((uint32_t)sl);
    rem = sl - pr * a.rsg;
    pa = (0x001102 >> (4 * pr)) & 0xF;
    pb = (0x010120 >> (4 * pr)) & 0xF;
  }
  int tap = (int)a.f_Gc.div((uint32_t)rem);
  const int g = rem - tap * a.Gc;
  t = 0;
  if (D3) {  // C3D: tap = (t, r, s)
    t = (int)a.f_RS3.div((uint32_t)tap);
    tap -= t * a.RS3;
  }
  r = (int)a.f_S.div((uint32_t)tap);
  sx = tap - r * a.S;
  gA = pa * a.Gc + g + a.a_goff;
  gB = pb * a.Gc + g;
}

template <bool D3>
__device__ __forceinline__ void coords(const OperandMap &m, const int32_t (&v)[NVAR], int32_t (&c)[5]) {
#pragma unroll
  for (int d = 0; d < 5; d++) {
    int32_t s = 0;
#pragma unroll
    for (int k = 0; k < (D3 ? NVAR : V_DO); k++) s += m.coef[d][k] * v[k];
    c[d] = s;
  }
}

__device__ __forceinline__ void named_bar(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
// two floats -> packed bf16x2 (lo = a), optionally with ReLU in the convert
__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  uint32_t r;
  asm("cvt.rn.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
  return r;
}
__device__ __forceinline__ uint32_t pack_bf16x2_relu(float a, float b) {
  uint32_t r;
  asm("cvt.rn.relu.bf16x2.f32 %0, %1, %2;" : "=r"(r) : "f"(b), "f"(a));
  return r;
}
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tma_store_5d(const CUtensorMap *m, const void *src, int32_t c0, int32_t c1,
                                             int32_t c2, int32_t c3, int32_t c4) {
  asm volatile(
      "cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];" ::"l"(
          reinterpret_cast<uint64_t>(m)),
      "r"(sm100::smem_u32(src)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4)
      : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait0() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }

// Out-of-line slow paths of the epilogue (kept out of the hot loop body).
// residual values of one row's 32 channels, read through the residual layout
static __device__ __noinline__ void residual_chunk(const EpiParams &e, int is_conv, int K, int n, int p, int q,
                                                   int kb, int koff, float *out) {
  const uint16_t *res = static_cast<const uint16_t *>(e.residual);
  for (int j = 0; j < 32; j++) {
    const int k = kb + j;
    float r = 0.f;
    if (k < K) {
      const int64_t o = is_conv ? e.res.off4(n, koff + k, p, q) : e.res.off2(q, koff + k);
      if (o >= 0) r = bf16_to_f32(__ldg(res + o));
    }
    out[j] = r;
  }
}
// fp32 residual (split-operand path)
static __device__ __noinline__ void residual_chunk_f32(const EpiParams &e, int is_conv, int K, int n, int p, int q,
                                                       int kb, int koff, float *out) {
  const float *res = static_cast<const float *>(e.residual);
  for (int j = 0; j < 32; j++) {
    const int k = kb + j;
    float r = 0.f;
    if (k < K) {
      const int64_t o = is_conv ? e.res.off4(n, koff + k, p, q) : e.res.off2(q, koff + k);
      if (o >= 0) r = __ldg(res + o);
    }
    out[j] = r;
  }
}
// fp32 output: one row's 32 channels, direct 16-byte stores of 4 channels
// (out_mode 2) or through the generic writer
static __device__ __noinline__ void store_chunk_f32(const TcArgs &a, float *y, int64_t yrow, int n, int p, int q,
                                                    int kb, const float *v) {
  if (a.out_mode == 2) {
    for (int c = 0; c < 8; c++) {
      const int k = kb + 4 * c;
      if (k >= a.K) break;
      float *dst = y + yrow + __ldg(a.yr.rd[1] + a.y_koff + k);
      asm volatile("st.global.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(dst), "f"(v[4 * c]), "f"(v[4 * c + 1]),
                   "f"(v[4 * c + 2]), "f"(v[4 * c + 3])
                   : "memory");
    }
    return;
  }
  for (int j = 0; j < 32; j++) {
    const int k = kb + j;
    if (k >= a.K) break;
    if (a.is_conv) write4<float>(a.yw, y, n, a.y_koff + k, p, q, v[j]);
    else write2<float>(a.yw, y, q, a.y_koff + k, v[j]);
  }
}
// one row's 32 channels into a layout with pads / unfold copies whose
// channel dim runs in 16-byte-aligned groups of 8 (NCHW[x]c tiled templates):
// every physical copy of the (n, p, q) row gets four 16-byte stores; pad
// positions the row owns get zeros (or are skipped under pads_zero)
static __device__ __noinline__ void write_chunk_vec(const TcArgs &a, uint16_t *y, int n, int p, int q, int kb,
                                                    const uint32_t *pk) {
  const Writer &w = a.yw;
  int64_t ch[4];
#pragma unroll
  for (int c = 0; c < 4; c++) {
    const int k = kb + 8 * c;
    ch[c] = k < a.K ? __ldg(a.yr.rd[1] + a.y_koff + k) : -1;
  }
  const int d0 = a.is_conv ? n : q;
  const int32_t a0 = __ldg(w.wptr[0] + d0), a1 = __ldg(w.wptr[0] + d0 + 1);
  int32_t b0 = 0, b1 = 1, c0 = 0, c1 = 1;
  if (a.is_conv) {
    b0 = __ldg(w.wptr[2] + p); b1 = __ldg(w.wptr[2] + p + 1);
    c0 = __ldg(w.wptr[3] + q); c1 = __ldg(w.wptr[3] + q + 1);
  }
  for (int32_t i = a0; i < a1; i++) {
    const int64_t ca = __ldg(w.wlist[0] + i);
    for (int32_t j = b0; j < b1; j++) {
      const int64_t cb = a.is_conv ? __ldg(w.wlist[2] + j) : 0;
      for (int32_t l = c0; l < c1; l++) {
        const int64_t cc = a.is_conv ? __ldg(w.wlist[3] + l) : 0;
        const bool zero = ((ca | cb | cc) & 1) != 0;
        if (zero && a.pads_zero) continue;
        const int64_t base = (ca >> 1) + (cb >> 1) + (cc >> 1);
#pragma unroll
        for (int c = 0; c < 4; c++) {
          if (ch[c] < 0) break;
          uint16_t *dst = y + base + ch[c];
          if (zero)
            asm volatile("st.global.v4.b32 [%0], {%1, %1, %1, %1};" ::"l"(dst), "r"(0u) : "memory");
          else
            asm volatile("st.global.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(dst), "r"(pk[4 * c]), "r"(pk[4 * c + 1]),
                         "r"(pk[4 * c + 2]), "r"(pk[4 * c + 3])
                         : "memory");
        }
      }
    }
  }
}
// one row's 32 channels through the generic writer (pads, unfold copies)
static __device__ __noinline__ void write_chunk(const Writer &w, int is_conv, int K, uint16_t *y, int n, int p,
                                                int q, int kb, int koff, const uint32_t *pk) {
  for (int j = 0; j < 32; j++) {
    const int k = kb + j;
    if (k >= K) break;
    const uint16_t h = (uint16_t)(j & 1 ? pk[j >> 1] >> 16 : pk[j >> 1] & 0xffff);
    if (is_conv) write4<uint16_t>(w, y, n, koff + k, p, q, h);
    else write2<uint16_t>(w, y, q, koff + k, h);
  }
}

// split-K: the tile's value = sum of the splits' partials in split order
// (this CTA's own split taken from its accumulator, the others read back
// from the workspace), so the result does not depend on which CTA finishes
// last.  Workspace layout per CTA tile and split: [BN/32][8][128] float4
// (32-column chunk, float4 slot, row): a warp's 32 rows are 512 contiguous
// bytes, so partial stores and loads are fully coalesced.  Out of line: the
// split path is rare and must not cost the common path registers.
static __device__ __noinline__ void split_total(const float *wt, int splits, int own, int BN, int cb, int row,
                                                const uint32_t *mine, float *out) {
  float t[32];
#pragma unroll
  for (int j = 0; j < 32; j++) t[j] = 0.f;
  for (int s = 0; s < splits; s++) {
    if (s == own) {
#pragma unroll
      for (int j = 0; j < 32; j++) t[j] += __uint_as_float(mine[j]);
      continue;
    }
    const float4 *src = reinterpret_cast<const float4 *>(wt + (size_t)s * (128 * BN)) + (size_t)(cb >> 5) * 8 * 128 + row;
    float4 f[8];
#pragma unroll
    for (int j = 0; j < 8; j++) f[j] = __ldcg(src + j * 128);
#pragma unroll
    for (int j = 0; j < 8; j++) {
      t[4 * j] += f[j].x; t[4 * j + 1] += f[j].y; t[4 * j + 2] += f[j].z; t[4 * j + 3] += f[j].w;
    }
  }
#pragma unroll
  for (int j = 0; j < 32; j++) out[j] = t[j];
}

// work unit -> (output tile mn, split index sp, reduction range [kb, ke))
struct UnitInfo { int mn, sp, kb, ke; bool split; };
__device__ __forceinline__ UnitInfo unit_info(const TcArgs &a, int tile) {
  UnitInfo u;
  if (tile < a.full_units) {
    u.mn = tile; u.sp = 0; u.kb = 0; u.ke = a.num_iters; u.split = false;
    return u;
  }
  const int t = tile - a.full_units;
  const int q = (int)a.f_spl.div((uint32_t)t);
  u.mn = a.full_units + q;
  u.sp = t - q * a.splits;
  u.split = a.splits > 1;
  u.kb = u.split ? u.sp * a.num_iters / a.splits : 0;
  u.ke = u.split ? (u.sp + 1) * a.num_iters / a.splits : a.num_iters;
  return u;
}

struct TileCoord { int n0, p0, q0, k0, d0; };
// work unit `tile` -> this CTA's 128-row M tile and the unit's N tile; with a
// CTA pair (CG = 2) a unit is two consecutive M tiles, one per CTA rank
template <bool D3>
__device__ __forceinline__ TileCoord tile_coord(const TcArgs &a, int tile, int BN, int CG, int rank) {
  const int mq = (int)a.f_nnt.div((uint32_t)tile);
  const int mt = mq * CG + rank, nt = tile - mq * a.num_n_tiles;
  const int mw = (int)a.f_mtw.div((uint32_t)mt);
  const int tw_i = mt - mw * a.mt_w;
  const int tn_i = (int)a.f_mth.div((uint32_t)mw);
  const int th_i = mw - tn_i * a.mt_h;
  if (D3) {  // C3D: the batch index of a tile is (n, od), one output depth slice per tile
    const int n = (int)a.f_Do3.div((uint32_t)tn_i);
    return {n, th_i * a.tile_h, tw_i * a.tile_w, nt * BN, tn_i - n * a.Do3};
  }
  return {tn_i * a.tile_n, th_i * a.tile_h, tw_i * a.tile_w, nt * BN, 0};
}

// RV: epilogue reads the residual as 16-byte vectors (a separate
// instantiation keeps the residual-free epilogue's register allocation).
// SC > 1: cluster split-K — the SC reduction ranges of one output tile run as
// the SC CTAs of a thread-block cluster (one tile per CTA, no workspace); each
// CTA drains its fp32 partial into its own (then idle) smem ring, and after a
// cluster barrier CTA r reduces rows [r * 128 / SC, (r + 1) * 128 / SC) of all
// SC partials through distributed shared memory in split order, applies the
// epilogue and stores them — the reduction and the epilogue are split SC ways.
template <int BN, int STAGES, int CG, bool RV, int SC, int HS = 0, bool D3 = false, int HR = 0>
__global__ void __launch_bounds__(kThreads, 1)
    k_tc_conv(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
              const __grid_constant__ CUtensorMap tmY, const __grid_constant__ TcArgs a, uint16_t *__restrict__ y) {
  using namespace sm100;
  using L = TcSmem<BN, STAGES, CG, HS, HR>;
  const int rank = CG == 2 ? (int)cluster_ctarank() : 0;
  const int unit0 = blockIdx.x / CG, unit_step = gridDim.x / CG;
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char *smem = reinterpret_cast<unsigned char *>(
      (reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  unsigned char *sA = smem;
  unsigned char *sB = smem + STAGES * L::kAst;
  unsigned char *sOut = smem + L::kOut;
  const uint32_t sSB = sm100::smem_u32(smem + L::kSB);  // scale [BN] then bias [BN] (fp32)
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + L::kBar);
  uint64_t *empty = full + STAGES;
  uint64_t *tfull = empty + STAGES;   // [2]
  constexpr int NACC = Nacc<BN>::value;
  uint64_t *tempty = tfull + NACC;    // [NACC]
  uint32_t *tmem_slot = reinterpret_cast<uint32_t *>(tempty + NACC);
  volatile int32_t *last_flag = reinterpret_cast<volatile int32_t *>(tmem_slot + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) { DBG(0); }
  if (warp == 0 && lane == 0) {
    tma_prefetch(&tmA);
    tma_prefetch(&tmB);
    if (a.out_mode == 1) tma_prefetch(&tmY);
    for (int s = 0; s < STAGES; s++) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < NACC; s++) {
      mbar_init(&tfull[s], 1);
      mbar_init(&tempty[s], kEpiWarps * CG);  // every epilogue warp of the pair
    }
    fence_mbar_init();
    DBG(33);
  }
  if (warp == 1) tmem_alloc<tmem_cols(NACC * BN), CG>(tmem_slot);
  if (threadIdx.x == 32) { DBG(34); }
  // slab table (see kTabSlabs): slab -> (tap r, s; channel slab g = (gt, gr))
  int32_t *tab = reinterpret_cast<int32_t *>(smem + L::kTab);
  const int padded_slabs = a.num_iters * a.spi;
  const bool use_tab = padded_slabs <= kTabSlabs;
  if (use_tab) {
    for (int sl = threadIdx.x; sl < padded_slabs; sl += kThreads) {
      const bool valid = sl < a.total_slabs;
      const int s0 = valid ? sl : 0;
      int r, sx, tt, gA, gB;
      slab_decode<D3>(a, s0, r, sx, tt, gA, gB);
#pragma unroll
      for (int o = 0; o < 2; o++) {
        const OperandMap &om = o == 0 ? a.A : a.B;
        const int ga = o == 0 ? gA : gB;
        const int gt = (int)om.fg.div((uint32_t)ga), gr = ga - gt * om.divg;
#pragma unroll
        for (int d = 0; d < 5; d++)
          tab[sl * 16 + o * 8 + d] = om.coef[d][V_R] * r + om.coef[d][V_S] * sx + om.coef[d][V_T] * tt +
                                     om.coef[d][V_GT] * gt + om.coef[d][V_GR] * gr;
        if (!valid) tab[sl * 16 + o * 8] = om.oob0;  // all-zero box (dim 0 has no tile term)
      }
    }
  }
  if (threadIdx.x == 0) { DBG(35); }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync();  // peer barriers initialised before any remote arrive
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // programmatic dependent launch: the prologue above overlapped the previous
  // kernel's tail; no global memory is touched before it has completed
  if (threadIdx.x == 0) { DBG(32); }
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  if (threadIdx.x == 0) { DBG(1); }

  if (warp == 0) {
    // -------------------------------------------------------- TMA producer
    // lane j < 8 issues A slab j of a stage, lane 16 + j issues B slab j:
    // the box coordinates of all slabs are computed in parallel.
    const bool isA = lane < 16;
    const int j = lane & 15;
    const OperandMap &om = isA ? a.A : a.B;
    const CUtensorMap *tmap = isA ? &tmA : &tmB;
    unsigned char *sbase = isA ? sA : sB;
    const int sbytes = isA ? L::kAst : L::kB;
    // issues per stage: (group, channel slab) pairs; a K-major operand has
    // one group, an MN-major one ng groups of mnw rows (planner: <= 16);
    // halo mode: B issues one box per (tap s, slab), lane j -> s = j / spi
    // 2-D halo (HR): B issues one box per tap (r, s), lane j -> (j / S, j % S)
    const int hsb = (HS && !isA) ? HS * (HR ? HR : 1) : 1;
    const bool active = j < om.ng * a.spi * hsb;
    const int hs_t = (HS && !isA) ? j / a.spi : 0;  // the lane's tap slot
    const int hs_s = HR ? hs_t % HS : hs_t, hr_r = HR ? hs_t / HS : 0;
    const int jj = (HS && !isA) ? j - hs_t * a.spi : j;
    const int gi = om.mnw ? jj % om.ng : 0, si = om.mnw ? jj / om.ng : jj;
    const int32_t hs_c[5] = {om.coef[0][V_S] * hs_s + om.coef[0][V_R] * hr_r, om.coef[1][V_S] * hs_s + om.coef[1][V_R] * hr_r,
                             om.coef[2][V_S] * hs_s + om.coef[2][V_R] * hr_r, om.coef[3][V_S] * hs_s + om.coef[3][V_R] * hr_r,
                             om.coef[4][V_S] * hs_s + om.coef[4][V_R] * hr_r};
    const uint32_t hs_off = (uint32_t)(hs_t * (BN / CG) * 128);
    // this lane's group: rows [gi * mnw, (gi + 1) * mnw) of the tile
    int g_dn = 0, g_dh = 0, g_dw = 0;
    if (om.mnw && isA) {
      const int r = gi * om.mnw;
      g_dn = r / (a.tile_h * a.tile_w);
      g_dh = (r / a.tile_w) % a.tile_h;
      g_dw = r % a.tile_w;
    } else if (om.mnw) {
      g_dw = gi * om.mnw;
    }
    const uint32_t goff = (uint32_t)(gi * om.gbytes);
    int it = 0, ti = 0;
    for (int tile = unit0; tile < a.num_tiles; tile += unit_step, ti++) {
      const UnitInfo ui = unit_info(a, tile);
      const TileCoord tc = tile_coord<D3>(a, ui.mn, BN, CG, rank);
      const int k_begin = ui.kb, k_end = ui.ke;
      int32_t v[NVAR];
      // B rows of this CTA: its 1/CG share of the unit's BN output channels
      const int pp = isA ? tc.p0 + g_dh : 0, qq = (isA ? tc.q0 : tc.k0 + rank * (BN / CG) + a.b_koff) + g_dw;
      v[V_N0] = isA ? tc.n0 + g_dn : 0;
      v[V_DO] = isA ? tc.d0 : 0;
      v[V_PT] = (int)om.fp.div((uint32_t)pp); v[V_PR] = pp - v[V_PT] * om.divp;
      v[V_QT] = (int)om.fq.div((uint32_t)qq); v[V_QR] = qq - v[V_QT] * om.divq;
      v[V_ONE] = 1;
      if (use_tab) {
        // the tile's part of the box coordinates, once per tile
        int32_t base[5];
        {
          int32_t vt[NVAR];
#pragma unroll
          for (int k = 0; k < NVAR; k++) vt[k] = v[k];
          vt[V_R] = 0; vt[V_S] = 0; vt[V_T] = 0; vt[V_GT] = 0; vt[V_GR] = 0;
          coords<D3>(om, vt, base);
        }
        const uint32_t trow = smem_u32(tab) + (uint32_t)((isA ? 0 : 8) * 4 + si * 64);
        int stage = it % a.nst;
        uint32_t ph = (uint32_t)((it / a.nst) & 1);
        const bool bload = !(a.b_res && ti > 0);  // resident B: loaded with the first tile only
        for (int kit = k_begin; kit < k_end; kit++, it++) {
          if (it >= a.nst) mbar_wait(&empty[stage], ph ^ 1);
          if (lane == 0 && rank == 0) mbar_expect_tx(&full[stage], CG * (a.a_bytes + (bload ? L::kB : 0)));
          __syncwarp();
          if (active && (isA || bload)) {
            const uint32_t ta = trow + (uint32_t)(kit * a.spi * 64);
            int32_t o0, o1, o2, o3, o4;
            asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(o0), "=r"(o1), "=r"(o2), "=r"(o3) : "r"(ta));
            asm volatile("ld.shared.b32 %0, [%1];" : "=r"(o4) : "r"(ta + 16));
            unsigned char *dst = sbase + stage * sbytes + goff + hs_off + si * om.slab_bytes;
            if constexpr (CG == 2)
              tma_load_5d_2cta(dst, tmap, &full[stage], base[0] + o0 + hs_c[0], base[1] + o1 + hs_c[1],
                               base[2] + o2 + hs_c[2], base[3] + o3 + hs_c[3], base[4] + o4 + hs_c[4]);
            else
              tma_load_5d(dst, tmap, &full[stage], base[0] + o0 + hs_c[0], base[1] + o1 + hs_c[1],
                          base[2] + o2 + hs_c[2], base[3] + o3 + hs_c[3], base[4] + o4 + hs_c[4]);
          }
          if (++stage == a.nst) { stage = 0; ph ^= 1u; }
        }
        continue;
      }
      for (int kit = k_begin; kit < k_end; kit++, it++) {
        const int stage = it % a.nst, round = it / a.nst;
        if (lane == 0 && ti == ALT_DBG_TILE && kit == k_begin) { DBG(24); }
        if (round > 0) mbar_wait(&empty[stage], (round - 1) & 1);
        if (lane == 0 && ti == ALT_DBG_TILE && kit == k_begin) { DBG(25); }
        // the leader's full barrier counts the bytes of both CTAs of a pair
        const bool bload = !(a.b_res && ti > 0);
        if (lane == 0 && rank == 0) mbar_expect_tx(&full[stage], CG * (a.a_bytes + (bload ? L::kB : 0)));
        __syncwarp();
        if (active && (isA || bload)) {
          const int slab = kit * a.spi + si;
          const bool valid = slab < a.total_slabs;
          const int sl = valid ? slab : 0;
          int gA, gB;
          slab_decode<D3>(a, sl, v[V_R], v[V_S], v[V_T], gA, gB);
          const int ga = isA ? gA : gB;
          v[V_GT] = (int)om.fg.div((uint32_t)ga); v[V_GR] = ga - v[V_GT] * om.divg;
          int32_t c[5];
          v[V_S] += hs_s;  // halo mode: this lane's tap s (B); 0 otherwise
          v[V_R] += hr_r;  // 2-D halo: this lane's tap r (B)
          coords<D3>(om, v, c);
          if (!valid) c[0] = om.oob0;
          if constexpr (CG == 2)
            tma_load_5d_2cta(sbase + stage * sbytes + goff + hs_off + si * om.slab_bytes, tmap, &full[stage], c[0], c[1],
                             c[2], c[3], c[4]);
          else
            tma_load_5d(sbase + stage * sbytes + goff + hs_off + si * om.slab_bytes, tmap, &full[stage], c[0], c[1], c[2],
                        c[3], c[4]);
        }
      }
    }
    if constexpr (SC > 1) { __syncwarp(); cluster_sync(); cluster_sync(); }  // rings free; partials pushed
  } else if (warp == 1) {
    if (lane == 0 && rank == 0) {
      // ------------------------------------------------------ MMA issuer
      // (the leader CTA issues for the pair: M = 128 * CG)
      // a_major / b_major (bits 15 / 16): MN-major operands
      const uint32_t idesc = idesc_f32acc(1 /*bf16*/, 128 * CG, BN) | (a.A.mnw ? 1u << 15 : 0u) |
                             (a.B.mnw ? 1u << 16 : 0u);
      const int sw = a.sw;
      // descriptors of stage 0's four K=16 steps; stage s adds s * stage bytes
      // to the start-address field (addr >> 4 in bits 0-13, no carry out)
      auto desc = [&](const OperandMap &om, uint32_t base, int kk) -> uint64_t {
        const int kc = kk * 16;
        if (om.mnw == 0) {
          // K-major: slab = sw channels x rows, each row one sw-channel run
          const uint32_t layout = sw == 8 ? 0u : (sw == 16 ? 6u : (sw == 32 ? 4u : 2u));
          const uint32_t sbo = sw == 8 ? 128u : (uint32_t)(8 * sw * 2);
          const uint32_t lbo = sw == 8 ? (uint32_t)om.slab_bytes : 16u;
          return smem_desc(base + (uint32_t)((kc / sw) * om.slab_bytes + (kc % sw) * 2), lbo, sbo, layout);
        }
        // MN-major: K row k of a group at k * mnw * 2 bytes; groups of mnw
        // rows gbytes apart.  Swizzled: LBO = group stride, SBO = 8 K rows;
        // interleaved (mnw = 8): SBO = group stride, LBO = 8 K rows (128 B)
        const uint32_t rowb = (uint32_t)om.mnw * 2;
        const uint32_t addr = base + (uint32_t)kc * rowb;
        if (om.mnw == 8) return smem_desc(addr, 128u, (uint32_t)om.gbytes, 0u);
        const uint32_t layout = om.mnw == 16 ? 6u : (om.mnw == 32 ? 4u : 2u);
        return smem_desc(addr, (uint32_t)om.gbytes, 8u * rowb, layout);
      };
      uint64_t dA[4], dB[4];
#pragma unroll
      for (int kk = 0; kk < 4; kk++) {
        dA[kk] = desc(a.A, smem_u32(sA), kk);
        dB[kk] = desc(a.B, smem_u32(sB), kk);
      }
      int it = 0, i = 0;
      for (int tile = unit0; tile < a.num_tiles; tile += unit_step, i++) {
        const int acc = i % NACC, use = i / NACC;
        if (i == ALT_DBG_TILE) { DBG(26); }
        if (use > 0) mbar_wait(&tempty[acc], (use - 1) & 1);
        if (i == ALT_DBG_TILE) { DBG(27); }
        tc_fence_after();
        const uint32_t d = tmem + (uint32_t)(acc * BN);
        const UnitInfo ui = unit_info(a, tile);
        const int k_begin = ui.kb, k_end = ui.ke;
        int stage = it % a.nst;
        uint32_t ph = (uint32_t)((it / a.nst) & 1);
        for (int kit = k_begin; kit < k_end; kit++, it++) {
          mbar_wait(&full[stage], ph);
          if (i == ALT_DBG_TILE && kit == k_begin) { DBG(28); }
          tc_fence_after();
          // resident B: this k iteration's slabs sit in B slot (kit - k_begin)
          const uint64_t oA = (uint64_t)((stage * L::kAst) >> 4),
                         oB = (uint64_t)(((a.b_res ? kit - k_begin : stage) * L::kB) >> 4);
          if (a.epi_dbg != 3) {  // developer knob 3: the TMA pipeline alone (no MMA, no drain)
#pragma unroll
            for (int ht = 0; ht < (HS ? HS : 1) * (HR ? HR : 1); ht++) {
              // halo: tap s reads A rows shifted by s (128-byte rows: + s * 8
              // in 16-byte units; base-offset field = s when requested); 2-D
              // halo: tap (r, s) reads rows shifted by r tile_w + s (r tile_w
              // rows are whole 1024-byte swizzle atoms)
              const int hs = HR ? ht % HS : ht, hr = HR ? ht / HS : 0;
              const uint64_t sA_off = HS ? (uint64_t)((hr * a.tile_w + hs) * 8) | (a.hboff ? ((uint64_t)hs << 49) : 0ull)
                                         : 0ull;
              const uint64_t sB_off = HS ? (uint64_t)((ht * (BN / CG) * 128) >> 4) : 0ull;
#pragma unroll
              for (int kk = 0; kk < 4; kk++) {
                const uint32_t accum = (kit != k_begin || kk != 0 || ht != 0) ? 1u : 0u;
                if constexpr (CG == 2) mma_bf16_2cta(d, dA[kk] + oA + sA_off, dB[kk] + oB + sB_off, idesc, accum);
                else mma_bf16(d, dA[kk] + oA + sA_off, dB[kk] + oB + sB_off, idesc, accum);
              }
            }
          }
          if constexpr (CG == 2) mma_commit_2cta(&empty[stage], 0x3);  // frees the stage in both CTAs
          else mma_commit(&empty[stage]);
          if (++stage == a.nst) { stage = 0; ph ^= 1u; }
        }
        if constexpr (CG == 2) mma_commit_2cta(&tfull[acc], 0x3);
        else mma_commit(&tfull[acc]);
        if (i == ALT_DBG_TILE) { DBG(29); }
        if (i == 0) { DBG(3); }
      }
    }
    if constexpr (SC > 1) { __syncwarp(); cluster_sync(); cluster_sync(); }  // rings free; partials pushed
  } else {
    // -------------------------------------------------------- epilogue
    // 8 warps: warp w reads TMEM lane quarter (w % 4) (hardware rule) and
    // column half (w - 2) / 4 of every 64-column chunk.
    const int et = threadIdx.x - 64;       // 0..255
    const int wq = warp & 3;
    const int half = (warp - 2) >> 2;      // column part (0 .. kParts - 1)
    const int row = wq * 32 + lane;        // accumulator row = tile row
    const int tn = a.tile_h * a.tile_w;
    const int sw_o = a.out_mode == 1 ? a.O.sw : 32;
    const int pitch = sw_o * 2;            // bytes per row in a staging slab
    const int swz = pitch == 128 ? 3 : (pitch == 64 ? 2 : (pitch == 32 ? 1 : 0));
    // this thread's four 16-byte pieces inside a (swizzled) staging buffer
    auto soff = [&](int c) -> uint32_t {
      const int ch = c * 8;
      uint32_t off = (uint32_t)(lane * pitch + (ch & (sw_o - 1)) * 2);
      off ^= ((off >> 7) & ((1u << swz) - 1u)) << 4;
      return (uint32_t)((ch / sw_o) * 32 * pitch) + off;
    };
    const uint32_t wbuf = smem_u32(sOut) + (uint32_t)((warp - 2) * 4096);
    const int act = a.epi.act;
    // scale / bias of a tile's BN channels, one per thread, fetched one tile
    // ahead into registers and staged in smem (ragged channels clamp)
    auto fetch_sb = [&](int tile, float &fs, float &fb) {
      fs = 1.f; fb = 0.f;
      if (tile < a.num_tiles && et < BN) {
        const int k = min(tile_coord<D3>(a, unit_info(a, tile).mn, BN, CG, rank).k0 + et, a.K - 1);
        fs = __ldg(a.epi.scale + k);
        fb = epi_bias(a.epi, k);
      }
    };
    float pf_s, pf_b;
    fetch_sb(unit0, pf_s, pf_b);
    // this thread's row and its warp's 32-row sub-box origin inside a tile
    // (tile rows are (n, h, w) with w fastest): divisions once per thread
    const int rn = row / tn, rp = (row / a.tile_w) % a.tile_h, rq = row % a.tile_w;
    const int r0 = wq * 32;
    const int sn0 = r0 / tn, sp0 = (r0 / a.tile_w) % a.tile_h, sq0 = r0 % a.tile_w;
    // per-thread constants of the store path (no divisions in the chunk loop)
    uint32_t so[4];
#pragma unroll
    for (int c = 0; c < 4; c++) so[c] = soff(c);
    // round stores: this thread's four 16-byte pieces in a 16 KB round buffer
    // [64 / sw_o slabs][128 rows][sw_o channels], rows swizzled as the store box
    if (a.out_round) {
#pragma unroll
      for (int c = 0; c < 4; c++) {
        const int ch = half * 32 + c * 8;
        uint32_t off = (uint32_t)(row * pitch + (ch & (sw_o - 1)) * 2);
        off ^= ((off >> 7) & ((1u << swz) - 1u)) << 4;
        so[c] = (uint32_t)((ch / sw_o) * 128 * pitch) + off;
      }
    }
    const uint32_t rbase = smem_u32(sOut);
    uint32_t round_ctr = 0;  // round-store buffer parity (across tiles)
    const int lg_sw = sw_o == 64 ? 6 : (sw_o == 32 ? 5 : (sw_o == 16 ? 4 : 3));  // sw_o is 8 .. 64
    const int nslab = 32 >> lg_sw;
    int32_t ocg[5], ocr[5];  // store coordinates per channel slab (tile, in-tile)
    uint32_t sbuf_ctr = 0;   // TMA-store staging buffer parity (per warp, across tiles)
#pragma unroll
    for (int d = 0; d < 5; d++) { ocg[d] = a.O.coef[d][V_GT]; ocr[d] = a.O.coef[d][V_GR]; }
    int i = 0;
    for (int tile = unit0; tile < a.num_tiles; tile += unit_step, i++) {
      const int acc = i % NACC, use = i / NACC;
      const UnitInfo ui = unit_info(a, tile);
      const int mn = ui.mn, ksp = ui.sp;
      const TileCoord tc = tile_coord<D3>(a, mn, BN, CG, rank);
      named_bar(2, kEpiThreads);  // every epilogue warp is done with the previous tile's values
      if (et < BN) {  // explicit shared-space stores (the aligned base is a generic pointer)
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sSB + 4u * et), "f"(pf_s) : "memory");
        asm volatile("st.shared.f32 [%0], %1;" ::"r"(sSB + 4u * (BN + et)), "f"(pf_b) : "memory");
      }
      named_bar(2, kEpiThreads);
      if (et == 0 && i == ALT_DBG_TILE) { DBG(30); }
      fetch_sb(tile + unit_step, pf_s, pf_b);
      const int n = tc.n0 + rn, p = tc.p0 + rp, q = tc.q0 + rq;
      const bool vrow = n < a.N && p < a.Ho && q < a.Wo;
      // the pair's second M tile past the last one (odd M-tile count): its
      // rows alias image n0 >= N, which a GEMM view (no image dim) maps back
      // onto rows 0..127 — such a tile stores nothing
      const bool tile_ok = tc.n0 < a.N;
      // per-warp stores: this warp's 32-row sub-box lies inside the output.
      // When y has a size-1 spatial dim the store view drops it, so a sub-box
      // of rows past Ho (or N) would otherwise land on row 0 (TMA clips only
      // the dims the view keeps)
      const bool sub_ok = tc.n0 + sn0 < a.N && tc.p0 + sp0 < a.Ho && tc.q0 + sq0 < a.Wo;
      // TMA-store coordinates of this warp's 32-row sub-box (tile part),
      // computed while the MMA may still be running
      int32_t cbase[5] = {0, 0, 0, 0, 0};
      if (a.out_mode == 1 && lane == 0) {
        // round stores: the box is the whole tile (origin n0, p0, q0)
        const int sn = tc.n0 + (a.out_round ? 0 : sn0), sp = tc.p0 + (a.out_round ? 0 : sp0),
                  sq = tc.q0 + (a.out_round ? 0 : sq0);
        int32_t vo[NVAR];
        vo[V_N0] = sn;
        vo[V_PT] = (int)a.O.fp.div((uint32_t)sp); vo[V_PR] = sp - vo[V_PT] * a.O.divp;
        vo[V_QT] = (int)a.O.fq.div((uint32_t)sq); vo[V_QR] = sq - vo[V_QT] * a.O.divq;
        vo[V_GT] = 0; vo[V_GR] = 0; vo[V_R] = 0; vo[V_S] = 0; vo[V_ONE] = 1; vo[V_DO] = tc.d0; vo[V_T] = 0;
        coords<D3>(a.O, vo, cbase);
      }
      int64_t yrow = 0;  // out_mode 2: offset of this thread's output row
      if (a.out_mode == 2 && vrow)
        yrow = a.is_conv ? __ldg(a.yr.rd[0] + n) + __ldg(a.yr.rd[2] + p) + __ldg(a.yr.rd[3] + q) : __ldg(a.yr.rd[0] + q);
      // residual rows (res_vec): this thread's 32 channels of a chunk are four
      // 16-byte vectors; chunk 0's are requested before the MMA completes,
      // chunk c + 1's while chunk c is converted
      int64_t rrow = -1;
      if (RV && vrow)
        rrow = a.is_conv ? __ldg(a.epi.res.rd[0] + n) + __ldg(a.epi.res.rd[2] + p) + __ldg(a.epi.res.rd[3] + q)
                         : __ldg(a.epi.res.rd[0] + q);
      uint4 rq[4];
      auto load_res = [&](int cbx) {
        const uint16_t *res = static_cast<const uint16_t *>(a.epi.residual);
#pragma unroll
        for (int c = 0; c < 4; c++) {
          const int k = tc.k0 + cbx + 8 * c;
          rq[c] = make_uint4(0u, 0u, 0u, 0u);
          if (rrow >= 0 && k < a.K)
            rq[c] = __ldg(reinterpret_cast<const uint4 *>(res + rrow + __ldg(a.epi.res.rd[1] + a.y_koff + k)));
        }
      };
      if constexpr (RV) load_res(half * 32);
      mbar_wait(&tfull[acc], use & 1);
      if (et == 0 && i == ALT_DBG_TILE) { DBG(2); }
      tc_fence_after();
      if constexpr (SC > 1) {
        // cluster split-K, phase 1: this CTA's fp32 partial rows are pushed
        // (fire-and-forget DSMEM stores) into the ring of the CTA that
        // finishes them — lane quarter q belongs to split q * SC / 4 — as
        // slice [my split][quarter within the owner][32-column chunk], each
        // 32 rows x 128 B with the 16-byte slots XOR-swizzled by (row & 7);
        // phase 2 then reduces from local shared memory only
        // every CTA's MMAs must be complete (its ring consumed) before any
        // peer writes into it: a cluster barrier after the accumulator is full
        __syncwarp();
        cluster_sync();
        {
          constexpr int NQ = 4 / SC;
          const int my_split = (int)cluster_ctarank();
          const int owner = (wq * SC) / 4, qi = wq - owner * NQ;
#pragma unroll 1
          for (int c0 = 0; c0 < BN; c0 += kStep) {
            const int cb = c0 + half * 32;
            if (cb >= BN) continue;
            uint32_t raw[32];
            tmem_ld_32x32b_x32(tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN + cb), raw);
            tmem_ld_wait();
            const uint32_t slice = (uint32_t)(((my_split * NQ + qi) * (BN / 32) + (cb >> 5)) * 4096);
            uint32_t ra;
            asm("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(smem) + slice + lane * 128), "r"(owner));
#pragma unroll
            for (int j4 = 0; j4 < 8; j4++)
              asm volatile("st.shared::cluster.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(ra + (uint32_t)((j4 ^ (lane & 7)) * 16)),
                           "r"(raw[4 * j4]), "r"(raw[4 * j4 + 1]), "r"(raw[4 * j4 + 2]), "r"(raw[4 * j4 + 3])
                           : "memory");
          }
        }
        if (et == 0) { DBG(36); }
        continue;  // one tile per CTA; phase 2 after the cluster barrier
      }
      const float *wsl = nullptr;  // this CTA tile's partials (split-K)
      int coop_rows = -1;          // cooperative split: 1 = this warp finishes its rows, 0 = another CTA does
      if (SC == 1 && ui.split) {
        const size_t cta_tile = (size_t)(mn - a.full_units) * CG + rank;
        float *wt = a.ws + cta_tile * (size_t)a.splits * (128 * BN);
        float *mine = wt + (size_t)ksp * (128 * BN);
#pragma unroll 1
        for (int c0 = 0; c0 < BN; c0 += kStep) {
          const int cb = c0 + half * 32;
          if (cb >= BN) continue;
          uint32_t raw[32];
          tmem_ld_32x32b_x32(tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN + cb), raw);
          tmem_ld_wait();
          uint4 *dst = reinterpret_cast<uint4 *>(mine) + (size_t)(cb >> 5) * 8 * 128 + row;
#pragma unroll
          for (int j = 0; j < 8; j++)
            __stcg(dst + j * 128, make_uint4(raw[4 * j], raw[4 * j + 1], raw[4 * j + 2], raw[4 * j + 3]));
        }
        __threadfence();
        if (et == 0 && i == ALT_DBG_TILE) { DBG(4); }
        named_bar(1, kEpiThreads);
        if (a.coop) {
          // every piece of the tile is resident (planner-checked): wait for all
          // partials, release the accumulator, then finish the rows of the
          // lane quarters this split owns (quarter q -> split q * splits / 4)
          if (et == 0) {
            atomicAdd(a.cnt + cta_tile, 1);
            int seen = 0;
            do {
              asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(seen) : "l"(a.cnt + cta_tile) : "memory");
              if (seen < a.splits) __nanosleep(64);
            } while (seen < a.splits);
          }
          named_bar(1, kEpiThreads);
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            if constexpr (CG == 2) mbar_arrive_cluster(&tempty[acc], 0);
            else mbar_arrive(&tempty[acc]);
          }
          coop_rows = (wq * a.splits) / 4 == ksp;
          wsl = wt;
        } else {
        if (et == 0) *last_flag = atomicAdd(a.cnt + cta_tile, 1) == a.splits - 1;
        named_bar(1, kEpiThreads);
        if (et == 0 && i == ALT_DBG_TILE) { DBG(7); }
        if (!*last_flag) {  // another CTA finishes this tile: free the accumulator
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            if constexpr (CG == 2) mbar_arrive_cluster(&tempty[acc], 0);
            else mbar_arrive(&tempty[acc]);
          }
          continue;
        }
        __threadfence();
        if (et == 0) a.cnt[cta_tile] = 0;  // ready for the next launch
        wsl = wt;
        }
      }
      // TMEM reads are software-pipelined (TMEM read is 32 B/clk per SM):
      // on the plain path (TMA-store output, no residual, no split) chunk
      // c + 1's load is issued as soon as chunk c's values are consumed, so
      // it overlaps chunk c's conversion and store.  That variant makes no
      // function calls while a load is in flight (a call would save / restore
      // the registers the asynchronous load is writing); the other variant
      // issues the next load at the end of the chunk.
      if (a.epi_dbg == 2 || a.epi_dbg == 3) {
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if constexpr (CG == 2) mbar_arrive_cluster(&tempty[acc], 0);
          else mbar_arrive(&tempty[acc]);
        }
        continue;
      }
      auto chunk_loop = [&](auto early_tag, auto res_tag) {
        constexpr bool EARLY = decltype(early_tag)::value;
        constexpr bool RESV = decltype(res_tag)::value;  // 16-byte residual vectors
        if (coop_rows == 0) return;  // cooperative split: another CTA finishes these rows
        if (half * 32 >= BN) {  // this warp's column part is past BLOCK_N: nothing to drain
          if (coop_rows >= 0) return;  // accumulator already released
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {
            if constexpr (CG == 2) mbar_arrive_cluster(&tempty[acc], 0);
            else mbar_arrive(&tempty[acc]);
          }
          return;
        }
        uint32_t raw[32];
        tmem_ld_32x32b_x32(tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN + half * 32), raw);
#pragma unroll 1
        for (int c0 = 0; c0 < BN; c0 += kStep) {
          const int cb = c0 + half * 32;     // first column of this thread's 32
          const int kb = tc.k0 + cb;
          const uint32_t next = tmem + ((uint32_t)(wq * 32) << 16) + (uint32_t)(acc * BN + cb + kStep);
          tmem_ld_wait();
#pragma unroll
          for (int j = 0; j < 32; j++) asm volatile("" : "+r"(raw[j]));  // uses stay after the wait
          if (et == 0 && i == ALT_DBG_TILE) { DBG(8 + (c0 / kStep) * 4); }
          if constexpr (!EARLY) {
            if (wsl) {
              float tot[32];
              split_total(wsl, a.splits, coop_rows >= 0 ? -1 : ksp, BN, cb, row, raw, tot);
#pragma unroll
              for (int j = 0; j < 32; j++) raw[j] = __float_as_uint(tot[j]);
            }
          }
          float v[32];
          {
#pragma unroll
            for (int j = 0; j < 8; j++) {
              float4 x, y;
              asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                           : "=f"(x.x), "=f"(x.y), "=f"(x.z), "=f"(x.w)
                           : "r"(sSB + 4u * (cb + 4 * j)));
              asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                           : "=f"(y.x), "=f"(y.y), "=f"(y.z), "=f"(y.w)
                           : "r"(sSB + 4u * (BN + cb + 4 * j)));
              v[4 * j + 0] = fmaf(__uint_as_float(raw[4 * j + 0]), x.x, y.x);
              v[4 * j + 1] = fmaf(__uint_as_float(raw[4 * j + 1]), x.y, y.y);
              v[4 * j + 2] = fmaf(__uint_as_float(raw[4 * j + 2]), x.z, y.z);
              v[4 * j + 3] = fmaf(__uint_as_float(raw[4 * j + 3]), x.w, y.w);
            }
          }
          if constexpr (RESV) {
#pragma unroll
            for (int c = 0; c < 4; c++) {
              const uint32_t w4[4] = {rq[c].x, rq[c].y, rq[c].z, rq[c].w};
#pragma unroll
              for (int h = 0; h < 4; h++) {
                v[8 * c + 2 * h] += __uint_as_float(w4[h] << 16);
                v[8 * c + 2 * h + 1] += __uint_as_float(w4[h] & 0xffff0000u);
              }
            }
            if (c0 + kStep < BN) load_res(cb + kStep);
          }
          if constexpr (EARLY) {
            if (c0 + kStep < BN) tmem_ld_32x32b_x32(next, raw);
          }
          if (c0 + kStep >= BN && coop_rows < 0) {  // accumulator buffer drained: MMA may reuse it
            tc_fence_before();
            __syncwarp();
            if (lane == 0) {
              if constexpr (CG == 2) mbar_arrive_cluster(&tempty[acc], 0);  // the leader's MMA waits
              else mbar_arrive(&tempty[acc]);
            }
          }
          if constexpr (!EARLY) {
            if (!RV && a.epi.residual && vrow) {
              float rv[32];  // local memory, touched only when a residual exists
              if (a.out_f32) residual_chunk_f32(a.epi, a.is_conv, a.K, n, p, q, kb, a.y_koff, rv);
              else residual_chunk(a.epi, a.is_conv, a.K, n, p, q, kb, a.y_koff, rv);
#pragma unroll
              for (int j = 0; j < 32; j++) v[j] += rv[j];
            }
            if (a.out_f32) {  // fp32 result (split-operand path): act, store
#pragma unroll
              for (int j = 0; j < 32; j++) v[j] = act == 1 ? fmaxf(v[j], 0.f) : (act == 2 ? fminf(fmaxf(v[j], 0.f), 6.f) : v[j]);
              if (vrow) store_chunk_f32(a, reinterpret_cast<float *>(y), yrow, n, p, q, kb, v);
              if (c0 + kStep < BN) tmem_ld_32x32b_x32(next, raw);
              continue;
            }
          }
          // activation folded into the bf16 conversion (cvt .relu)
          uint32_t pk[16];
          if (act == 1) {
#pragma unroll
            for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2_relu(v[2 * j], v[2 * j + 1]);
          } else if (act == 2) {
#pragma unroll
            for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2_relu(fminf(v[2 * j], 6.f), fminf(v[2 * j + 1], 6.f));
          } else {
#pragma unroll
            for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2(v[2 * j], v[2 * j + 1]);
          }
          if (et == 0 && i == ALT_DBG_TILE) { DBG(9 + (c0 / kStep) * 4); }
          if (a.epi_dbg == 1) {
            if (pk[0] == 0x7fff1234u) y[0] = 0;  // keep the values live
          } else if (a.out_mode == 2) {
            // direct 16-byte stores: 8 channels are contiguous in y
            if (vrow) {
#pragma unroll
              for (int c = 0; c < 4; c++) {
                const int k = kb + 8 * c;
                if (k < a.K) {
                  uint16_t *dst = y + yrow + __ldg(a.yr.rd[1] + a.y_koff + k);
                  asm volatile("st.global.v4.b32 [%0], {%1, %2, %3, %4};" ::"l"(dst), "r"(pk[4 * c]),
                               "r"(pk[4 * c + 1]), "r"(pk[4 * c + 2]), "r"(pk[4 * c + 3])
                               : "memory");
                }
              }
            }
          } else if (a.out_mode == 1 && a.out_round) {
            // Round store: every epilogue warp writes its 32 x 32 piece of the
            // round's 128 x 64 block into one of two 16 KB buffers; thread 0
            // then stores the block with one TMA store per channel slab.
            // Buffer reuse: thread 0 waits (before the "free" barrier) until
            // the store issued two rounds ago has read its buffer.
            const uint32_t rbuf = rbase + (uint32_t)(round_ctr++ & 1u) * 16384u;
            if (et == 0) bulk_wait_read1();
            named_bar(3, kEpiThreads);
#pragma unroll
            for (int c = 0; c < 4; c++)
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(rbuf + so[c]), "r"(pk[4 * c]),
                           "r"(pk[4 * c + 1]), "r"(pk[4 * c + 2]), "r"(pk[4 * c + 3])
                           : "memory");
            fence_async_smem();
            named_bar(4, kEpiThreads);
            if (et == 0) {
              const int kr = tc.k0 + c0;  // the round's first channel
              for (int j = 0; j < (64 >> lg_sw) && tile_ok; j++) {
                if (kr + (j << lg_sw) >= a.K) break;
                const int g = ((kr + a.y_koff) >> lg_sw) + j;
                const int gt = (int)a.O.fg.div((uint32_t)g), gr = g - gt * a.O.divg;
                int32_t co[5];
#pragma unroll
                for (int d = 0; d < 5; d++) co[d] = cbase[d] + ocg[d] * gt + ocr[d] * gr;
                asm volatile(
                    "cp.async.bulk.tensor.5d.global.shared::cta.tile.bulk_group [%0, {%2, %3, %4, %5, %6}], [%1];" ::"l"(
                        reinterpret_cast<uint64_t>(&tmY)),
                    "r"(rbuf + (uint32_t)(j * 128 * pitch)), "r"(co[0]), "r"(co[1]), "r"(co[2]), "r"(co[3]), "r"(co[4])
                    : "memory");
              }
              bulk_commit();
            }
          } else if (a.out_mode == 1) {
            // Each warp stores its own 32-row x 32-channel sub-tile: private
            // double-buffered staging, swizzled rows, one TMA store per slab;
            // no CTA-wide barrier.  Buffer `buf` is free once the store issued
            // two chunks ago has read it (<= 1 store group in flight per warp).
            // alternate the two buffers across every chunk this warp stores
            // (not per tile: with BLOCK_N 64 a tile is one chunk, and the
            // previous tile's store may still be reading the other buffer)
            const uint32_t buf = (uint32_t)(sbuf_ctr++ & 1u) * 2048u;
            if (lane == 0) bulk_wait_read1();
            __syncwarp();
#pragma unroll
            for (int c = 0; c < 4; c++)
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(wbuf + buf + so[c]), "r"(pk[4 * c]),
                           "r"(pk[4 * c + 1]), "r"(pk[4 * c + 2]), "r"(pk[4 * c + 3])
                           : "memory");
            if (et == 0 && i == ALT_DBG_TILE) { DBG(10 + (c0 / kStep) * 4); }
            fence_async_smem();
            __syncwarp();
            if (lane == 0) {
              for (int j = 0; j < nslab && tile_ok && sub_ok; j++) {
                if (kb + (j << lg_sw) >= a.K) break;  // channels past K: nothing to store
                const int g = ((kb + a.y_koff) >> lg_sw) + j;
                const int gt = (int)a.O.fg.div((uint32_t)g), gr = g - gt * a.O.divg;
                int32_t co[5];
#pragma unroll
                for (int d = 0; d < 5; d++) co[d] = cbase[d] + ocg[d] * gt + ocr[d] * gr;
                tma_store_5d(&tmY, sOut + (warp - 2) * 4096 + buf + j * (32 << (lg_sw + 1)), co[0], co[1], co[2], co[3],
                             co[4]);
              }
              bulk_commit();
              if (et == 0 && i == ALT_DBG_TILE) { DBG(11 + (c0 / kStep) * 4); }
            }
          } else if constexpr (!EARLY) {
            // generic layouts: every copy / pad position through the writer
            if (vrow) {
              if (a.yvec) write_chunk_vec(a, y, n, p, q, kb, pk);
              else write_chunk(a.yw, a.is_conv, a.K, y, n, p, q, kb, a.y_koff, pk);
            }
          }
          if constexpr (!EARLY) {
            if (c0 + kStep < BN) tmem_ld_32x32b_x32(next, raw);
          }
        }
      };
      if constexpr (RV) {
        if (a.out_mode != 0 && !wsl) chunk_loop(std::true_type{}, std::true_type{});
        else chunk_loop(std::false_type{}, std::true_type{});
      } else {
        if (a.out_mode != 0 && !a.epi.residual && !wsl && !a.out_f32) chunk_loop(std::true_type{}, std::false_type{});
        else chunk_loop(std::false_type{}, std::false_type{});
      }
      if (coop_rows >= 0) {
        // cooperative split: the last CTA of the tile to finish resets the
        // counters for the next launch (every CTA is past its wait by then)
        named_bar(1, kEpiThreads);
        if (et == 0) {
          const size_t cta_tile = (size_t)(mn - a.full_units) * CG + rank;
          if (atomicAdd(a.done + cta_tile, 1) == a.splits - 1) {
            a.cnt[cta_tile] = 0;
            a.done[cta_tile] = 0;
          }
        }
      }
      if (et == 0 && i == ALT_DBG_TILE) { DBG(31); }
    }
    if constexpr (SC > 1) {
      // cluster split-K, phase 2 (out_mode 1): CTA `crank` owns TMEM lane
      // quarters [crank * 4 / SC, (crank + 1) * 4 / SC) of the tile; work item
      // = (quarter, 32-column chunk), one per warp at a time; the SC partials
      // are read through DSMEM and summed in split order
      __syncwarp();
      cluster_sync();
      if (et == 0) { DBG(37); }
      const int crank = (int)cluster_ctarank();
      const TileCoord tc = tile_coord<D3>(a, unit_info(a, unit0).mn, BN, CG, rank);
      constexpr int NQ = 4 / SC, NCH = BN / 32;
      const int ew = warp - 2;
      int cnt = 0;
      for (int item = ew; item < NQ * NCH; item += kEpiWarps, cnt++) {
        const int qq = crank * NQ + item / NCH, ch = item % NCH;
        const int cb = ch * 32, kb = tc.k0 + cb;
        float t[32];
#pragma unroll
        for (int j = 0; j < 32; j++) t[j] = 0.f;
        // the SC slices of these rows were pushed here in phase 1: local reads
        const int qi = qq - crank * NQ;
#pragma unroll
        for (int sp2 = 0; sp2 < SC; sp2++) {
          const uint32_t ra = smem_u32(smem) + (uint32_t)(((sp2 * NQ + qi) * NCH + ch) * 4096 + lane * 128);
          float4 f[8];
#pragma unroll
          for (int j4 = 0; j4 < 8; j4++)
            asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                         : "=f"(f[j4].x), "=f"(f[j4].y), "=f"(f[j4].z), "=f"(f[j4].w)
                         : "r"(ra + (uint32_t)((j4 ^ (lane & 7)) * 16)));
#pragma unroll
          for (int j4 = 0; j4 < 8; j4++) {
            t[4 * j4] += f[j4].x; t[4 * j4 + 1] += f[j4].y; t[4 * j4 + 2] += f[j4].z; t[4 * j4 + 3] += f[j4].w;
          }
        }
        if (et == 0 && cnt == 0) { DBG(38); }
        float v[32];
#pragma unroll
        for (int j = 0; j < 8; j++) {
          float4 x, yb;
          asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                       : "=f"(x.x), "=f"(x.y), "=f"(x.z), "=f"(x.w) : "r"(sSB + 4u * (cb + 4 * j)));
          asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                       : "=f"(yb.x), "=f"(yb.y), "=f"(yb.z), "=f"(yb.w) : "r"(sSB + 4u * (BN + cb + 4 * j)));
          v[4 * j + 0] = fmaf(t[4 * j + 0], x.x, yb.x);
          v[4 * j + 1] = fmaf(t[4 * j + 1], x.y, yb.y);
          v[4 * j + 2] = fmaf(t[4 * j + 2], x.z, yb.z);
          v[4 * j + 3] = fmaf(t[4 * j + 3], x.w, yb.w);
        }
        uint32_t pk[16];
        if (act == 1) {
#pragma unroll
          for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2_relu(v[2 * j], v[2 * j + 1]);
        } else if (act == 2) {
#pragma unroll
          for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2_relu(fminf(v[2 * j], 6.f), fminf(v[2 * j + 1], 6.f));
        } else {
#pragma unroll
          for (int j = 0; j < 16; j++) pk[j] = pack_bf16x2(v[2 * j], v[2 * j + 1]);
        }
        const uint32_t buf = (uint32_t)(sbuf_ctr++ & 1u) * 2048u;
        if (lane == 0) bulk_wait_read1();
        __syncwarp();
#pragma unroll
        for (int c = 0; c < 4; c++)
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(wbuf + buf + so[c]), "r"(pk[4 * c]),
                       "r"(pk[4 * c + 1]), "r"(pk[4 * c + 2]), "r"(pk[4 * c + 3])
                       : "memory");
        fence_async_smem();
        __syncwarp();
        if (lane == 0) {
          // store coordinates of this quarter's 32-row sub-box
          const int r0 = qq * 32;
          const int sn = tc.n0 + r0 / tn, spp = tc.p0 + (r0 / a.tile_w) % a.tile_h, sq = tc.q0 + r0 % a.tile_w;
          int32_t vo[NVAR], cbq[5];
          vo[V_N0] = sn;
          vo[V_PT] = (int)a.O.fp.div((uint32_t)spp); vo[V_PR] = spp - vo[V_PT] * a.O.divp;
          vo[V_QT] = (int)a.O.fq.div((uint32_t)sq); vo[V_QR] = sq - vo[V_QT] * a.O.divq;
          vo[V_GT] = 0; vo[V_GR] = 0; vo[V_R] = 0; vo[V_S] = 0; vo[V_ONE] = 1; vo[V_DO] = tc.d0; vo[V_T] = 0;
          coords<D3>(a.O, vo, cbq);
          const bool q_ok = sn < a.N && spp < a.Ho && sq < a.Wo;  // as sub_ok above
          for (int j = 0; j < nslab && q_ok; j++) {
            if (kb + (j << lg_sw) >= a.K) break;
            const int g = ((kb + a.y_koff) >> lg_sw) + j;
            const int gt = (int)a.O.fg.div((uint32_t)g), gr = g - gt * a.O.divg;
            int32_t co[5];
#pragma unroll
            for (int d = 0; d < 5; d++) co[d] = cbq[d] + ocg[d] * gt + ocr[d] * gr;
            tma_store_5d(&tmY, sOut + (warp - 2) * 4096 + buf + j * (32 << (lg_sw + 1)), co[0], co[1], co[2], co[3],
                         co[4]);
          }
          bulk_commit();
        }
        if (et == 0 && cnt == 0) { DBG(39); }
      }
    }
    if (et == 0) { DBG(5); }
    if (lane == 0 && a.out_mode == 1) bulk_wait_read0();  // smem reads done; the global writes complete with the grid
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2 || SC > 1) cluster_sync();  // the pair's MMAs / the peers' DSMEM reads are done
  if (warp == 1) tmem_dealloc<tmem_cols(NACC * BN), CG>(tmem);
  if (threadIdx.x == 32) { DBG(6); }
}

// =========================================================== host planner ==
enum Role { R_NONE = 0, R_N, R_H, R_W, R_C, R_TR, R_TS, R_D, R_TT };  // R_D / R_TT: C3D depth / depth tap

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

// The part of a compiled layout a TMA view needs: physical extents / strides
// and the affine map i_d = sum_p coef_p j_p + off_d (separable layouts).
// Physical dims of extent 1 are ignored, which is how fold_window() below
// drops a dim it merged into another.
struct LView {
  bool ok = false;
  int lrank = 0, prank = 0;
  int64_t pshape[kMaxP] = {}, pstride[kMaxP] = {}, coef[kMaxP] = {};
  int32_t owner[kMaxP] = {};
  int64_t off[kMaxL] = {};
  int64_t lext[kMaxL] = {};  // logical extents
};

static LView lview(const Layout &L) {
  LView v;
  v.ok = L.separable && L.aff.ok;
  v.lrank = L.lrank;
  v.prank = L.prank;
  for (int p = 0; p < L.prank; p++) {
    v.pshape[p] = L.pshape[p];
    v.pstride[p] = L.pstride[p];
    v.coef[p] = L.aff.coef[p];
    v.owner[p] = L.pdim_owner[p];
  }
  for (int d = 0; d < L.lrank; d++) {
    v.off[d] = L.aff.off[d];
    v.lext[d] = L.lshape[d];
  }
  return v;
}

// Window folding (unfold with one conv window per layout tile):
// when x's W dim is unfold(B = E >= S, step = conv stride) of the conv-padded
// row, stored [.. Wt][Wi][C] with the channel run innermost, the (Wi, C)
// pair is one contiguous run of E*C elements per output column — the whole
// filter row's reduction.  With the weights stored [.. S'][C] (S padded to E)
// the conv is the same sum as a conv with S = 1, stride 1, no W padding and
// E*C channels: x'(n, s*C + c, h, q) = x(n, c, h, V q + s - pad).  This turns
// a few-channel layer (conv1, C = 3) into 64-element K rows instead of
// 16-byte slabs per tap.
static bool fold_window(const LView &x, const LView &w, int64_t S, int Vw, int pw, int64_t Wo, LView *xo,
                        LView *wo, int64_t *Cfold) {
  if (!x.ok || !w.ok || x.lrank != 4 || w.lrank != 4) return false;
  int xw[kMaxP], nxw = 0, xc = -1, nxc = 0, ws = -1, nws = 0, wc = -1, nwc = 0;
  for (int p = 0; p < x.prank; p++) {
    if (x.pshape[p] == 1) continue;
    if (x.owner[p] == 3) xw[nxw++] = p;
    if (x.owner[p] == 1) { xc = p; nxc++; }
  }
  for (int p = 0; p < w.prank; p++) {
    if (w.pshape[p] == 1) continue;
    if (w.owner[p] == 3) { ws = p; nws++; }
    if (w.owner[p] == 1) { wc = p; nwc++; }
  }
  if (nxw != 2 || nxc != 1 || nws != 1 || nwc != 1) return false;
  // Wi = the inner of the two (stride 1 unfolds give both coefficient 1)
  const int wi = x.pstride[xw[0]] < x.pstride[xw[1]] ? xw[0] : xw[1], wt = wi == xw[0] ? xw[1] : xw[0];
  if (x.coef[wi] != 1 || x.coef[wt] != Vw || x.off[3] != -pw || x.pshape[wt] < Wo) return false;
  const int64_t E = x.pshape[wi], C = x.pshape[xc];
  if (E < S || x.pstride[xc] != 1 || x.coef[xc] != 1 || x.off[1] != 0 || x.pstride[wi] != C) return false;
  if (w.pshape[ws] != E || w.coef[ws] != 1 || w.off[3] != 0 || w.pstride[ws] != C) return false;
  if (w.pshape[wc] != C || w.pstride[wc] != 1 || w.coef[wc] != 1 || w.off[1] != 0) return false;
  *xo = x;
  *wo = w;
  xo->pshape[xc] = E * C;
  xo->pshape[wi] = 1;
  xo->coef[wt] = 1;
  xo->off[3] = 0;
  wo->pshape[wc] = E * C;
  wo->pshape[ws] = 1;
  *Cfold = E * C;
  return true;
}

// Cut a TMA view out of a compiled layout: per logical dim a role (rows n/h/w,
// channel c, filter taps r/s).  Requires the layout's affine map (split /
// reorder / pad / unfold sequences); see DESIGN.md §5.
// mnw > 0 builds an MN-major view: the R_W role's in-tile dim must be the
// stride-1 dim (box = mnw, the caller sets that role's tile to mnw and the
// other row roles' tiles to 1: one box per group of mnw rows), the channel
// dim is an ordinary box dim of sw channels.
// clip: an output view of a padded layout (ALT_EPI_PADS_ZERO stores): each
// spatial dim's extent ends at the last element row, so TMA drops the rows
// of a tile past Ho / Wo instead of writing them into the hi pad
static bool build_view(const LView &L, const RoleInfo *roles, int sw, View *out, char *why, int mnw = 0,
                       bool clip = false) {
  auto fail = [&](const char *m) { snprintf(why, 160, "%s", m); return false; };
  if (!L.ok) return fail("layout not separable-affine");
  View v;
  int nphys[kMaxL] = {};
  int plist[kMaxL][kMaxP];
  for (int p = 0; p < L.prank; p++) {
    if (L.pshape[p] == 1) continue;
    const int d = L.owner[p];
    plist[d][nphys[d]++] = p;
  }
  for (int d = 0; d < L.lrank; d++) {
    const RoleInfo &ri = roles[d];
    const int64_t off = L.off[d];
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
          if (L.coef[p] == 1) plo = p; else phi = p;
        }
        if (plo < 0 || (!mnw && L.pstride[plo] != 1)) return fail("channel tile is not the innermost (stride-1) dim");
        const int64_t xlo = L.pshape[plo];
        if (xlo % sw) return fail("slab width does not divide channel tile");
        if (phi >= 0 && L.coef[phi] != xlo) return fail("channel digits not a plain split");
        v.xlo = xlo;
        v.divg = (int)(xlo / sw);
        VDim &lo = add(plo, sw, 1, mnw ? 5 : 0);
        lo.coef[V_GR] = sw;
        if (phi >= 0) {
          VDim &hi = add(phi, 1, 1, 100);
          hi.coef[V_GT] = 1;
        }
        break;
      }
      case R_N: {
        if (nphys[d] == 0) { if (ri.tile != 1) return fail("tile_n > 1 on a size-1 dim"); break; }
        if (nphys[d] != 1 || L.coef[plist[d][0]] != 1 || off != 0) return fail("batch dim must be plain");
        VDim &x = add(plist[d][0], ri.tile, 1, 50);
        x.coef[V_N0] = 1;
        break;
      }
      case R_TR:
      case R_TS:
      case R_TT: {
        if (nphys[d] == 0) break;
        if (nphys[d] != 1 || L.coef[plist[d][0]] != 1 || off != 0) return fail("filter tap dim must be plain");
        VDim &x = add(plist[d][0], 1, 1, 100);
        x.coef[ri.role == R_TR ? V_R : (ri.role == R_TS ? V_S : V_T)] = 1;
        break;
      }
      case R_D: {
        // C3D depth (box 1): input coordinate od Vd - pd + dd t (+ the
        // layout's own pad offset), output coordinate od; plain dim only
        if (nphys[d] == 0) { if (ri.V != 1 || ri.win != 1) return fail("depth window on a size-1 dim"); break; }
        if (nphys[d] != 1 || L.coef[plist[d][0]] != 1) return fail("depth dim must be plain (no split / unfold)");
        VDim &x = add(plist[d][0], 1, 1, 100);
        x.coef[V_DO] = ri.V;
        x.coef[V_T] = ri.tap;
        x.coef[V_ONE] = (int32_t)(-ri.pad - off);
        break;
      }
      case R_H:
      case R_W: {
        const bool isH = ri.role == R_H;
        const int VT = isH ? V_PT : V_QT, VR = isH ? V_PR : V_QR, VTAP = isH ? V_R : V_S;
        // MN-major: the W role's in-tile dim is the innermost box dim
        const int base_order = isH ? 20 : (mnw ? 0 : 10);
        if (mnw && !isH && ri.V != 1) return fail("MN-major operand with a strided M dim");
        // a box's start along the stride-1 dim must stay 16-byte aligned (a
        // filter tap / padding shift of the MN run traps in TMA): MN-major
        // activations take 1x1 unpadded convs (and GEMM rows) only
        if (mnw && !isH && (ri.win != 1 || ri.pad != 0 || off != 0))
          return fail("MN-major operand with filter taps / padding along its stride-1 dim");
        int &div = isH ? v.divp : v.divq;
        if (nphys[d] == 0) {
          if (ri.tile != 1 || ri.win != 1) return fail("tile > 1 on a size-1 spatial dim");
          break;
        }
        if (nphys[d] == 1) {
          const int p = plist[d][0];
          if (L.coef[p] != 1) return fail("spatial dim coefficient != 1");
          const int box = ri.tile * ri.V;
          if (box > 256) return fail("box > 256");
          VDim &x = add(p, box, ri.V, base_order);
          x.coef[VR] = ri.V;
          x.coef[VTAP] = ri.tap;
          x.coef[V_ONE] = (int32_t)(-ri.pad - off);
          if (clip) x.extent = std::min<int64_t>(x.extent, L.lext[d] - off);
          break;
        }
        if (nphys[d] != 2) return fail("spatial dim with >2 physical dims");
        int plo = -1, phi = -1;
        for (int i = 0; i < 2; i++) {
          const int p = plist[d][i], o = plist[d][1 - i];
          // the in-tile digit: coefficient 1, and the inner one when both are 1
          if (L.coef[p] == 1 && (L.coef[o] != 1 || L.pstride[p] < L.pstride[o])) plo = p; else phi = p;
        }
        if (plo < 0 || phi < 0) return fail("spatial digits without unit coefficient");
        const int64_t Elo = L.pshape[plo], ch = L.coef[phi];
        if (ch == Elo) {
          // plain split (GEMM-like): no window, no stride, no padding
          if (ri.V != 1 || ri.win != 1 || ri.pad != 0 || off != 0) return fail("split spatial dim with window/stride");
          if (mnw && !isH && ri.tile > Elo) return fail("MN-major group wider than the inner M tile");
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
          // unfold (overlapped tiles): the M tile must sit inside one
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
  if (mnw) {  // the group's mnw rows must be the stride-1 dim
    bool ok = false;
    for (int i = 0; i < v.rank; i++)
      if (v.d[i].order == 0 && v.d[i].stride == 1 && v.d[i].box == mnw && v.d[i].estride == 1) ok = true;
    if (!ok) return fail("MN-major: the M tile's run is not the stride-1 dim");
  }
  // order: dim 0 = channel run, then box>1 dims inner->outer, then box-1
  std::stable_sort(v.d, v.d + v.rank, [](const VDim &x, const VDim &y) { return x.order < y.order; });
  // merge box-1 dims adjacent in memory until rank <= 5
  while (v.rank > 5) {
    bool merged = false;
    for (int i = 1; i < v.rank && !merged; i++) {
      for (int j = 1; j < v.rank && !merged; j++) {
        if (i == j || v.d[i].box != 1 || v.d[j].box != 1) continue;
        if (v.d[i].stride != v.d[j].stride * v.d[j].extent) continue;  // i outer, j inner
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

// sw: channels per slab; the swizzle follows the innermost box dim (sw for a
// K-major view, the group width mnw for an MN-major one)
static bool encode_view(const View &v, const void *base, int esize, int sw, CUtensorMap *tm, OperandMap *om,
                        char *why, int mnw = 0) {
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
  const int row_bytes = (mnw ? mnw : sw) * esize;
  CUtensorMapSwizzle swz = row_bytes == 16 ? CU_TENSOR_MAP_SWIZZLE_NONE
                           : row_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B
                           : row_bytes == 64 ? CU_TENSOR_MAP_SWIZZLE_64B
                                             : CU_TENSOR_MAP_SWIZZLE_128B;
  auto enc = get_encode();
  if (!enc) { snprintf(why, 160, "cuTensorMapEncodeTiled unavailable"); return false; }
  static const CUtensorMapL2promotion promo = [] {
    const char *e = getenv("ALT_TMA_L2PROMO");  // developer A/B knob: 0 none, 64, 128, 256 (default)
    const int v = e ? atoi(e) : 256;
    return v == 0 ? CU_TENSOR_MAP_L2_PROMOTION_NONE
                  : v == 64 ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                            : v == 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  }();
  CUresult r = enc(tm, esize == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 5,
                   const_cast<void *>(base), dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz, promo,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) { snprintf(why, 160, "cuTensorMapEncodeTiled failed (%d)", (int)r); return false; }
  memset(om, 0, sizeof(*om));
  for (int i = 0; i < 5; i++)
    for (int k = 0; k < NVAR; k++) om->coef[i][k] = i < v.rank ? v.d[i].coef[k] : 0;
  om->divp = v.divp;
  om->divq = v.divq;
  om->divg = v.divg;
  om->fp = FastDiv((uint32_t)v.divp);
  om->fq = FastDiv((uint32_t)v.divq);
  om->fg = FastDiv((uint32_t)v.divg);
  int64_t rows = 1;
  for (int i = 1; i < v.rank; i++) rows *= (int64_t)((v.d[i].box + v.d[i].estride - 1) / v.d[i].estride);
  om->slab_bytes = (int32_t)(rows * row_bytes);
  om->oob0 = (int32_t)v.d[0].extent;
  om->sw = sw;
  om->mnw = mnw;
  om->ng = 1;
  om->gbytes = 0;
  return true;
}

alt_status make_reader(Layout *L, Reader *r);
alt_status make_writer(Layout *L, Writer *w);

// out_mode 2 needs every 8-channel group contiguous and 16-byte aligned:
// the output-channel dim (logical 1) innermost with a run that 8 divides,
// every other stride a multiple of 8 elements
static bool direct_store_ok(const LView &L) {
  if (!L.ok || L.lrank < 2) return false;
  int pc = -1;
  for (int p = 0; p < L.prank; p++) {
    if (L.pshape[p] == 1) continue;
    if (L.owner[p] == 1 && L.coef[p] == 1) pc = p;
  }
  if (pc < 0 || L.pstride[pc] != 1 || L.pshape[pc] % 8 || L.off[1] != 0) return false;
  for (int p = 0; p < L.prank; p++)
    if (p != pc && L.pshape[p] > 1 && L.pstride[p] % 8) return false;
  return true;
}
alt_status make_epi(const OpEpilogue &e, EpiParams *p);

// ---- optional per-CTA timestamps (env ALT_TC_DEBUG=1; developer tool)
static uint64_t *debug_buffer() {
  static uint64_t *buf = nullptr;
  static bool init = false;
  if (!init) {
    init = true;
    const char *e = getenv("ALT_TC_DEBUG");
    if (e && e[0] == '1' && cudaMalloc(&buf, (size_t)40 * 8 << 20) != cudaSuccess) buf = nullptr;
  }
  return buf;
}

}  // namespace alt
extern "C" int alt__debug_tc(uint64_t *host, int64_t n) {
  uint64_t *b = alt::debug_buffer();
  if (!b) return -1;
  return cudaMemcpy(host, b, (size_t)n * 8, cudaMemcpyDeviceToHost) == cudaSuccess ? 0 : -1;
}
namespace alt {

// per-device ones / zeros vectors (never freed: process lifetime)
alt_status identity_vectors(int64_t K, const float **ones, const float **zeros) {
  static std::mutex mu;
  struct Buf { int dev; int64_t cap; float *ones, *zeros; };
  static std::vector<Buf> bufs;
  int dev = 0;
  cudaGetDevice(&dev);
  std::lock_guard<std::mutex> g(mu);
  for (auto &b : bufs) {
    if (b.dev == dev && b.cap >= K) { *ones = b.ones; *zeros = b.zeros; return ALT_OK; }
  }
  const int64_t cap = std::max<int64_t>(K, 4096);
  std::vector<float> h1(cap, 1.f);
  float *d1 = nullptr, *d0 = nullptr;
  if (cudaMalloc(&d1, cap * 4) != cudaSuccess || cudaMalloc(&d0, cap * 4) != cudaSuccess) {
    cudaGetLastError();
    set_error("identity epilogue buffers: out of memory");
    return ALT_E_NOMEM;
  }
  cudaMemcpy(d1, h1.data(), cap * 4, cudaMemcpyHostToDevice);
  cudaMemset(d0, 0, cap * 4);
  bufs.push_back({dev, cap, d1, d0});
  *ones = d1;
  *zeros = d0;
  return ALT_OK;
}

static int num_sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <int BN, int STAGES, int CG_, bool RV, int SC = 1, int HS = 0, bool D3 = false, int HR = 0>
static cudaError_t launch_tc(const CUtensorMap &ta, const CUtensorMap &tb, const CUtensorMap &ty, const TcArgs &a,
                             uint16_t *y, int grid, cudaStream_t s) {
  constexpr int CG = CG_;
  auto kern = k_tc_conv<BN, STAGES, CG, RV, SC, HS, D3, HR>;
  const int smem = TcSmem<BN, STAGES, CG, HS, HR>::kBytes;
  static_assert(TcSmem<BN, STAGES, CG, HS, HR>::kBytes <= 232448, "smem budget");
  static bool attr_set = false;  // once per instantiation (not capture-safe to repeat)
  if (!attr_set) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (CG == 2) cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 0);
    attr_set = true;
  }
  static const bool pdl = [] {
    const char *e = getenv("ALT_PDL");
    return !(e && e[0] == '0');
  }();
  cudaLaunchConfig_t lc{};
  lc.gridDim = dim3((unsigned)grid);
  lc.blockDim = dim3(kThreads);
  lc.dynamicSmemBytes = smem;
  lc.stream = s;
  cudaLaunchAttribute at[2];
  int na = 0;
  if (CG * SC > 1) {
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = CG * SC;
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    na++;
  }
  if (pdl) {  // may start while the previous kernel in the stream drains
    at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[na].val.programmaticStreamSerializationAllowed = 1;
    na++;
  }
  lc.attrs = at;
  lc.numAttrs = na;
  cudaLaunchKernelEx(&lc, kern, ta, tb, ty, a, y);
  return cudaGetLastError();
}

// ---- launch-plan cache: everything the host derives for a call, keyed by
// the call's arguments (layout serials, pointers, geometry, epilogue, cfg)
struct TcKey {
  int64_t v[40];
  bool operator==(const TcKey &o) const { return memcmp(v, o.v, sizeof(v)) == 0; }
};
struct TcKeyHash {
  size_t operator()(const TcKey &k) const {
    uint64_t h = 1469598103934665603ull;
    for (int i = 0; i < 40; i++) h = (h ^ (uint64_t)k.v[i]) * 1099511628211ull;
    return (size_t)h;
  }
};
struct TcPlan {
  CUtensorMap ta, tb, ty;
  TcArgs a;
  int grid;
  int BN, stages, cg;
  int sc;  // cluster split-K factor (1 = off)
  int hs;  // halo mode: filter width S folded into row-shifted A reads (0 = off)
  int hr;  // 2-D halo: filter height R folded too (0 = off)
  alt_kernel_cfg used;
};
static std::mutex g_tc_mu;
static std::unordered_map<TcKey, TcPlan, TcKeyHash> g_tc_cache;

// smem-ring depth per (BLOCK_N, CTA group): the deepest ring that fits 227 KB
// next to the kEpiWarps staging buffers and the slab table
constexpr int stages_for(int BN, int CG) {
  return kEpiWarps == 8 ? (CG == 2 ? (BN == 128 ? 7 : 5) : (BN == 64 ? 7 : (BN == 128 ? 5 : (BN == 192 ? 4 : 3))))  // BN 192 pair: 5
                        : (CG == 2 ? (BN == 128 ? 5 : 4) : (BN == 64 ? 5 : (BN == 128 ? 4 : 3)));
}
// halo-mode ring depth (A stage + 8 spare rows, three B tap slabs per stage)
constexpr int stages_halo(int BN, int CG) { return BN / CG == 64 ? 4 : 2; }
// 2-D halo ring: 33 KB A stages next to one resident 72 KB B slot (BN 64)
constexpr int kStagesHalo2 = 3;
template <bool RV>
static cudaError_t launch_plan_rv(const TcPlan &pl, uint16_t *yy, cudaStream_t stream) {
  if (pl.hr == 3) return launch_tc<64, kStagesHalo2, 1, RV, 1, 3, false, 3>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  if (pl.hs == 3) {
    if (pl.cg == 2) {
      if (pl.BN == 128) return launch_tc<128, stages_halo(128, 2), 2, RV, 1, 3>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
      return launch_tc<256, stages_halo(256, 2), 2, RV, 1, 3>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    }
    if (pl.BN == 64) return launch_tc<64, stages_halo(64, 1), 1, RV, 1, 3>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    return launch_tc<128, stages_halo(128, 1), 1, RV, 1, 3>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  }
  if (pl.cg == 2) {
    if (pl.BN == 128) return launch_tc<128, stages_for(128, 2), 2, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    if (pl.BN == 192) return launch_tc<192, stages_for(192, 2), 2, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    return launch_tc<256, stages_for(256, 2), 2, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  }
  if (pl.BN == 64) return launch_tc<64, stages_for(64, 1), 1, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  if (pl.BN == 128) return launch_tc<128, stages_for(128, 1), 1, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  if (pl.BN == 192) return launch_tc<192, stages_for(192, 1), 1, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  return launch_tc<256, stages_for(256, 1), 1, RV>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
}
static cudaError_t launch_plan(const TcPlan &pl, void *y, cudaStream_t stream) {
  uint16_t *yy = static_cast<uint16_t *>(y);
  if (pl.sc > 1) {  // cluster split-K: one CTA, no residual vectors (planner-checked)
    if (pl.BN == 128)
      return pl.sc == 2 ? launch_tc<128, stages_for(128, 1), 1, false, 2>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream)
                        : launch_tc<128, stages_for(128, 1), 1, false, 4>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    return pl.sc == 2 ? launch_tc<256, stages_for(256, 1), 1, false, 2>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream)
                      : launch_tc<256, stages_for(256, 1), 1, false, 4>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  }
  if (pl.a.Do3) {  // C3D (planner: no residual, no split, no halo)
    if (pl.cg == 2) {
      if (pl.BN == 128) return launch_tc<128, stages_for(128, 2), 2, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
      if (pl.BN == 192) return launch_tc<192, stages_for(192, 2), 2, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
      return launch_tc<256, stages_for(256, 2), 2, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    }
    if (pl.BN == 64) return launch_tc<64, stages_for(64, 1), 1, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    if (pl.BN == 128) return launch_tc<128, stages_for(128, 1), 1, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    if (pl.BN == 192) return launch_tc<192, stages_for(192, 1), 1, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
    return launch_tc<256, stages_for(256, 1), 1, false, 1, 0, true>(pl.ta, pl.tb, pl.ty, pl.a, yy, pl.grid, stream);
  }
  return pl.a.res_vec ? launch_plan_rv<true>(pl, yy, stream) : launch_plan_rv<false>(pl, yy, stream);
}

// common driver for conv and GEMM
struct TcProblem {
  bool is_conv;
  Layout *al, *bl, *yl;
  LView va, vb, vy;           // what build_view sees (folded views for conv1-like layers)
  const void *a, *b;
  void *y;
  RoleInfo ra[kMaxL], rb[kMaxL], ry[kMaxL];
  int64_t N, K, Ho, Wo;       // output geometry (GEMM: 1, cols, 1, M)
  int64_t R, S, C;            // taps and reduction channels
  OpEpilogue epi;
  int64_t coff = 0, koff = 0; // grouped conv: this group's first input / output channel
  int64_t T = 1, Do = 0;      // C3D: depth taps, output depth (Do = 0: conv2d / GEMM)
  int pairs = 0;              // fp32 split operands: 6 plane products per slab (0 = bf16)
  bool out_f32 = false;       // fp32 output / residual
};

static alt_status tc_run(TcProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used,
                         int tile_n_fixed, int tile_h_fixed) {
  char why[160] = "";
  TcKey key;
  memset(&key, 0, sizeof(key));
  {
    int64_t *k = key.v;
    int i = 0;
    k[i++] = P.is_conv;
    k[i++] = (int64_t)P.al->serial; k[i++] = (int64_t)P.bl->serial; k[i++] = (int64_t)P.yl->serial;
    k[i++] = (int64_t)(uintptr_t)P.a; k[i++] = (int64_t)(uintptr_t)P.b; k[i++] = (int64_t)(uintptr_t)P.y;
    k[i++] = P.N; k[i++] = P.K; k[i++] = P.Ho; k[i++] = P.Wo; k[i++] = P.R; k[i++] = P.S; k[i++] = P.C;
    for (int d = 0; d < 5; d++) {
      k[i++] = ((int64_t)P.ra[d].role << 48) | ((int64_t)P.ra[d].V << 32) | ((int64_t)P.ra[d].pad << 16) |
               P.ra[d].win;
    }
    k[i++] = (P.T << 32) | P.Do;
    k[i++] = (int64_t)(uintptr_t)P.epi.scale; k[i++] = (int64_t)(uintptr_t)P.epi.bias;
    k[i++] = (int64_t)(uintptr_t)P.epi.bias_att;
    k[i++] = (int64_t)(uintptr_t)P.epi.residual;
    k[i++] = P.epi.residual_l ? (int64_t)P.epi.residual_l->serial : 0;
    k[i++] = P.epi.act;
    k[i++] = (P.coff << 32) | P.koff;
    k[i++] = P.pairs * 4 + (P.out_f32 ? 2 : 0) + (P.epi.pads_zero ? 1 : 0);
    if (cfg) {
      k[i++] = cfg->block_n; k[i++] = cfg->tile_n; k[i++] = cfg->tile_h; k[i++] = cfg->tile_w;
      k[i++] = cfg->stages;
      k[i++] = cfg->cta_pair;
      k[i++] = cfg->split_k;
      k[i++] = cfg->split_cluster;
      k[i++] = cfg->block_k;  // halo request / refusal
    }
    int dev = 0;
    cudaGetDevice(&dev);
    k[i++] = dev;
  }
  {
    std::lock_guard<std::mutex> g(g_tc_mu);
    auto it = g_tc_cache.find(key);
    if (it != g_tc_cache.end()) {
      cudaError_t e = launch_plan(it->second, P.y, stream);
      count_launch();
      if (e != cudaSuccess) { set_error("tc launch failed: %s", cudaGetErrorString(e)); return ALT_E_CUDA; }
      if (used) *used = it->second.used;
      return ALT_OK;
    }
  }
  const int esize = 2;
  // M-tile candidates (tile_n x tile_h x tile_w = 128 output pixels)
  struct Cand { int tn, th, tw; };
  std::vector<Cand> cands;
  if (cfg && cfg->tile_n * cfg->tile_h * cfg->tile_w == 128) {
    if (P.Do && cfg->tile_n != 1) { set_error("tc: C3D tiles hold one output depth slice (tile_n = 1)"); return ALT_E_UNSUPPORTED; }
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
    // least wasted rows first, then longer contiguous runs
    std::stable_sort(cands.begin(), cands.end(), [&](const Cand &x, const Cand &y) {
      auto cov = [&](const Cand &c) {
        return (double)((P.Ho + c.th - 1) / c.th * c.th) * ((P.Wo + c.tw - 1) / c.tw * c.tw) *
               ((P.N + c.tn - 1) / c.tn * c.tn);
      };
      double a = cov(x), b = cov(y);
      if (a != b) return a < b;
      return x.tw > y.tw;
    });
  }
  int BN = cfg && cfg->block_n ? cfg->block_n : (P.K > 128 ? 256 : (P.K > 64 ? 128 : 64));
  if (BN != 64 && BN != 128 && BN != 192 && BN != 256) { set_error("tc: block_n must be 64/128/192/256"); return ALT_E_UNSUPPORTED; }
  // CTA pair (tcgen05 cta_group::2, M = 256): cfg->cta_pair 1 = pair,
  // 2 = single CTA, 0 = pair when BLOCK_N >= 128
  const int cg = (cfg && cfg->cta_pair == 2) ? 1 : ((cfg && cfg->cta_pair == 1) || BN >= 128 ? 2 : 1);
  if (cg == 2 && BN < 128) { set_error("tc: a CTA pair needs block_n >= 128"); return ALT_E_UNSUPPORTED; }
  for (const Cand &c : cands) {
    RoleInfo ra[kMaxL], rb[kMaxL], ry[kMaxL];
    memcpy(ra, P.ra, sizeof(ra));
    memcpy(rb, P.rb, sizeof(rb));
    memcpy(ry, P.ry, sizeof(ry));
    for (int d = 0; d < kMaxL; d++) {
      if (ra[d].role == R_N) ra[d].tile = c.tn;
      if (ra[d].role == R_H) ra[d].tile = c.th;
      if (ra[d].role == R_W) ra[d].tile = c.tw;
      // output stores are per epilogue warp: a 32-row sub-box of the tile
      // (rows are (n, h, w) with w fastest, all extents powers of two)
      const int sw_w = c.tw >= 32 ? 32 : c.tw;
      const int sw_h = c.tw >= 32 ? 1 : (c.tw * c.th >= 32 ? 32 / c.tw : c.th);
      const int sw_n = 32 / (sw_w * sw_h);
      if (ry[d].role == R_N) ry[d].tile = sw_n;
      if (ry[d].role == R_H) ry[d].tile = sw_h;
      if (ry[d].role == R_W) ry[d].tile = sw_w;
      if (rb[d].role == R_W) rb[d].tile = BN / cg;
    }
    // halo mode (stride-1 3x3, 64-channel slabs, K-major A): the tile's W run
    // tw in {16, 32, 64} must leave S - 1 spare columns past Wo, so the row
    // shifts of the valid outputs stay inside their own W run
    static const int halo_env = [] { const char *e = getenv("ALT_TC_HALO"); return e ? atoi(e) : -1; }();
    const int halo_cfg = cfg && cfg->block_k == 1 ? 1 : (cfg && cfg->block_k == 2 ? 0 : -1);
    const int halo_want = halo_env >= 0 ? halo_env : (halo_cfg >= 0 ? halo_cfg : 0);
    const bool halo_ok = halo_want && P.is_conv && P.S == 3 && !P.pairs && P.ra[3].role == R_W && P.ra[3].V == 1 &&
                         P.ra[3].tap == 1 && (c.tw == 16 || c.tw == 32 || c.tw == 64) && P.Wo + P.S - 2 < c.tw &&
                         !(cfg && (cfg->split_k > 1 || cfg->split_cluster)) && BN / cg <= 128;
    // 2-D halo (hmode 2): R filter rows folded too — one 64-channel slab
    // (C <= 64), one 64-channel N tile per CTA, one image per tile (tile_n 1,
    // the tile's (tile_h + R - 1) x tile_w input rows in one box <= 256 rows)
    static const int hrow_env = [] { const char *e = getenv("ALT_TC_HROW"); return e ? atoi(e) : 1; }();
    const bool hrow_ok = halo_ok && hrow_env && P.R == 3 && P.C <= 64 && P.K <= 64 && BN == 64 && cg == 1 &&
                         c.tn == 1 && (c.th + P.R - 1) * c.tw <= 256 && P.ra[2].role == R_H && P.ra[2].V == 1 &&
                         P.ra[2].tap == 1 && P.T == 1 && !P.Do;
    for (int hmode = hrow_ok ? 2 : (halo_ok ? 1 : 0); hmode >= 0; hmode--)
    for (int sw = 64; sw >= 8; sw /= 2) {
      if (hmode && sw != 64) continue;
      RoleInfo rah[kMaxL];
      memcpy(rah, ra, sizeof(rah));
      if (hmode) rah[3].tap = 0;  // the A box does not move with the tap s
      if (hmode == 2) { rah[2].tap = 0; rah[2].tile = c.th + (int)P.R - 1; }  // nor with r: R - 1 extra rows
      View va, vb;
      // K-major first (the channel run innermost); otherwise an MN-major
      // view whose stride-1 dim is the M (A) / N (B) run: groups of mnw rows
      // (mnw = the widest of 64 / 32 / 16 / 8 that tiles the run), one TMA box
      // of mnw x sw per (group, slab)
      auto view_of = [&](const LView &L, const RoleInfo *roles, int rows, int run, View *v, int *mnw) -> bool {
        *mnw = 0;
        if (build_view(L, roles, sw, v, why)) return true;
        char why2[160];
        for (int w = 64; w >= 8; w /= 2) {
          if (run % w || rows % w || (rows / w) * (64 / sw) > 16) continue;
          RoleInfo rm[kMaxL];
          memcpy(rm, roles, sizeof(rm));
          for (int d = 0; d < kMaxL; d++) {
            if (rm[d].role == R_W) rm[d].tile = w;
            if (rm[d].role == R_H || rm[d].role == R_N) rm[d].tile = 1;
          }
          if (build_view(L, rm, sw, v, why2, w)) { *mnw = w; return true; }
        }
        return false;
      };
      int mnA = 0, mnB = 0;
      if (!view_of(P.va, rah, 128, c.tw, &va, &mnA)) continue;
      if (hmode && mnA) continue;
      if (!view_of(P.vb, rb, BN / cg, BN / cg, &vb, &mnB)) continue;
      // halo modes issue one B box per (tap, slab) from lanes 16..31: an
      // MN-major B (ng groups per slab) would need ng x taps boxes and its
      // tap index would run past the stage (found by the randomized stress:
      // an out-of-bounds shared-memory write with the paper's weight order)
      if (hmode && mnB) continue;
      // a group's weight rows start at b_koff: when the weight layout splits
      // K into tiles of divq rows the box origin must sit on a tile boundary
      // (a box covers whole tiles; found by the randomized stress: K / groups
      // = 144 on a K/32 weight layout read the wrong rows)
      if (vb.divq > 1 && vb.divq < (1 << 30) && P.koff % vb.divq) {
        snprintf(why, 160, "group weight offset %lld not a multiple of the weight k tile %d", (long long)P.koff, vb.divq);
        continue;
      }
      int64_t rowsA = 1, rowsB = 1;
      for (int i = 1; i < va.rank; i++) rowsA *= (va.d[i].box + va.d[i].estride - 1) / va.d[i].estride;
      for (int i = 1; i < vb.rank; i++) rowsB *= (vb.d[i].box + vb.d[i].estride - 1) / vb.d[i].estride;
      // K-major: a box holds the tile's rows; MN-major: sw K rows of one group
      const int64_t rowsA_want = mnA ? sw : (hmode == 2 ? (int64_t)(c.th + P.R - 1) * c.tw : 128);
      if (rowsA != rowsA_want || rowsB != (mnB ? sw : BN / cg)) {
        snprintf(why, 160, "rows A %lld B %lld", (long long)rowsA, (long long)rowsB);
        continue;
      }
      TcPlan pl;
      TcArgs &a = pl.a;
      memset(&a, 0, sizeof(a));
      if (!encode_view(va, P.a, esize, sw, &pl.ta, &a.A, why, mnA)) continue;
      if (!encode_view(vb, P.b, esize, sw, &pl.tb, &a.B, why, mnB)) continue;
      if (mnA) { a.A.ng = 128 / mnA; a.A.gbytes = 64 * mnA * esize; }
      if (mnB) { a.B.ng = BN / cg / mnB; a.B.gbytes = 64 * mnB * esize; }
      // output: TMA-store view when y holds one copy per element (no pads /
      // unfold duplicates) and a >= 8-channel contiguous run, else the writer
      a.out_mode = 0;
      memset(&pl.ty, 0, sizeof(pl.ty));
      static const int store_mode = [] {
        const char *e = getenv("ALT_TC_STORE");
        // default TMA stores (measured faster than direct 16-byte stores)
        return e && e[0] == 'd' ? 2 : (e && e[0] == 'g' ? 0 : 1);
      }();
      // fp32 output: direct 16-byte stores (4 channels) or the generic writer
      if ((store_mode == 2 || P.out_f32) && !(P.yl->flags & (ALT_HAS_PAD | ALT_HAS_UNFOLD)) && P.K % 8 == 0 &&
          P.koff % 8 == 0 && (reinterpret_cast<uintptr_t>(P.y) & 15) == 0 && direct_store_ok(P.vy)) {
        alt_status st2 = make_reader(P.yl, &a.yr);
        if (st2 != ALT_OK) return st2;
        a.out_mode = 2;
      }
      // TMA-store view: y holds one copy per element; pads only when the
      // caller guarantees they already hold 0 (ALT_EPI_PADS_ZERO)
      if (a.out_mode == 0 && store_mode != 0 && !P.out_f32 && !(P.yl->flags & ALT_HAS_UNFOLD) &&
          (!(P.yl->flags & ALT_HAS_PAD) || P.epi.pads_zero)) {
        char why2[160];
        // round stores (one 128-row box per channel slab and round) unless a
        // split-K / cluster form is requested (their epilogues skip rounds)
        static const bool rounds_on = [] { const char *e = getenv("ALT_TC_ROUND"); return !(e && e[0] == '0'); }();
        const bool want_round = rounds_on && !(cfg && (cfg->split_k > 1 || cfg->split_cluster)) && kEpiWarps == 8;
        for (int so = 64; so >= 8 && want_round && !a.out_mode; so /= 2) {
          if (P.koff % so) continue;
          if ((P.yl->flags & ALT_HAS_PAD) && P.yl->max_copies[1] != 1) break;
          RoleInfo rr[kMaxL];
          memcpy(rr, ry, sizeof(rr));
          for (int d = 0; d < kMaxL; d++) {
            if (rr[d].role == R_N) rr[d].tile = c.tn;
            if (rr[d].role == R_H) rr[d].tile = c.th;
            if (rr[d].role == R_W) rr[d].tile = c.tw;
          }
          View vy;
          if (!build_view(P.vy, rr, so, &vy, why2, 0, (P.yl->flags & ALT_HAS_PAD) != 0)) continue;
          int64_t rowsY = 1;
          for (int i = 1; i < vy.rank; i++) rowsY *= vy.d[i].box;
          if (rowsY != 128) continue;
          if (encode_view(vy, P.y, esize, so, &pl.ty, &a.O, why2)) { a.out_mode = 1; a.out_round = 1; }
        }
        for (int so = 32; so >= 8 && !a.out_mode; so /= 2) {
          if (P.koff % so) continue;  // a group's first channel must start a store slab
          View vy;
          if ((P.yl->flags & ALT_HAS_PAD) && P.yl->max_copies[1] != 1) break;  // padded channels: the writer
          if (!build_view(P.vy, ry, so, &vy, why2, 0, (P.yl->flags & ALT_HAS_PAD) != 0)) continue;
          int64_t rowsY = 1;
          for (int i = 1; i < vy.rank; i++) rowsY *= vy.d[i].box;
          if (rowsY != 32) continue;
          if (encode_view(vy, P.y, esize, so, &pl.ty, &a.O, why2)) a.out_mode = 1;
        }
      }
      // generic-writer layouts (pads / unfold copies) with 8-channel runs:
      // the vectorised writer (the channel dim itself must hold one copy
      // per channel, or its pad positions already be 0)
      a.pads_zero = P.epi.pads_zero;
      a.yvec = 0;
      if (a.out_mode == 0 && !P.out_f32 && P.yl->separable && P.K % 8 == 0 && P.koff % 8 == 0 &&
          (reinterpret_cast<uintptr_t>(P.y) & 15) == 0 && chan_vec8(*P.yl, true) &&
          (P.yl->max_copies[1] == 1 || P.epi.pads_zero)) {
        alt_status st2 = make_reader(P.yl, &a.yr);
        if (st2 != ALT_OK) return st2;
        a.yvec = 1;
      }
      if (P.Do && a.out_mode != 1) { snprintf(why, 160, "C3D needs a TMA-store output layout"); continue; }
      a.is_conv = P.is_conv;
      a.N = (int32_t)P.N; a.K = (int32_t)P.K; a.Ho = (int32_t)P.Ho; a.Wo = (int32_t)P.Wo;
      a.tile_n = c.tn; a.tile_h = c.th; a.tile_w = c.tw;
      a.mt_h = (int32_t)((P.Ho + c.th - 1) / c.th);
      a.mt_w = (int32_t)((P.Wo + c.tw - 1) / c.tw);
      const int64_t mt_n = (P.N * (P.Do ? P.Do : 1) + c.tn - 1) / c.tn;  // C3D: tiles over (n, od)
      const int64_t mtiles = mt_n * a.mt_h * a.mt_w;
      const int64_t ntiles = (P.K + BN - 1) / BN;
      if (mtiles * ntiles > 0x7fffffff) { set_error("tc: too many tiles"); return ALT_E_UNSUPPORTED; }
      a.num_n_tiles = (int32_t)ntiles;
      a.num_tiles = (int32_t)(((mtiles + cg - 1) / cg) * ntiles);  // work units
      a.S = (int32_t)(hmode ? 1 : P.S);  // halo: the slabs enumerate (r, g); the S taps ride in each stage
      const int64_t Rsl = hmode == 2 ? 1 : P.R;  // 2-D halo: the slabs enumerate g; all R x S taps ride in each stage
      a.a_bytes = (int32_t)((hmode == 2 ? rowsA_want : 128) * 64 * esize);  // one 64-channel stage
      a.Gc = (int32_t)((P.C + sw - 1) / sw);
      if (P.coff % sw) { snprintf(why, 160, "group channel offset %% slab"); continue; }
      a.a_goff = (int32_t)(P.coff / sw);
      a.b_koff = (int32_t)P.koff;
      a.y_koff = (int32_t)P.koff;
      a.rsg = (int32_t)(Rsl * a.S * a.Gc);
      a.pairs = P.pairs;
      a.out_f32 = P.out_f32 ? 1 : 0;
      if (P.pairs && P.C % sw) { snprintf(why, 160, "split planes not slab-aligned"); continue; }
      a.total_slabs = (int32_t)((P.pairs ? P.pairs : 1) * P.T * Rsl * a.S * a.Gc);
      a.Do3 = (int32_t)P.Do;
      a.RS3 = (int32_t)(Rsl * a.S);
      a.f_Do3 = FastDiv((uint32_t)std::max<int64_t>(1, P.Do));
      a.f_RS3 = FastDiv((uint32_t)std::max(1, a.RS3));
      pl.hs = hmode ? (int)P.S : 0;
      pl.hr = hmode == 2 ? (int)P.R : 0;
      {
        static const int hboff = [] { const char *e = getenv("ALT_HALO_BOFF"); return e ? atoi(e) : 0; }();
        a.hboff = hboff;
      }
      a.spi = 64 / sw;
      a.num_iters = (a.total_slabs + a.spi - 1) / a.spi;
      a.sw = sw;
      // split-K when the output tiles leave SMs idle (small M x N, long K)
      {
        const int64_t units = a.num_tiles;
        const int64_t slots = num_sms() / cg;
        int64_t sk = 1;
        if (cfg && cfg->split_k > 0) sk = cfg->split_k;
        // auto: no split (measured: the serial partial reduction costs more
        // than the idle SMs it recovers on the ResNet-50 set; tuned per layer)
        sk = std::max<int64_t>(1, std::min<int64_t>(sk, a.num_iters));
        a.splits = (int32_t)sk;
        a.full_units = 0;
        a.ws = nullptr;
        a.cnt = nullptr;
        // tail split (split_cluster == 2): whole waves run unsplit, only the
        // output tiles of the last, partial wave are split sk ways
        int64_t split_units = units;
        if (cfg && cfg->split_cluster == 2 && sk > 1) {
          const int64_t tail = units % slots;
          split_units = units > slots ? tail : units;
          a.full_units = (int32_t)(units - split_units);
          if (split_units == 0) { sk = 1; a.splits = 1; }
        }
        // cluster split-K: the sk ranges of a tile as one cluster, reduced
        // through DSMEM (single CTA, TMA-store output, no residual, sk 2 / 4)
        pl.sc = 1;
        if (cfg && cfg->split_cluster == 1 && sk > 1) {
          if (cg != 1 || (sk != 2 && sk != 4) || BN < 128 || BN == 192 || a.out_mode != 1 || P.epi.residual) {
            set_error("tc: cluster split-K needs one CTA, block_n 128/256, split 2/4, a TMA-store output and no residual");
            return ALT_E_UNSUPPORTED;
          }
          pl.sc = (int)sk;
          a.num_tiles = (int32_t)(units * sk);
        } else if (sk > 1) {
          if ((int64_t)a.num_tiles * sk > 0x7fffffff) { set_error("tc: too many tiles"); return ALT_E_UNSUPPORTED; }
          // per-plan workspace (lives as long as the process: captured graphs
          // may replay the plan after the cache forgets it)
          const size_t wsb = (size_t)split_units * cg * sk * 128 * BN * sizeof(float);
          // bounded: plans (and their workspaces) live for the process, so a
          // tuner sweeping many split points must not exhaust the device
          static std::mutex ws_mu;
          static size_t ws_total = 0;
          {
            std::lock_guard<std::mutex> g(ws_mu);
            if (ws_total + wsb > ((size_t)4 << 30)) {
              set_error("tc: split-K workspace budget (4 GiB per process) exhausted");
              return ALT_E_NOMEM;
            }
            ws_total += wsb;
          }
          // cooperative reduction (tail split, 2 / 4 splits, every piece in one
          // round of the persistent grid so all pieces of a tile are resident)
          a.coop = (cfg && cfg->split_cluster == 2 && (sk == 2 || sk == 4) &&
                    split_units * sk <= slots) ? 1 : 0;
          a.done = nullptr;
          if (cudaMalloc(&a.ws, wsb) != cudaSuccess || cudaMalloc(&a.cnt, (size_t)split_units * cg * 4) != cudaSuccess ||
              cudaMemset(a.cnt, 0, (size_t)split_units * cg * 4) != cudaSuccess ||
              (a.coop && (cudaMalloc(&a.done, (size_t)split_units * cg * 4) != cudaSuccess ||
                          cudaMemset(a.done, 0, (size_t)split_units * cg * 4) != cudaSuccess))) {
            cudaGetLastError();
            set_error("tc: split-K workspace: out of memory");
            return ALT_E_NOMEM;
          }
          a.num_tiles = (int32_t)(a.full_units + split_units * sk);
        }
      }
      a.f_nnt = FastDiv((uint32_t)a.num_n_tiles);
      a.f_mtw = FastDiv((uint32_t)a.mt_w);
      a.f_mth = FastDiv((uint32_t)a.mt_h);
      a.f_spl = FastDiv((uint32_t)a.splits);
      a.f_Gc = FastDiv((uint32_t)a.Gc);
      a.f_rsg = FastDiv((uint32_t)std::max(1, a.rsg));
      a.f_S = FastDiv((uint32_t)a.S);
      alt_status st;
      if ((st = make_epi(P.epi, &a.epi)) != ALT_OK) return st;
      a.res_vec = P.epi.residual && !P.out_f32 && a.epi.res.sep && chan_vec8(*P.epi.residual_l, true) &&
                  (reinterpret_cast<uintptr_t>(P.epi.residual) & 15) == 0 ? 1 : 0;
      // the kernel always applies scale * acc + bias: absent ones become the
      // identity (device-resident ones / zeros, grown on demand)
      if (!a.epi.scale || !a.epi.bias) {
        const float *ones = nullptr, *zeros = nullptr;
        if ((st = identity_vectors(P.K, &ones, &zeros)) != ALT_OK) return st;
        if (!a.epi.scale) a.epi.scale = ones;
        if (!a.epi.bias) a.epi.bias = zeros;
      }
      if ((st = make_writer(P.yl, &a.yw)) != ALT_OK) return st;
      a.dbg = debug_buffer();
      {
        static const int epi_dbg = [] { const char *e = getenv("ALT_TC_EPI_DBG"); return e ? atoi(e) : 0; }();
        a.epi_dbg = epi_dbg;
      }
      pl.grid = pl.sc > 1 ? a.num_tiles  // one tile per CTA
                          : (int)std::min<int64_t>((int64_t)a.num_tiles * cg, num_sms() / cg * cg);
      pl.BN = BN;
      pl.cg = cg;
      pl.stages = pl.hr ? kStagesHalo2 : (pl.hs ? stages_halo(BN, cg) : stages_for(BN, cg));
      // a shallower ring than the instantiation's (tuner knob; 2 .. STAGES)
      a.nst = (cfg && cfg->stages >= 2 && cfg->stages < pl.stages) ? cfg->stages : pl.stages;
      {
        // resident weights (see TcArgs::b_res): a CTA's units keep one N tile
        // when its unit stride is a multiple of the N-tile count (N fastest)
        static const bool no_res = getenv("ALT_TC_NO_BRES") != nullptr;  // developer A/B knob
        const int64_t ustep = pl.grid / cg;
        a.b_res = (!no_res && pl.sc == 1 && a.splits == 1 && a.full_units == 0 && a.num_iters <= a.nst &&
                   ustep % a.num_n_tiles == 0 && a.num_tiles > ustep) ? 1 : 0;
        // 2-D halo: B lives in its one resident slot (the CTA keeps its N tile,
        // the reduction is one stage), else this plan is not valid
        if (pl.hr) {
          if (!(pl.sc == 1 && a.splits == 1 && a.full_units == 0 && a.num_iters == 1 && ustep % a.num_n_tiles == 0)) {
            snprintf(why, 160, "2-D halo needs one reduction stage and a fixed N tile per CTA");
            continue;
          }
          a.b_res = 1;
        }
      }
      alt_kernel_cfg u{};
      u.path = ALT_PATH_TC;
      u.block_m = 128 * cg;
      u.cta_pair = cg == 2 ? 1 : 2;
      u.block_n = BN;
      u.block_k = 64;
      u.stages = a.nst;
      u.tile_n = c.tn; u.tile_h = c.th; u.tile_w = c.tw;
      u.split_k = a.splits;
      u.split_cluster = pl.sc > 1 ? 1 : (a.full_units > 0 && a.splits > 1 ? 2 : 0);
      u.block_k = pl.hr ? 3 : (pl.hs ? 1 : 64);  // 1 = halo, 3 = 2-D halo (cfg->block_k: 1 request, 2 refuse)
      pl.used = u;
      cudaError_t e = launch_plan(pl, P.y, stream);
      count_launch();
      if (e != cudaSuccess) { set_error("tc launch failed: %s", cudaGetErrorString(e)); return ALT_E_CUDA; }
      {
        std::lock_guard<std::mutex> g(g_tc_mu);
        if (g_tc_cache.size() > 4096) g_tc_cache.clear();
        g_tc_cache.emplace(key, pl);
      }
      if (used) *used = u;
      return ALT_OK;
    }
  }
  set_error("tc path unavailable: %s", why);
  return ALT_E_UNSUPPORTED;
}

// ---- fp32 on the tensor cores (reading A27, split3.cu): each fp32 operand is
// split into three bf16 planes stored reduction-innermost ([outer][3 Cp]) in
// stream-ordered scratch, the conv / GEMM runs the six plane products of
// every reduction slab on the bf16 kernel, and the epilogue writes fp32.
alt_status split3_launch(Layout *L, const float *src, int red, int64_t C, int64_t Cp, uint16_t *dst,
                         cudaStream_t stream);

// compiled internal layouts of the split planes, by logical shape (stable
// serials keep the launch-plan cache hit across calls)
static Layout *split_layout(int lrank, const int64_t *lshape, int nprims, const alt_prim *prims) {
  static std::mutex mu;
  static std::vector<std::pair<std::vector<int64_t>, Layout *>> cache;
  std::vector<int64_t> key(lshape, lshape + lrank);
  key.push_back(nprims ? prims[0].v[0] * 16 + prims[0].v[1] : -1);
  std::lock_guard<std::mutex> g(mu);
  for (auto &e : cache)
    if (e.first == key) return e.second;
  Layout *L = new Layout();
  if (compile_layout(lrank, lshape, prims, nprims, L) != ALT_OK) { delete L; return nullptr; }
  cache.push_back({key, L});
  return L;
}

struct SplitScratch {
  void *p[2] = {nullptr, nullptr};
  cudaStream_t s;
  ~SplitScratch() { for (void *q : p) if (q) cudaFreeAsync(q, s); }
};

static alt_status tc_conv_f32(const ConvProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream,
                              alt_kernel_cfg *used) {
  if (P.groups > 1) { set_error("tc path: fp32 grouped conv runs on the generic path"); return ALT_E_UNSUPPORTED; }
  const int64_t Cp = (P.C + 7) / 8 * 8;
  alt_prim nhwc{};
  nhwc.kind = ALT_REORDER; nhwc.n = 4; nhwc.v[0] = 0; nhwc.v[1] = 2; nhwc.v[2] = 3; nhwc.v[3] = 1;
  const int64_t xs[4] = {P.N, 3 * Cp, P.H, P.W}, ws[4] = {P.K, 3 * Cp, P.R, P.S};
  Layout *XL = split_layout(4, xs, 1, &nhwc), *WL = split_layout(4, ws, 1, &nhwc);
  if (!XL || !WL) return ALT_E_NOMEM;
  SplitScratch sc;
  sc.s = stream;
  if (cudaMallocAsync(&sc.p[0], (size_t)XL->pnumel * 2, stream) != cudaSuccess ||
      cudaMallocAsync(&sc.p[1], (size_t)WL->pnumel * 2, stream) != cudaSuccess) {
    cudaGetLastError();
    set_error("tc fp32: split scratch allocation failed");
    return ALT_E_NOMEM;
  }
  alt_status st = split3_launch(P.xl, static_cast<const float *>(P.x), 1, P.C, Cp,
                                static_cast<uint16_t *>(sc.p[0]), stream);
  if (st == ALT_OK)
    st = split3_launch(P.wl, static_cast<const float *>(P.w), 1, P.C, Cp, static_cast<uint16_t *>(sc.p[1]), stream);
  if (st != ALT_OK) return st;
  TcProblem T{};
  T.is_conv = true;
  T.al = XL; T.bl = WL; T.yl = P.yl;
  T.a = sc.p[0]; T.b = sc.p[1]; T.y = P.y;
  T.ra[0].role = R_N;
  T.ra[1].role = R_C;
  T.ra[2] = RoleInfo{R_H, 1, P.Vh, P.ph, (int)((P.R - 1) * P.dh + 1), P.dh};
  T.ra[3] = RoleInfo{R_W, 1, P.Vw, P.pw, (int)((P.S - 1) * P.dw + 1), P.dw};
  T.rb[0] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.rb[1].role = R_C;
  T.rb[2].role = R_TR;
  T.rb[3].role = R_TS;
  T.ry[0].role = R_N;
  T.ry[1].role = R_C;
  T.ry[2] = RoleInfo{R_H, 1, 1, 0, 1, 0};
  T.ry[3] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.N = P.N; T.K = P.K; T.Ho = P.Ho; T.Wo = P.Wo;
  T.R = P.R; T.S = P.S; T.C = Cp;
  T.epi = P.epi;
  T.va = lview(*XL); T.vb = lview(*WL); T.vy = lview(*P.yl);
  T.pairs = 6;
  T.out_f32 = true;
  if (P.N * P.Ho * P.Wo >= (1ll << 31)) { set_error("tc: too many output pixels"); return ALT_E_UNSUPPORTED; }
  return tc_run(T, cfg, stream, used, 0, 0);
}

static alt_status tc_gemm_f32(const GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream,
                              alt_kernel_cfg *used) {
  const int64_t Kp = (P.K + 7) / 8 * 8;
  alt_prim tr{};
  tr.kind = ALT_REORDER; tr.n = 2; tr.v[0] = 1; tr.v[1] = 0;
  const int64_t as[2] = {P.M, 3 * Kp}, bs[2] = {3 * Kp, P.N};
  Layout *AL = split_layout(2, as, 0, nullptr), *BL = split_layout(2, bs, 1, &tr);
  if (!AL || !BL) return ALT_E_NOMEM;
  SplitScratch sc;
  sc.s = stream;
  if (cudaMallocAsync(&sc.p[0], (size_t)AL->pnumel * 2, stream) != cudaSuccess ||
      cudaMallocAsync(&sc.p[1], (size_t)BL->pnumel * 2, stream) != cudaSuccess) {
    cudaGetLastError();
    set_error("tc fp32: split scratch allocation failed");
    return ALT_E_NOMEM;
  }
  // A [M, K]: reduction dim 1; B [K(+1), N]: reduction dim 0, rows k < K
  alt_status st = split3_launch(P.al, static_cast<const float *>(P.a), 1, P.K, Kp,
                                static_cast<uint16_t *>(sc.p[0]), stream);
  if (st == ALT_OK)
    st = split3_launch(P.bl, static_cast<const float *>(P.b), 0, P.K, Kp, static_cast<uint16_t *>(sc.p[1]), stream);
  if (st != ALT_OK) return st;
  TcProblem T{};
  T.is_conv = false;
  T.al = AL; T.bl = BL; T.yl = P.cl;
  T.a = sc.p[0]; T.b = sc.p[1]; T.y = P.c;
  T.ra[0] = RoleInfo{R_W, 128, 1, 0, 1, 0};
  T.ra[1].role = R_C;
  T.rb[0].role = R_C;
  T.rb[1] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.ry[0] = RoleInfo{R_W, 128, 1, 0, 1, 0};
  T.ry[1].role = R_C;
  T.N = 1; T.K = P.N; T.Ho = 1; T.Wo = P.M;
  T.R = 1; T.S = 1; T.C = Kp;
  T.epi = P.epi;
  T.va = lview(*AL); T.vb = lview(*BL); T.vy = lview(*P.cl);
  T.pairs = 6;
  T.out_f32 = true;
  if (P.M >= (1ll << 31)) { set_error("tc: M too large"); return ALT_E_UNSUPPORTED; }
  return tc_run(T, cfg, stream, used, 1, 1);
}

// C3D on the tensor cores: the conv2d kernel with a depth role — each M tile
// is one output depth slice od of one image n (tile_n = 1, tiles over
// (n, od)), the reduction runs over (t, r, s, channel slab) and the depth tap
// t moves the A box along D (od Vd - pd + dd t; out of range = TMA zero fill)
static alt_status tc_conv3d(const ConvProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream,
                            alt_kernel_cfg *used) {
  if (P.dtype != ALT_BF16) { set_error("tc path: C3D is bf16 (fp32 runs on the generic path)"); return ALT_E_UNSUPPORTED; }
  if (P.groups > 1) { set_error("tc path: grouped C3D runs on the generic path"); return ALT_E_UNSUPPORTED; }
  if (P.epi.residual) { set_error("tc path: C3D with a residual runs on the generic path"); return ALT_E_UNSUPPORTED; }
  if (cfg && (cfg->split_k > 1 || cfg->split_cluster)) { set_error("tc path: C3D has no split-K"); return ALT_E_UNSUPPORTED; }
  TcProblem T{};
  T.is_conv = true;
  T.al = P.xl; T.bl = P.wl; T.yl = P.yl;
  T.a = P.x; T.b = P.w; T.y = P.y;
  // x (n, c, d, h, w); w (k, c, t, r, s); y (n, k, od, oh, ow)
  T.ra[0].role = R_N;
  T.ra[1].role = R_C;
  T.ra[2] = RoleInfo{R_D, 1, P.Vd, P.pd, (int)((P.T - 1) * P.dd + 1), P.dd};
  T.ra[3] = RoleInfo{R_H, 1, P.Vh, P.ph, (int)((P.R - 1) * P.dh + 1), P.dh};
  T.ra[4] = RoleInfo{R_W, 1, P.Vw, P.pw, (int)((P.S - 1) * P.dw + 1), P.dw};
  T.rb[0] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.rb[1].role = R_C;
  T.rb[2].role = R_TT;
  T.rb[3].role = R_TR;
  T.rb[4].role = R_TS;
  T.ry[0].role = R_N;
  T.ry[1].role = R_C;
  T.ry[2] = RoleInfo{R_D, 1, 1, 0, 1, 0};
  T.ry[3] = RoleInfo{R_H, 1, 1, 0, 1, 0};
  T.ry[4] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.N = P.N; T.K = P.K; T.Ho = P.Ho; T.Wo = P.Wo;
  T.R = P.R; T.S = P.S; T.C = P.C;
  T.T = P.T; T.Do = P.Do;
  T.epi = P.epi;
  T.va = lview(*P.xl); T.vb = lview(*P.wl); T.vy = lview(*P.yl);
  if (P.N * P.Do * P.Ho * P.Wo >= (1ll << 31)) { set_error("tc: too many output pixels"); return ALT_E_UNSUPPORTED; }
  return tc_run(T, cfg, stream, used, 1, 0);
}

alt_status tc_conv(const ConvProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used) {
  if (P.c3d) return tc_conv3d(P, cfg, stream, used);
  if (P.dtype == ALT_F32) return tc_conv_f32(P, cfg, stream, used);
  if (P.dtype != ALT_BF16) { set_error("tc path: bf16 / fp32 only"); return ALT_E_UNSUPPORTED; }
  const int64_t G = P.groups < 1 ? 1 : P.groups;
  const int64_t Cg = P.C / G, Kg = P.K / G;
  if (G > 1 && (Cg % 8 || Kg % 8 || G == P.C)) {
    set_error("tc path: grouped conv needs C/groups and K/groups multiples of 8 (depthwise: the dw kernel)");
    return ALT_E_UNSUPPORTED;
  }
  TcProblem T{};
  T.is_conv = true;
  T.al = P.xl; T.bl = P.wl; T.yl = P.yl;
  T.a = P.x; T.b = P.w; T.y = P.y;
  // x logical (n, c, h, w); w logical (k, c, r, s); y logical (n, k, p, q)
  T.ra[0].role = R_N;
  T.ra[1].role = R_C;
  // dilation d: tap r adds d r to the box coordinate (the TMA coordinate
  // rule's V_R coefficient) and the window spans d (R - 1) + 1 rows
  T.ra[2] = RoleInfo{R_H, 1, P.Vh, P.ph, (int)((P.R - 1) * P.dh + 1), P.dh};
  T.ra[3] = RoleInfo{R_W, 1, P.Vw, P.pw, (int)((P.S - 1) * P.dw + 1), P.dw};
  T.rb[0] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.rb[1].role = R_C;
  T.rb[2].role = R_TR;
  T.rb[3].role = R_TS;
  T.ry[0].role = R_N;
  T.ry[1].role = R_C;
  T.ry[2] = RoleInfo{R_H, 1, 1, 0, 1, 0};
  T.ry[3] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.N = P.N; T.K = Kg; T.Ho = P.Ho; T.Wo = P.Wo;
  T.R = P.R; T.S = P.S; T.C = Cg;
  T.epi = P.epi;
  T.va = lview(*P.xl); T.vb = lview(*P.wl); T.vy = lview(*P.yl);
  {
    LView xf, wf;
    int64_t Cf = 0;
    if (G == 1 && P.dw == 1 && fold_window(T.va, T.vb, P.S, P.Vw, P.pw, P.Wo, &xf, &wf, &Cf)) {
      T.va = xf; T.vb = wf;
      T.ra[3] = RoleInfo{R_W, 1, 1, 0, 1, 0};
      T.S = 1; T.C = Cf;
    }
  }
  if (P.N * P.Ho * P.Wo >= (1ll << 31)) { set_error("tc: too many output pixels"); return ALT_E_UNSUPPORTED; }
  if (G == 1) return tc_run(T, cfg, stream, used, 0, 0);
  // grouped conv: one launch per group (the paper's GRP operator), each a
  // Cg -> Kg implicit GEMM reading its channel slabs of x, its weight rows
  // and writing its output channels through the same layouts
  for (int64_t g = 0; g < G; g++) {
    TcProblem Tg = T;
    Tg.coff = g * Cg;
    Tg.koff = g * Kg;
    if (T.epi.scale) Tg.epi.scale = T.epi.scale + g * Kg;
    if (T.epi.bias) Tg.epi.bias = T.epi.bias + g * Kg;
    const alt_status st = tc_run(Tg, cfg, stream, used, 0, 0);
    if (st != ALT_OK) return st;
  }
  return ALT_OK;
}

alt_status tc_gemm(const GemmProblem &P, const alt_kernel_cfg *cfg, cudaStream_t stream, alt_kernel_cfg *used) {
  if (P.dtype == ALT_F32) return tc_gemm_f32(P, cfg, stream, used);
  if (P.dtype != ALT_BF16) { set_error("tc path: bf16 / fp32 only"); return ALT_E_UNSUPPORTED; }
  TcProblem T{};
  T.is_conv = false;
  T.al = P.al; T.bl = P.bl; T.yl = P.cl;
  T.a = P.a; T.b = P.b; T.y = P.c;
  // A logical (m, k): m = rows (W role), k = reduction; B logical (k, n); C (m, n)
  T.ra[0] = RoleInfo{R_W, 128, 1, 0, 1, 0};
  T.ra[1].role = R_C;
  T.rb[0].role = R_C;
  T.rb[1] = RoleInfo{R_W, 1, 1, 0, 1, 0};
  T.ry[0] = RoleInfo{R_W, 128, 1, 0, 1, 0};
  T.ry[1].role = R_C;
  T.N = 1; T.K = P.N; T.Ho = 1; T.Wo = P.M;
  T.R = 1; T.S = 1; T.C = P.K;
  T.epi = P.epi;
  T.va = lview(*P.al); T.vb = lview(*P.bl); T.vy = lview(*P.cl);
  if (P.M >= (1ll << 31)) { set_error("tc: M too large"); return ALT_E_UNSUPPORTED; }
  return tc_run(T, cfg, stream, used, 1, 1);
}

}  // namespace alt
