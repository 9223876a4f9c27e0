// relayout.cu — the layout-conversion operator (paper Fig. 5a):
//   dst[j] = G_dst(j) is a structural zero ? 0 : src[F_src(G_dst(j))]
// for every physical position j of dst.  HBM-bound bit copy.
//
// Kernels (chosen on the host from the compiled layouts):
//   K_TILE    both layouts separable and dst's innermost logical dim (a)
//             differs from src's innermost logical dim (b): 2-D tiles over
//             (dst dim of b's lowest digit) x (dst innermost dim), staged
//             through shared memory so both the reads (contiguous along b in
//             src) and the writes (contiguous along a in dst) coalesce.  All
//             index math is two per-tile 1-D offset tables in smem.
//   K_VEC     both separable, runs of the dst innermost dim are contiguous
//             in src: one 4/8/16-byte vector per thread.
//   K_SEP     both separable, anything else: per-element table lookups.
//   K_GENERIC any layouts (e.g. fuse across logical dims): the
//             primitive interpreter per element.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdlib>
#include <mutex>
#include <vector>
#include <cstdio>

#include "common.cuh"

namespace alt {

struct SepPair {
  // dst physical dims (innermost last)
  int32_t prank;
  FastDiv pdiv[kMaxP];
  int32_t powner[kMaxP];
  int32_t prad[kMaxP];
  int32_t lrank;
  const int32_t *rev[kMaxL];   // dst reverse tables
  const int64_t *rd[kMaxL];    // src owner offsets
};

template <typename T>
__device__ __forceinline__ uint4 ld16(const T *p) { return __ldg(reinterpret_cast<const uint4 *>(p)); }

// Warp-cooperative store of per-lane contiguous runs.  Lane l holds NVO
// 16-byte vectors forming one contiguous dst run that starts at element
// offset off (-1: the lane stores nothing).  Written straight from registers,
// store instruction k would touch 32 runs 16 bytes each (32 partial lines per
// instruction); staged through this warp's shared buffer st[32 * NVO], store
// instruction k moves the warp's vectors [32k, 32k + 32) in lane order — one
// 512-byte span when the lanes' runs are adjacent, which they are except
// where a warp straddles a batch boundary.  Slots are XOR-swizzled so both
// the staging writes and the reads hit distinct banks per 8-lane phase.
template <typename T, int NVO>
__device__ __forceinline__ void warp_store_runs(uint4 *st, const uint4 (&w)[NVO], int64_t off, T *dst, int lane) {
  constexpr int VE = 16 / sizeof(T);
  auto key = [](int s) { return ((s * NVO) >> 3) & (NVO - 1); };
#pragma unroll
  for (int k = 0; k < NVO; k++) st[lane * NVO + (k ^ key(lane))] = w[k];
  __syncwarp();
#pragma unroll
  for (int k = 0; k < NVO; k++) {
    const int j = k * 32 + lane, s = j / NVO, r = j % NVO;
    const long long so = __shfl_sync(0xffffffffu, (long long)off, s);
    if (so >= 0) *reinterpret_cast<uint4 *>(dst + so + (int64_t)r * VE) = st[s * NVO + (r ^ key(s))];
  }
  __syncwarp();
}

// ------------------------------------------------------------------ K_SEP --
template <typename T, int V>
__global__ void __launch_bounds__(256) k_relayout_sep(SepPair P, const T *__restrict__ src,
                                                      T *__restrict__ dst, uint32_t nvec) {
  using Vec = typename std::conditional<
      V * sizeof(T) == 16, uint4,
      typename std::conditional<V * sizeof(T) == 8, uint2,
                                typename std::conditional<V * sizeof(T) == 4, uint32_t, T>::type>::type>::type;
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += gridDim.x * blockDim.x) {
    uint32_t rem = v * V;
    int32_t combo[kMaxL];
#pragma unroll
    for (int d = 0; d < kMaxL; d++) combo[d] = 0;
    for (int p = P.prank - 1; p >= 0; p--) {
      uint32_t q, r;
      P.pdiv[p].divmod(rem, q, r);
      combo[P.powner[p]] += (int32_t)r * P.prad[p];
      rem = q;
    }
    int64_t off = 0;
    bool ok = true;
    for (int d = 0; d < P.lrank; d++) {
      int32_t i = __ldg(P.rev[d] + combo[d]);
      if (i < 0) { ok = false; break; }
      off += __ldg(P.rd[d] + i);
    }
    Vec val;
    if (ok) val = *reinterpret_cast<const Vec *>(src + off);
    else memset(&val, 0, sizeof(Vec));
    reinterpret_cast<Vec *>(dst)[v] = val;
  }
}

// --------------------------------------------------------------- K_GATHER --
// One 16-byte dst vector per thread along the dst innermost dim (logical dim
// a); the other dims are decoded once per vector, the V elements gather
// through a's tables.  Neighbouring threads hold neighbouring vectors, so each
// of the V gathers is coalesced across the warp.  Serves pad / unfold layouts.
template <typename T>
__global__ void __launch_bounds__(256) k_relayout_gather(SepPair P, int32_t a, const T *__restrict__ src,
                                                         T *__restrict__ dst, uint32_t nvec) {
  constexpr int V = 16 / sizeof(T);
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += gridDim.x * blockDim.x) {
    uint32_t rem = v * V;
    int32_t combo[kMaxL];
#pragma unroll
    for (int d = 0; d < kMaxL; d++) combo[d] = 0;
    for (int p = P.prank - 1; p >= 0; p--) {
      uint32_t q, r;
      P.pdiv[p].divmod(rem, q, r);
      combo[P.powner[p]] += (int32_t)r * P.prad[p];
      rem = q;
    }
    int64_t base = 0;
    bool ok = true;
    for (int d = 0; d < P.lrank; d++) {
      if (d == a) continue;
      const int32_t i = __ldg(P.rev[d] + combo[d]);
      if (i < 0) { ok = false; break; }
      base += __ldg(P.rd[d] + i);
    }
    T val[V];
#pragma unroll
    for (int j = 0; j < V; j++) {
      val[j] = 0;
      if (ok) {
        const int32_t i = __ldg(P.rev[a] + combo[a] + j);
        if (i >= 0) val[j] = src[base + __ldg(P.rd[a] + i)];
      }
    }
    reinterpret_cast<uint4 *>(dst)[v] = *reinterpret_cast<const uint4 *>(val);
  }
}

// ----------------------------------------------------------------- K_GVEC --
// One 16-byte dst vector per thread for layouts whose innermost dst dims are
// too short for K_GATHER / K_TILE (e.g. a 4-channel run inside an unfolded
// window, reading A23): the physical coordinate is decoded once per vector
// and then stepped with carries; only the logical dims whose coordinate
// changed are looked up again.
template <typename T>
__global__ void __launch_bounds__(256) k_relayout_gvec(SepPair P, const T *__restrict__ src,
                                                       T *__restrict__ dst, uint32_t nvec) {
  // all per-dim arrays are indexed with compile-time indices (registers)
  constexpr int V = 16 / sizeof(T);
  for (uint32_t v = blockIdx.x * blockDim.x + threadIdx.x; v < nvec; v += gridDim.x * blockDim.x) {
    uint32_t rem = v * V;
    int32_t coord[kMaxP];
    int32_t combo[kMaxL];
#pragma unroll
    for (int d = 0; d < kMaxL; d++) combo[d] = 0;
#pragma unroll
    for (int p = kMaxP - 1; p >= 0; p--) {
      coord[p] = 0;
      if (p < P.prank) {
        uint32_t q, r;
        P.pdiv[p].divmod(rem, q, r);
        coord[p] = (int32_t)r;
#pragma unroll
        for (int d = 0; d < kMaxL; d++)
          if (P.powner[p] == d) combo[d] += (int32_t)r * P.prad[p];
        rem = q;
      }
    }
    int64_t part[kMaxL];
    uint32_t zero = 0;  // bit d: logical dim d sits on a structural zero
#pragma unroll
    for (int d = 0; d < kMaxL; d++) {
      part[d] = 0;
      if (d < P.lrank) {
        const int32_t i = __ldg(P.rev[d] + combo[d]);
        if (i < 0) zero |= 1u << d;
        else part[d] = __ldg(P.rd[d] + i);
      }
    }
    T val[V];
#pragma unroll
    for (int j = 0; j < V; j++) {
      int64_t off = 0;
#pragma unroll
      for (int d = 0; d < kMaxL; d++) off += part[d];
      val[j] = zero ? T(0) : src[off];
      if (j + 1 < V) {
        uint32_t dirty = 0;
        bool carry = true;
#pragma unroll
        for (int p = kMaxP - 1; p >= 0; p--) {
          if (carry && p < P.prank) {
            const int o = P.powner[p];
            dirty |= 1u << o;
            const int32_t c = coord[p] + 1;
            const bool wrap = c >= (int32_t)P.pdiv[p].d;
            coord[p] = wrap ? 0 : c;
            const int32_t delta = wrap ? -(c - 1) * P.prad[p] : P.prad[p];
#pragma unroll
            for (int d = 0; d < kMaxL; d++)
              if (o == d) combo[d] += delta;
            carry = wrap;
          }
        }
#pragma unroll
        for (int d = 0; d < kMaxL; d++) {
          if (d < P.lrank && (dirty >> d & 1)) {
            const int32_t i = __ldg(P.rev[d] + combo[d]);
            part[d] = i < 0 ? 0 : __ldg(P.rd[d] + i);
            zero = i < 0 ? (zero | 1u << d) : (zero & ~(1u << d));
          }
        }
      }
    }
    reinterpret_cast<uint4 *>(dst)[v] = *reinterpret_cast<const uint4 *>(val);
  }
}

// ----------------------------------------------------------------- K_TILE --
struct TilePlan {
  SepPair P;
  int32_t p0, p1;        // dst dims: innermost (x) and b's lowest digit (y)
  int32_t a, b;          // logical dims of p0 / p1
  int32_t TX, TY;        // tile extents along p0 / p1
  int32_t nx, ny;        // number of chunks along p0 / p1
  int64_t dstride_p1;    // dst stride of p1
  uint32_t ntiles;
  int32_t nouter;        // dims other than p0, p1 (outer first)
  int32_t outer[kMaxP];
  FastDiv odiv[kMaxP];
  int64_t ostride[kMaxP];
  FastDiv nxdiv, nydiv;
  int32_t ey_total;      // extent of p1
};

template <typename T>
__global__ void __launch_bounds__(256) k_relayout_tile(TilePlan TP, const T *__restrict__ src,
                                                       T *__restrict__ dst) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  const int TX = TP.TX, TY = TP.TY;
  const int LD = TX + (sizeof(T) == 2 ? 2 : 1);        // row pitch (elements), breaks bank conflicts
  T *tile = reinterpret_cast<T *>(smem_raw);
  int64_t *offA = reinterpret_cast<int64_t *>(smem_raw + (((size_t)TY * LD * sizeof(T) + 15) & ~size_t(15)));
  int64_t *offB = offA + TX;
  __shared__ int64_t s_src_base, s_dst_base;
  __shared__ int32_t s_comboA, s_comboB, s_ok, s_ey;
  const SepPair &P = TP.P;

  for (uint32_t t = blockIdx.x; t < TP.ntiles; t += gridDim.x) {
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t rem = t, q, r;
      TP.nxdiv.divmod(rem, q, r);
      const int32_t cx = (int32_t)r;
      rem = q;
      TP.nydiv.divmod(rem, q, r);
      const int32_t cy = (int32_t)r;
      rem = q;
      int32_t combo[kMaxL];
      for (int d = 0; d < kMaxL; d++) combo[d] = 0;
      int64_t dbase = (int64_t)cx * TX + (int64_t)cy * TY * TP.dstride_p1;
      for (int k = TP.nouter - 1; k >= 0; k--) {
        const int p = TP.outer[k];
        TP.odiv[k].divmod(rem, q, r);
        rem = q;
        combo[P.powner[p]] += (int32_t)r * P.prad[p];
        dbase += (int64_t)r * TP.ostride[k];
      }
      int64_t sbase = 0;
      int ok = 1;
      for (int d = 0; d < P.lrank; d++) {
        if (d == TP.a || d == TP.b) continue;
        const int32_t i = P.rev[d][combo[d]];
        if (i < 0) { ok = 0; break; }
        sbase += P.rd[d][i];
      }
      s_src_base = sbase;
      s_dst_base = dbase;
      s_comboA = combo[TP.a] + cx * TX * P.prad[TP.p0];
      s_comboB = combo[TP.b] + cy * TY * P.prad[TP.p1];
      s_ok = ok;
      s_ey = min(TY, TP.ey_total - cy * TY);
    }
    __syncthreads();
    const int64_t dbase = s_dst_base;
    const int ok = s_ok;
    const int ey = s_ey;
    if (ok) {
      for (int x = threadIdx.x; x < TX; x += blockDim.x) {
        int32_t i = P.rev[TP.a][s_comboA + x * P.prad[TP.p0]];
        offA[x] = i < 0 ? INT64_MIN / 4 : P.rd[TP.a][i];
      }
      for (int y = threadIdx.x; y < TY; y += blockDim.x) {
        int32_t i = y < ey ? P.rev[TP.b][s_comboB + y * P.prad[TP.p1]] : -1;
        offB[y] = i < 0 ? INT64_MIN / 4 : P.rd[TP.b][i];
      }
      __syncthreads();
      const int64_t sbase = s_src_base;
      // read phase: consecutive threads walk y (contiguous in src)
      for (int e = threadIdx.x; e < TX * TY; e += blockDim.x) {
        int y = e % TY, x = e / TY;
        int64_t o = offA[x] + offB[y];
        T v = 0;
        if (o >= 0) v = src[sbase + o];
        tile[y * LD + x] = v;
      }
    } else {
      for (int e = threadIdx.x; e < TX * TY; e += blockDim.x) tile[(e / TX) * LD + (e % TX)] = 0;
    }
    __syncthreads();
    // write phase: consecutive threads walk x (contiguous in dst)
    for (int e = threadIdx.x; e < TX * ey; e += blockDim.x) {
      int x = e % TX, y = e / TX;
      dst[dbase + (int64_t)y * TP.dstride_p1 + x] = tile[y * LD + x];
    }
  }
}

// -------------------------------------------------------------- K_GENERIC --
template <typename T>
__global__ void __launch_bounds__(256) k_relayout_generic(const LayoutDesc *__restrict__ S,
                                                          const LayoutDesc *__restrict__ D,
                                                          const T *__restrict__ src, T *__restrict__ dst,
                                                          int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n;
       j += (int64_t)gridDim.x * blockDim.x) {
    int64_t c[kStageRank];
    int64_t rem = j;
    for (int p = D->prank - 1; p >= 0; p--) {
      int64_t e = D->shp[D->np][p];
      c[p] = rem % e;
      rem /= e;
    }
    T v = 0;
    if (dev_G(*D, c)) {
      int64_t o = dev_F_offset(*S, c);
      if (o >= 0) v = src[o];
    }
    dst[j] = v;
  }
}

// ------------------------------------------------------------------- host --
static int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

static bool fill_pair(Layout *S, Layout *D, const SepDev &ss, const SepDev &ds, SepPair *P) {
  if (D->pnumel >= (1ll << 31)) return false;
  P->prank = D->prank;
  for (int p = 0; p < D->prank; p++) {
    P->pdiv[p] = FastDiv((uint32_t)D->pshape[p]);
    P->powner[p] = D->pdim_owner[p];
    P->prad[p] = D->pdim_rad[p];
  }
  P->lrank = D->lrank;
  for (int d = 0; d < D->lrank; d++) {
    P->rev[d] = ds.rev[d];
    P->rd[d] = ss.rd[d];
  }
  return true;
}


// ------------------------------------------------------------------ K_ROW --
// dst's innermost physical dims hold only the src-contiguous logical dim b
// (any pad / unfold / split of it) and one dim p0 of logical dim a (dst
// innermost, X elements).  For every combination of the other ("outer") dst
// dims the CTA stages the X src rows it needs — a index rev_a(outer_a + j),
// the window of b the block touches, read coalesced (16-byte vectors) along
// b — into shared memory as [X][window], then writes the contiguous dst block
// of that outer index as 16-byte vectors made of whole X-runs, each X-run's
// b index looked up through rev_b(outer_b + suffix_b(pos)).  Serves the conv
// input templates (pad + unfold + NCHW[x]c, Fig. 5 / §5.1), padded-channel
// and window-folded image layouts.
struct RowPlan {
  int32_t a, b;            // logical dims of p0 / of the suffix
  int32_t X, Lb;           // extent of p0, logical extent of b
  int32_t LbS;             // staged row pitch (elements, multiple of 16 B)
  int32_t span;            // staged window length (elements, multiple of V)
  int32_t npos;            // dst positions per outer index (excluding p0)
  int32_t nout;            // outer dims (innermost last)
  FastDiv odiv[kMaxP];
  int32_t oowner[kMaxP], orad[kMaxP];
  uint32_t nouter;         // number of outer indices
  int32_t per_iter;        // outer indices staged per CTA iteration
  int32_t lrank;
  const int32_t *rev[kMaxL];   // dst reverse tables
  const int64_t *rd[kMaxL];    // src owner offsets
  const int32_t *sbc;          // [npos] suffix part of b's combo
  const int32_t *blo;          // [footprint_b] window start per outer b combo
  int32_t vec_load;            // src rows loadable as 16-byte vectors along b
  int32_t lgX;                 // log2 X
  FastDiv f_nv, f_span, f_vpb;  // span / V, span, blk / V
  int32_t bstatic;             // b has no outer dims: sbc holds the b index itself (or -1)
};

// RB = 0: rows staged as [X][window] (any X).  RB = 8 / 16 (X * sizeof(T)
// bytes, vector loads): each thread loads one 16-byte b-vector of all X rows
// and transposes it in registers, so the stage holds [window][X] — every
// X-run of the dst is one 8 / 16-byte shared load in the write phase.  Runs
// are stored at slot b ^ ((b / V) & (V - 1)) within each V-run group, which
// spreads a warp's stores (lane stride V runs) over the banks.
template <typename T, int RB>
__global__ void __launch_bounds__(256) k_relayout_row(RowPlan R, const T *__restrict__ src, T *__restrict__ dst) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  T *rows = reinterpret_cast<T *>(smem_raw);  // [per_iter][X][LbS]
  __shared__ int64_t s_base[64];              // per staged outer index: src offset of (a, b) = (0, 0)
  __shared__ int32_t s_acombo[64];            // outer part of a's combo, or -1 for an all-zero block
  __shared__ int32_t s_bcombo[64], s_lo[64];  // outer part of b's combo, window start
  constexpr int V = 16 / sizeof(T);
  pdl_wait();
  const int X = R.X, LbS = R.LbS, span = R.span;
  const int blk = R.npos * X;                 // dst elements per outer index
  const int rows_per = X * LbS;
  for (uint32_t o0 = blockIdx.x * R.per_iter; o0 < R.nouter; o0 += gridDim.x * R.per_iter) {
    const int cnt = (int)min((uint32_t)R.per_iter, R.nouter - o0);
    __syncthreads();
    if (threadIdx.x < cnt) {
      uint32_t rem = o0 + threadIdx.x;
      int32_t combo[kMaxL];
#pragma unroll
      for (int d = 0; d < kMaxL; d++) combo[d] = 0;
      for (int k = R.nout - 1; k >= 0; k--) {
        uint32_t q, r;
        R.odiv[k].divmod(rem, q, r);
        combo[R.oowner[k]] += (int32_t)r * R.orad[k];
        rem = q;
      }
      int64_t base = 0;
      bool ok = true;
      for (int d = 0; d < R.lrank; d++) {
        if (d == R.a || d == R.b) continue;
        const int32_t i = __ldg(R.rev[d] + combo[d]);
        if (i < 0) { ok = false; break; }
        base += __ldg(R.rd[d] + i);
      }
      s_base[threadIdx.x] = base;
      s_acombo[threadIdx.x] = ok ? combo[R.a] : -1;
      s_bcombo[threadIdx.x] = combo[R.b];
      s_lo[threadIdx.x] = __ldg(R.blo + combo[R.b]);
    }
    __syncthreads();
    // stage: element (o, j, bi) -> rows[o][j][bi - lo]; flat over (row, vector)
    // so every thread has work for any window length; b fastest (coalesced)
    if constexpr (RB > 0) {
      constexpr int XR = RB / sizeof(T);  // == X
      const int nv = span / V;
      for (int e = threadIdx.x; e < cnt * nv; e += blockDim.x) {
        const int o = (int)R.f_nv.div((uint32_t)e), bv = e - o * nv;
        const int ac = s_acombo[o];
        const int b0 = s_lo[o] + bv * V;
        uint4 u[XR];
#pragma unroll
        for (int j = 0; j < XR; j++) {
          const int32_t ai = (ac < 0 || b0 >= R.Lb) ? -1 : __ldg(R.rev[R.a] + ac + j);
          u[j] = make_uint4(0u, 0u, 0u, 0u);
          if (ai >= 0) u[j] = __ldg(reinterpret_cast<const uint4 *>(src + s_base[o] + __ldg(R.rd[R.a] + ai) + b0));
        }
        unsigned char *ob = reinterpret_cast<unsigned char *>(rows + (size_t)o * rows_per);
#pragma unroll
        for (int k = 0; k < V; k++) {
          const int bl = bv * V + k;
          const int slot = bl ^ ((bl / V) & (V - 1));
          uint32_t w[RB / 4];
          if constexpr (sizeof(T) == 2) {
            // run k = element k of every row j: 16-bit transpose with byte_perm
            const uint32_t sel = (k & 1) ? 0x7632u : 0x5410u;
#pragma unroll
            for (int jp = 0; jp < XR / 2; jp++) {
              const uint32_t *a0 = reinterpret_cast<const uint32_t *>(&u[2 * jp]);
              const uint32_t *a1 = reinterpret_cast<const uint32_t *>(&u[2 * jp + 1]);
              w[jp] = __byte_perm(a0[k >> 1], a1[k >> 1], sel);
            }
          } else {
#pragma unroll
            for (int j = 0; j < XR; j++) w[j] = reinterpret_cast<const uint32_t *>(&u[j])[k];
          }
          if constexpr (RB == 16)
            *reinterpret_cast<uint4 *>(ob + (size_t)slot * 16) = make_uint4(w[0], w[1], w[2], w[3]);
          else
            *reinterpret_cast<uint2 *>(ob + (size_t)slot * 8) = make_uint2(w[0], w[1]);
        }
      }
    } else if (R.vec_load) {
      const int nv = span / V;
      for (int e = threadIdx.x; e < cnt * X * nv; e += blockDim.x) {
        const int row = (int)R.f_nv.div((uint32_t)e), bv = e - row * nv;
        const int o = row >> R.lgX, j = row & (X - 1);
        const int ac = s_acombo[o];
        const int b0 = s_lo[o] + bv * V;
        const int32_t ai = (ac < 0 || b0 >= R.Lb) ? -1 : __ldg(R.rev[R.a] + ac + j);
        uint4 u = make_uint4(0u, 0u, 0u, 0u);
        if (ai >= 0) u = __ldg(reinterpret_cast<const uint4 *>(src + s_base[o] + __ldg(R.rd[R.a] + ai) + b0));
        *reinterpret_cast<uint4 *>(rows + (size_t)o * rows_per + (size_t)j * LbS + bv * V) = u;
      }
    } else {
      for (int e = threadIdx.x; e < cnt * X * span; e += blockDim.x) {
        const int row = (int)R.f_span.div((uint32_t)e), bl = e - row * span;
        const int o = row >> R.lgX, j = row & (X - 1);
        const int ac = s_acombo[o];
        const int bi = s_lo[o] + bl;
        const int32_t ai = (ac < 0 || bi >= R.Lb) ? -1 : __ldg(R.rev[R.a] + ac + j);
        rows[(size_t)o * rows_per + (size_t)j * LbS + bl] =
            ai < 0 ? T(0) : src[s_base[o] + __ldg(R.rd[R.a] + ai) + bi];
      }
    }
    __syncthreads();
    // write: 16-byte vectors of the contiguous dst blocks of the cnt outer
    // indices (they are consecutive, so the cnt blocks are one dst range)
    T *dblk = dst + (int64_t)o0 * blk;
    const int vpb = blk / V;  // vectors per block
    for (int v = threadIdx.x; v < cnt * vpb; v += blockDim.x) {
      const int o = (int)R.f_vpb.div((uint32_t)v), w = (v - o * vpb) * V;
      const T *rb = rows + (size_t)o * rows_per;
      const int bc = s_bcombo[o], lo = s_lo[o];
      T val[V] = {};
      if constexpr (RB > 0) {
        const unsigned char *ob = reinterpret_cast<const unsigned char *>(rb);
        constexpr int RUNS = 16 / RB;  // X-runs per 16-byte dst vector
        uint32_t wv[4];
#pragma unroll
        for (int r = 0; r < RUNS; r++) {
          const int pos = (w >> R.lgX) + r;
          const int32_t bi = R.bstatic ? __ldg(R.sbc + pos) : __ldg(R.rev[R.b] + bc + __ldg(R.sbc + pos));
          const int bl = bi - lo;
          const int slot = bl ^ ((bl / V) & (V - 1));
          if constexpr (RB == 16) {
            uint4 q = make_uint4(0u, 0u, 0u, 0u);
            if (bi >= 0) q = *reinterpret_cast<const uint4 *>(ob + (size_t)slot * 16);
            wv[0] = q.x; wv[1] = q.y; wv[2] = q.z; wv[3] = q.w;
          } else {
            uint2 q = make_uint2(0u, 0u);
            if (bi >= 0) q = *reinterpret_cast<const uint2 *>(ob + (size_t)slot * 8);
            wv[2 * r] = q.x; wv[2 * r + 1] = q.y;
          }
        }
        *reinterpret_cast<uint4 *>(dblk + (int64_t)v * V) = make_uint4(wv[0], wv[1], wv[2], wv[3]);
        continue;
      } else if (X >= V) {
        const int pos = w >> R.lgX, j0 = w & (X - 1);
        const int32_t bi = R.bstatic ? __ldg(R.sbc + pos) : __ldg(R.rev[R.b] + bc + __ldg(R.sbc + pos));
#pragma unroll
        for (int k = 0; k < V; k++) val[k] = bi < 0 ? T(0) : rb[(size_t)(j0 + k) * LbS + (bi - lo)];
      } else {
        const int pos0 = w >> R.lgX;
#pragma unroll
        for (int k = 0; k < V; k++) {
          const int pos = pos0 + (k >> R.lgX), j = k & (X - 1);
          const int32_t bi = R.bstatic ? __ldg(R.sbc + pos) : __ldg(R.rev[R.b] + bc + __ldg(R.sbc + pos));
          val[k] = bi < 0 ? T(0) : rb[(size_t)j * LbS + (bi - lo)];
        }
      }
      *reinterpret_cast<uint4 *>(dblk + (int64_t)v * V) = *reinterpret_cast<const uint4 *>(val);
    }
  }
}


// K_ROW, identity suffix (dst positions = the b indices in order, e.g. the
// padded-channel image layout N C/8 H W 8c) with 16- or 32-byte X-runs: no
// shared-memory transpose —
// a thread loads one 16-byte b-vector of each of the X rows (pad rows are
// zeros), transposes it in registers and stores the V runs, which are
// adjacent in dst.  Neighbouring threads take neighbouring b-vectors.
// X = V (16-byte runs) or, for fp32, 2 V (32-byte runs: 8 channels); a
// thread's V runs (V X elements) are one contiguous dst span, written through
// warp_store_runs.
template <typename T, int X>
__global__ void __launch_bounds__(256) k_relayout_row_ident(RowPlan R, const T *__restrict__ src,
                                                            T *__restrict__ dst, uint32_t nthr) {
  pdl_wait();
  constexpr int V = 16 / sizeof(T);
  constexpr int NVO = X;  // 16-byte output vectors per thread: V runs of X elements
  __shared__ uint4 stage[8][32 * NVO];
  const int lane = threadIdx.x & 31;
  uint4 *st = stage[threadIdx.x >> 5];
  const uint32_t nv = (uint32_t)(R.Lb / V);
  for (uint32_t t0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u); t0 < nthr; t0 += gridDim.x * blockDim.x) {
    const uint32_t t = t0 + lane;
    uint4 w[NVO];
    int64_t off = -1;
    if (t < nthr) {
    const uint32_t o = t / nv, bv = t - o * nv;
    uint32_t rem = o;
    int32_t combo[kMaxL];
#pragma unroll
    for (int d = 0; d < kMaxL; d++) combo[d] = 0;
    for (int k = R.nout - 1; k >= 0; k--) {
      uint32_t q, r;
      R.odiv[k].divmod(rem, q, r);
      combo[R.oowner[k]] += (int32_t)r * R.orad[k];
      rem = q;
    }
    int64_t base = 0;
    bool ok = true;
    for (int d = 0; d < R.lrank; d++) {
      if (d == R.a || d == R.b) continue;
      const int32_t i = __ldg(R.rev[d] + combo[d]);
      if (i < 0) { ok = false; break; }
      base += __ldg(R.rd[d] + i);
    }
    uint4 u[X];
#pragma unroll
    for (int j = 0; j < X; j++) {
      const int32_t ai = ok ? __ldg(R.rev[R.a] + combo[R.a] + j) : -1;
      u[j] = ai < 0 ? make_uint4(0u, 0u, 0u, 0u)
                    : __ldg(reinterpret_cast<const uint4 *>(src + base + __ldg(R.rd[R.a] + ai) + (int64_t)bv * V));
    }
    // run k = element k of rows 0 .. X-1 (X / V vectors)
#pragma unroll
    for (int k = 0; k < V; k++) {
#pragma unroll
      for (int h = 0; h < X / V; h++) {
        uint32_t ww[4];
        if constexpr (sizeof(T) == 2) {
          const uint32_t sel = (k & 1) ? 0x7632u : 0x5410u;
#pragma unroll
          for (int jp = 0; jp < 4; jp++)
            ww[jp] = __byte_perm(reinterpret_cast<const uint32_t *>(&u[h * V + 2 * jp])[k >> 1],
                                 reinterpret_cast<const uint32_t *>(&u[h * V + 2 * jp + 1])[k >> 1], sel);
        } else {
#pragma unroll
          for (int j = 0; j < 4; j++) ww[j] = reinterpret_cast<const uint32_t *>(&u[h * V + j])[k];
        }
        w[k * (X / V) + h] = make_uint4(ww[0], ww[1], ww[2], ww[3]);
      }
    }
    off = (int64_t)o * (R.npos * X) + (int64_t)bv * V * X;
    }
    warp_store_runs<T, NVO>(st, w, off, dst, lane);
  }
}

// ------------------------------------------------------------------ K_WIN --
// Group form of K_ROW for the conv input templates (pad + unfold of H and W
// + NCHW[x]c, Fig. 5 / §5.1; window-folded images).  dst's
// innermost physical dims G = [pg, p0] (p0: the X-run of logical dim a) are
// one contiguous dst block per outer index.  The rows the block reads are
// the combinations of G's dims not owned by the src-contiguous dim b (x the
// X run); each is staged once per block over the b window the block touches
// (whole rows when G holds every b dim), 16-byte coalesced loads, pad rows
// as zeros.  The write phase then emits every X-run of the block as 16-byte
// vectors with one b-table lookup per run.  K_ROW stages a separate window
// per innermost outer index (for the 8 x 8 unfold template: 10 x overlapping
// windows and per-element lookups; ncu: instruction-bound at 62 % SM busy).
constexpr int kWinG = 6;
struct WinPlan {
  int32_t a, b;
  int32_t X, Lb, LbS, span;    // run length, b extent, staged row pitch, window (elements)
  int32_t nvs;                 // 16-byte vectors per staged row
  int32_t ng;                  // G dims above p0 (dst order, innermost last)
  FastDiv gdiv[kWinG];
  int32_t gowner[kWinG], grad[kWinG];
  int32_t nrq;                 // row groups (product of G's non-b dims above p0)
  int32_t nrun;                // X-runs per block
  int32_t nbg;                 // combinations of G's b coordinates
  int32_t nout;
  FastDiv odiv[kMaxP];
  int32_t oowner[kMaxP], orad[kMaxP];
  uint32_t nouter;
  int32_t lrank;
  const int32_t *rev[kMaxL];
  const int64_t *rd[kMaxL];
  const int32_t *blo;          // window start per outer b combo
  FastDiv f_x, f_nvs;
  // per-block offset tables: for every logical dim d != b owning G dims (a
  // always: p0 is its innermost), T_d[local] = rd_d[rev_d(outer_d + G part)]
  // over d's G coordinates (mixed radix, innermost first); a staged row's src
  // offset is base + sum_d T_d[local_d] — a few dozen lookups per block
  // instead of a dependent rev -> rd chain per dim for each of its rows
  int32_t nt;                  // tables
  int32_t tdim[kMaxL];         // logical dim of table t
  int32_t toff[kMaxL + 1];     // entry offsets (prefix sums)
  int32_t tn[kMaxL];           // coordinates of table t
  FastDiv text[kMaxL][kWinG + 1];
  int32_t trad[kMaxL][kWinG + 1];
  int32_t gti[kWinG];          // table of G dim k's owner (-1: b)
  int32_t gmul[kWinG];         // place value of G dim k in its table's local index
  int32_t ati;                 // table of a (local index = a's G part * X + j)
  uint32_t notab;              // bit d: logical dim d (!= b) has no G dims (block base only)
};

// outer index o -> per-logical-dim combos of the outer dims
__device__ __forceinline__ void win_outer(const WinPlan &P, uint32_t o, int32_t (&combo)[kMaxL]) {
#pragma unroll
  for (int d = 0; d < kMaxL; d++) combo[d] = 0;
  for (int k = P.nout - 1; k >= 0; k--) {
    uint32_t q, r;
    P.odiv[k].divmod(o, q, r);
    combo[P.oowner[k]] += (int32_t)r * P.orad[k];
    o = q;
  }
}

template <typename T, int X>
__global__ void __launch_bounds__(512) k_relayout_win(WinPlan P, const T *__restrict__ src, T *__restrict__ dst) {
  extern __shared__ __align__(16) unsigned char win_smem[];
  const int ntab = P.toff[P.nt];
  int64_t *s_tab = reinterpret_cast<int64_t *>(win_smem);                     // [ntab]
  int32_t *s_bsl = reinterpret_cast<int32_t *>(win_smem + (size_t)ntab * 8);  // [nbg] run slot of G's b coords
  // runs staged transposed: [rq][window slot][X], the slots of a row
  // XOR-swizzled within each V-run group (conflict-free staging stores)
  uint4 *runs = reinterpret_cast<uint4 *>(win_smem + (((size_t)ntab * 8 + (size_t)P.nbg * 4 + 15) & ~size_t(15)));
  __shared__ int64_t s_base;
  constexpr int V = 16 / sizeof(T);
  constexpr int NV = X / V;                         // 16-byte vectors per run (1 or 2)
  auto slot = [](int bl) { return bl ^ ((bl / V) & (V - 1)); };
  pdl_wait();
  const int64_t blk = (int64_t)P.nrun * X;
  for (uint32_t o = blockIdx.x; o < P.nouter; o += gridDim.x) {
    int32_t oc[kMaxL];
    win_outer(P, o, oc);
    const int lo = __ldg(P.blo + oc[P.b]);
    __syncthreads();  // the previous block's runs are consumed
    if (threadIdx.x == 0) {
      int64_t base = 0;
      for (int d = 0; d < P.lrank; d++) {
        if (!((P.notab >> d) & 1u)) continue;
        const int32_t i = __ldg(P.rev[d] + oc[d]);
        if (i < 0) { base = -1; break; }
        base += __ldg(P.rd[d] + i);
      }
      s_base = base;
    }
    for (int e = threadIdx.x; e < ntab; e += blockDim.x) {
      int t = 0;
      while (e >= P.toff[t + 1]) t++;
      uint32_t rem = (uint32_t)(e - P.toff[t]);
      int32_t sub = 0;
      for (int k = 0; k < P.tn[t]; k++) {
        uint32_t q, r;
        P.text[t][k].divmod(rem, q, r);
        sub += (int32_t)r * P.trad[t][k];
        rem = q;
      }
      const int d = P.tdim[t];
      const int32_t i = __ldg(P.rev[d] + oc[d] + sub);
      s_tab[e] = i < 0 ? -1 : __ldg(P.rd[d] + i);
    }
    for (int g = threadIdx.x; g < P.nbg; g += blockDim.x) {
      uint32_t rem = (uint32_t)g;
      int32_t cb = oc[P.b];
      for (int k = P.ng - 1; k >= 0; k--) {
        if (P.gowner[k] != P.b) continue;
        uint32_t q, rr;
        P.gdiv[k].divmod(rem, q, rr);
        cb += (int32_t)rr * P.grad[k];
        rem = q;
      }
      const int32_t bi = __ldg(P.rev[P.b] + cb);
      s_bsl[g] = bi < 0 ? -1 : slot(bi - lo);
    }
    __syncthreads();
    const int64_t base = s_base;
    // stage: item (rq, b-vector v) loads the X rows' 16-byte vectors at
    // b0 = lo + v V and transposes them into V runs of X elements
    for (int e = threadIdx.x; e < P.nrq * P.nvs; e += blockDim.x) {
      const int rq = (int)P.f_nvs.div((uint32_t)e), v = e - rq * P.nvs;
      const int b0 = lo + v * V;
      int loc[kMaxL];
#pragma unroll
      for (int t = 0; t < kMaxL; t++) loc[t] = 0;
      uint32_t rem = (uint32_t)rq;
      for (int k = P.ng - 1; k >= 0; k--) {
        if (P.gti[k] < 0) continue;
        uint32_t q, rr;
        P.gdiv[k].divmod(rem, q, rr);
        loc[P.gti[k]] += (int)rr * P.gmul[k];
        rem = q;
      }
      int64_t off = base;
      for (int t = 0; t < P.nt && off >= 0; t++) {
        if (t == P.ati) continue;
        const int64_t x = s_tab[P.toff[t] + loc[t]];
        off = x < 0 ? -1 : off + x;
      }
      const int64_t *ta = s_tab + P.toff[P.ati] + loc[P.ati] * X;
      uint4 u[X];
#pragma unroll
      for (int j = 0; j < X; j++) {
        const int64_t xa = ta[j];
        u[j] = (off < 0 || xa < 0 || b0 >= P.Lb) ? make_uint4(0u, 0u, 0u, 0u) : ld16(src + off + xa + b0);
      }
      uint4 *rrow = runs + (size_t)rq * P.LbS * NV;
#pragma unroll
      for (int k = 0; k < V; k++) {
        const int sl = slot(v * V + k);
#pragma unroll
        for (int h = 0; h < NV; h++) {
          uint32_t ww[4];
          if constexpr (sizeof(T) == 2) {
            const uint32_t sel = (k & 1) ? 0x7632u : 0x5410u;
#pragma unroll
            for (int jp = 0; jp < 4; jp++)
              ww[jp] = __byte_perm(reinterpret_cast<const uint32_t *>(&u[h * V + 2 * jp])[k >> 1],
                                   reinterpret_cast<const uint32_t *>(&u[h * V + 2 * jp + 1])[k >> 1], sel);
          } else {
#pragma unroll
            for (int jj = 0; jj < 4; jj++) ww[jj] = reinterpret_cast<const uint32_t *>(&u[h * V + jj])[k];
          }
          rrow[sl * NV + h] = make_uint4(ww[0], ww[1], ww[2], ww[3]);
        }
      }
    }
    __syncthreads();
    T *db = dst + (int64_t)o * blk;
    for (int q = threadIdx.x; q < P.nrun; q += blockDim.x) {
      uint32_t rem = (uint32_t)q;
      int rq = 0, rmul = 1, gb = 0, gmul = 1;
      for (int k = P.ng - 1; k >= 0; k--) {
        uint32_t qq, rr;
        P.gdiv[k].divmod(rem, qq, rr);
        if (P.gowner[k] == P.b) { gb += (int)rr * gmul; gmul *= (int)P.gdiv[k].d; }
        else { rq += (int)rr * rmul; rmul *= (int)P.gdiv[k].d; }
        rem = qq;
      }
      const int sl = s_bsl[gb];
      const uint4 *rr = runs + ((size_t)rq * P.LbS + (sl < 0 ? 0 : sl)) * NV;
#pragma unroll
      for (int h = 0; h < NV; h++)
        *reinterpret_cast<uint4 *>(db + (int64_t)q * X + h * V) = sl < 0 ? make_uint4(0u, 0u, 0u, 0u) : rr[h];
    }
  }
}

// host side of K_WIN: false (nothing launched) when the layouts do not fit
static bool win_launch(Layout *S, const void *src, Layout *D, void *dst, int wb, const SepDev &ss,
                       const SepDev &ds, cudaStream_t stream, int nsm, alt_status *st) {
  const int V = 16 / wb;
  if (D->prank < 3 || D->pnumel >= (1ll << 31)) return false;
  if ((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src)) & 15) return false;
  const int p0 = D->prank - 1;
  const int a = D->pdim_owner[p0];
  const int b = S->pdim_owner[S->prank - 1];
  if (D->pdim_rad[p0] != 1 || a == b || D->pdim_owner[p0 - 1] != b) return false;
  const int64_t X = D->pshape[p0];
  if (!(X * wb == 16 || X * wb == 32)) return false;
  // measured (R3, 256 x 64 x 56 x 56, 512-thread CTAs): bf16 101 us vs
  // K_ROW 167 us; fp32 316 us at this budget (its whole-row group does not
  // fit) and 200 us at 200 KB, i.e. no better than K_ROW's 194 us, so fp32
  // stays on K_ROW unless forced (ALT_WIN_FP32=1)
  static const bool win_f32 = getenv("ALT_WIN_FP32") != nullptr;
  if (wb == 4 && !win_f32) return false;
  const int64_t Lb = S->lshape[b];
  if (Lb % V || Lb >= (1 << 20)) return false;
  for (int64_t i = 0; i < Lb; i++) if (S->rd[b][i] != i) return false;  // b contiguous in src
  for (int d = 0; d < S->lrank; d++) {
    if (d == b) continue;
    for (int64_t o : S->rd[d]) if (o >= 0 && o % V) return false;   // rows start on 16 bytes
  }
  // the largest group G = [pg, p0] whose staged rows fit the budget
  // budget: staged bytes per CTA (a larger group removes the window overlap
  // between neighbouring blocks but lowers residency); developer knob
  static const size_t budget = getenv("ALT_WIN_BUDGET") ? (size_t)atol(getenv("ALT_WIN_BUDGET")) : 110 * 1000;
  int best_pg = -1;
  int64_t best_span = 0, best_nrq = 0, best_ngb = 0;
  std::vector<int32_t> best_blo;
  for (int pg = p0 - 1; pg >= 1 && p0 - pg <= kWinG; pg--) {
    int64_t nrq = 1;
    for (int p = pg; p < p0; p++) if (D->pdim_owner[p] != b) nrq *= D->pshape[p];
    // window per outer b combo: the b indices the block's G coordinates reach
    std::vector<int> bo, bg;
    for (int p = 0; p < pg; p++) if (D->pdim_owner[p] == b) bo.push_back(p);
    for (int p = pg; p < p0; p++) if (D->pdim_owner[p] == b) bg.push_back(p);
    int64_t nob = 1, ngb = 1;
    for (int p : bo) nob *= D->pshape[p];
    for (int p : bg) ngb *= D->pshape[p];
    if (nob * ngb > (1 << 22)) continue;
    std::vector<int32_t> blo((size_t)D->rev[b].size(), 0);
    int64_t span = 0;
    for (int64_t k = 0; k < nob; k++) {
      int64_t rem = k, ob = 0;
      for (int t = (int)bo.size() - 1; t >= 0; t--) {
        ob += (rem % D->pshape[bo[(size_t)t]]) * D->pdim_rad[bo[(size_t)t]];
        rem /= D->pshape[bo[(size_t)t]];
      }
      int64_t lo = INT64_MAX, hi = -1;
      for (int64_t g = 0; g < ngb; g++) {
        int64_t rg = g, cbv = ob;
        for (int t = (int)bg.size() - 1; t >= 0; t--) {
          cbv += (rg % D->pshape[bg[(size_t)t]]) * D->pdim_rad[bg[(size_t)t]];
          rg /= D->pshape[bg[(size_t)t]];
        }
        const int32_t bi = D->rev[b][(size_t)cbv];
        if (bi >= 0) { lo = std::min<int64_t>(lo, bi); hi = std::max<int64_t>(hi, bi); }
      }
      if (hi < 0) lo = hi = 0;
      lo = lo / V * V;
      blo[(size_t)ob] = (int32_t)lo;
      span = std::max<int64_t>(span, hi - lo + 1);
    }
    span = (span + V - 1) / V * V;
    const size_t smem = (((size_t)nrq * X * 8 + (size_t)ngb * 4 + 15) & ~size_t(15)) + (size_t)nrq * X * span * wb;
    if (smem > budget || nrq * X > 8192) break;
    best_pg = pg; best_span = span; best_nrq = nrq; best_ngb = ngb; best_blo.swap(blo);
  }
  if (best_pg < 0 || best_nrq == 1) return false;  // one row group: K_ROW's forms serve it
  const int pg = best_pg;
  WinPlan P{};
  int tabn = 0;
  P.a = a; P.b = b;
  P.X = (int32_t)X; P.Lb = (int32_t)Lb; P.span = (int32_t)best_span;
  const int64_t LbS = best_span;  // run slots per staged row group
  P.LbS = (int32_t)LbS;
  P.nvs = (int32_t)(best_span / V);
  P.ng = p0 - pg;
  int64_t nrun = 1;
  for (int p = pg; p < p0; p++) {
    const int k = p - pg;
    P.gdiv[k] = FastDiv((uint32_t)D->pshape[p]);
    P.gowner[k] = D->pdim_owner[p];
    P.grad[k] = D->pdim_rad[p];
    nrun *= D->pshape[p];
  }
  P.nrq = (int32_t)best_nrq;
  P.nrun = (int32_t)nrun;
  int k = 0;
  int64_t nouter = 1;
  for (int p = 0; p < pg; p++) {
    P.odiv[k] = FastDiv((uint32_t)D->pshape[p]);
    P.oowner[k] = D->pdim_owner[p];
    P.orad[k] = D->pdim_rad[p];
    nouter *= D->pshape[p];
    k++;
  }
  P.nout = k;
  P.nouter = (uint32_t)nouter;
  P.lrank = D->lrank;
  for (int d = 0; d < D->lrank; d++) { P.rev[d] = ds.rev[d]; P.rd[d] = ss.rd[d]; }
  P.f_x = FastDiv((uint32_t)X);
  P.f_nvs = FastDiv((uint32_t)P.nvs);
  P.nbg = (int32_t)best_ngb;
  {
    // per-logical-dim offset tables over the G coordinates (see WinPlan)
    int nt = 0, tot = 0;
    P.notab = 0;
    for (int d = 0; d < D->lrank; d++) {
      if (d == b) continue;
      std::vector<int> gd;  // G dims of d above p0, innermost first
      for (int p = p0 - 1; p >= pg; p--) if (D->pdim_owner[p] == d) gd.push_back(p);
      if (d != a && gd.empty()) { P.notab |= 1u << d; continue; }
      if (nt >= kMaxL || (int)gd.size() + 1 > kWinG + 1) return false;
      P.tdim[nt] = d;
      P.toff[nt] = tot;
      int k = 0, sz = 1;
      if (d == a) { P.text[nt][k] = FastDiv((uint32_t)X); P.trad[nt][k] = 1; k++; sz *= (int)X; P.ati = nt; }
      for (int p : gd) {
        P.text[nt][k] = FastDiv((uint32_t)D->pshape[p]);
        P.trad[nt][k] = D->pdim_rad[p];
        P.gti[p - pg] = nt;
        P.gmul[p - pg] = sz / (d == a ? (int)X : 1);
        sz *= (int)D->pshape[p];
        k++;
      }
      P.tn[nt] = k;
      tot += sz;
      nt++;
    }
    for (int p = pg; p < p0; p++) if (D->pdim_owner[p] == b) P.gti[p - pg] = -1;
    P.nt = nt;
    P.toff[nt] = tot;
    if (tot > 4096) return false;
    tabn = tot;
  }
  const size_t smem = (((size_t)tabn * 8 + (size_t)best_ngb * 4 + 15) & ~size_t(15)) + (size_t)best_nrq * X * LbS * wb;
  // device copy of the window-start table, cached per (layout pair, device)
  static std::mutex mu;
  struct Ent { uint64_t s, d; int dev; int32_t *ptr; };
  static std::vector<Ent> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  int32_t *dt = nullptr;
  {
    std::lock_guard<std::mutex> g(mu);
    for (auto &e : cache) if (e.s == S->serial && e.d == D->serial && e.dev == dev) dt = e.ptr;
    if (!dt) {
      if (cudaMalloc(&dt, best_blo.size() * 4) != cudaSuccess) { cudaGetLastError(); return false; }
      if (cudaMemcpy(dt, best_blo.data(), best_blo.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) { cudaGetLastError(); return false; }
      cache.push_back({S->serial, D->serial, dev, dt});
    }
  }
  P.blo = dt;
  // threads per CTA: each block's three phases are latency-bound, so more
  // threads per block shorten them (developer knob ALT_WIN_THREADS)
  static const int win_threads = [] {
    const int t = getenv("ALT_WIN_THREADS") ? atoi(getenv("ALT_WIN_THREADS")) : 512;
    return t <= 128 ? 128 : (t <= 256 ? 256 : 512);  // the kernel's launch bound is 512
  }();
  const int per_sm = std::max(1, (int)std::min<size_t>(2048 / win_threads, (size_t)(200 * 1024) / smem));
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(nouter, (int64_t)nsm * per_sm));
#define WIN_LAUNCH(T, XX)                                                                                 \
  do {                                                                                                   \
    cudaFuncSetAttribute(k_relayout_win<T, XX>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
    launch_pdl(k_relayout_win<T, XX>, grid, win_threads, smem, stream, P, (const T *)src, (T *)dst);     \
  } while (0)
  if (wb == 2) {
    if (X == 8) WIN_LAUNCH(uint16_t, 8); else WIN_LAUNCH(uint16_t, 16);
  } else {
    if (X == 4) WIN_LAUNCH(uint32_t, 4); else WIN_LAUNCH(uint32_t, 8);
  }
#undef WIN_LAUNCH
  count_launch();
  *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
  if (*st != ALT_OK) set_error("relayout (window group) launch failed");
  return true;
}

// position q of the suffix holds b index q (no pad / unfold of b)
static bool bmap_static_is(const Layout *D, int b, const std::vector<int32_t> &sbc, int64_t q) {
  return D->rev[b][sbc[(size_t)q]] == q;
}

// host side of K_ROW: returns false (nothing launched) when not applicable
static bool row_launch(Layout *S, const void *src, Layout *D, void *dst, int wb, const SepDev &ss,
                       const SepDev &ds, cudaStream_t stream, int nsm, alt_status *st) {
  const int V = 16 / wb;
  if (D->pnumel >= (1ll << 31)) return false;
  if ((reinterpret_cast<uintptr_t>(dst) & 15) || D->pnumel % V) return false;
  const int p0 = D->prank - 1;
  const int a = D->pdim_owner[p0];
  const int b = S->pdim_owner[S->prank - 1];
  if (a == b || D->pdim_rad[p0] != 1) return false;
  const int64_t Lb = S->lshape[b];
  for (int64_t i = 0; i < Lb; i++) if (S->rd[b][i] != i) return false;  // b contiguous in src
  // suffix: dims just above p0 owned by b
  int ps = p0;
  while (ps - 1 >= 0 && D->pdim_owner[ps - 1] == b) ps--;
  if (ps == p0) return false;
  const int64_t X = D->pshape[p0];
  if (X < V ? (V % X != 0) : (X % V != 0)) return false;
  if (X & (X - 1)) return false;  // power of two (shift / mask decode)
  int64_t npos = 1;
  for (int p = ps; p < p0; p++) npos *= D->pshape[p];
  if (npos * X % V || npos > (1 << 20)) return false;
  // suffix part of b's combo per position
  std::vector<int32_t> sbc((size_t)npos);
  for (int64_t pos = 0; pos < npos; pos++) {
    int64_t rem = pos, combo = 0;
    for (int p = p0 - 1; p >= ps; p--) {
      combo += (rem % D->pshape[p]) * D->pdim_rad[p];
      rem /= D->pshape[p];
    }
    sbc[(size_t)pos] = (int32_t)combo;
  }
  // every outer combo of b (mixed radix over b's outer dims): the b window
  // its block touches, start aligned down to a vector
  std::vector<int> bouter;
  for (int p = 0; p < ps; p++) if (D->pdim_owner[p] == b) bouter.push_back(p);
  const int64_t fb = (int64_t)D->rev[b].size();
  std::vector<int32_t> blo((size_t)fb, 0);
  int64_t span = 0;
  {
    int64_t nob = 1;
    for (int p : bouter) nob *= D->pshape[p];
    for (int64_t k = 0; k < nob; k++) {
      int64_t rem = k, ob = 0;
      for (int t = (int)bouter.size() - 1; t >= 0; t--) {
        const int p = bouter[t];
        ob += (rem % D->pshape[p]) * D->pdim_rad[p];
        rem /= D->pshape[p];
      }
      int64_t lo = INT64_MAX, hi = -1;
      for (int64_t pos = 0; pos < npos; pos++) {
        const int32_t bi = D->rev[b][ob + sbc[(size_t)pos]];
        if (bi >= 0) { lo = std::min<int64_t>(lo, bi); hi = std::max<int64_t>(hi, bi); }
      }
      if (hi < 0) lo = hi = 0;
      lo = lo / V * V;
      blo[(size_t)ob] = (int32_t)lo;
      span = std::max<int64_t>(span, hi - lo + 1);
    }
  }
  span = (span + V - 1) / V * V;
  int64_t LbS = span;
  if ((LbS * wb) % 128 == 0) LbS += V;  // rows j and j + 1 on different banks
  // transposed staging when an X-run is 8 or 16 bytes and rows load as vectors
  bool vl0 = Lb % V == 0 && (reinterpret_cast<uintptr_t>(src) & 15) == 0;
  for (int d = 0; d < S->lrank && vl0; d++) {
    if (d == b) continue;
    for (int64_t o : S->rd[d]) if (o >= 0 && o % V) { vl0 = false; break; }
  }
  static const bool no_tr = getenv("ALT_RELAYOUT_NOTR") != nullptr;  // developer A/B knob
  // (measured: a win for 8-byte runs, e.g. the window-folded image 5.5x; for
  // 16-byte runs the [X][window] form's wider stage parallelism is faster)
  const int RB = (!no_tr && vl0 && X * wb == 8) ? 8 : 0;
  if (RB) LbS = span;  // [window][X] runs, no row padding
  const size_t blk_smem = (size_t)X * LbS * wb;
  if (blk_smem > 32768) return false;
  RowPlan R{};
  R.a = a; R.b = b; R.X = (int32_t)X; R.Lb = (int32_t)Lb; R.npos = (int32_t)npos;
  R.LbS = (int32_t)LbS; R.span = (int32_t)span;
  R.lrank = D->lrank;
  int k = 0;
  int64_t nouter = 1;
  for (int p = 0; p < ps; p++) {
    R.odiv[k] = FastDiv((uint32_t)D->pshape[p]);
    R.oowner[k] = D->pdim_owner[p];
    R.orad[k] = D->pdim_rad[p];
    nouter *= D->pshape[p];
    k++;
  }
  R.nout = k;
  R.nouter = (uint32_t)nouter;
  for (int d = 0; d < D->lrank; d++) { R.rev[d] = ds.rev[d]; R.rd[d] = ss.rd[d]; }
  // device copies of the two tables, cached per (layout pair, device)
  static std::mutex mu;
  struct Ent { uint64_t s, d; int dev; int32_t *ptr; };
  static std::vector<Ent> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  int32_t *dt = nullptr;
  {
    std::lock_guard<std::mutex> g(mu);
    for (auto &e : cache) if (e.s == S->serial && e.d == D->serial && e.dev == dev) dt = e.ptr;
    if (!dt) {
      std::vector<int32_t> h(sbc);
      if (bouter.empty())  // static b map: store the b index itself
        for (size_t q = 0; q < h.size(); q++) h[q] = D->rev[b][h[q]] < 0 ? -1 : D->rev[b][h[q]];
      h.insert(h.end(), blo.begin(), blo.end());
      if (cudaMalloc(&dt, h.size() * 4) != cudaSuccess) { cudaGetLastError(); return false; }
      if (cudaMemcpy(dt, h.data(), h.size() * 4, cudaMemcpyHostToDevice) != cudaSuccess) { cudaGetLastError(); return false; }
      cache.push_back({S->serial, D->serial, dev, dt});
    }
  }
  R.sbc = dt;
  R.blo = dt + npos;
  R.lgX = 0;
  while ((1ll << R.lgX) < X) R.lgX++;
  R.bstatic = bouter.empty() ? 1 : 0;
  R.f_nv = FastDiv((uint32_t)(span / V));
  R.f_span = FastDiv((uint32_t)span);
  R.f_vpb = FastDiv((uint32_t)(npos * X / V));
  bool vl = Lb % V == 0 && (reinterpret_cast<uintptr_t>(src) & 15) == 0;
  for (int d = 0; d < S->lrank && vl; d++) {
    if (d == b) continue;
    for (int64_t o : S->rd[d]) if (o >= 0 && o % V) { vl = false; break; }
  }
  R.vec_load = vl ? 1 : 0;
  // identity suffix with 16- or 32-byte runs: the register-transpose form
  {
    bool ident = R.bstatic && npos == Lb && (X * wb == 16 || (X * wb == 32 && wb == 4)) && vl0;
    for (int64_t q = 0; q < npos && ident; q++) ident = bmap_static_is(D, b, sbc, q);
    static const bool no_id = getenv("ALT_RELAYOUT_NOID") != nullptr;  // developer A/B knob
    if (ident && !no_id) {
      const int64_t nthr = nouter * (Lb / V);
      if (nthr < (1ll << 31)) {
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((nthr + 255) / 256, (int64_t)nsm * 16));
        const bool x2 = X * wb == 32;
        if (wb == 2 && !x2) launch_pdl(k_relayout_row_ident<uint16_t, 8>, grid, 256, 0, stream, R, (const uint16_t *)src, (uint16_t *)dst, (uint32_t)nthr);
        else if (!x2) launch_pdl(k_relayout_row_ident<uint32_t, 4>, grid, 256, 0, stream, R, (const uint32_t *)src, (uint32_t *)dst, (uint32_t)nthr);
        else launch_pdl(k_relayout_row_ident<uint32_t, 8>, grid, 256, 0, stream, R, (const uint32_t *)src, (uint32_t *)dst, (uint32_t)nthr);
        count_launch();
        *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
        if (*st != ALT_OK) set_error("relayout (row, identity) launch failed");
        return true;
      }
    }
  }
  int per = (int)std::max<int64_t>(1, std::min<int64_t>(64, 16384 / (int64_t)blk_smem));
  R.per_iter = per;
  const size_t smem = (size_t)per * blk_smem;
  const int64_t iters = (nouter + per - 1) / per;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(iters, (int64_t)nsm * 8));
#define ROW_LAUNCH(T, RBV)                                                                               \
  do {                                                                                                   \
    cudaFuncSetAttribute(k_relayout_row<T, RBV>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem); \
    launch_pdl(k_relayout_row<T, RBV>, grid, 256, smem, stream, R, (const T *)src, (T *)dst);           \
  } while (0)
  if (wb == 2) {
    if (RB == 8) ROW_LAUNCH(uint16_t, 8);
    else ROW_LAUNCH(uint16_t, 0);
  } else {
    if (RB == 8) ROW_LAUNCH(uint32_t, 8);
    else ROW_LAUNCH(uint32_t, 0);
  }
#undef ROW_LAUNCH
  count_launch();
  *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
  if (*st != ALT_OK) set_error("relayout (row) launch failed");
  return true;
}

// ===================================================== strided permutation ==
// Fast path for layouts built from split / reorder only (no pad, no unfold):
// both are permutations of a common refinement of the logical digits, so the
// conversion is a strided permutation copy.  Dims are coalesced, then either
//   K_PCOPY  (dst-innermost == src-innermost): 16-byte vector copy, or
//   K_PTRANS (they differ): 2-D tiles staged through shared memory with
//            16-byte global loads along the src-contiguous dim and 16-byte
//            global stores along the dst-contiguous dim.
struct PermDims {
  int32_t nd;                  // batch dims (outer, excluding X / Y)
  FastDiv ext[kMaxP];
  int64_t sstr[kMaxP], dstr[kMaxP];
  int64_t ex, ey;              // extents of X (dst stride 1) and Y (src stride 1)
  int64_t sx, dy;              // src stride of X, dst stride of Y
};

struct RDim { int64_t ext, sstr, dstr; };

static bool refine_perm(const Layout &S, const Layout &D, std::vector<RDim> &out) {
  const uint32_t bad = ALT_HAS_PAD | ALT_HAS_UNFOLD;
  if (!S.separable || !D.separable || !S.aff.ok || !D.aff.ok || (S.flags & bad) || (D.flags & bad)) return false;
  if (!(S.flags & ALT_LOSSLESS) || !(D.flags & ALT_LOSSLESS)) return false;
  out.clear();
  for (int d = 0; d < S.lrank; d++) {
    struct Dig { int64_t coef, ext, str; };
    auto digits = [&](const Layout &L) {
      std::vector<Dig> v;
      for (int p = 0; p < L.prank; p++)
        if (L.pdim_owner[p] == d && L.pshape[p] > 1) v.push_back({L.aff.coef[p], L.pshape[p], L.pstride[p]});
      std::sort(v.begin(), v.end(), [](const Dig &a, const Dig &b) { return a.coef < b.coef; });
      return v;
    };
    std::vector<Dig> sd = digits(S), dd = digits(D);
    if (S.lshape[d] == 1) continue;
    // place values of both digit systems must form one divisibility chain
    std::vector<int64_t> pv;
    for (auto &g : sd) { pv.push_back(g.coef); pv.push_back(g.coef * g.ext); }
    for (auto &g : dd) { pv.push_back(g.coef); pv.push_back(g.coef * g.ext); }
    std::sort(pv.begin(), pv.end());
    pv.erase(std::unique(pv.begin(), pv.end()), pv.end());
    if (pv.empty() || pv.front() != 1 || pv.back() != S.lshape[d]) return false;
    for (size_t i = 0; i + 1 < pv.size(); i++) {
      if (pv[i + 1] % pv[i]) return false;
      const int64_t v = pv[i], e = pv[i + 1] / pv[i];
      auto stride_in = [&](const std::vector<Dig> &ds, int64_t *str) {
        for (auto &g : ds)
          if (v >= g.coef && v < g.coef * g.ext) {
            if (v % g.coef) return false;
            *str = g.str * (v / g.coef);
            return (v * e) <= g.coef * g.ext;
          }
        return false;
      };
      RDim r{e, 0, 0};
      if (!stride_in(sd, &r.sstr) || !stride_in(dd, &r.dstr)) return false;
      out.push_back(r);
    }
  }
  // dst row-major order, then coalesce dims nested in both layouts
  std::sort(out.begin(), out.end(), [](const RDim &a, const RDim &b) { return a.dstr > b.dstr; });
  std::vector<RDim> c;
  for (const RDim &r : out) {
    if (!c.empty() && c.back().dstr == r.dstr * r.ext && c.back().sstr == r.sstr * r.ext) {
      c.back().ext *= r.ext;
      c.back().dstr = r.dstr;
      c.back().sstr = r.sstr;
    } else {
      c.push_back(r);
    }
  }
  out = c;
  return true;
}


// vector copy: each thread moves VPT vectors of 16 bytes along X (contiguous
// in both layouts); batch dims decoded per vector
template <typename T>
__global__ void __launch_bounds__(256) k_perm_copy(PermDims P, const T *__restrict__ src, T *__restrict__ dst,
                                                   uint32_t nvec) {
  constexpr int V = 16 / sizeof(T);
  const uint32_t vx = (uint32_t)(P.ex / V);  // vectors per X run
  for (uint32_t v0 = blockIdx.x * blockDim.x * 4 + threadIdx.x; v0 < nvec; v0 += gridDim.x * blockDim.x * 4) {
    uint4 val[4];
    int64_t doff[4];
    bool ok[4];
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const uint32_t v = v0 + u * blockDim.x;
      ok[u] = v < nvec;
      if (!ok[u]) continue;
      uint32_t rem = v / vx;
      const uint32_t xi = (v - rem * vx) * V;
      int64_t so = (int64_t)xi * P.sx;
      for (int k = P.nd - 1; k >= 0; k--) {
        uint32_t q, r;
        P.ext[k].divmod(rem, q, r);
        so += (int64_t)r * P.sstr[k];
        rem = q;
      }
      doff[u] = (int64_t)v * V;
      val[u] = ld16(src + so);
    }
#pragma unroll
    for (int u = 0; u < 4; u++)
      if (ok[u]) *reinterpret_cast<uint4 *>(dst + doff[u]) = val[u];
  }
}

// transpose tiles: X (dst stride 1) x Y (src stride 1), TX x TY elements
template <typename T, int TX, int TY>
__global__ void __launch_bounds__(256) k_perm_trans(PermDims P, const T *__restrict__ src, T *__restrict__ dst,
                                                    uint32_t ntiles) {
  constexpr int V = 16 / sizeof(T);
  // rows of TY elements; the 16-byte vector slots of row x are XOR-swizzled
  // by (x / 8) so the column walks of the store phase spread over the banks
  constexpr int NV = TY / V;
  __shared__ __align__(16) T tile[TX * TY];
  auto at = [](int x, int y) { return x * TY + ((((y / V) ^ ((x >> 3) % NV)) * V) + (y % V)); };
  const uint32_t tx_n = (uint32_t)((P.ex + TX - 1) / TX), ty_n = (uint32_t)((P.ey + TY - 1) / TY);
  for (uint32_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
    uint32_t rem = t;
    const uint32_t cx = rem % tx_n;
    rem /= tx_n;
    const uint32_t cy = rem % ty_n;
    rem /= ty_n;
    int64_t sb = 0, db = 0;
    for (int k = P.nd - 1; k >= 0; k--) {
      uint32_t q, r;
      P.ext[k].divmod(rem, q, r);
      sb += (int64_t)r * P.sstr[k];
      db += (int64_t)r * P.dstr[k];
      rem = q;
    }
    const int64_t x0 = (int64_t)cx * TX, y0 = (int64_t)cy * TY;
    const int nx = (int)(P.ex - x0 < TX ? P.ex - x0 : TX), ny = (int)(P.ey - y0 < TY ? P.ey - y0 : TY);
    sb += x0 * P.sx + y0;
    db += y0 * P.dy + x0;
    __syncthreads();
    if constexpr (TY >= 4 * V) {
      // wide Y: tile rows x; 16-byte loads along y, column-walk stores
      for (int e = threadIdx.x; e < TX * (TY / V); e += blockDim.x) {
        const int x = e / (TY / V), y = (e % (TY / V)) * V;
        if (x >= nx || y >= ny) continue;
        const T *s = src + sb + (int64_t)x * P.sx + y;
        if (y + V <= ny && ((reinterpret_cast<uintptr_t>(s) & 15) == 0)) {
          *reinterpret_cast<uint4 *>(&tile[at(x, y)]) = ld16(s);
        } else {
          for (int j = 0; j < V && y + j < ny; j++) tile[at(x, y + j)] = s[j];
        }
      }
      __syncthreads();
      for (int e = threadIdx.x; e < TY * (TX / V); e += blockDim.x) {
        const int y = e / (TX / V), x = (e % (TX / V)) * V;
        if (y >= ny || x >= nx) continue;
        T *d = dst + db + (int64_t)y * P.dy + x;
        if (x + V <= nx && ((reinterpret_cast<uintptr_t>(d) & 15) == 0)) {
          T v[V];
#pragma unroll
          for (int j = 0; j < V; j++) v[j] = tile[at(x + j, y)];
          *reinterpret_cast<uint4 *>(d) = *reinterpret_cast<const uint4 *>(v);
        } else {
          for (int j = 0; j < V && x + j < nx; j++) d[j] = tile[at(x + j, y)];
        }
      }
    } else {
      // narrow Y (a few vectors per src run): tile rows y; neighbouring
      // threads load neighbouring x (coalesced when the runs are adjacent) and
      // scatter into rows y, stores are 16-byte vectors along x
      for (int e = threadIdx.x; e < TX * (TY / V); e += blockDim.x) {
        const int x = e % TX, y = (e / TX) * V;
        if (x >= nx || y >= ny) continue;
        const T *s = src + sb + (int64_t)x * P.sx + y;
        if (y + V <= ny && ((reinterpret_cast<uintptr_t>(s) & 15) == 0)) {
          const uint4 u = ld16(s);
          const T *uv = reinterpret_cast<const T *>(&u);
#pragma unroll
          for (int j = 0; j < V; j++) tile[(y + j) * TX + x] = uv[j];
        } else {
          for (int j = 0; j < V && y + j < ny; j++) tile[(y + j) * TX + x] = s[j];
        }
      }
      __syncthreads();
      for (int e = threadIdx.x; e < TY * (TX / V); e += blockDim.x) {
        const int y = e / (TX / V), x = (e % (TX / V)) * V;
        if (y >= ny || x >= nx) continue;
        T *d = dst + db + (int64_t)y * P.dy + x;
        if (x + V <= nx && ((reinterpret_cast<uintptr_t>(d) & 15) == 0)) {
          *reinterpret_cast<uint4 *>(d) = *reinterpret_cast<const uint4 *>(&tile[y * TX + x]);
        } else {
          for (int j = 0; j < V && x + j < nx; j++) d[j] = tile[y * TX + x + j];
        }
      }
    }
  }
}


// register transpose: one thread moves a V x V block (V = 16 / sizeof(T)):
// V 16-byte loads along Y (src-contiguous) from V consecutive X rows, a
// V x V transpose in registers (byte_perm for 16-bit words), V 16-byte stores
// along X (dst-contiguous).  Neighbouring threads take neighbouring Y blocks,
// so both the loads (per X row) and the stores (per Y row, when dst rows of
// consecutive y are adjacent, e.g. NCHW -> NCHW[V]c) coalesce; no shared
// memory and no barriers.  Needs ex % V == ey % V == 0 and V-aligned strides.
// Lane mapping: a warp covers LX x-blocks by LY y-blocks (LX * LY = 32,
// y-blocks fastest), so a load instruction reads LY * 16 contiguous bytes of
// each of the lanes' src rows and a store instruction writes LX * 16
// contiguous bytes of each dst row.
template <typename T>
__global__ void __launch_bounds__(256) k_perm_rt(PermDims P, const T *__restrict__ src, T *__restrict__ dst,
                                               uint32_t nblk, int lgLY) {
  pdl_wait();  // launched with launch_pdl: no global access before the previous grid completes
  constexpr int V = 16 / sizeof(T);
  // lgLY < 0: flat mapping (y-blocks, then x-blocks, then batch, fastest
  // first) — used when a thread's V stores are adjacent (dy == V) or there is
  // one y-block (ey == V) and the warp tiling does not divide the extents
  const int lg = lgLY < 0 ? 0 : lgLY;
  const uint32_t LY = 1u << lg, LX = 32u >> lg;
  const uint32_t byn = (uint32_t)(P.ey / V), bxn = (uint32_t)(P.ex / V);
  const uint32_t gyn = (byn + LY - 1) / LY, gxn = bxn / LX;  // warp tiles along y (ragged) / x
  for (uint32_t t = blockIdx.x * blockDim.x + threadIdx.x; t < nblk; t += gridDim.x * blockDim.x) {
    uint32_t rem, by, bx;
    if (lgLY < 0) {
      rem = t;
      by = rem % byn;
      rem /= byn;
      bx = rem % bxn;
      rem /= bxn;
    } else {
      const uint32_t lane = t & 31u;
      rem = t >> 5;
      const uint32_t gy = rem % gyn;
      rem /= gyn;
      const uint32_t gx = rem % gxn;
      rem /= gxn;
      by = gy * LY + (lane & (LY - 1));
      bx = gx * LX + (lane >> lg);
      if (by >= byn) continue;  // ragged last y tile
    }
    int64_t sb = 0, db = 0;
    for (int k = P.nd - 1; k >= 0; k--) {
      uint32_t q, r;
      P.ext[k].divmod(rem, q, r);
      sb += (int64_t)r * P.sstr[k];
      db += (int64_t)r * P.dstr[k];
      rem = q;
    }
    const int64_t x0 = (int64_t)bx * V, y0 = (int64_t)by * V;
    uint4 u[V];
#pragma unroll
    for (int j = 0; j < V; j++) u[j] = ld16(src + sb + (x0 + j) * P.sx + y0);
#pragma unroll
    for (int k = 0; k < V; k++) {
      uint32_t w[4];
      if constexpr (sizeof(T) == 2) {
        const uint32_t sel = (k & 1) ? 0x7632u : 0x5410u;
#pragma unroll
        for (int jp = 0; jp < 4; jp++)
          w[jp] = __byte_perm(reinterpret_cast<const uint32_t *>(&u[2 * jp])[k >> 1],
                              reinterpret_cast<const uint32_t *>(&u[2 * jp + 1])[k >> 1], sel);
      } else {
#pragma unroll
        for (int j = 0; j < 4; j++) w[j] = reinterpret_cast<const uint32_t *>(&u[j])[k];
      }
      *reinterpret_cast<uint4 *>(dst + db + (y0 + k) * P.dy + x0) = make_uint4(w[0], w[1], w[2], w[3]);
    }
  }
}

// k_perm_rt, flat mapping with ex == V and dy == V (e.g. NCHW -> NCHW[V]c):
// a thread's V x V block is one contiguous dst run of V vectors, stored
// through warp_store_runs (512-byte spans per store instruction instead of
// 32 lanes x 16 bytes at a 128-byte stride: measured 0.68 -> see DESIGN §5).
template <typename T>
__global__ void __launch_bounds__(256) k_perm_rt_ws(PermDims P, const T *__restrict__ src, T *__restrict__ dst,
                                                  uint32_t nblk) {
  pdl_wait();
  constexpr int V = 16 / sizeof(T);
  __shared__ uint4 stage[8][32 * V];
  const int lane = threadIdx.x & 31;
  uint4 *st = stage[threadIdx.x >> 5];
  const uint32_t byn = (uint32_t)(P.ey / V);
  for (uint32_t t0 = blockIdx.x * blockDim.x + (threadIdx.x & ~31u); t0 < nblk; t0 += gridDim.x * blockDim.x) {
    const uint32_t t = t0 + lane;
    uint4 w[V];
    int64_t off = -1;
    if (t < nblk) {
      uint32_t rem = t / byn;
      const uint32_t by = t - rem * byn;
      int64_t sb = 0, db = 0;
      for (int k = P.nd - 1; k >= 0; k--) {
        uint32_t q, r;
        P.ext[k].divmod(rem, q, r);
        sb += (int64_t)r * P.sstr[k];
        db += (int64_t)r * P.dstr[k];
        rem = q;
      }
      const int64_t y0 = (int64_t)by * V;
      uint4 u[V];
#pragma unroll
      for (int j = 0; j < V; j++) u[j] = ld16(src + sb + j * P.sx + y0);
#pragma unroll
      for (int k = 0; k < V; k++) {
        uint32_t ww[4];
        if constexpr (sizeof(T) == 2) {
          const uint32_t sel = (k & 1) ? 0x7632u : 0x5410u;
#pragma unroll
          for (int jp = 0; jp < 4; jp++)
            ww[jp] = __byte_perm(reinterpret_cast<const uint32_t *>(&u[2 * jp])[k >> 1],
                                 reinterpret_cast<const uint32_t *>(&u[2 * jp + 1])[k >> 1], sel);
        } else {
#pragma unroll
          for (int j = 0; j < 4; j++) ww[j] = reinterpret_cast<const uint32_t *>(&u[j])[k];
        }
        w[k] = make_uint4(ww[0], ww[1], ww[2], ww[3]);
      }
      off = db + y0 * V;
    }
    warp_store_runs<T, V>(st, w, off, dst, lane);
  }
}

// K_PBLOCK: the X x Y transpose tile would be mostly empty (X and Y both
// short, e.g. weights KCRS -> KCRS16k16c: X = 16 c, Y = R S = 9), so the tile
// grows by the batch dims nearest to dst-contiguity until it holds up to
// 4096 elements; a CTA iteration moves one such block: scalar loads in src
// order (coalesced along the src runs) into shared memory at the block's
// compact dst position, then 16-byte stores of the block (contiguous in dst
// when the block dims nest, which the selection favours) or scalar stores.
constexpr int kPbMax = 6;
struct PermBlock {
  int32_t nb;                     // block dims
  int32_t bsize;                  // elements per block
  FastDiv sext[kPbMax];           // block dims in src order (innermost first)
  int64_t ssrc[kPbMax];           //   their src strides
  int32_t sloc[kPbMax];           //   their compact dst-order (local) strides
  FastDiv dext[kPbMax];           // block dims in dst order (innermost first)
  int64_t ddst[kPbMax];           //   their dst strides
  int32_t dcontig;                // block is one contiguous dst range
  int32_t nd;                     // batch dims
  FastDiv ext[kMaxP];
  int64_t sstr[kMaxP], dstr[kMaxP];
  uint32_t nbatch;
};

template <typename T>
__global__ void __launch_bounds__(256) k_perm_block(PermBlock B, const T *__restrict__ src, T *__restrict__ dst) {
  pdl_wait();
  extern __shared__ __align__(16) unsigned char pb_smem[];
  T *tile = reinterpret_cast<T *>(pb_smem);
  constexpr int V = 16 / sizeof(T);
  for (uint32_t bi = blockIdx.x; bi < B.nbatch; bi += gridDim.x) {
    uint32_t rem = bi;
    int64_t sb = 0, db = 0;
    for (int k = B.nd - 1; k >= 0; k--) {
      uint32_t q, r;
      B.ext[k].divmod(rem, q, r);
      sb += (int64_t)r * B.sstr[k];
      db += (int64_t)r * B.dstr[k];
      rem = q;
    }
    __syncthreads();
    // eight loads in flight per thread before the shared stores
    for (int e0 = threadIdx.x; e0 < B.bsize; e0 += blockDim.x * 8) {
      T val[8];
      int loc[8];
#pragma unroll
      for (int u = 0; u < 8; u++) {
        const int e = e0 + u * (int)blockDim.x;
        loc[u] = -1;
        if (e >= B.bsize) continue;
        uint32_t re = (uint32_t)e;
        int lc = 0;
        int64_t so = 0;
        for (int i = 0; i < B.nb; i++) {
          uint32_t q, ii;
          B.sext[i].divmod(re, q, ii);
          re = q;
          so += (int64_t)ii * B.ssrc[i];
          lc += (int)ii * B.sloc[i];
        }
        loc[u] = lc;
        val[u] = src[sb + so];
      }
#pragma unroll
      for (int u = 0; u < 8; u++)
        if (loc[u] >= 0) tile[loc[u]] = val[u];
    }
    __syncthreads();
    if (B.dcontig && ((db % V) == 0)) {
      for (int v = threadIdx.x; v < B.bsize / V; v += blockDim.x)
        *reinterpret_cast<uint4 *>(dst + db + (int64_t)v * V) = *reinterpret_cast<const uint4 *>(tile + v * V);
    } else {
      for (int l = threadIdx.x; l < B.bsize; l += blockDim.x) {
        uint32_t rl = (uint32_t)l;
        int64_t dof = 0;
        for (int i = 0; i < B.nb; i++) {
          uint32_t q, ii;
          B.dext[i].divmod(rl, q, ii);
          rl = q;
          dof += (int64_t)ii * B.ddst[i];
        }
        dst[db + dof] = tile[l];
      }
    }
  }
}

// host side of K_PBLOCK over the refined dims r (X = ix, Y = iy); false when
// the block would not beat the transpose tiles
static bool pblock_launch(const std::vector<RDim> &r, int ix, int iy, const void *src, void *dst, int wb,
                          cudaStream_t stream, int nsm) {
  const int V = 16 / wb;
  std::vector<int> in = {ix, iy};
  int64_t bsize = r[ix].ext * r[iy].ext;
  if (bsize > 4096) return false;  // the X x Y tile alone exceeds a block: transpose tiles
  for (;;) {
    int best = -1;
    for (int i = 0; i < (int)r.size(); i++) {
      if (std::find(in.begin(), in.end(), i) != in.end()) continue;
      if (best < 0 || r[i].dstr < r[best].dstr) best = i;
    }
    if (best < 0 || bsize * r[best].ext > 4096 || (int)in.size() >= kPbMax) break;
    in.push_back(best);
    bsize *= r[best].ext;
  }
  if (bsize < 256 || bsize % V) return false;
  PermBlock B{};
  B.nb = (int)in.size();
  B.bsize = (int32_t)bsize;
  std::vector<int> so(in), dor(in);
  std::sort(so.begin(), so.end(), [&](int a, int b) { return r[a].sstr < r[b].sstr; });
  std::sort(dor.begin(), dor.end(), [&](int a, int b) { return r[a].dstr < r[b].dstr; });
  std::vector<int64_t> loc(r.size(), 0);
  int64_t acc = 1;
  bool contig = true;
  for (int k = 0; k < B.nb; k++) {
    const int i = dor[(size_t)k];
    loc[(size_t)i] = acc;
    if (r[i].dstr != acc) contig = false;
    B.dext[k] = FastDiv((uint32_t)r[i].ext);
    B.ddst[k] = r[i].dstr;
    acc *= r[i].ext;
  }
  for (int k = 0; k < B.nb; k++) {
    const int i = so[(size_t)k];
    B.sext[k] = FastDiv((uint32_t)r[i].ext);
    B.ssrc[k] = r[i].sstr;
    B.sloc[k] = (int32_t)loc[(size_t)i];
  }
  B.dcontig = contig ? 1 : 0;
  int nd = 0;
  int64_t nbatch = 1;
  for (int i = 0; i < (int)r.size(); i++) {
    if (std::find(in.begin(), in.end(), i) != in.end()) continue;
    if (nd >= kMaxP) return false;
    B.ext[nd] = FastDiv((uint32_t)r[i].ext);
    B.sstr[nd] = r[i].sstr;
    B.dstr[nd] = r[i].dstr;
    nbatch *= r[i].ext;
    nd++;
  }
  if (nbatch >= (1ll << 31)) return false;
  B.nd = nd;
  B.nbatch = (uint32_t)nbatch;
  const size_t smem = (size_t)bsize * wb;
  const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(nbatch, (int64_t)nsm * 8));
  if (wb == 2) launch_pdl(k_perm_block<uint16_t>, grid, 256, smem, stream, B, (const uint16_t *)src, (uint16_t *)dst);
  else launch_pdl(k_perm_block<uint32_t>, grid, 256, smem, stream, B, (const uint32_t *)src, (uint32_t *)dst);
  return true;
}

static bool perm_launch(Layout *S, const void *src, Layout *D, void *dst, int wb, cudaStream_t stream, int nsm,
                        alt_status *st) {
  std::vector<RDim> r;
  if (!refine_perm(*S, *D, r)) return false;
  int ix = -1, iy = -1;
  for (int i = 0; i < (int)r.size(); i++) {
    if (r[i].dstr == 1) ix = i;
    if (r[i].sstr == 1) iy = i;
  }
  if (ix < 0 || iy < 0) return false;
  const int V = 16 / wb;
  PermDims P{};
  int nd = 0;
  for (int i = 0; i < (int)r.size(); i++) {
    if (i == ix || i == iy) continue;
    if (nd >= kMaxP || r[i].ext >= (1ll << 31)) return false;
    P.ext[nd] = FastDiv((uint32_t)r[i].ext);
    P.sstr[nd] = r[i].sstr;
    P.dstr[nd] = r[i].dstr;
    nd++;
  }
  P.nd = nd;
  P.ex = r[ix].ext;
  P.sx = r[ix].sstr;
  if ((reinterpret_cast<uintptr_t>(src) | reinterpret_cast<uintptr_t>(dst)) & 15) return false;
  if (ix == iy) {
    // same innermost dim: vector copy (needs whole vectors and aligned runs)
    if (P.ex % V) return false;
    for (int k = 0; k < nd; k++)
      if (P.sstr[k] % V) return false;
    const int64_t nvec = D->pnumel / V;
    if (nvec >= (1ll << 31)) return false;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((nvec + 1023) / 1024, (int64_t)nsm * 8));
    if (wb == 2) k_perm_copy<uint16_t><<<grid, 256, 0, stream>>>(P, (const uint16_t *)src, (uint16_t *)dst, (uint32_t)nvec);
    else k_perm_copy<uint32_t><<<grid, 256, 0, stream>>>(P, (const uint32_t *)src, (uint32_t *)dst, (uint32_t)nvec);
  } else {
    P.ey = r[iy].ext;
    P.dy = r[iy].dstr;
    static const bool no_rt = getenv("ALT_RELAYOUT_NORT") != nullptr;  // developer A/B knob
    // both the loads (LY y-blocks per src row) and the stores (LX x-blocks
    // per dst row) coalesce for any V-divisible extents (lane mapping below)
    bool rt = !no_rt && P.ex % V == 0 && P.ey % V == 0 && P.sx % V == 0 && P.dy % V == 0;
    for (int k = 0; k < nd && rt; k++) rt = P.sstr[k] % V == 0 && P.dstr[k] % V == 0;
    // lanes per y-row: as many y-blocks as there are (<= 32), the rest along x
    int lgLY = 5;
    if (rt) {
      const int64_t byn = P.ey / V, bxn = P.ex / V;
      // LX x-blocks (<= 8, dividing bxn) per dst row and LY = 32 / LX y-blocks
      // per src row: both sides move >= 64 contiguous bytes per instruction
      int LX = 1;
      while (LX < 8 && bxn % (LX * 2) == 0) LX *= 2;
      lgLY = 5;
      while ((32 >> lgLY) < LX) lgLY--;
      if ((1ll << lgLY) > byn * 2 || LX == 1) {  // most y lanes idle / one x-block
        if (P.dy == V || P.ey == V) lgLY = -1;   // flat mapping coalesces here
        else if (LX == 1) rt = false;
      }
    }
    int64_t nblk = rt ? D->pnumel / (V * V) : 0;
    if (rt && lgLY >= 0) {  // threads = 32 x warp tiles x batch (the last y tile may be ragged)
      const int64_t byn = P.ey / V, bxn = P.ex / V, LY = 1ll << lgLY, LX = 32 >> lgLY;
      nblk = 32 * ((byn + LY - 1) / LY) * (bxn / LX) * (D->pnumel / (P.ex * P.ey));
    }
    if (rt && nblk < (1ll << 31)) {
      const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((nblk + 255) / 256, (int64_t)nsm * 16));
      static const bool no_ws = getenv("ALT_RELAYOUT_NOWS") != nullptr;  // developer A/B knob
      if (lgLY < 0 && P.ex == V && P.dy == V && !no_ws) {
        if (wb == 2) launch_pdl(k_perm_rt_ws<uint16_t>, grid, 256, 0, stream, P, (const uint16_t *)src, (uint16_t *)dst, (uint32_t)nblk);
        else launch_pdl(k_perm_rt_ws<uint32_t>, grid, 256, 0, stream, P, (const uint32_t *)src, (uint32_t *)dst, (uint32_t)nblk);
      } else if (wb == 2) launch_pdl(k_perm_rt<uint16_t>, grid, 256, 0, stream, P, (const uint16_t *)src, (uint16_t *)dst, (uint32_t)nblk, lgLY);
      else launch_pdl(k_perm_rt<uint32_t>, grid, 256, 0, stream, P, (const uint32_t *)src, (uint32_t *)dst, (uint32_t)nblk, lgLY);
      count_launch();
      *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
      if (*st != ALT_OK) set_error("relayout (register transpose) launch failed");
      return true;
    }
    // tile shape: TX x TY elements (16 KB), the pair wasting
    // the fewest elements on ragged edges (larger square-ish tiles on ties)
    const int64_t area = 16384 / wb;  // 16 KB of shared memory per tile
    int TX = 8;
    double best = 1e30;
    for (int tx = 8; tx <= (wb == 2 ? 1024 : 512); tx *= 2) {
      const int64_t ty = area / tx;
      if (ty < 8) break;
      const double waste = (double)((P.ex + tx - 1) / tx * tx) * ((P.ey + ty - 1) / ty * ty) / ((double)P.ex * P.ey);
      const double score = waste * 1.0 + 1e-3 * std::abs(std::log2((double)tx / ty));
      if (score < best) { best = score; TX = tx; }
    }
    static const bool no_pb = getenv("ALT_RELAYOUT_NOPB") != nullptr;  // developer A/B knob
    if (best > 2.0 && !no_pb && pblock_launch(r, ix, iy, src, dst, wb, stream, nsm)) {
      count_launch();
      *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
      if (*st != ALT_OK) set_error("relayout (permutation block) launch failed");
      return true;
    }
    const int64_t TY = area / TX;
    const int64_t tiles = ((P.ex + TX - 1) / TX) * ((P.ey + TY - 1) / TY) * (D->pnumel / (P.ex * P.ey));
    if (tiles >= (1ll << 31)) return false;
    const int grid = (int)std::max<int64_t>(1, std::min<int64_t>(tiles, (int64_t)nsm * 8));
    const uint32_t nt = (uint32_t)tiles;
#define PT(T, X, A) k_perm_trans<T, X, A / X><<<grid, 256, 0, stream>>>(P, (const T *)src, (T *)dst, nt)
    if (wb == 2) {
      switch (TX) {
        case 8: PT(uint16_t, 8, 8192); break;
        case 16: PT(uint16_t, 16, 8192); break;
        case 32: PT(uint16_t, 32, 8192); break;
        case 64: PT(uint16_t, 64, 8192); break;
        case 128: PT(uint16_t, 128, 8192); break;
        case 256: PT(uint16_t, 256, 8192); break;
        case 512: PT(uint16_t, 512, 8192); break;
        default: PT(uint16_t, 1024, 8192); break;
      }
    } else {
      switch (TX) {
        case 8: PT(uint32_t, 8, 4096); break;
        case 16: PT(uint32_t, 16, 4096); break;
        case 32: PT(uint32_t, 32, 4096); break;
        case 64: PT(uint32_t, 64, 4096); break;
        case 128: PT(uint32_t, 128, 4096); break;
        case 256: PT(uint32_t, 256, 4096); break;
        default: PT(uint32_t, 512, 4096); break;
      }
    }
#undef PT
  }
  count_launch();
  *st = cudaGetLastError() == cudaSuccess ? ALT_OK : ALT_E_CUDA;
  if (*st != ALT_OK) set_error("relayout (permutation) launch failed");
  return true;
}

alt_status relayout_launch(Layout *S, const void *src, Layout *D, void *dst, int wb,
                           cudaStream_t stream) {
  if (S->lrank != D->lrank) { set_error("alt_relayout: logical ranks differ"); return ALT_E_SHAPE; }
  for (int d = 0; d < S->lrank; d++)
    if (S->lshape[d] != D->lshape[d]) { set_error("alt_relayout: logical shapes differ (dim %d)", d); return ALT_E_SHAPE; }
  SepDev ss{}, ds{};
  const LayoutDesc *sdesc = nullptr, *ddesc = nullptr;
  alt_status st = device_tables(S, &ss, &sdesc);
  if (st != ALT_OK) return st;
  st = device_tables(D, &ds, &ddesc);
  if (st != ALT_OK) return st;
  const int nsm = sm_count();
  {
    alt_status pst = ALT_OK;
    if (perm_launch(S, src, D, dst, wb, stream, nsm, &pst)) return pst;
  }

  if (S->separable && D->separable) {
    // every element dst holds must have a copy in src
    for (int d = 0; d < D->lrank; d++)
      for (int32_t v : D->rev[d])
        if (v >= 0 && S->rd[d][v] < 0) { set_error("alt_relayout: source layout has no copy of an element dst needs"); return ALT_E_LOSSY; }
    {
      alt_status rst = ALT_OK;
      static const bool no_row = getenv("ALT_RELAYOUT_NOROW") != nullptr;  // developer A/B knob
      static const bool no_win = getenv("ALT_RELAYOUT_NOWIN") != nullptr;  // developer A/B knob
      if (!no_win && win_launch(S, src, D, dst, wb, ss, ds, stream, nsm, &rst)) return rst;
      if (!no_row && row_launch(S, src, D, dst, wb, ss, ds, stream, nsm, &rst)) return rst;
    }
    SepPair P{};
    if (fill_pair(S, D, ss, ds, &P)) {
      const int p0 = D->prank - 1;
      const int a = D->pdim_owner[p0];
      // src innermost physical dim and its logical dim
      const int b = S->pdim_owner[S->prank - 1];
      const int64_t E0 = D->pshape[p0];
      // ---- K_VEC: dst runs along p0 are contiguous in src
      int V = 16 / wb;
      while (V > 1) {
        bool good = (E0 % V == 0);
        for (int d = 0; d < D->lrank && good; d++) {
          if (d == a) continue;
          for (int64_t o : S->rd[d]) if (o >= 0 && o % V) { good = false; break; }
        }
        const auto &rev = D->rev[a];
        const auto &rd = S->rd[a];
        for (size_t c0 = 0; c0 < rev.size() && good; c0 += V) {
          int32_t i0 = rev[c0];
          if (i0 >= 0 && rd[i0] % V) good = false;
          for (int v = 1; v < V && good; v++) {
            int32_t iv = rev[c0 + v];
            if ((i0 < 0) != (iv < 0)) good = false;
            else if (i0 >= 0 && (iv != i0 + v || rd[iv] != rd[i0] + v)) good = false;
          }
        }
        if (good) break;
        V >>= 1;
      }
      const int64_t elems = D->pnumel;
      if (V > 1 || a == b) {
        uint32_t nvec = (uint32_t)(elems / V);
        int grid = (int)std::min<int64_t>((nvec + 255) / 256, (int64_t)nsm * 16);
        if (grid < 1) grid = 1;
#define LAUNCH_SEP(T, VV) k_relayout_sep<T, VV><<<grid, 256, 0, stream>>>(P, (const T *)src, (T *)dst, nvec)
        if (wb == 2) {
          if (V == 8) LAUNCH_SEP(uint16_t, 8); else if (V == 4) LAUNCH_SEP(uint16_t, 4);
          else if (V == 2) LAUNCH_SEP(uint16_t, 2); else LAUNCH_SEP(uint16_t, 1);
        } else {
          if (V == 4) LAUNCH_SEP(uint32_t, 4); else if (V == 2) LAUNCH_SEP(uint32_t, 2);
          else LAUNCH_SEP(uint32_t, 1);
        }
#undef LAUNCH_SEP
        count_launch();
        if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
        return ALT_OK;
      }
      // ---- K_TILE: transpose through shared memory
      int p1 = -1;
      for (int p = 0; p < D->prank; p++)
        if (D->pdim_owner[p] == b && D->pdim_rad[p] == 1 && D->pshape[p] > 1) p1 = p;
      const bool gvec_ok = elems % (16 / wb) == 0 && (reinterpret_cast<uintptr_t>(dst) & 15) == 0;
      if (gvec_ok && E0 < 16 / wb) {
        // ---- K_GVEC: short innermost runs (one 16-byte vector spans dims)
        const uint32_t nv = (uint32_t)(elems / (16 / wb));
        const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((nv + 255) / 256, (int64_t)nsm * 16));
        if (wb == 2) k_relayout_gvec<uint16_t><<<grid, 256, 0, stream>>>(P, (const uint16_t *)src, (uint16_t *)dst, nv);
        else k_relayout_gvec<uint32_t><<<grid, 256, 0, stream>>>(P, (const uint32_t *)src, (uint32_t *)dst, nv);
        count_launch();
        if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
        return ALT_OK;
      }
      if (p1 >= 0 && p1 != p0 && E0 % (16 / wb) != 0) {  // else K_GATHER below is faster
        TilePlan TP{};
        TP.P = P;
        TP.p0 = p0;
        TP.p1 = p1;
        TP.a = a;
        TP.b = b;
        TP.TX = (int32_t)std::min<int64_t>(E0, 64);
        while (E0 % TP.TX) TP.TX--;
        const int64_t Ey = D->pshape[p1];
        TP.TY = (int32_t)std::min<int64_t>(Ey, std::max<int64_t>(8, 4096 / TP.TX));
        if (TP.TY > 256) TP.TY = 256;
        TP.nx = (int32_t)(E0 / TP.TX);
        TP.ny = (int32_t)((Ey + TP.TY - 1) / TP.TY);
        TP.dstride_p1 = D->pstride[p1];
        TP.ey_total = (int32_t)Ey;
        TP.nxdiv = FastDiv(TP.nx);
        TP.nydiv = FastDiv(TP.ny);
        int64_t nt = (int64_t)TP.nx * TP.ny;
        int k = 0;
        for (int p = 0; p < D->prank; p++) {
          if (p == p0 || p == p1) continue;
          TP.outer[k] = p;
          TP.odiv[k] = FastDiv((uint32_t)D->pshape[p]);
          TP.ostride[k] = D->pstride[p];
          nt *= D->pshape[p];
          k++;
        }
        TP.nouter = k;
        TP.ntiles = (uint32_t)nt;
        const int LD = TP.TX + (wb == 2 ? 2 : 1);
        size_t smem = (((size_t)TP.TY * LD * wb + 15) & ~size_t(15)) + (size_t)(TP.TX + TP.TY) * 8;
        int grid = (int)std::min<int64_t>(nt, (int64_t)nsm * 8);
        if (wb == 2) {
          cudaFuncSetAttribute(k_relayout_tile<uint16_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
          k_relayout_tile<uint16_t><<<grid, 256, smem, stream>>>(TP, (const uint16_t *)src, (uint16_t *)dst);
        } else {
          cudaFuncSetAttribute(k_relayout_tile<uint32_t>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
          k_relayout_tile<uint32_t><<<grid, 256, smem, stream>>>(TP, (const uint32_t *)src, (uint32_t *)dst);
        }
        count_launch();
        if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
        return ALT_OK;
      }
      // ---- K_GATHER: 16-byte dst vectors along the dst innermost dim
      {
        const int VV = 16 / wb;
        bool ok = E0 % VV == 0 && D->pdim_rad[p0] == 1 && ((reinterpret_cast<uintptr_t>(dst) & 15) == 0);
        if (ok) {
          const uint32_t nv = (uint32_t)(elems / VV);
          const int grid = (int)std::max<int64_t>(1, std::min<int64_t>((nv + 255) / 256, (int64_t)nsm * 16));
          if (wb == 2) k_relayout_gather<uint16_t><<<grid, 256, 0, stream>>>(P, a, (const uint16_t *)src, (uint16_t *)dst, nv);
          else k_relayout_gather<uint32_t><<<grid, 256, 0, stream>>>(P, a, (const uint32_t *)src, (uint32_t *)dst, nv);
          count_launch();
          if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
          return ALT_OK;
        }
      }
      // ---- K_SEP scalar
      uint32_t nvec = (uint32_t)elems;
      int grid = (int)std::min<int64_t>((nvec + 255) / 256, (int64_t)nsm * 16);
      if (wb == 2) k_relayout_sep<uint16_t, 1><<<grid, 256, 0, stream>>>(P, (const uint16_t *)src, (uint16_t *)dst, nvec);
      else k_relayout_sep<uint32_t, 1><<<grid, 256, 0, stream>>>(P, (const uint32_t *)src, (uint32_t *)dst, nvec);
      count_launch();
      if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
      return ALT_OK;
    }
  }
  // ---- K_GENERIC
  if (!(S->flags & ALT_LOSSLESS)) {
    // the generic path cannot cheaply prove dst only needs present elements;
    // a lossy source is only accepted on the table path
    set_error("alt_relayout: lossy non-separable source");
    return ALT_E_LOSSY;
  }
  int64_t n = D->pnumel;
  int grid = (int)std::min<int64_t>((n + 255) / 256, (int64_t)nsm * 16);
  if (grid < 1) grid = 1;
  if (wb == 2) k_relayout_generic<uint16_t><<<grid, 256, 0, stream>>>(sdesc, ddesc, (const uint16_t *)src, (uint16_t *)dst, n);
  else k_relayout_generic<uint32_t><<<grid, 256, 0, stream>>>(sdesc, ddesc, (const uint32_t *)src, (uint32_t *)dst, n);
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("relayout launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

}  // namespace alt
