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

  if (S->separable && D->separable) {
    // every element dst holds must have a copy in src
    for (int d = 0; d < D->lrank; d++)
      for (int32_t v : D->rev[d])
        if (v >= 0 && S->rd[d][v] < 0) { set_error("alt_relayout: source layout has no copy of an element dst needs"); return ALT_E_LOSSY; }
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
      if (p1 >= 0 && p1 != p0) {
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
