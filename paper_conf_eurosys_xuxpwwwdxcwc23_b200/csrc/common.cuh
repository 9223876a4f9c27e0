// common.cuh — small device helpers shared by the kernels.
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdlib>
#include <utility>

#include "layout.h"

namespace alt {

// Programmatic dependent launch for the CUDA-core kernels of a chain: the
// kernel may be scheduled while the previous kernel in the stream drains
// (its launch latency, and the next tensor-core kernel's prologue, overlap
// work); pdl_wait() at the top of the kernel orders every global access after
// the previous grid's completion.  Without the attribute both are no-ops.
__device__ __forceinline__ void pdl_wait() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kern)(KArgs...), int grid, int block, size_t smem, cudaStream_t s,
                              Args &&...args) {
  cudaLaunchConfig_t lc{};
  lc.gridDim = dim3((unsigned)grid);
  lc.blockDim = dim3((unsigned)block);
  lc.dynamicSmemBytes = smem;
  lc.stream = s;
  static const bool on = [] { const char *e = getenv("ALT_PDL_CC"); return !(e && e[0] == '0'); }();
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  lc.attrs = at;
  lc.numAttrs = on ? 1 : 0;
  return cudaLaunchKernelEx(&lc, kern, std::forward<Args>(args)...);
}

// Unsigned 32-bit division by a run-time constant (Granlund-Montgomery):
// q = mulhi(n, mul) >> shr, valid for n, d < 2^31.
// m = ceil(2^(32+l) / d), l = ceil(log2 d): exact for every n < 2^32.
struct FastDiv {
  uint32_t d = 1, shr = 0;
  uint64_t mul64 = 0;
  FastDiv() = default;
  explicit FastDiv(uint32_t div) : d(div) {
    if (div <= 1) { d = 1; return; }
    uint32_t l = 0;
    while ((1ull << l) < div) l++;
    mul64 = ((1ull << (32 + l)) + div - 1) / div;
    shr = l;
  }
  __host__ __device__ __forceinline__ uint32_t div(uint32_t n) const {
#ifdef __CUDA_ARCH__
    if (d == 1) return n;
    return (uint32_t)(((uint64_t)n * mul64) >> (32 + shr));
#else
    return n / d;
#endif
  }
  __host__ __device__ __forceinline__ void divmod(uint32_t n, uint32_t &q, uint32_t &r) const {
    q = div(n);
    r = n - q * d;
  }
};

// bit-exact element copy types
template <int B> struct Word;
template <> struct Word<2> { using T = uint16_t; };
template <> struct Word<4> { using T = uint32_t; };

__device__ __forceinline__ float bf16_to_f32(uint16_t h) { return __uint_as_float(((uint32_t)h) << 16); }
// round-to-nearest-even fp32 -> bf16 bits (NaN stays NaN)
__device__ __forceinline__ uint16_t f32_to_bf16_rne(float f) {
  return __bfloat16_as_ushort(__float2bfloat16_rn(f));
}

// Generic interpreter on device: phys coords -> logical (false = zero).
static __device__ __noinline__ bool dev_G(const LayoutDesc &D, int64_t *cur) {
  int64_t prev[kStageRank];
  for (int s = D.np - 1; s >= 0; s--) {
    const int64_t *E = D.shp[s];
    int rp = D.rank[s], k = D.dim[s];
    switch (D.kind[s]) {
      case ALT_SPLIT: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        int64_t i = 0;
        for (int l = 0; l < m; l++) i = i * D.v[s][l] + cur[k + l];
        prev[k] = i;
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + m - 1];
        break;
      }
      case ALT_REORDER:
        for (int j = 0; j < rp; j++) prev[D.v[s][j]] = cur[j];
        break;
      case ALT_FUSE: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        int64_t e = cur[k];
        for (int l = m - 1; l >= 0; l--) { prev[k + l] = e % E[k + l]; e /= E[k + l]; }
        for (int d = k + m; d < rp; d++) prev[d] = cur[d - m + 1];
        break;
      }
      case ALT_UNFOLD: {
        for (int d = 0; d < k; d++) prev[d] = cur[d];
        int64_t i = cur[k] * D.v[s][1] + cur[k + 1];
        if (i >= E[k]) return false;
        prev[k] = i;
        for (int d = k + 1; d < rp; d++) prev[d] = cur[d + 1];
        break;
      }
      case ALT_PAD: {
        for (int d = 0; d < rp; d++) prev[d] = cur[d];
        int64_t i = cur[k] - D.v[s][0];
        if (i < 0 || i >= E[k]) return false;
        prev[k] = i;
        break;
      }
    }
    for (int d = 0; d < rp; d++) cur[d] = prev[d];
  }
  return true;
}

// logical coords -> owner physical linear offset (-1 = no copy)
static __device__ __noinline__ int64_t dev_F_offset(const LayoutDesc &D, const int64_t *logical) {
  int64_t cur[kStageRank], nxt[kStageRank];
  for (int d = 0; d < D.lrank; d++) cur[d] = logical[d];
  for (int s = 0; s < D.np; s++) {
    int r = D.rank[s], k = D.dim[s];
    const int64_t *E = D.shp[s];
    switch (D.kind[s]) {
      case ALT_SPLIT: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t i = cur[k];
        for (int l = m - 1; l >= 0; l--) { nxt[k + l] = i % D.v[s][l]; i /= D.v[s][l]; }
        for (int d = k + 1; d < r; d++) nxt[d + m - 1] = cur[d];
        break;
      }
      case ALT_REORDER:
        for (int j = 0; j < r; j++) nxt[j] = cur[D.v[s][j]];
        break;
      case ALT_FUSE: {
        int m = D.n[s];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t e = 0;
        for (int l = 0; l < m; l++) e = e * E[k + l] + cur[k + l];
        nxt[k] = e;
        for (int d = k + m; d < r; d++) nxt[d - m + 1] = cur[d];
        break;
      }
      case ALT_UNFOLD: {
        int64_t B = D.v[s][0], S = D.v[s][1], T = D.shp[s + 1][k];
        for (int d = 0; d < k; d++) nxt[d] = cur[d];
        int64_t t = cur[k] / S;
        if (t > T - 1) t = T - 1;
        int64_t b = cur[k] - t * S;
        if (b >= B) return -1;
        nxt[k] = t;
        nxt[k + 1] = b;
        for (int d = k + 1; d < r; d++) nxt[d + 1] = cur[d];
        break;
      }
      case ALT_PAD:
        for (int d = 0; d < r; d++) nxt[d] = cur[d];
        nxt[k] = cur[k] + D.v[s][0];
        break;
    }
    for (int d = 0; d < D.rank[s + 1]; d++) cur[d] = nxt[d];
  }
  int64_t off = 0;
  for (int d = 0; d < D.prank; d++) off += cur[d] * D.pstride[d];
  return off;
}

// launch accounting (alt_launch_count)
void count_launch(int n = 1);

}  // namespace alt
