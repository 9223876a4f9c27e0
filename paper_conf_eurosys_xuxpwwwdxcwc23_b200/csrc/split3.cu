// split3.cu — fp32 operands for the tensor cores (reading A27).
//
// The paper's GPU arithmetic is fp32.  An fp32 value splits
// exactly into three bf16 terms, x = h + m + l + e with
//   h = bf16(x), m = bf16(x - h), l = bf16(x - h - m)   (RNE; each difference
//   is exact in fp32), |e| <= 2^-24 |x|,
// so x y = sum of the nine plane products; the six of weight > 2^-24 (hh, hm,
// mh, hl, mm, lh) run as bf16 tcgen05 MMAs with fp32 accumulation — the same
// tensor-core work as 3xTF32 (tf32 MMAs run at half the bf16 rate) with a
// smaller dropped remainder (2^-24 vs 2^-22).
//
// This kernel reads an fp32 operand through its declared layout (the Reader
// tables, any ALT layout) and writes the three planes as one bf16 tensor
// whose reduction dim is tripled and padded to Cp (multiple of 8): plane p
// holds channels [p Cp, p Cp + C), zeros up to (p + 1) Cp.  The planes are
// stored reduction-innermost ([outer][3 Cp], K-major for the MMA), written
// as 16-byte vectors.
#include <cuda_runtime.h>

#include <algorithm>

#include "epilogue.cuh"
#include "ops.h"

namespace alt {

alt_status make_reader(Layout *L, Reader *r);

struct Split3Args {
  Reader r;
  int32_t mode;            // 0: rank 4 (o0, c, o2, o3); 1: rank 2 (o, c); 2: rank 2 (c, o)
  int64_t D0, D2, D3;      // outer extents (rank 2: D2 = D3 = 1)
  int64_t C, Cp;           // reduction extent read / padded plane width
};

__device__ __forceinline__ uint16_t bf16_rn(float v) { return f32_to_bf16_rne(v); }

__global__ void k_split3(const Split3Args a, const float *__restrict__ src, uint16_t *__restrict__ dst) {
  const int64_t groups = a.Cp / 8;
  const int64_t total = a.D0 * a.D2 * a.D3 * groups;
  for (int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t o = t / groups, c0 = (t - o * groups) * 8;
    const int64_t i3 = o % a.D3, i2 = (o / a.D3) % a.D2, i0 = o / (a.D3 * a.D2);
    uint32_t ph[4], pm[4], pl[4];
#pragma unroll
    for (int j = 0; j < 8; j++) {
      const int64_t c = c0 + j;
      float x = 0.f;
      if (c < a.C) {
        const int64_t off = a.mode == 0 ? a.r.off4(i0, c, i2, i3) : (a.mode == 1 ? a.r.off2(i0, c) : a.r.off2(c, i0));
        if (off >= 0) x = __ldg(src + off);
      }
      const uint16_t h = bf16_rn(x);
      const float r1 = x - bf16_to_f32(h);
      const uint16_t m = bf16_rn(r1);
      const float r2 = r1 - bf16_to_f32(m);
      const uint16_t l = bf16_rn(r2);
      const int w = j >> 1, sh = (j & 1) * 16;
      if (sh == 0) { ph[w] = h; pm[w] = m; pl[w] = l; }
      else { ph[w] |= (uint32_t)h << 16; pm[w] |= (uint32_t)m << 16; pl[w] |= (uint32_t)l << 16; }
    }
    uint16_t *row = dst + o * 3 * a.Cp + c0;
    *reinterpret_cast<uint4 *>(row) = make_uint4(ph[0], ph[1], ph[2], ph[3]);
    *reinterpret_cast<uint4 *>(row + a.Cp) = make_uint4(pm[0], pm[1], pm[2], pm[3]);
    *reinterpret_cast<uint4 *>(row + 2 * a.Cp) = make_uint4(pl[0], pl[1], pl[2], pl[3]);
  }
}

// Split one fp32 operand (layout L, logical rank 4 with the reduction dim 1,
// or rank 2 with the reduction dim `red`) restricted to C reduction entries
// into dst (bf16, [outer][3 Cp]).
alt_status split3_launch(Layout *L, const float *src, int red, int64_t C, int64_t Cp, uint16_t *dst,
                         cudaStream_t stream) {
  Split3Args a{};
  alt_status st = make_reader(L, &a.r);
  if (st != ALT_OK) return st;
  a.C = C;
  a.Cp = Cp;
  if (L->lrank == 4) {
    a.mode = 0;
    a.D0 = L->lshape[0]; a.D2 = L->lshape[2]; a.D3 = L->lshape[3];
  } else {
    a.mode = red == 1 ? 1 : 2;
    a.D0 = L->lshape[red == 1 ? 0 : 1];
    a.D2 = a.D3 = 1;
  }
  const int64_t total = a.D0 * a.D2 * a.D3 * (Cp / 8);
  if (total == 0) return ALT_OK;
  const int grid = (int)std::min<int64_t>((total + 255) / 256, 148 * 16);
  k_split3<<<grid, 256, 0, stream>>>(a, src, dst);
  count_launch();
  if (cudaGetLastError() != cudaSuccess) { set_error("split3 launch failed"); return ALT_E_CUDA; }
  return ALT_OK;
}

}  // namespace alt
