// epilogue.cuh — reading operands through, and writing results into, any
// compiled ALT layout from device code.
//
// The writer is the producer half of layout propagation (Fig. 5b,
// P:870-879): a conv / GEMM epilogue stores each result element at every
// physical position its output layout holds it (all unfold copies), and
// writes 0 into the structural-zero positions it owns (pad / overhang,
// reading A8), so the consumer reads its tuned layout with no conversion op.
#pragma once
#include "common.cuh"

namespace alt {

// Offsets of logical elements in a layout: separable tables or interpreter.
struct Reader {
  int32_t sep;
  int32_t lrank;
  const int64_t *rd[4];
  const LayoutDesc *desc;
  __device__ __forceinline__ int64_t off4(int64_t i0, int64_t i1, int64_t i2, int64_t i3) const {
    if (sep) {
      int64_t a = __ldg(rd[0] + i0), b = __ldg(rd[1] + i1), c = __ldg(rd[2] + i2), d = __ldg(rd[3] + i3);
      if ((a | b | c | d) < 0) return -1;
      return a + b + c + d;
    }
    int64_t l[4] = {i0, i1, i2, i3};
    return dev_F_offset(*desc, l);
  }
  __device__ __forceinline__ int64_t off2(int64_t i0, int64_t i1) const {
    if (sep) {
      int64_t a = __ldg(rd[0] + i0), b = __ldg(rd[1] + i1);
      if ((a | b) < 0) return -1;
      return a + b;
    }
    int64_t l[2] = {i0, i1};
    return dev_F_offset(*desc, l);
  }
};

// Rank-5 reader / writer (C3D operands): owner offsets of a separable layout,
// or the primitive interpreter; every position an element owns.
struct Reader5 {
  int32_t sep;
  const int64_t *rd[5];
  const LayoutDesc *desc;
  __device__ __forceinline__ int64_t off5(int64_t i0, int64_t i1, int64_t i2, int64_t i3, int64_t i4) const {
    if (sep) {
      const int64_t a = __ldg(rd[0] + i0), b = __ldg(rd[1] + i1), c = __ldg(rd[2] + i2), d = __ldg(rd[3] + i3),
                    e = __ldg(rd[4] + i4);
      if ((a | b | c | d | e) < 0) return -1;
      return a + b + c + d + e;
    }
    int64_t l[5] = {i0, i1, i2, i3, i4};
    return dev_F_offset(*desc, l);
  }
};
struct Writer5 {
  const int32_t *wptr[5];
  const int64_t *wlist[5];
};

// Every physical position owned by a logical element (separable layouts).
struct Writer {
  int32_t lrank;
  const int32_t *wptr[4];
  const int64_t *wlist[4];
};

struct EpiParams {
  const float *scale;
  const float *bias;
  const void *residual;
  Reader res;
  int32_t act;
  // bias attached to the weight by store_at: the bias of output
  // channel k is batt[batt_base + batt_rd[k]] (bf16 or fp32), read in place
  const void *batt;
  const int64_t *batt_rd;
  int64_t batt_base;
  int32_t batt_bf16;
};

__device__ __forceinline__ float epi_bias(const EpiParams &e, int64_t k) {
#ifndef ALT_NO_BATT  // developer A/B knob: build without the attached-bias read
  if (e.batt) {
    const int64_t o = e.batt_base + __ldg(e.batt_rd + k);
    return e.batt_bf16 ? bf16_to_f32(__ldg(static_cast<const uint16_t *>(e.batt) + o))
                       : __ldg(static_cast<const float *>(e.batt) + o);
  }
#endif
  return __ldg(e.bias + k);
}

__device__ __forceinline__ float apply_act(float v, int act) {
  if (act == 1) v = fmaxf(v, 0.f);
  else if (act == 2) v = fminf(fmaxf(v, 0.f), 6.f);
  return v;
}

template <typename T>
__device__ __forceinline__ float load_as_f32(const T *p, int64_t o);
template <>
__device__ __forceinline__ float load_as_f32<float>(const float *p, int64_t o) { return __ldg(p + o); }
template <>
__device__ __forceinline__ float load_as_f32<uint16_t>(const uint16_t *p, int64_t o) {
  return bf16_to_f32(__ldg(p + o));
}

template <typename T>
__device__ __forceinline__ T from_f32(float v);
template <>
__device__ __forceinline__ float from_f32<float>(float v) { return v; }
template <>
__device__ __forceinline__ uint16_t from_f32<uint16_t>(float v) { return f32_to_bf16_rne(v); }

// store one rank-4 logical element (conv y[n,k,p,q]) through the writer
template <typename T>
__device__ __forceinline__ void write4(const Writer &W, T *y, int64_t i0, int64_t i1, int64_t i2,
                                       int64_t i3, T v) {
  const int32_t a0 = __ldg(W.wptr[0] + i0), a1 = __ldg(W.wptr[0] + i0 + 1);
  const int32_t b0 = __ldg(W.wptr[1] + i1), b1 = __ldg(W.wptr[1] + i1 + 1);
  const int32_t c0 = __ldg(W.wptr[2] + i2), c1 = __ldg(W.wptr[2] + i2 + 1);
  const int32_t d0 = __ldg(W.wptr[3] + i3), d1 = __ldg(W.wptr[3] + i3 + 1);
  for (int32_t a = a0; a < a1; a++) {
    const int64_t ca = __ldg(W.wlist[0] + a);
    for (int32_t b = b0; b < b1; b++) {
      const int64_t cb = __ldg(W.wlist[1] + b);
      for (int32_t c = c0; c < c1; c++) {
        const int64_t cc = __ldg(W.wlist[2] + c);
        for (int32_t d = d0; d < d1; d++) {
          // each code is 2*offset + is_zero
          const int64_t cd = __ldg(W.wlist[3] + d);
          const int64_t off = (ca >> 1) + (cb >> 1) + (cc >> 1) + (cd >> 1);
          y[off] = ((ca | cb | cc | cd) & 1) ? T(0) : v;
        }
      }
    }
  }
}

template <typename T>
__device__ __forceinline__ void write2(const Writer &W, T *y, int64_t i0, int64_t i1, T v) {
  const int32_t a0 = __ldg(W.wptr[0] + i0), a1 = __ldg(W.wptr[0] + i0 + 1);
  const int32_t b0 = __ldg(W.wptr[1] + i1), b1 = __ldg(W.wptr[1] + i1 + 1);
  for (int32_t a = a0; a < a1; a++) {
    const int64_t ca = __ldg(W.wlist[0] + a);
    for (int32_t b = b0; b < b1; b++) {
      const int64_t cb = __ldg(W.wlist[1] + b);
      y[(ca >> 1) + (cb >> 1)] = ((ca | cb) & 1) ? T(0) : v;
    }
  }
}

}  // namespace alt
