// store_at.cu — the store_at / decouple_at layout primitives (paper §4.1,
// P:783-795) on device, and the attached-bias row read of the GEMM that
// consumes a store_at weight ("attach each element of the bias
// vector to each column of the weight matrix ... the inner product and the
// bias addition in GMM may be computed together").
//
// Reading A26: Z = store_at(A, b, dim) has A's logical shape with
// extent E_dim + 1 along dim; Z[i] = A[i] for i_dim < E_dim, and
// Z[i] = b[i without dim] (b dense row-major) for i_dim == E_dim.  Z and A are
// stored through arbitrary compiled layouts (generic interpreter: dev_G on
// the destination, dev_F_offset on the source), so the fused tensor can put
// each bias element next to its weight column (e.g. Z stored [N, K + pad]).
#include <cuda_runtime.h>

#include "common.cuh"
#include "ops.h"

namespace alt {

void count_launch(int n);

namespace {

template <typename T>
__global__ void __launch_bounds__(256) k_store_at(const LayoutDesc *__restrict__ A, const LayoutDesc *__restrict__ Z,
                                                  const T *__restrict__ a, const T *__restrict__ b,
                                                  T *__restrict__ z, int32_t dim, int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    int64_t c[kStageRank];
    int64_t rem = j;
    for (int p = Z->prank - 1; p >= 0; p--) {
      const int64_t e = Z->shp[Z->np][p];
      c[p] = rem % e;
      rem /= e;
    }
    T v = 0;
    if (dev_G(*Z, c)) {
      const int64_t E = Z->shp[0][dim] - 1;  // A's extent along dim
      if (c[dim] < E) {
        const int64_t o = dev_F_offset(*A, c);
        if (o >= 0) v = a[o];
      } else {
        int64_t lin = 0;  // b[i without dim], row-major
        for (int d = 0; d < Z->lrank; d++)
          if (d != dim) lin = lin * Z->shp[0][d] + c[d];
        v = b[lin];
      }
    }
    z[j] = v;
  }
}

// a (through A's layout, every physical position incl. pad zeros) from Z
template <typename T>
__global__ void __launch_bounds__(256) k_decouple_a(const LayoutDesc *__restrict__ A, const LayoutDesc *__restrict__ Z,
                                                    const T *__restrict__ z, T *__restrict__ a, int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    int64_t c[kStageRank];
    int64_t rem = j;
    for (int p = A->prank - 1; p >= 0; p--) {
      const int64_t e = A->shp[A->np][p];
      c[p] = rem % e;
      rem /= e;
    }
    T v = 0;
    if (dev_G(*A, c)) {
      const int64_t o = dev_F_offset(*Z, c);
      if (o >= 0) v = z[o];
    }
    a[j] = v;
  }
}

// b (dense row-major over Z's dims without dim) = Z[.., E_dim, ..]; with
// to_f32 the bf16 / f32 value is widened to fp32 (the attached-bias read of
// the GEMM epilogue)
template <typename T, typename O>
__global__ void __launch_bounds__(256) k_decouple_b(const LayoutDesc *__restrict__ Z, const T *__restrict__ z,
                                                    O *__restrict__ b, int32_t dim, int64_t n) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    int64_t c[kMaxL];
    int64_t rem = j;
    for (int d = Z->lrank - 1; d >= 0; d--) {
      if (d == dim) { c[d] = Z->shp[0][d] - 1; continue; }
      const int64_t e = Z->shp[0][d];
      c[d] = rem % e;
      rem /= e;
    }
    const int64_t o = dev_F_offset(*Z, c);
    O v = 0;
    if (o >= 0) {
      if constexpr (sizeof(O) == sizeof(T)) v = z[o];
      else v = (O)bf16_to_f32((uint16_t)z[o]);
    }
    b[j] = v;
  }
}

int grid_for(int64_t n) {
  static int nsm = 0;
  if (!nsm) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    if (nsm <= 0) nsm = 148;
  }
  int64_t g = (n + 255) / 256;
  const int64_t cap = (int64_t)nsm * 8;
  if (g > cap) g = cap;
  return (int)(g < 1 ? 1 : g);
}

alt_status launched(const char *what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) { set_error("%s: launch failed: %s", what, cudaGetErrorString(e)); return ALT_E_CUDA; }
  count_launch(1);
  return ALT_OK;
}

}  // namespace

alt_status store_at_launch(Layout *A, const void *a, const void *b, int32_t dim, Layout *Z, void *z, int wb,
                           cudaStream_t s) {
  SepDev sa{}, sz{};
  const LayoutDesc *da = nullptr, *dz = nullptr;
  alt_status st = device_tables(A, &sa, &da);
  if (st != ALT_OK) return st;
  if ((st = device_tables(Z, &sz, &dz)) != ALT_OK) return st;
  const int64_t n = Z->pnumel;
  if (wb == 2)
    k_store_at<uint16_t><<<grid_for(n), 256, 0, s>>>(da, dz, (const uint16_t *)a, (const uint16_t *)b,
                                                     (uint16_t *)z, dim, n);
  else
    k_store_at<uint32_t><<<grid_for(n), 256, 0, s>>>(da, dz, (const uint32_t *)a, (const uint32_t *)b,
                                                     (uint32_t *)z, dim, n);
  return launched("alt_store_at");
}

alt_status decouple_at_launch(Layout *Z, const void *z, int32_t dim, Layout *A, void *a, void *b, int wb,
                              cudaStream_t s) {
  SepDev sa{}, sz{};
  const LayoutDesc *da = nullptr, *dz = nullptr;
  alt_status st = device_tables(A, &sa, &da);
  if (st != ALT_OK) return st;
  if ((st = device_tables(Z, &sz, &dz)) != ALT_OK) return st;
  const int64_t na = A->pnumel;
  const int64_t nb = Z->lnumel / Z->lshape[dim];
  if (wb == 2) {
    k_decouple_a<uint16_t><<<grid_for(na), 256, 0, s>>>(da, dz, (const uint16_t *)z, (uint16_t *)a, na);
    if ((st = launched("alt_decouple_at")) != ALT_OK) return st;
    k_decouple_b<uint16_t, uint16_t><<<grid_for(nb), 256, 0, s>>>(dz, (const uint16_t *)z, (uint16_t *)b, dim, nb);
  } else {
    k_decouple_a<uint32_t><<<grid_for(na), 256, 0, s>>>(da, dz, (const uint32_t *)z, (uint32_t *)a, na);
    if ((st = launched("alt_decouple_at")) != ALT_OK) return st;
    k_decouple_b<uint32_t, uint32_t><<<grid_for(nb), 256, 0, s>>>(dz, (const uint32_t *)z, (uint32_t *)b, dim, nb);
  }
  return launched("alt_decouple_at");
}

alt_status attached_row_f32(Layout *Z, const void *z, int32_t dim, int wb, float *out, cudaStream_t s) {
  SepDev sz{};
  const LayoutDesc *dz = nullptr;
  alt_status st = device_tables(Z, &sz, &dz);
  if (st != ALT_OK) return st;
  const int64_t nb = Z->lnumel / Z->lshape[dim];
  if (wb == 2)
    k_decouple_b<uint16_t, float><<<grid_for(nb), 256, 0, s>>>(dz, (const uint16_t *)z, out, dim, nb);
  else
    k_decouple_b<float, float><<<grid_for(nb), 256, 0, s>>>(dz, (const float *)z, out, dim, nb);
  return launched("alt_matmul_store_at");
}

}  // namespace alt
