// TMEM read throughput microbenchmark: W warps per CTA, each loops tcgen05.ld
// (shape per template) + wait over its lane quarter; one CTA per SM.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "sm100.cuh"
using namespace alt::sm100;

template <int MODE>
__global__ void k(int iters, unsigned long long *out, uint32_t *sink) {
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (warp == 0) tmem_alloc<512, 1>(&slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot;
  uint32_t x = 0;
  const uint32_t base = tmem + ((uint32_t)((warp & 3) * 32) << 16);
  const int colbase = (warp >> 2) * 128;
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
    if (MODE == 0) {
      uint32_t r[32];
      tmem_ld_32x32b_x32(base + colbase + (it & 3) * 32, r);
      tmem_ld_wait();
      x ^= r[lane] + r[(lane + 7) & 31];
    } else if (MODE == 1) {
      uint32_t r[4][32];
#pragma unroll
      for (int c = 0; c < 4; c++) tmem_ld_32x32b_x32(base + colbase + c * 32, r[c]);
      tmem_ld_wait();
#pragma unroll
      for (int c = 0; c < 4; c++) x ^= r[c][lane];
    } else if (MODE == 3 || MODE == 4) {
      // MODE 3: load, then independent ALU work, then use; MODE 4: ALU work only
      uint32_t r[32];
      if (MODE == 3) tmem_ld_32x32b_x32(base + colbase + (it & 3) * 32, r);
      float f = __uint_as_float(x) + 1.0f;
#pragma unroll
      for (int k = 0; k < 64; k++) f = fmaf(f, 1.0001f, 0.5f);
      x ^= __float_as_uint(f);
      if (MODE == 3) {
        tmem_ld_wait();
        x ^= r[lane] + r[(lane + 7) & 31];
      }
    } else {
      uint32_t r[64];
      tmem_ld_32x32b_x64(base + colbase + (it & 1) * 64, r);
      tmem_ld_wait();
      x ^= r[lane] + r[(lane + 33) & 63];
    }
  }
  unsigned long long t1 = clock64();
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = t1 - t0;
  if (x == 0x12345678u) sink[0] = x;
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512, 1>(tmem);
}

int main() {
  unsigned long long *d;
  uint32_t *s;
  cudaMalloc(&d, 148 * 8);
  cudaMalloc(&s, 4);
  const int iters = 4096;
  for (int mode = 0; mode < 5; mode++)
    for (int warps = 4; warps <= 8; warps += 4) {
      void (*kern)(int, unsigned long long *, uint32_t *) =
          mode == 0 ? k<0> : (mode == 1 ? k<1> : (mode == 2 ? k<2> : (mode == 3 ? k<3> : k<4>)));
      kern<<<148, warps * 32>>>(iters, d, s);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[148];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      const double bytes_per_iter = (mode == 0 || mode == 3 ? 4096.0 : (mode == 1 ? 16384.0 : (mode == 2 ? 8192.0 : 0.0))) * warps;
      printf("mode %d warps %d: %s  %.1f cycles/iter  %.1f B/clk per SM\n", mode, warps, cudaGetErrorString(e),
             (double)h[0] / iters, bytes_per_iter * iters / h[0]);
    }
  return 0;
}
