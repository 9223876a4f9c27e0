// TMEM -> register throughput vs warps / loads in flight / load shape.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include "sm100.cuh"
using namespace alt::sm100;

__device__ __forceinline__ void ld128(uint32_t taddr, uint32_t (&r)[128]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x128.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31, %32, %33, %34, %35, %36, %37, %38, %39, %40, %41, %42, %43, %44, %45, %46, %47, %48, %49, %50, %51, %52, %53, %54, %55, %56, %57, %58, %59, %60, %61, %62, %63, %64, %65, %66, %67, %68, %69, %70, %71, %72, %73, %74, %75, %76, %77, %78, %79, %80, %81, %82, %83, %84, %85, %86, %87, %88, %89, %90, %91, %92, %93, %94, %95, %96, %97, %98, %99, %100, %101, %102, %103, %104, %105, %106, %107, %108, %109, %110, %111, %112, %113, %114, %115, %116, %117, %118, %119, %120, %121, %122, %123, %124, %125, %126, %127}, [%128];"
    : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]), "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]), "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]), "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]), "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]), "=r"(r[61]), "=r"(r[62]), "=r"(r[63]), "=r"(r[64]), "=r"(r[65]), "=r"(r[66]), "=r"(r[67]), "=r"(r[68]), "=r"(r[69]), "=r"(r[70]), "=r"(r[71]), "=r"(r[72]), "=r"(r[73]), "=r"(r[74]), "=r"(r[75]), "=r"(r[76]), "=r"(r[77]), "=r"(r[78]), "=r"(r[79]), "=r"(r[80]), "=r"(r[81]), "=r"(r[82]), "=r"(r[83]), "=r"(r[84]), "=r"(r[85]), "=r"(r[86]), "=r"(r[87]), "=r"(r[88]), "=r"(r[89]), "=r"(r[90]), "=r"(r[91]), "=r"(r[92]), "=r"(r[93]), "=r"(r[94]), "=r"(r[95]), "=r"(r[96]), "=r"(r[97]), "=r"(r[98]), "=r"(r[99]), "=r"(r[100]), "=r"(r[101]), "=r"(r[102]), "=r"(r[103]), "=r"(r[104]), "=r"(r[105]), "=r"(r[106]), "=r"(r[107]), "=r"(r[108]), "=r"(r[109]), "=r"(r[110]), "=r"(r[111]), "=r"(r[112]), "=r"(r[113]), "=r"(r[114]), "=r"(r[115]), "=r"(r[116]), "=r"(r[117]), "=r"(r[118]), "=r"(r[119]), "=r"(r[120]), "=r"(r[121]), "=r"(r[122]), "=r"(r[123]), "=r"(r[124]), "=r"(r[125]), "=r"(r[126]), "=r"(r[127])
    : "r"(taddr));
}

// MODE 0: x32 ld+wait; 1: x64; 2: x128; 3: two x32 in flight then wait
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
  const int nw = blockDim.x / 32;
  const uint32_t base = tmem + ((uint32_t)((warp & 3) * 32) << 16);
  const int colbase = ((warp >> 2) * 512 / (nw / 4)) & 511;  // spread the warps of a quarter over columns
  __syncthreads();
  unsigned long long t0 = clock64();
  for (int it = 0; it < iters; it++) {
    if (MODE == 0) {
      uint32_t r[32];
      tmem_ld_32x32b_x32(base + ((colbase + (it & 3) * 32) & 511), r);
      tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; j++) x += r[j];
    } else if (MODE == 1) {
      uint32_t r[64];
      tmem_ld_32x32b_x64(base + ((colbase + (it & 1) * 64) & 511), r);
      tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 64; j++) x += r[j];
    } else if (MODE == 2) {
      uint32_t r[128];
      ld128(base + (colbase & 384), r);
      tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 128; j++) x += r[j];
    } else {
      uint32_t r[32], s[32];
      tmem_ld_32x32b_x32(base + (colbase & 511), r);
      tmem_ld_32x32b_x32(base + ((colbase + 32) & 511), s);
      tmem_ld_wait();
#pragma unroll
      for (int j = 0; j < 32; j++) x += r[j] ^ s[j];
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
  const int iters = 2048;
  for (int mode = 0; mode < 4; mode++)
    for (int warps : {4, 8, 16}) {
      void (*kern)(int, unsigned long long *, uint32_t *) = mode == 0 ? k<0> : mode == 1 ? k<1> : mode == 2 ? k<2> : k<3>;
      kern<<<148, warps * 32>>>(iters, d, s);
      cudaError_t e = cudaDeviceSynchronize();
      unsigned long long h[148];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      const double bytes_per_iter_warp = mode == 0 ? 4096.0 : mode == 1 ? 8192.0 : mode == 2 ? 16384.0 : 8192.0;
      printf("mode %d (%s) warps %2d: %s  %7.1f cycles/iter  %6.1f B/clk per SM\n", mode,
             mode == 0 ? "x32" : mode == 1 ? "x64" : mode == 2 ? "x128" : "2 x32", warps, cudaGetErrorString(e),
             (double)h[0] / iters, bytes_per_iter_warp * warps * iters / h[0]);
    }
  return 0;
}
