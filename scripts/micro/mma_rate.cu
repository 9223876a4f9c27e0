// tcgen05.mma issue-rate microbenchmark (developer tool, not product code):
// one thread issues ITER x 4 MMAs (M = 128, N = 64 / 128 / 256, K = 4 x 16
// over one 64-channel SW128 K-major slab, both operands in shared memory, as
// the conv kernel does) into one TMEM accumulator, commits, waits, and
// reports cycles per MMA; variants with the halo kernel's row-shifted A start
// (+ s rows, with and without the descriptor base-offset field).
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I../../paper_conf_eurosys_xuxpwwwdxcwc23_b200/csrc mma_rate.cu -o mma_rate
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "sm100.cuh"
using namespace alt::sm100;

template <int N>
__global__ void __launch_bounds__(128, 1) k_mma(int iters, int shift, int hboff, unsigned long long *out) {
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char *smem = reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  unsigned char *sA = smem;                 // 136 rows x 128 B
  unsigned char *sB = smem + 136 * 128 + 1024 - (136 * 128) % 1024;
  __shared__ uint64_t bar;
  __shared__ uint32_t tslot;
  for (int i = threadIdx.x; i < (136 * 128 + N * 128 + 2048) / 16; i += blockDim.x)
    reinterpret_cast<uint4 *>(smem)[i] = make_uint4(0x3f803f80u, 0, 0, 0);
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_mbar_init(); }
  if (threadIdx.x < 32) tmem_alloc<256>(&tslot);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tslot;
  if (threadIdx.x == 0) {
    const uint32_t idesc = idesc_f32acc(1, 128, N);
    uint64_t dA[4], dB[4];
    for (int kk = 0; kk < 4; kk++) {
      dA[kk] = smem_desc(smem_u32(sA) + kk * 32, 16, 1024, 2);
      dB[kk] = smem_desc(smem_u32(sB) + kk * 32, 16, 1024, 2);
    }
    const uint64_t aoff = (uint64_t)(shift * 8) | (hboff ? ((uint64_t)shift << 49) : 0ull);
    unsigned long long t0 = clock64();
    for (int it = 0; it < iters; it++)
#pragma unroll
      for (int kk = 0; kk < 4; kk++) mma_bf16(tmem, dA[kk] + aoff, dB[kk], idesc, (it | kk) ? 1u : 0u);
    unsigned long long t1 = clock64();
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    unsigned long long t2 = clock64();
    out[blockIdx.x * 2] = t1 - t0;
    out[blockIdx.x * 2 + 1] = t2 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc<256>(tmem);
}

template <int N>
void run(int ctas, int shift, int hboff) {
  unsigned long long *d, h[2 * 148];
  cudaMalloc(&d, sizeof(h));
  const int smem = 136 * 128 + N * 128 + 4096;
  cudaFuncSetAttribute(k_mma<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const int iters = 2000;
  k_mma<N><<<ctas, 128, smem>>>(100, shift, hboff, d);
  k_mma<N><<<ctas, 128, smem>>>(iters, shift, hboff, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("N %d: %s\n", N, cudaGetErrorString(e)); return; }
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  const double cyc = (double)h[1] / (iters * 4);
  printf("N %3d ctas %3d shift %d hboff %d: %.1f cycles / MMA (issue %.1f), floor 128*N/256 = %d, %.0f FLOP/clk/SM\n", N, ctas,
         shift, hboff, cyc, (double)h[0] / (iters * 4), 128 * N / 256, 2.0 * 128 * N * 16 / cyc);
  cudaFree(d);
}

int main() {
  for (int ctas : {1, 148}) {
    run<64>(ctas, 0, 0);
    run<128>(ctas, 0, 0);
    run<256>(ctas, 0, 0);
    run<64>(ctas, 1, 1);
    run<64>(ctas, 2, 1);
    run<64>(ctas, 1, 0);
    run<128>(ctas, 1, 1);
  }
  return 0;
}
