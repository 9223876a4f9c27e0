// Issue cost of the mbarrier / TMA operations a producer loop is made of
// (single thread, clock64 around N repetitions).  Developer tool.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include "sm100.cuh"
using namespace alt::sm100;

__global__ void k(const __grid_constant__ CUtensorMap tm, long long *out) {
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char *smem = reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar[4];
  if (threadIdx.x != 0) return;
  mbar_init(&bar[0], 1); mbar_init(&bar[1], 1 << 19); mbar_init(&bar[2], 1); mbar_init(&bar[3], 1);
  fence_mbar_init();
  const int N = 256;
  long long t0, t1;
  // (a) try_wait on a completed phase: complete phase 0 of bar[0] first
  mbar_arrive(&bar[0]);
  t0 = clock64();
  for (int i = 0; i < N; i++) mbar_wait(&bar[0], 0);
  t1 = clock64(); out[0] = (t1 - t0) / N;
  // (b) arrive (no completion: count 1<<20)
  t0 = clock64();
  for (int i = 0; i < N; i++) mbar_arrive(&bar[1]);
  t1 = clock64(); out[1] = (t1 - t0) / N;
  // (c) expect_tx on bar[1]
  t0 = clock64();
  for (int i = 0; i < N; i++) mbar_expect_tx(&bar[1], 16);
  mbar_arrive(&bar[0]);
  t1 = clock64(); out[2] = (t1 - t0) / N;
  // (d) TMA issue: 16 KB boxes into one buffer tracked by bar[2] (expect N*16KB first)
  asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(&bar[2])), "r"(32 * 16384) : "memory");
  t0 = clock64();
  for (int i = 0; i < 32; i++) tma_load_5d(smem, &tm, &bar[2], 0, (i & 63) * 128, 0, 0, 0);
  t1 = clock64(); out[3] = (t1 - t0) / 32;
  mbar_arrive(&bar[2]);
  mbar_wait(&bar[2], 0);
  long long t2 = clock64(); out[4] = t2 - t1;  // drain time after the last issue
  // (e) round trip: expect_tx + 1 TMA + wait, serial
  t0 = clock64();
  for (int i = 0; i < 32; i++) {
    mbar_expect_tx(&bar[3], 16384);
    tma_load_5d(smem, &tm, &bar[3], 0, (i & 63) * 128, 0, 0, 0);
    mbar_wait(&bar[3], i & 1);
  }
  t1 = clock64(); out[5] = (t1 - t0) / 32;
}

// tcgen05.mma issue cost and completion time (M = 128, N = NN, K = 16 each)
template <int NN>
__global__ void kmma(long long *out) {
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char *smem = reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32;
  if (warp == 0) tmem_alloc<512, 1>(&slot);
  if (threadIdx.x == 32) { mbar_init(&bar, 1); fence_mbar_init(); }
  for (int i = threadIdx.x; i < 48 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t *>(smem)[i] = 0;
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (threadIdx.x == 32) {
    const uint32_t tmem = slot;
    constexpr uint32_t idesc = idesc_f32acc(1, 128, NN);
    const uint32_t a = smem_u32(smem), b = smem_u32(smem + 16384);
    const int N = 64;
    long long t0 = clock64();
    for (int i = 0; i < N; i++) {
      const uint64_t ad = smem_desc(a + (i & 3) * 32, 16, 1024, 2);
      const uint64_t bd = smem_desc(b + (i & 3) * 32, 16, 1024, 2);
      mma_bf16(tmem, ad, bd, idesc, i > 0);
    }
    long long t1 = clock64();
    mma_commit(&bar);
    mbar_wait(&bar, 0);
    long long t2 = clock64();
    out[0] = (t1 - t0) / N;
    out[1] = (t2 - t0) / N;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc<512, 1>(slot);
}

int main() {
  void *buf; cudaMalloc(&buf, 1 << 24); cudaMemset(buf, 0, 1 << 24);
  long long *out; cudaMalloc(&out, 64 * 8);
  cudaDriverEntryPointQueryResult q; void *p = nullptr;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  auto enc = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  CUtensorMap tm;
  cuuint64_t d[5] = {64, 1 << 16, 1, 1, 1}, st[4] = {128, 128ull << 16, 128ull << 16, 128ull << 16};
  cuuint32_t b[5] = {64, 128, 1, 1, 1}, e[5] = {1, 1, 1, 1, 1};
  enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, buf, d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
      CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  for (int rep = 0; rep < 2; rep++) {
    k<<<1, 32, 20 * 1024>>>(tm, out);
    cudaError_t err = cudaDeviceSynchronize();
    if (err != cudaSuccess) { printf("%s\n", cudaGetErrorString(err)); return 1; }
  }
  cudaFuncSetAttribute(kmma<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  cudaFuncSetAttribute(kmma<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  long long hm[2];
  for (int rep = 0; rep < 2; rep++) kmma<64><<<1, 64, 50 * 1024>>>(out + 16);
  cudaDeviceSynchronize();
  cudaMemcpy(hm, out + 16, sizeof(hm), cudaMemcpyDeviceToHost);
  printf("mma N=64: issue %lld clk/instr, completion %lld clk/instr\n", hm[0], hm[1]);
  for (int rep = 0; rep < 2; rep++) kmma<256><<<1, 64, 50 * 1024>>>(out + 16);
  if (cudaDeviceSynchronize() != cudaSuccess) printf("mma kernel failed\n");
  cudaMemcpy(hm, out + 16, sizeof(hm), cudaMemcpyDeviceToHost);
  printf("mma N=256: issue %lld clk/instr, completion %lld clk/instr\n", hm[0], hm[1]);
  long long h[6];
  cudaMemcpy(h, out, sizeof(h), cudaMemcpyDeviceToHost);
  printf("try_wait (done phase) %lld clk\narrive %lld clk\nexpect_tx %lld clk\nTMA issue 16KB %lld clk\ndrain %lld clk\n"
         "serial expect+TMA+wait round trip %lld clk\n", h[0], h[1], h[2], h[3], h[4], h[5]);
  return 0;
}
