// TMA load throughput microbenchmark (developer tool, not product code).
// One CTA per SM: lane 0 of warp 0 streams boxes through an S-stage smem
// ring (expect_tx + cp.async.bulk.tensor), lane 0 of warp 1 waits on each
// stage's full barrier and frees it at once.  Reports chip GB/s and bytes
// per SM clock for several box shapes / footprints.
// build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I../../paper_conf_eurosys_xuxpwwwdxcwc23_b200/csrc tma_bw.cu -o tma_bw
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstdint>
#include <vector>

#include "sm100.cuh"
using namespace alt::sm100;

constexpr int MAXST = 16;

struct Pat {
  int rank;
  int box_bytes;
  int32_t ext[5];   // coordinate extents to sweep (in box units per dim: start = idx * step)
  int32_t step[5];
  int loads;        // loads per stage
  int stages;
};

__device__ __forceinline__ void mbar_spin(uint64_t *bar, uint32_t parity) {
  const uint32_t a = smem_u32(bar);
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(a),
      "r"(parity)
      : "memory");
}
template <int MODE>
__global__ void __launch_bounds__(64, 1) k_tma(const __grid_constant__ CUtensorMap tm, Pat p, int iters,
                                               unsigned long long *cyc) {
  extern __shared__ __align__(1024) unsigned char smem_raw[];
  unsigned char *smem = reinterpret_cast<unsigned char *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[MAXST], empty[MAXST];
  const int STAGES = p.stages;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int sbytes = p.box_bytes * p.loads;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; s++) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    fence_mbar_init();
    tma_prefetch(&tm);
  }
  __syncthreads();
  unsigned long long t0 = clock64();
  if (MODE == 7 || MODE == 8) {
    // one box per lane: lanes 0 .. loads-1 of warp 0 issue the boxes of a
    // stage concurrently (the conv kernel's producer pattern)
    if (warp == 0) {
      int stage = 0; uint32_t ph = 0;
      for (int it = 0; it < iters; it++) {
        if (it >= STAGES) mbar_wait(&empty[stage], ph ^ 1);
        if (lane == 0) mbar_expect_tx(&full[stage], sbytes);
        __syncwarp();
        const int32_t cc = ((blockIdx.x * 37 + it * p.loads + lane) & 63);
        if (lane < p.loads)
          tma_load_5d(smem + stage * sbytes + lane * p.box_bytes, &tm, &full[stage], 0,
                      MODE == 7 ? cc * p.step[1] : 0, MODE == 8 ? cc * p.step[2] : 0, 0, 0);
        if (++stage == STAGES) { stage = 0; ph ^= 1; }
      }
    } else if (warp == 1 && lane == 0) {
      int stage = 0; uint32_t ph = 0;
      for (int it = 0; it < iters; it++) {
        if (MODE == 9) mbar_spin(&full[stage], ph); else mbar_wait(&full[stage], ph);
        mbar_arrive(&empty[stage]);
        if (++stage == STAGES) { stage = 0; ph ^= 1; }
      }
    }
  } else if (MODE == 6 || MODE == 9) {
    // MODE 9: both sides spin on test_wait instead of try_wait
    if (warp == 0 && lane == 0) {
      int stage = 0; uint32_t ph = 0;
      for (int it = 0; it < iters; it++) {
        if (it >= STAGES) { if (MODE == 9) mbar_spin(&empty[stage], ph ^ 1); else mbar_wait(&empty[stage], ph ^ 1); }
        mbar_expect_tx(&full[stage], sbytes);
        for (int l = 0; l < p.loads; l++)
          tma_load_5d(smem + stage * sbytes + l * p.box_bytes, &tm, &full[stage], 0, ((blockIdx.x * 37 + it * p.loads + l) & 63) * p.step[1], 0, 0, 0);
        if (++stage == STAGES) { stage = 0; ph ^= 1; }
      }
    } else if (warp == 1 && lane == 0) {
      int stage = 0; uint32_t ph = 0;
      for (int it = 0; it < iters; it++) {
        if (MODE == 9) mbar_spin(&full[stage], ph); else mbar_wait(&full[stage], ph);
        mbar_arrive(&empty[stage]);
        if (++stage == STAGES) { stage = 0; ph ^= 1; }
      }
    }
  } else
  if (warp == 0 && lane == 0) {
    for (int it = 0; it < iters; it++) {
      const int stage = it % STAGES, round = it / STAGES;
      if (round > 0) { if (MODE >= 4) mbar_spin(&empty[stage], (round - 1) & 1); else mbar_wait(&empty[stage], (round - 1) & 1); }
      mbar_expect_tx(&full[stage], sbytes);
      for (int l = 0; l < p.loads; l++) {
        // linear box index -> coordinates (mixed radix over ext)
        int32_t c[5] = {0, 0, 0, 0, 0};
        if (MODE == 0 || MODE == 1 || MODE == 5) {
          uint32_t idx = (uint32_t)((blockIdx.x * 7919u + it * p.loads + l) * 2654435761u);
          for (int d = 0; d < p.rank; d++) {
            c[d] = (int32_t)(idx % (uint32_t)p.ext[d]) * p.step[d];
            idx /= (uint32_t)p.ext[d];
          }
        } else {
          c[1] = ((blockIdx.x * 37 + it * p.loads + l) & 63) * p.step[1];
        }
        void *dst = smem + stage * sbytes + l * p.box_bytes;
        if (MODE == 1 || MODE == 3) {
          asm volatile(
              "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
              " [%0], [%1, {%3, %4}], [%2];" ::"r"(smem_u32(dst)),
              "l"(reinterpret_cast<uint64_t>(&tm)), "r"(smem_u32(&full[stage])), "r"(c[0]), "r"(c[1])
              : "memory");
        } else {
          tma_load_5d(dst, &tm, &full[stage], c[0], c[1], c[2], c[3], c[4]);
        }
      }
    }
  } else if (warp == 1 && lane == 0) {
    for (int it = 0; it < iters; it++) {
      const int stage = it % STAGES, round = it / STAGES;
      if (MODE >= 4) mbar_spin(&full[stage], round & 1); else mbar_wait(&full[stage], round & 1);
      mbar_arrive(&empty[stage]);
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) cyc[blockIdx.x] = clock64() - t0;
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  cudaDriverEntryPointQueryResult q;
  void *p = nullptr;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q);
  return reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
}

// rank-5 map over a bf16 tensor with dims (innermost first) and box; element strides 1
static CUtensorMap make_map(void *base, std::vector<uint64_t> dims, std::vector<uint32_t> box, int swz_bytes,
                            std::vector<uint32_t> es = {}, int rank = 5) {
  CUtensorMap tm;
  cuuint64_t d[5], st[4];
  cuuint32_t b[5], e[5];
  uint64_t prev = 2;
  for (int i = 0; i < 5; i++) {
    d[i] = i < (int)dims.size() ? dims[i] : 1;
    b[i] = i < (int)box.size() ? box[i] : 1;
    e[i] = i < (int)es.size() ? es[i] : 1;
    if (i > 0) st[i - 1] = prev;
    prev *= d[i];
  }
  auto swz = swz_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE;
  CUresult r = get_encode()(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, rank, base, d, st, b, e, CU_TENSOR_MAP_INTERLEAVE_NONE,
                            swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) printf("encode failed %d\n", (int)r);
  return tm;
}

int main() {
  int nsm;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  const size_t big = (size_t)1 << 30;
  void *buf;
  cudaMalloc(&buf, big);
  cudaMemset(buf, 0, big);
  unsigned long long *cyc;
  cudaMalloc(&cyc, 4 * nsm * sizeof(unsigned long long));
  for (auto f : {k_tma<0>, k_tma<1>, k_tma<2>, k_tma<3>, k_tma<4>, k_tma<5>, k_tma<6>, k_tma<7>, k_tma<8>, k_tma<9>}) if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 210 * 1024) != cudaSuccess) printf("attr failed\n");
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char *name, std::vector<uint64_t> dims, std::vector<uint32_t> box, Pat p, int ctas_per_sm, int mode = 0) {
    CUtensorMap tm = make_map(buf, dims, box, 128, {}, (mode == 1 || mode == 3) ? 2 : 5);
    auto kern = mode == 0 ? k_tma<0> : mode == 1 ? k_tma<1> : mode == 2 ? k_tma<2> : mode == 3 ? k_tma<3> : mode == 4 ? k_tma<4> : mode == 5 ? k_tma<5> : mode == 6 ? k_tma<6> : mode == 7 ? k_tma<7> : mode == 8 ? k_tma<8> : k_tma<9>;
    const int iters = 2048;
    const int smem = p.stages * p.box_bytes * p.loads + 1024;
    const int grid = nsm * ctas_per_sm;
    kern<<<grid, 64, smem>>>(tm, p, 64, cyc);
    cudaEventRecord(e0);
    kern<<<grid, 64, smem>>>(tm, p, iters, cyc);
    cudaEventRecord(e1);
    cudaError_t err = cudaGetLastError();
    if (err == cudaSuccess) err = cudaDeviceSynchronize();
    if (err != cudaSuccess) { printf("%s: %s\n", name, cudaGetErrorString(err)); exit(1); }
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    const double bytes = (double)grid * iters * p.box_bytes * p.loads;
    printf("mode %d %-44s box %5d B x%d, %2d st, %d CTA/SM: %8.1f GB/s %6.1f B/clk/SM@1.965\n", mode, name, p.box_bytes, p.loads,
           p.stages, ctas_per_sm, bytes / ms / 1e6, bytes / ms / 1e6 / nsm / 1.965);
  };
  if (getenv("TMA_ALL")) {
    uint64_t R = (uint64_t)1 << 22;
    int cfgs[][3] = {{128, 1, 6}, {128, 2, 4}, {64, 2, 6}, {32, 4, 6}, {16, 8, 6}, {128, 3, 3}, {64, 4, 4},
                     {32, 8, 4}, {128, 4, 3}, {256, 1, 4}, {256, 2, 3}};
    for (auto &c : cfgs) {
      Pat p = {2, c[0] * 128, {1, (int32_t)(R / c[0])}, {0, c[0]}, c[1], c[2]};
      run("2D [R][64] concurrent lanes", {64, R}, {64, (uint32_t)c[0]}, p, 1, 7);
    }
  }
  // single-lane issue, L2-resident boxes (64 distinct): try_wait (6) vs spin (9),
  // boxes per stage, stage depth
  for (int mode : {6, 9}) {
    uint64_t R = (uint64_t)1 << 22;
    for (int rows : {64, 128, 256}) for (int st : {2, 4, 8}) for (int nl : {1, 2}) {
      if (st * rows * 128 * nl > 200 * 1024) continue;
      Pat p = {2, rows * 128, {1, (int32_t)(R / rows)}, {0, rows}, nl, st};
      run("2D [R][64] L2-resident", {64, R}, {64, (uint32_t)rows}, p, 1, mode);
    }
  }
  return 0;
}
