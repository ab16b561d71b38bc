// Microbenchmark: TMA / bulk-copy throughput per SM for the decode GEMV's unit shapes
// (16 KB per stage), from HBM (streamed) and from L2 (a 4 MB window re-read).
//   P0 2-D fp16 box {64, 128}, SWIZZLE_128B      (128 rows of 128 B: the activation slice)
//   P1 4-D u8 box {64, 16, 2, 8}, SWIZZLE_64B     (256 rows of 64 B: INT4 T16 weights, UG=2)
//   P2 2-D u64 box {256, 8}, no swizzle           (8 rows of 2 KB)
//   P3 one cp.async.bulk of 16 KB
//   P4 8 cp.async.bulk of 2 KB
// One CTA per SM: warp 0 (elected lane) issues into an 8-stage ring, warp 1 releases.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -I include \
//      -I paper_conf_cluster_zhaowplw25_b200/csrc tools/mb_tma.cu -o tools/mb_tma
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#include "sq_common.cuh"

using namespace sq;

constexpr int MAXST = 13;
int STAGE = 16384;
__constant__ int d_stage = 16384;

__global__ void __launch_bounds__(64, 1) k_tma(const __grid_constant__ CUtensorMap tm, const uint8_t* src,
                                                int pattern, int iters, uint64_t span_units, int STAGES, uint32_t stage_bytes) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[MAXST], empty[MAXST];
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    fence_barrier_init();
  }
  __syncthreads();
  if (warp == 0) {
    for (int i = 0; i < iters; ++i) {
      const int s = i % STAGES, ph = (i / STAGES) & 1;
      mbar_wait(&empty[s], ph ^ 1);
      if (elect_one()) {
        const uint64_t unit = ((uint64_t)blockIdx.x * iters + i) % span_units;  // stage-sized unit index
        uint8_t* dst = smem + s * stage_bytes;
        mbar_arrive_expect_tx(&full[s], stage_bytes);
        if ((pattern & 15) == 0) tma_load_2d(dst, &tm, &full[s], 0, (int)(unit * (pattern >> 4)));
        else if (pattern == 1 || pattern >= 5 && pattern <= 7) tma_load_4d(dst, &tm, &full[s], 0, 0, 0, (int)(unit * 8));
        else if (pattern == 8)
          for (int j = 0; j < 16; ++j) bulk_load(dst + j * 1024, src + unit * stage_bytes + j * 1024, 1024, &full[s]);
        else if (pattern == 2) tma_load_2d(dst, &tm, &full[s], 0, (int)(unit * 8));
        else if ((pattern & 15) == 3) bulk_load(dst, src + unit * stage_bytes, stage_bytes, &full[s]);
        else
          for (int j = 0; j < 8; ++j) bulk_load(dst + j * 2048, src + unit * stage_bytes + j * 2048, 2048, &full[s]);
      }
      __syncwarp();
    }
  } else {
    for (int i = 0; i < iters; ++i) {
      const int s = i % STAGES, ph = (i / STAGES) & 1;
      mbar_wait(&full[s], ph);
      __syncwarp();
      if (elect_one()) mbar_arrive(&empty[s]);
      __syncwarp();
    }
  }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  void* f = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  EncodeFn enc = reinterpret_cast<EncodeFn>(f);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const uint64_t big = 4ull << 30;  // 4 GB streamed
  uint8_t* buf;
  cudaMalloc(&buf, big);
  cudaMemset(buf, 1, big);
  const int iters = 2048;
  const char* names[9] = {"2D fp16 {64,128} SW128", "4D u8 {64,16,2,8} SW64", "2D u64 {256,8}", "bulk 16KB x1",
                          "bulk 2KB x8", "4D u8 {128,8,2,8} SW128", "4D u8 {48,16,2,8} none (12KB)",
                          "4D u8 {128,6,2,8} none (12KB)", "bulk 1KB x16"};
  for (int cfg = 0; cfg < 6; ++cfg) {
    const int sb = cfg < 3 ? 8192 << cfg : 8192 << (cfg - 3);
    const int p = cfg < 3 ? 0 : 3;
    const int STAGES = sb <= 16384 ? 8 : 6;
    const int smem = STAGES * sb + 2048;
    cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    const uint64_t span = big / sb;
    CUtensorMap tm{};
    cuuint32_t es[4] = {1, 1, 1, 1};
    if (p == 0) {
      cuuint64_t d[2] = {64, big / 128}, st[1] = {128};
      cuuint32_t b[2] = {64, (cuuint32_t)(sb / 128)};
      enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    k_tma<<<sms, 64, smem>>>(tm, buf, p + 16 * (sb / 128), 64, span, STAGES, sb);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    k_tma<<<sms, 64, smem>>>(tm, buf, p + 16 * (sb / 128), iters, span, STAGES, sb);
    cudaEventRecord(e1);
    cudaError_t err = cudaDeviceSynchronize();
    if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    const double bytes = (double)sms * iters * sb;
    printf("stage %6d B x%d %s: %8.1f GB/s  %6.1f GB/s per SM  %.3f us per stage\n", sb, STAGES, p == 0 ? "2D box" : "bulk  ",
           bytes / (ms * 1e-3) / 1e9, bytes / (ms * 1e-3) / 1e9 / sms, ms * 1e3 / iters);
  }
  return 0;
}
