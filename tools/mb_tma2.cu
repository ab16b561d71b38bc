// Microbenchmark: whole-GPU TMA streaming rate vs ring depth, one CTA per SM (one elected
// producer lane, one consumer warp that releases slots as soon as they land).  Patterns:
//   A  bulk copy of the whole stage (contiguous)
//   B  3-D box {128 B, L lines, 8 tiles}, SWIZZLE_128B, tiles kg KB apart (the K2c INT4 weight stage)
//   C  2-D fp16 boxes {64, 128} SW128 x (stage / 16 KB), rows k*2 bytes apart (the K2c fp16 stage)
// Each CTA streams its own contiguous slice of a 4 GB buffer (like a k-split panel).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I paper_conf_cluster_zhaowplw25_b200/csrc -I include tools/mb_tma2.cu -o tools/mb_tma2 -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#include "sq_common.cuh"

using namespace sq;

constexpr int MAXST = 24;

__global__ void __launch_bounds__(64, 1) k_stream(const __grid_constant__ CUtensorMap tm, const uint8_t* src, int pattern,
                                                   int iters, int STAGES, uint32_t stage_bytes, int kg) {
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
        uint8_t* dst = smem + s * stage_bytes;
        mbar_arrive_expect_tx(&full[s], stage_bytes);
        if (pattern == 0) {
          bulk_load(dst, src + ((uint64_t)blockIdx.x * iters + i) * stage_bytes, stage_bytes, &full[s]);
        } else if (pattern == 1) {
          // CTA b owns 8 tiles (rows of T16 units) x its k range: tile row = blockIdx.x * 8, line = i * L
          const int L = stage_bytes / 1024;  // 128-B lines per tile = stage / (8 tiles x 128 B)
          tma_load_3d(dst, &tm, &full[s], 0, i * L, blockIdx.x * 8);
        } else {
          // fp16 rows: CTA b owns 128 rows; stage = nb boxes of {64 halves, 128 rows}
          const int nb = stage_bytes / 16384;
          for (int j = 0; j < nb; ++j) tma_load_2d(dst + j * 16384, &tm, &full[s], (i * nb + j) * 64, blockIdx.x * 128);
        }
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
  const uint64_t big = 4ull << 30;
  uint8_t* buf;
  cudaMalloc(&buf, big);
  cudaMemset(buf, 1, big);
  cudaFuncSetAttribute(k_stream, cudaFuncAttributeMaxDynamicSharedMemorySize, 226 * 1024);
  const char* names[3] = {"bulk", "3D-lines-SW128", "2D-fp16-SW128"};
  for (int pattern = 0; pattern < 3; ++pattern) {
    for (int sb : {16384, 32768}) {
      for (int st : {4, 6, 8, 10, 12, 13}) {
        if ((size_t)st * sb + 1024 > 226 * 1024) continue;
        const uint64_t per_cta = big / sms / sb * sb;
        const int iters = (int)(per_cta / sb);
        CUtensorMap tm{};
        cuuint32_t es[3] = {1, 1, 1};
        if (pattern == 1) {
          // [tiles = sms*8][lines = per_cta/8/128][128 B]
          const uint64_t lines = per_cta / 8 / 128;
          cuuint64_t d[3] = {128, lines, (cuuint64_t)sms * 8}, stv[2] = {128, lines * 128};
          cuuint32_t b[3] = {128, (cuuint32_t)(sb / 1024), 8};
          enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, buf, d, stv, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        } else if (pattern == 2) {
          const uint64_t k = per_cta / 128 / 2;  // halves per row
          cuuint64_t d[2] = {k, (cuuint64_t)sms * 128}, stv[1] = {k * 2};
          cuuint32_t b[2] = {64, 128};
          enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, stv, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
              CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        }
        const int smem = st * sb + 1024;
        k_stream<<<sms, 64, smem>>>(tm, buf, pattern, 64, st, sb, 0);
        cudaError_t le = cudaGetLastError();
        if (le != cudaSuccess) { printf("launch error %s\n", cudaGetErrorString(le)); return 1; }
        le = cudaDeviceSynchronize();
        if (le != cudaSuccess) { printf("run error %s\n", cudaGetErrorString(le)); return 1; }
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        k_stream<<<sms, 64, smem>>>(tm, buf, pattern, iters, st, sb, 0);
        cudaEventRecord(e1);
        cudaError_t err = cudaDeviceSynchronize();
        if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        const double bytes = (double)sms * iters * sb;
        printf("{\"pattern\": \"%s\", \"stage\": %d, \"stages\": %d, \"inflight_KB\": %d, \"ms\": %.3f, \"GBps\": %.1f, \"per_SM\": %.1f}\n",
               names[pattern], sb, st, st * sb / 1024, ms, bytes / (ms * 1e-3) / 1e9, bytes / (ms * 1e-3) / 1e9 / sms);
      }
    }
  }
  return 0;
}
