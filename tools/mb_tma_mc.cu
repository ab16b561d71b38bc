// Microbenchmark: is the ~45 GB/s-per-SM TMA ingest limit on the SM side or the L2 side?
// Clusters of CS CTAs (one per SM) stream 16-KB stages; each CTA fetches 1/CS of every stage
// with .multicast::cluster to all CS CTAs, so L2 serves each byte once per cluster while every
// SM still receives every byte.  Reported: bytes delivered per SM per second.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -I include \
//      -I paper_conf_cluster_zhaowplw25_b200/csrc tools/mb_tma_mc.cu -o tools/mb_tma_mc -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#include "sq_common.cuh"

using namespace sq;

constexpr int STAGES = 8, STAGE = 16384;

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ void remote_arrive(uint64_t* bar, uint32_t cta) {
  uint32_t ra;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(ra) : "r"(smem_u32(bar)), "r"(cta));
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(ra) : "memory");
}

__global__ void __launch_bounds__(64, 1) k_mc(const __grid_constant__ CUtensorMap tm, int iters, int cs, int l2rows) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t full[STAGES], empty[STAGES];
  const int warp = threadIdx.x >> 5;
  const uint32_t rank = cs > 1 ? cluster_rank() : 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < STAGES; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], cs); }
    fence_barrier_init();
  }
  __syncthreads();
  if (cs > 1) cluster_sync();
  const int cluster = blockIdx.x / cs;
  const int rows_per = 128 / cs;  // this CTA's share of the 128 x 128 B stage
  if (warp == 0) {
    for (int i = 0; i < iters; ++i) {
      const int s = i % STAGES, ph = (i / STAGES) & 1;
      mbar_wait(&empty[s], ph ^ 1);  // every CTA of the cluster released slot s
      if (elect_one()) {
        mbar_arrive_expect_tx(&full[s], STAGE);
        const int row = (int)((((int64_t)cluster * iters + i) * 128) % l2rows) + rank * rows_per;
        uint8_t* dst = smem + s * STAGE + rank * rows_per * 128;
        if (cs == 1) {
          tma_load_2d(dst, &tm, &full[s], 0, row);
        } else {
          const uint16_t mask = (uint16_t)((1u << cs) - 1);
          asm volatile(
              "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.multicast::cluster"
              " [%0], [%1, {%3, %4}], [%2], %5;" ::"r"(smem_u32(dst)),
              "l"(&tm), "r"(smem_u32(&full[s])), "r"(0), "r"(row), "h"(mask)
              : "memory");
        }
      }
      __syncwarp();
    }
  } else {
    for (int i = 0; i < iters; ++i) {
      const int s = i % STAGES, ph = (i / STAGES) & 1;
      mbar_wait(&full[s], ph);
      __syncwarp();
      if (elect_one()) {
        if (cs == 1) mbar_arrive(&empty[s]);
        else for (int c = 0; c < cs; ++c) remote_arrive(&empty[s], c);
      }
      __syncwarp();
    }
  }
  __syncthreads();
  if (cs > 1) cluster_sync();
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
  const int smem = STAGES * STAGE + 2048;
  cudaFuncSetAttribute(k_mc, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_mc, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int l2 = 0; l2 < 2; ++l2) {
    for (int cs : {1, 2, 4, 8}) {
      CUtensorMap tm{};
      cuuint32_t es[2] = {1, 1};
      cuuint64_t d[2] = {64, big / 128}, st[1] = {128};
      cuuint32_t b[2] = {64, (cuuint32_t)(128 / cs)};
      enc(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, buf, d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      const int grid = (sms / cs) * cs;
      const int iters = 2048;
      const int l2rows = l2 ? (4 << 20) / 128 : (int)(big / 128);
      cudaLaunchConfig_t cfg{};
      cfg.gridDim = dim3(grid);
      cfg.blockDim = dim3(64);
      cfg.dynamicSmemBytes = smem;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = cs;
      at[0].val.clusterDim.y = 1;
      at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      cudaLaunchKernelEx(&cfg, k_mc, tm, 64, cs, l2rows);
      cudaEvent_t e0, e1;
      cudaEventCreate(&e0); cudaEventCreate(&e1);
      cudaEventRecord(e0);
      cudaError_t le = cudaLaunchKernelEx(&cfg, k_mc, tm, iters, cs, l2rows);
      cudaEventRecord(e1);
      cudaError_t err = cudaDeviceSynchronize();
      if (le != cudaSuccess || err != cudaSuccess) {
        printf("cs=%d error %s %s\n", cs, cudaGetErrorString(le), cudaGetErrorString(err));
        return 1;
      }
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      const double per_sm = (double)iters * STAGE / (ms * 1e-3) / 1e9;
      printf("%s cluster=%d grid=%d: %.1f GB/s delivered per SM (%.0f GB/s total delivered, %.0f GB/s from L2)\n",
             l2 ? "L2 " : "HBM", cs, grid, per_sm, per_sm * grid, per_sm * grid / cs);
    }
  }
  return 0;
}
