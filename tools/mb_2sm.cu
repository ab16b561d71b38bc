// Semantics check for the 2-SM (cta_group::2) tensor-core path planned for K3: a CTA pair computes
// D[256 rows x 256 tokens] = A[256 x 64] . B[256 x 64]^T with
//   * A (fp16) written by each CTA's warps into its OWN tensor memory (rows 128 r .. 128 r + 127),
//   * B (fp16) loaded by each CTA's TMA (tokens 128 r .. 128 r + 127) with .cta_group::2, both loads
//     completing on the LEADER's mbarrier,
//   * the peer's "A ready" signalled by a remote mbarrier arrive on the leader,
//   * tcgen05.mma.cta_group::2 (M = 256, N = 256, K = 16, A from TMEM) issued by the leader only,
//   * a multicast commit to both CTAs' barriers, each CTA reading its 128 rows of D from its TMEM.
// Prints the max abs error against a host fp32 product, and the cycles per MMA of a long loop.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_cluster_zhaowplw25_b200/csrc \
//        -I include tools/mb_2sm.cu -o tools/mb_2sm -lcuda
#include <cuda.h>
#include <cuda_fp16.h>
#include <cstdio>
#include <cstdlib>
#include <cmath>
#include <vector>

#include "sq_tc.cuh"

using namespace sq;
using namespace sq::tc;

__device__ __forceinline__ uint32_t cta_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
  uint32_t o;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
  return o;
}
__device__ __forceinline__ void wait_cl(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  while (!ok)
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void arrive_remote(uint32_t cl_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cl_addr) : "memory");
}
__device__ __forceinline__ void tma2_2d(uint32_t dst, const void* tmap, uint32_t mbar_cl, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
               ::"r"(dst), "l"(tmap), "r"(mbar_cl), "r"(c0), "r"(c1) : "memory");
}
__device__ __forceinline__ void mma2_ts(uint32_t d, uint32_t a, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\ttcgen05.mma.cta_group::2.kind::f16 [%0], [%1], %2, %3, p;\n\t}"
               ::"r"(d), "r"(a), "l"(bdesc), "r"(idesc), "r"(acc) : "memory");
}
__device__ __forceinline__ void commit2_mc(uint64_t* bar, uint16_t mask) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
               ::"r"(smem_u32(bar)), "h"(mask) : "memory");
}

constexpr int NT = 128;  // threads per CTA: 4 warps (one per TMEM lane quadrant)

__global__ void __launch_bounds__(NT, 1)
    k_2sm(const __grid_constant__ CUtensorMap tmb, const __half* A, float* D, int reps, long long* cyc) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  __shared__ uint64_t full_x, full_a, d_full;
  __shared__ uint32_t tslot;
  const uint32_t rank = cta_rank();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    mbar_init(&full_x, 1);
    mbar_init(&full_a, 8);
    mbar_init(&d_full, 1);
    fence_barrier_init();
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tslot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  tc_fence_after();
  const uint32_t tmem = tslot;
  // B half: tokens [128 rank, 128 rank + 128) x 64 k, SW128, completes on the leader's full_x
  if (threadIdx.x == 0) {
    if (rank == 0) mbar_arrive_expect_tx(&full_x, 2 * 128 * 128);
    tma2_2d(smem_u32(smem), &tmb, mapa(smem_u32(&full_x), 0), 0, 128 * rank);
  }
  // A rows of this CTA -> own TMEM, column c = k pair (2c, 2c + 1); 64 k = 32 columns at column 256
  {
    const int row = rank * 128 + warp * 32 + lane;
    uint32_t v[16];
    for (int h = 0; h < 2; ++h) {
      for (int c = 0; c < 16; ++c) {
        __half2 p = __halves2half2(A[row * 64 + (h * 16 + c) * 2], A[row * 64 + (h * 16 + c) * 2 + 1]);
        v[c] = *reinterpret_cast<uint32_t*>(&p);
      }
      tmem_st16(tmem + ((uint32_t)(warp * 32) << 16) + 256 + h * 16, v);
    }
    tc_wait_st();
    tc_fence_before();
    __syncwarp();
    if (lane == 0) arrive_remote(mapa(smem_u32(&full_a), 0));
  }
  constexpr uint32_t idesc = make_idesc(256, 256);
  if (rank == 0 && warp == 1) {
    wait_cl(&full_a, 0);
    wait_cl(&full_x, 0);
    tc_fence_after();
    long long t0 = clock64();
    if (elect_one()) {
      for (int r = 0; r < reps; ++r)
        for (int kk = 0; kk < 4; ++kk)
          mma2_ts(tmem, tmem + 256 + kk * 8, make_sw128_desc(smem_u32(smem) + kk * 32), idesc, (r | kk) != 0);
      commit2_mc(&d_full, 0x3);
    }
    __syncwarp();
    wait_cl(&d_full, 0);
    if (lane == 0) *cyc = clock64() - t0;
  }
  wait_cl(&d_full, 0);
  tc_fence_after();
  {
    const int row = rank * 128 + warp * 32 + lane;
    for (int c = 0; c < 256; c += 16) {
      uint32_t v[16];
      tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + c, v);
      tc_wait_ld();
      for (int i = 0; i < 16; ++i) D[row * 256 + c + i] = __uint_as_float(v[i]);
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem) : "memory");
  }
}

int main() {
  std::vector<__half> a(256 * 64), b(256 * 64);
  srand(1);
  for (auto& v : a) v = __float2half((rand() % 17 - 8) / 8.f);
  for (auto& v : b) v = __float2half((rand() % 17 - 8) / 8.f);
  __half *da, *db;
  float* dd;
  long long* dc;
  cudaMalloc(&da, a.size() * 2);
  cudaMalloc(&db, b.size() * 2);
  cudaMalloc(&dd, 256 * 256 * 4);
  cudaMalloc(&dc, 8);
  cudaMemcpy(da, a.data(), a.size() * 2, cudaMemcpyHostToDevice);
  cudaMemcpy(db, b.data(), b.size() * 2, cudaMemcpyHostToDevice);
  CUtensorMap tm;
  const cuuint64_t dims[2] = {64, 256}, strides[1] = {128};
  const cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
  CUresult cr = cuTensorMapEncodeTiled(&tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 2, db, dims, strides, box, es,
                                       CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                                       CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (cr != CUDA_SUCCESS) { printf("encode failed %d\n", (int)cr); return 1; }
  cudaFuncSetAttribute(k_2sm, cudaFuncAttributeMaxDynamicSharedMemorySize, 32768);
  const int cy = getenv("CY") ? atoi(getenv("CY")) : 0;
  for (int reps : {1, 1000}) {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = cy ? dim3(1, 2) : dim3(2, 1);
    cfg.blockDim = dim3(NT);
    cfg.dynamicSmemBytes = 32768;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = cy ? 1 : 2;
    at[0].val.clusterDim.y = cy ? 2 : 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, k_2sm, tm, (const __half*)da, dd, reps, dc);
    if (e != cudaSuccess) { printf("launch error %s\n", cudaGetErrorString(e)); return 1; }
    e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("kernel error %s\n", cudaGetErrorString(e)); return 1; }
    std::vector<float> d(256 * 256);
    long long cyc = 0;
    cudaMemcpy(d.data(), dd, d.size() * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(&cyc, dc, 8, cudaMemcpyDeviceToHost);
    double err = 0;
    for (int i = 0; i < 256; ++i)
      for (int t = 0; t < 256; ++t) {
        double s = 0;
        for (int k = 0; k < 64; ++k) s += (double)__half2float(a[i * 64 + k]) * __half2float(b[t * 64 + k]);
        err = std::max(err, std::fabs(d[i * 256 + t] - reps * s));
      }
    printf("reps %d: max abs err %.3g; %.1f cycles per M256 N256 K16 MMA\n", reps, err, (double)cyc / (reps * 4));
  }
  return 0;
}
