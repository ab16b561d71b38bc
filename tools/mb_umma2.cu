// Microbenchmark: tcgen05.mma kind::f16 M=128 N=32 K=16 (A from TMEM) issue/execute rate under the
// K2c decode kernel's conditions: (a) alone, same accumulator; (b) the accumulator switching among
// 4 row tiles every 16 MMAs (panels of P = 4); (c) = (b) while W warps stream tcgen05.st into the
// TMEM A ring (the dequant warps' traffic: 64 KB per 16 MMAs at full speed).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I paper_conf_cluster_zhaowplw25_b200/csrc -I include tools/mb_umma2.cu -o tools/mb_umma2
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "sq_tc.cuh"

using namespace sq;
using namespace sq::tc;

__global__ void __launch_bounds__(32 * 18, 1) k_umma2(long long* out, int iters, int mode, int st_warps) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  __shared__ volatile int done;
  const int warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 16384 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); done = 0; }
  if (warp == 0) tmem_alloc(&tbase, 512);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  constexpr uint32_t idesc = make_idesc(128, 32);
  if (warp == 0) {
    long long t0 = 0, t1 = 0;
    if (elect_one()) {
      const uint64_t bdesc = make_sw128_desc(smem_u32(smem));
      t0 = clock64();
      for (int i = 0; i < iters; i += 16) {
        const uint32_t d = mode >= 1 ? ((i >> 4) & 3) * 32 : 0;
        const uint32_t a = 128 + ((i >> 4) & 1) * 128;
#pragma unroll
        for (int kk = 0; kk < 16; ++kk) tc_mma_ts(d, a + kk * 8, bdesc + (kk & 3) * 2, idesc, 1u);
      }
      tc_commit(&bar);
    }
    __syncwarp();
    mbar_wait(&bar, 0);
    t1 = clock64();
    if (threadIdx.x < 32) {
      long long a = __shfl_sync(0xffffffff, t0, __ffs(__ballot_sync(0xffffffff, t0 != 0)) - 1);
      if (threadIdx.x == 0) { out[2 * blockIdx.x] = a; out[2 * blockIdx.x + 1] = t1; done = 1; }
    }
  } else if (mode == 2 && warp - 1 < st_warps) {
    // stream tcgen05.st into the A ring (columns 128..383), lane quadrant = warp % 4
    const uint32_t lane_base = (uint32_t)((warp & 3) * 32) << 16;
    uint32_t v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = 0u;
    int c = 0;
    while (!done) {
      tmem_st16(lane_base + 128 + ((c * 16 + (warp >> 2) * 64) & 255), v);
      tc_wait_st();
      ++c;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(0, 512); }
}

// pure tcgen05.st throughput: W warps each issue `iters` st.32x32b.x16 (2 KB per warp-instruction),
// with a wait::st every `batch` stores; bytes per cycle per SM from clock64 on warp 0
__global__ void __launch_bounds__(32 * 17, 1) k_st(long long* out, int iters, int batch, int nwarps) {
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) tmem_alloc(&tbase, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  long long t0 = clock64();
  if (warp < nwarps) {
    const uint32_t lane_base = (uint32_t)((warp & 3) * 32) << 16;
    uint32_t v[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) v[i] = (uint32_t)i;
    for (int i = 0; i < iters; ++i) {
      tmem_st16(lane_base + ((i * 16 + (warp >> 2) * 128) & 511), v);
      if ((i + 1) % batch == 0) tc_wait_st();
    }
    tc_wait_st();
  }
  __syncthreads();
  long long t1 = clock64();
  if (threadIdx.x == 0) { out[2 * blockIdx.x] = t0; out[2 * blockIdx.x + 1] = t1; }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(0, 512); }
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  long long* d;
  cudaMalloc(&d, 2 * sms * sizeof(long long));
  cudaFuncSetAttribute(k_umma2, cudaFuncAttributeMaxDynamicSharedMemorySize, 20 * 1024);
  const int iters = 16384;
  struct { int mode, w; } cases[] = {{0, 0}, {1, 0}, {2, 4}, {2, 8}, {2, 16}};
  for (auto cs : cases) {
    k_umma2<<<sms, 32 * 18, 20 * 1024>>>(d, iters, cs.mode, cs.w);
    cudaError_t err = cudaDeviceSynchronize();
    if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
    long long h[2];
    cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
    printf("mode %d (%s) st_warps %2d: %.1f cycles per M128 N32 K16 MMA\n", cs.mode,
           cs.mode == 0 ? "same D" : (cs.mode == 1 ? "D over 4 tiles" : "D over 4 tiles + tcgen05.st"), cs.w,
           (double)(h[1] - h[0]) / iters);
  }
  for (int w : {4, 8, 16}) {
    for (int batch : {1, 4, 16}) {
      const int iters = 4096;
      k_st<<<sms, 32 * 17>>>(d, iters, batch, w);
      cudaError_t err = cudaDeviceSynchronize();
      if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); return 1; }
      long long h[2];
      cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
      const double bytes = (double)w * iters * 2048;
      printf("tcgen05.st.32x32b.x16: %2d warps, wait every %2d: %.1f B/cycle per SM\n", w, batch, bytes / (double)(h[1] - h[0]));
    }
  }
  return 0;
}
