// Microbenchmark: tcgen05.mma kind::f16 issue/execute rate on sm_100a for the decode
// shapes (M = 128 weight rows, N = 32..256 tokens, K = 16), A from TMEM (TS) or SMEM (SS).
// One CTA per SM; one elected thread issues ITERS MMAs back to back, then a commit;
// cycles per MMA = (commit arrival - first issue) / ITERS.  Operand data are zeros.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_cluster_zhaowplw25_b200/csrc tools/mb_umma.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

#include "sq_tc.cuh"

using namespace sq;
using namespace sq::tc;

template <int N, bool TS>
__global__ void __launch_bounds__(128, 1) k_umma(long long* out, int iters) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x >> 5;
  for (int i = threadIdx.x; i < 65536 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(smem)[i] = 0;
  if (threadIdx.x == 0) { mbar_init(&bar, 1); fence_barrier_init(); }
  if (warp == 0) tmem_alloc(&tbase, 512);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  constexpr uint32_t idesc = make_idesc(128, N);
  if (warp == 0) {
    long long t0 = 0, t1 = 0;
    if (elect_one()) {
      const uint64_t adesc = make_sw128_desc(smem_u32(smem));
      const uint64_t bdesc = make_sw128_desc(smem_u32(smem + 16384));
      t0 = clock64();
      for (int i = 0; i < iters; i += 16) {
#pragma unroll
        for (int kk = 0; kk < 16; ++kk) {
          if constexpr (TS) tc_mma_ts(0, 256 + (kk & 3) * 8, bdesc + (kk & 3) * 2, idesc, 1u);
          else tc_mma_ss(0, adesc + (kk & 3) * 2, bdesc + (kk & 3) * 2, idesc, 1u);
        }
      }
      tc_commit(&bar);
    }
    __syncwarp();
    mbar_wait(&bar, 0);
    t1 = clock64();
    if (threadIdx.x == 0 || (t0 && blockIdx.x == 0)) {}
    if (elect_one()) {}
    if (threadIdx.x < 32) {
      long long a = __shfl_sync(0xffffffff, t0, __ffs(__ballot_sync(0xffffffff, t0 != 0)) - 1);
      if (threadIdx.x == 0) { out[2 * blockIdx.x] = a; out[2 * blockIdx.x + 1] = t1; }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) { tc_fence_after(); tmem_dealloc(0, 512); }
}

template <int N, bool TS>
void run(int iters, int sms) {
  long long* d;
  cudaMalloc(&d, 2 * sms * sizeof(long long));
  auto k = k_umma<N, TS>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 66 * 1024);
  k<<<sms, 128, 66 * 1024>>>(d, iters);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<<<sms, 128, 66 * 1024>>>(d, iters);
  cudaEventRecord(e1);
  cudaError_t err = cudaDeviceSynchronize();
  if (err != cudaSuccess) { printf("error %s\n", cudaGetErrorString(err)); exit(1); }
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  long long h[2];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  const double cyc = (double)(h[1] - h[0]) / iters;
  const double flops = 2.0 * 128 * N * 16 * (double)iters * sms;
  printf("%s N=%3d: %.1f cycles/MMA (CTA 0), %.1f TFLOP/s over %d SMs (%.1f us)\n", TS ? "TS" : "SS", N, cyc,
         flops / (ms * 1e-3) / 1e12, sms, ms * 1e3);
  cudaFree(d);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int iters = 16384;
  run<32, true>(iters, sms);
  run<64, true>(iters, sms);
  run<128, true>(iters, sms);
  run<256, true>(iters, sms);
  run<32, false>(iters, sms);
  run<64, false>(iters, sms);
  run<128, false>(iters, sms);
  run<256, false>(iters, sms);
  return 0;
}
