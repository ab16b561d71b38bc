// Microbenchmark: does the activation stream of the tcgen05 decode GEMV (K2c) eat into the per-SM
// ingest its weight stream needs?  One CTA per SM streams K2c-INT4-shaped weight stages (3-D box of
// 128-B lines, SWIZZLE_128B, 24 KB per unit) and, optionally,
//   meta : a 2-D box of 8 rows x 192 B per unit (the unit's scales/zeros),
//   x    : per k-step (every P units) an activation slice box {64 k, R rows, 6 k-blocks} from a small
//          L2-resident buffer holding `m` valid rows (rows >= m are out of bounds -> zero fill).
// A consumer warp releases every slot as soon as it lands.  Reports weight GB/s and total ingest.
// Also prints cudaOccupancyMaxActiveClusters for a K2c-sized CTA (704 threads, ~225 KB smem).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr \
//        -I paper_conf_cluster_zhaowplw25_b200/csrc -I include tools/mb_ingest.cu -o tools/mb_ingest -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>

#include "sq_common.cuh"

using namespace sq;

constexpr int MAXST = 16;
constexpr int WST = 24 * 1024;   // weight stage bytes
constexpr int XST = 24 * 1024;   // activation stage bytes (32 rows x 384 k x 2 B)

__global__ void __launch_bounds__(64, 1) k_ingest(const __grid_constant__ CUtensorMap tw, const __grid_constant__ CUtensorMap tm,
                                                   const __grid_constant__ CUtensorMap tx, int iters, int SW, int SX,
                                                   int P, int use_meta, int use_x, uint32_t xbytes, int ksteps_x) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t fw[MAXST], ew[MAXST], fx[MAXST], ex[MAXST];
  const int warp = threadIdx.x >> 5;
  uint8_t* wring = smem;
  uint8_t* mring = smem + SW * WST;
  uint8_t* xring = mring + SW * 1536;
  if (threadIdx.x == 0) {
    for (int i = 0; i < SW; ++i) { mbar_init(&fw[i], 1); mbar_init(&ew[i], 1); }
    for (int i = 0; i < SX; ++i) { mbar_init(&fx[i], 1); mbar_init(&ex[i], 1); }
    fence_barrier_init();
  }
  __syncthreads();
  const int tile0 = blockIdx.x * 8;
  if (warp == 0) {
    int qx = 0;
    for (int i = 0; i < iters; ++i) {
      if (use_x && i % P == 0) {
        const int sx = qx % SX, ph = (qx / SX) & 1;
        mbar_wait(&ex[sx], ph ^ 1);
        if (elect_one()) {
          mbar_arrive_expect_tx(&fx[sx], xbytes);
          tma_load_3d(xring + sx * XST, &tx, &fx[sx], 0, 0, (qx % ksteps_x) * 6);
        }
        __syncwarp();
        ++qx;
      }
      const int s = i % SW, ph = (i / SW) & 1;
      mbar_wait(&ew[s], ph ^ 1);
      if (elect_one()) {
        mbar_arrive_expect_tx(&fw[s], WST + (use_meta ? 1536 : 0));
        tma_load_3d(wring + s * WST, &tw, &fw[s], 0, i * 24, tile0);
        if (use_meta) tma_load_2d(mring + s * 1536, &tm, &fw[s], (i % 1000) * 48, tile0);
      }
      __syncwarp();
    }
  } else {
    int qx = 0;
    for (int i = 0; i < iters; ++i) {
      if (use_x && i % P == 0) {
        const int sx = qx % SX, ph = (qx / SX) & 1;
        mbar_wait(&fx[sx], ph);
        __syncwarp();
        if (elect_one()) mbar_arrive(&ex[sx]);
        __syncwarp();
        ++qx;
      }
      const int s = i % SW, ph = (i / SW) & 1;
      mbar_wait(&fw[s], ph);
      __syncwarp();
      if (elect_one()) mbar_arrive(&ew[s]);
      __syncwarp();
    }
  }
}

__global__ void __launch_bounds__(704, 1) k_dummy(int* p) {
  extern __shared__ uint8_t s[];
  if (p) p[threadIdx.x] = s[threadIdx.x];
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
  // cluster residency of a K2c-sized CTA
  cudaFuncSetAttribute(k_dummy, cudaFuncAttributeMaxDynamicSharedMemorySize, 225 * 1024);
  cudaFuncSetAttribute(k_dummy, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int cs = 1; cs <= 16; cs *= 2) {
    for (int c2 : {cs, cs + (cs == 2 ? 1 : 0)}) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(c2 * 16);
      cfg.blockDim = dim3(704);
      cfg.dynamicSmemBytes = 225 * 1024;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = c2; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      int ncl = -1;
      cudaError_t e = cudaOccupancyMaxActiveClusters(&ncl, k_dummy, &cfg);
      printf("{\"cluster\": %d, \"max_active_clusters\": %d, \"ctas\": %d, \"err\": \"%s\"}\n", c2, ncl, ncl * c2,
             cudaGetErrorString(e));
      cudaGetLastError();
      if (cs != 2) break;
    }
  }
  for (int z : {5, 6, 7}) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(z * 16);
    cfg.blockDim = dim3(704);
    cfg.dynamicSmemBytes = 225 * 1024;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = z; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    int ncl = -1;
    cudaOccupancyMaxActiveClusters(&ncl, k_dummy, &cfg);
    cudaGetLastError();
    printf("{\"cluster\": %d, \"max_active_clusters\": %d, \"ctas\": %d}\n", z, ncl, ncl * z);
  }

  const uint64_t big = 4ull << 30;
  uint8_t *buf, *mbuf, *xbuf;
  cudaMalloc(&buf, big);
  cudaMemset(buf, 1, big);
  cudaMalloc(&mbuf, 256ull << 20);
  cudaMemset(mbuf, 2, 256ull << 20);
  const int K = 36864;  // activation k extent (fc2-like), fp16
  cudaMalloc(&xbuf, 32ull * K * 2);
  cudaMemset(xbuf, 0, 32ull * K * 2);
  const int max_dyn = 227 * 1024 - 1024;  // opt-in limit minus the static barriers
  if (cudaFuncSetAttribute(k_ingest, cudaFuncAttributeMaxDynamicSharedMemorySize, max_dyn) != cudaSuccess) {
    printf("attribute error\n");
    return 1;
  }
  cuuint32_t es[3] = {1, 1, 1};
  for (int ctas : {sms, 144}) {
    const uint64_t per_cta = big / sms / WST * WST;
    const int iters = (int)(per_cta / WST);
    const uint64_t lines = per_cta / 8 / 128;
    CUtensorMap tw{}, tm{};
    {
      cuuint64_t d[3] = {128, lines, (cuuint64_t)sms * 8}, stv[2] = {128, lines * 128};
      cuuint32_t b[3] = {128, 24, 8};
      enc(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, 3, buf, d, stv, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    {
      // meta: [tiles][48000 u32]; box {48 u32, 8 rows}
      const uint64_t cols = (256ull << 20) / 4 / ((uint64_t)sms * 8);
      cuuint64_t d[2] = {cols, (cuuint64_t)sms * 8}, stv[1] = {cols * 4};
      cuuint32_t b[2] = {48, 8};
      CUresult r = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, mbuf, d, stv, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                       CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r != CUDA_SUCCESS) printf("meta encode failed %d\n", (int)r);
    }
    struct V { const char* name; int meta, x, P, m, rows, SW, SX; };
    const V vs[] = {
        {"w", 0, 0, 1, 0, 0, 7, 1},          {"w+meta", 1, 0, 1, 0, 0, 7, 1},
        {"w+meta+x32/P2", 1, 1, 2, 32, 32, 6, 2}, {"w+meta+x32/P4", 1, 1, 4, 32, 32, 6, 2},
        {"w+meta+x1box32/P2", 1, 1, 2, 1, 32, 6, 2}, {"w+meta+x16box16/P2", 1, 1, 2, 16, 16, 6, 2},
        {"w+meta+x8box8/P2", 1, 1, 2, 8, 8, 6, 2}, {"w+meta+x32/P2/SX3", 1, 1, 2, 32, 32, 5, 3},
        {"w+meta+x16box16/P8", 1, 1, 8, 16, 16, 6, 2}, {"w/SW4", 0, 0, 1, 0, 0, 4, 1},
        {"w/SW5", 0, 0, 1, 0, 0, 5, 1},
    };
    for (const V& v : vs) {
      CUtensorMap tx{};
      {
        cuuint64_t d[3] = {64, (cuuint64_t)v.m > 0 ? (cuuint64_t)v.m : 1, (cuuint64_t)K / 64}, stv[2] = {(cuuint64_t)K * 2, 128};
        cuuint32_t b[3] = {64, (cuuint32_t)(v.rows > 0 ? v.rows : 32), 6};
        CUresult r = enc(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, 3, xbuf, d, stv, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
        if (r != CUDA_SUCCESS) printf("x encode failed %d\n", (int)r);
      }
      const uint32_t xbytes = 64 * 2 * 6 * (v.rows > 0 ? v.rows : 32);
      const int smem = v.SW * (WST + 1536) + v.SX * XST + 1024;
      if (smem > max_dyn) { printf("skip %s\n", v.name); continue; }
      k_ingest<<<ctas, 64, smem>>>(tw, tm, tx, 64, v.SW, v.SX, v.P, v.meta, v.x, xbytes, K / 384);
      cudaError_t le = cudaGetLastError();
      if (le == cudaSuccess) le = cudaDeviceSynchronize();
      if (le != cudaSuccess) { printf("error %s: %s\n", v.name, cudaGetErrorString(le)); return 1; }
      float best = 1e30f;
      for (int r = 0; r < 3; ++r) {
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        k_ingest<<<ctas, 64, smem>>>(tw, tm, tx, iters, v.SW, v.SX, v.P, v.meta, v.x, xbytes, K / 384);
        cudaEventRecord(e1);
        if (cudaGetLastError() != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) { printf("run error\n"); return 1; }
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
      }
      const double wbytes = (double)ctas * iters * WST;
      const double tot = (double)ctas * iters * (WST + (v.meta ? 1536 : 0)) + (v.x ? (double)ctas * (iters / v.P) * xbytes : 0);
      printf("{\"variant\": \"%s\", \"ctas\": %d, \"weights_GBps\": %.1f, \"ingest_GBps\": %.1f, \"ingest_per_SM\": %.1f}\n",
             v.name, ctas, wbytes / (best * 1e-3) / 1e9, tot / (best * 1e-3) / 1e9, tot / (best * 1e-3) / 1e9 / ctas);
    }
  }
  return 0;
}
