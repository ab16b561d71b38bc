// f4 — W8A8 linear (weight-activation INT8, the SmoothQuant / bitsandbytes scheme of P:93; DESIGN.md
// R26): symmetric per-output-channel INT8 weights, symmetric per-token INT8 activations (dynamic),
// exact int32 accumulation on the tcgen05 tensor cores (kind::i8), y = acc * s_x[t] * s_w[n] (+ bias).
//
//   K9  k_quant_w8     one CTA per weight row: max |w| (fixed-order tree), s = fp16(amax / 127),
//                      codes = clamp(rint(w / s), -127, 127).  Load time.
//   K10 k_quant_act8   the same per token row, scale kept fp32.  Per call, HBM-bound.
//   K11 k_gemm_i8      D[128 weight rows x BT tokens] int32 in TMEM += A[128 x 32 int8] . B[BT x 32]^T:
//                      tcgen05.mma.cta_group::1.kind::i8 (M = 128, N = BT, K = 32), A and B straight from
//                      shared memory (SW128, 128-byte k rows) filled by TMA -- no dequantization at all;
//                      4-warp epilogue (TMEM -> registers: int32 -> fp32 scale, bias, act / residual).
//                      Split-k (Z slices, for grids narrower than the GPU) writes exact int32 partials;
//                      k_i8_reduce sums them in integers (order-independent, hence deterministic) and
//                      applies the same epilogue.
// Warp roles of K11: 0 TMA producer, 1 MMA issuer (+ TMEM alloc), 2..5 epilogue.
#include <cuda.h>

#include "sq_tc.cuh"

namespace sq {
namespace {
using namespace tc;

constexpr int W8_THREADS = 256;

__device__ __forceinline__ float block_max(float v, float* red) {
#pragma unroll
  for (int o = 16; o; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) red[w] = v;
  __syncthreads();
  float r = red[0];
  for (int i = 1; i < W8_THREADS / 32; ++i) r = fmaxf(r, red[i]);
  __syncthreads();
  return r;
}

__device__ __forceinline__ int8_t code127(float v, float s) {
  if (s == 0.0f) return 0;
  float q = rintf(__fdiv_rn(v, s));
  q = fminf(fmaxf(q, -127.0f), 127.0f);
  return (int8_t)(int)q;
}

// ACT = false: weight row, fp16 scale; ACT = true: token row (row stride ld), fp32 scale
template <bool ACT>
__global__ void __launch_bounds__(W8_THREADS) k_quant8(const __half* __restrict__ src, int64_t k, int64_t ld,
                                                       int8_t* __restrict__ codes, void* __restrict__ scales) {
  __shared__ float red[W8_THREADS / 32];
  const int64_t row = blockIdx.x;
  const __half* p = src + row * ld;
  float amax = 0.f;
  for (int64_t j = threadIdx.x; j < k; j += W8_THREADS) amax = fmaxf(amax, fabsf(__half2float(p[j])));
  amax = block_max(amax, red);
  float s;
  if constexpr (ACT) {
    s = __fdiv_rn(amax, 127.0f);
    if (threadIdx.x == 0) static_cast<float*>(scales)[row] = s;
  } else {
    const __half s16 = __float2half_rn(__fdiv_rn(amax, 127.0f));
    s = __half2float(s16);
    if (threadIdx.x == 0) static_cast<__half*>(scales)[row] = s16;
  }
  for (int64_t j = threadIdx.x; j < k; j += W8_THREADS) codes[row * k + j] = code127(__half2float(p[j]), s);
}

// instruction descriptor, kind::i8: D = s32 (2), A = B = s8 (1), K-major, M x N
constexpr uint32_t make_idesc_i8(int M, int N) {
  return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void tc_mma_ss_i8(uint32_t d_tmem, uint64_t a_desc, uint64_t b_desc, uint32_t idesc,
                                             uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n\t}" ::"r"(d_tmem),
      "l"(a_desc), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}

constexpr int I8_BN = 128;              // weight rows per tile (MMA M)
constexpr int I8_KS = 128;              // k per stage (one 128-B SW128 row)
constexpr int I8_THREADS = 32 * 6;

template <int BT>
struct I8Cfg {
  static constexpr int A_BYTES = I8_BN * I8_KS, B_BYTES = BT * I8_KS, STAGE = A_BYTES + B_BYTES;
  static constexpr int S = (200 * 1024) / STAGE > 8 ? 8 : (200 * 1024) / STAGE;
  static constexpr int BARS = 2 * S + 1;
  static constexpr int SMEM = S * STAGE + BARS * 8 + 16 + 1024;
  static constexpr int TMEM_COLS = BT < 32 ? 32 : BT;
};

struct I8P {
  const __half* sw;    // [n] fp16 weight scales
  const float* sx;     // [m] fp32 token scales
  const __half* bias;  // [n] or null
  void* y;             // fp16 / fp32 [m, ldy], or int32 partials [Z][m][n]
  int64_t ldy;
  int m, n, kst;       // tokens, rows, k-stages of the whole k
  int Z;               // k slices (blockIdx.z); Z > 1 -> raw int32 partials
};

template <int EPI>
__device__ __forceinline__ void i8_store(const I8P& p, int t, int row, int32_t acc) {
  const float v = (float)acc * p.sx[t] * __half2float(p.sw[row]) + (p.bias ? __half2float(p.bias[row]) : 0.f);
  if constexpr (EPI == SQ_EPI_F32_ACCUM) {
    float* y = static_cast<float*>(p.y) + (int64_t)t * p.ldy + row;
    *y += v;
  } else {
    static_cast<__half*>(p.y)[(int64_t)t * p.ldy + row] = __float2half_rn(apply_act<EPI>(v));
  }
}

// EPI >= 0: fused epilogue; EPI = -1: raw int32 (partials [z][m][n], or the accumulator for testing)
template <int BT, int EPI>
__global__ void __launch_bounds__(I8_THREADS, 1)
    k_gemm_i8(const __grid_constant__ CUtensorMap tm_w, const __grid_constant__ CUtensorMap tm_x, const I8P p) {
  using C = I8Cfg<BT>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::S * C::STAGE);
  uint64_t* empty = full + C::S;
  uint64_t* d_full = empty + C::S;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(d_full + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int row0 = blockIdx.x * I8_BN, t0 = blockIdx.y * BT, z = blockIdx.z;
  const int ks0 = (int)((int64_t)z * p.kst / p.Z), ks1 = (int)((int64_t)(z + 1) * p.kst / p.Z);
  if (threadIdx.x == 0) {
    for (int i = 0; i < C::S; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(d_full, 1);
    fence_barrier_init();
    prefetch_tmap(&tm_w);
    prefetch_tmap(&tm_x);
  }
  if (warp == 1) tmem_alloc(tmem_slot, C::TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp == 0) {
    for (int j = ks0, i = 0; j < ks1; ++j, ++i) {
      const int s = i % C::S, ph = (i / C::S) & 1;
      mbar_wait(&empty[s], ph ^ 1);
      if (elect_one()) {
        uint8_t* st = smem + s * C::STAGE;
        mbar_arrive_expect_tx(&full[s], C::STAGE);
        tma_load_2d(st, &tm_w, &full[s], j * I8_KS, row0);
        tma_load_2d(st + C::A_BYTES, &tm_x, &full[s], j * I8_KS, t0);
      }
      __syncwarp();
    }
  } else if (warp == 1) {
    constexpr uint32_t idesc = make_idesc_i8(I8_BN, BT);
    for (int j = ks0, i = 0; j < ks1; ++j, ++i) {
      const int s = i % C::S, ph = (i / C::S) & 1;
      mbar_wait(&full[s], ph);
      tc_fence_after();
      if (elect_one()) {
        const uint32_t st = smem_u32(smem + s * C::STAGE);
        const uint64_t ad = make_sw128_desc(st), bd = make_sw128_desc(st + C::A_BYTES);
#pragma unroll
        for (int kk = 0; kk < I8_KS / 32; ++kk)
          tc_mma_ss_i8(tmem, ad + (uint64_t)((kk * 32) >> 4), bd + (uint64_t)((kk * 32) >> 4), idesc,
                       (j == ks0 && kk == 0) ? 0u : 1u);
        tc_commit(&empty[s]);
        if (j == ks1 - 1) tc_commit(d_full);
      }
      __syncwarp();
    }
  } else {
    const int sp = warp & 3;
    const int row = row0 + sp * 32 + lane;
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    mbar_wait_sleepy(d_full, 0);
    tc_fence_after();
#pragma unroll 1
    for (int c = 0; c < BT; c += 16) {
      uint32_t v[16];
      tmem_ld16(tmem + lane_base + c, v);
      tc_wait_ld();
#pragma unroll
      for (int i = 0; i < 16; ++i) {
        const int t = t0 + c + i;
        if (t >= p.m) continue;
        const int32_t acc = (int32_t)v[i];
        if constexpr (EPI < 0) static_cast<int32_t*>(p.y)[((int64_t)z * p.m + t) * p.n + row] = acc;
        else i8_store<EPI>(p, t, row, acc);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, C::TMEM_COLS);
  }
}

// sum the Z int32 partials (exact) and apply the epilogue; one thread per output
template <int EPI>
__global__ void __launch_bounds__(256) k_i8_reduce(const int32_t* __restrict__ part, int Z, const I8P p) {
  const int64_t idx = (int64_t)blockIdx.x * 256 + threadIdx.x;
  if (idx >= (int64_t)p.m * p.n) return;
  const int t = (int)(idx / p.n), row = (int)(idx % p.n);
  int32_t acc = 0;
  for (int z = 0; z < Z; ++z) acc += part[(int64_t)z * p.m * p.n + idx];
  if constexpr (EPI < 0) static_cast<int32_t*>(p.y)[idx] = acc;
  else i8_store<EPI>(p, t, row, acc);
}

template <int BT, int EPI>
cudaError_t launch_i8(const CUtensorMap& tw, const CUtensorMap& tx, const I8P& p, cudaStream_t s) {
  auto kern = k_gemm_i8<BT, EPI>;
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, I8Cfg<BT>::SMEM);
    if (e != cudaSuccess) return e;
    set = true;
  }
  dim3 grid((unsigned)(p.n / I8_BN), (unsigned)((p.m + BT - 1) / BT), (unsigned)p.Z);
  kern<<<grid, I8_THREADS, I8Cfg<BT>::SMEM, s>>>(tw, tx, p);
  return cudaGetLastError();
}

template <int BT>
cudaError_t launch_i8_epi(const CUtensorMap& tw, const CUtensorMap& tx, const I8P& p, int epi, cudaStream_t s) {
  switch (epi) {
    case SQ_EPI_F16: return launch_i8<BT, SQ_EPI_F16>(tw, tx, p, s);
    case SQ_EPI_F16_RELU: return launch_i8<BT, SQ_EPI_F16_RELU>(tw, tx, p, s);
    case SQ_EPI_F16_GELU: return launch_i8<BT, SQ_EPI_F16_GELU>(tw, tx, p, s);
    case SQ_EPI_F32_ACCUM: return launch_i8<BT, SQ_EPI_F32_ACCUM>(tw, tx, p, s);
    default: return launch_i8<BT, -1>(tw, tx, p, s);
  }
}

cudaError_t launch_i8_reduce(const int32_t* part, int Z, const I8P& p, int epi, cudaStream_t s) {
  const unsigned blocks = (unsigned)(((int64_t)p.m * p.n + 255) / 256);
  switch (epi) {
    case SQ_EPI_F16: k_i8_reduce<SQ_EPI_F16><<<blocks, 256, 0, s>>>(part, Z, p); break;
    case SQ_EPI_F16_RELU: k_i8_reduce<SQ_EPI_F16_RELU><<<blocks, 256, 0, s>>>(part, Z, p); break;
    case SQ_EPI_F16_GELU: k_i8_reduce<SQ_EPI_F16_GELU><<<blocks, 256, 0, s>>>(part, Z, p); break;
    case SQ_EPI_F32_ACCUM: k_i8_reduce<SQ_EPI_F32_ACCUM><<<blocks, 256, 0, s>>>(part, Z, p); break;
    default: k_i8_reduce<-1><<<blocks, 256, 0, s>>>(part, Z, p); break;
  }
  return cudaGetLastError();
}

int i8_bt(int64_t m) { return m <= 32 ? 32 : (m <= 64 ? 64 : (m <= 128 ? 128 : 256)); }

// k slices: enough CTAs for the GPU when the row x token grid is narrow (decode)
int i8_z(int64_t n, int64_t m, int64_t k) {
  const int64_t tiles = (n / I8_BN) * ((m + i8_bt(m) - 1) / i8_bt(m));
  const int64_t kst = k / I8_KS;
  int z = 1;
  while (tiles * z < num_sms() && z * 2 <= kst && z < 16) z *= 2;
  return z;
}

}  // namespace
}  // namespace sq

using namespace sq;

extern "C" {

sq_status sq_quantize_w8(const void* w_dev, int64_t n, int64_t k, int8_t* codes_dev, void* scales_dev,
                         sq_stream_t stream) {
  if (!w_dev || !codes_dev || !scales_dev || n < 1 || k < 1) return fail(SQ_EINVAL, "sq_quantize_w8: bad arguments");
  k_quant8<false><<<(unsigned)n, W8_THREADS, 0, (cudaStream_t)stream>>>((const __half*)w_dev, k, k, codes_dev, scales_dev);
  count_launch();
  return cuda_check(cudaGetLastError(), "sq_quantize_w8");
}

sq_status sq_quantize_act8(const void* x_dev, int64_t m, int64_t k, int64_t ldx, int8_t* codes_dev, float* scales_dev,
                           sq_stream_t stream) {
  if (!x_dev || !codes_dev || !scales_dev || m < 1 || k < 1 || ldx < k) return fail(SQ_EINVAL, "sq_quantize_act8: bad arguments");
  auto t = prof_begin(KC_GLUE, (double)m * k * 3, 0, (cudaStream_t)stream);
  k_quant8<true><<<(unsigned)m, W8_THREADS, 0, (cudaStream_t)stream>>>((const __half*)x_dev, k, ldx, codes_dev, scales_dev);
  prof_end(t, (cudaStream_t)stream);
  count_launch();
  return cuda_check(cudaGetLastError(), "sq_quantize_act8");
}

size_t sq_linear_w8a8_workspace_bytes(int64_t n, int64_t k, int64_t m) {
  if (n < 1 || k < 1 || m < 1) return 0;
  const int z = i8_z(n, m, k);
  return z > 1 ? (size_t)z * m * n * 4 : 0;
}

sq_status sq_linear_w8a8(const int8_t* wq_dev, const void* sw_dev, const void* bias_dev, int64_t n, int64_t k,
                         const int8_t* xq_dev, const float* sx_dev, int64_t m, void* y_dev, int64_t ldy, int mode,
                         void* ws_dev, size_t ws_bytes, sq_stream_t stream) {
  if (!wq_dev || !sw_dev || !xq_dev || !sx_dev || !y_dev) return fail(SQ_EINVAL, "sq_linear_w8a8: null pointer");
  if (n < 128 || n % 128 || k < 128 || k % 128 || m < 1 || m > (1 << 24))
    return fail(SQ_EINVAL, "sq_linear_w8a8: need n, k multiples of 128 (n=%lld k=%lld m=%lld)", (long long)n, (long long)k, (long long)m);
  if (mode < 0 || mode > SQ_W8A8_I32) return fail(SQ_EINVAL, "sq_linear_w8a8: mode %d", mode);
  if (mode != SQ_W8A8_I32 && ldy < n) return fail(SQ_EINVAL, "sq_linear_w8a8: ldy < n");
  if ((reinterpret_cast<uintptr_t>(wq_dev) | reinterpret_cast<uintptr_t>(xq_dev)) & 15u)
    return fail(SQ_EINVAL, "sq_linear_w8a8: codes must be 16-B aligned");
  const int z = i8_z(n, m, k);
  const size_t need = sq_linear_w8a8_workspace_bytes(n, k, m);
  if (z > 1 && (!ws_dev || ws_bytes < need)) return fail(SQ_ENOMEM, "sq_linear_w8a8: workspace %zu < %zu", ws_bytes, need);
  cudaStream_t s = (cudaStream_t)stream;
  const int bt = i8_bt(m);
  CUtensorMap tw, tx;
  {
    const uint64_t d[2] = {(uint64_t)k, (uint64_t)n}, st[1] = {(uint64_t)k};
    const uint32_t b[2] = {I8_KS, I8_BN};
    cudaError_t e = encode_nd(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, wq_dev, 2, d, st, b, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return cuda_check(e, "sq_linear_w8a8: weight tensor map");
  }
  {
    const uint64_t d[2] = {(uint64_t)k, (uint64_t)m}, st[1] = {(uint64_t)k};
    const uint32_t b[2] = {I8_KS, (uint32_t)bt};
    cudaError_t e = encode_nd(&tx, CU_TENSOR_MAP_DATA_TYPE_UINT8, xq_dev, 2, d, st, b, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return cuda_check(e, "sq_linear_w8a8: activation tensor map");
  }
  I8P p{};
  p.sw = static_cast<const __half*>(sw_dev);
  p.sx = sx_dev;
  p.bias = static_cast<const __half*>(bias_dev);
  p.y = z > 1 ? ws_dev : y_dev;
  p.ldy = ldy;
  p.m = (int)m;
  p.n = (int)n;
  p.kst = (int)(k / I8_KS);
  p.Z = z;
  const int epi = mode == SQ_W8A8_I32 ? -1 : mode;
  auto t = prof_begin(KC_GEMM, (double)n * k + (double)m * k, 2.0 * m * n * k, s);
  cudaError_t e;
  const int kepi = z > 1 ? -1 : epi;
  switch (bt) {
    case 32: e = launch_i8_epi<32>(tw, tx, p, kepi, s); break;
    case 64: e = launch_i8_epi<64>(tw, tx, p, kepi, s); break;
    case 128: e = launch_i8_epi<128>(tw, tx, p, kepi, s); break;
    default: e = launch_i8_epi<256>(tw, tx, p, kepi, s); break;
  }
  count_launch();
  if (e == cudaSuccess && z > 1) {
    I8P q = p;
    q.y = y_dev;
    e = launch_i8_reduce(static_cast<const int32_t*>(ws_dev), z, q, epi, s);
    count_launch();
  }
  prof_end(t, s);
  return cuda_check(e, "sq_linear_w8a8");
}

}  // extern "C"
