// f2 — inputs of SplitQuant's variance indicator (Proposition 1, eq. 3; Theorem 1,
// P:176-182):  omega_{i,b} = sum_o D_{W_o} S_{W_o}(b)^2 G(X_o),  G(X) = Var[X] / 4 for the
// deterministic (round-to-nearest) quantizer.
//
//  * k_scale_sq: one pass over W fp16 [n, k]; one warp per 128 weights (1, 2 or 4 groups of
//    128 / 64 / 32), per group the RTN scale of every candidate bit width b exactly as the
//    quantizer computes it (R5: s = fp16(fp32(mx - mn) / (2^b - 1)), canonical +0), and the sum
//    over groups of group * s(b)^2 -- D_W S_W(b)^2 with the per-group scale of reading R4
//    (R17).  fp64 partials per CTA in fixed warp order, then one CTA sums the
//    partials in fixed order: deterministic.
//  * k_moments: E[X] and Var[X] (population, over all elements) of calibration activations in
//    two passes (sum, then sum of squared deviations), fp64, same fixed-order reductions.
// HBM-bound: W is read once (2 B / weight) for all bit widths together.
#include "sq_common.cuh"

namespace sq {
namespace {

constexpr int kThr = 256;
constexpr int kMaxBits = 8;

__device__ __forceinline__ double block_sum_d(double v, double* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffff, v, o);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  double t = 0.0;
#pragma unroll
  for (int i = 0; i < kThr / 32; ++i) t += red[i];  // fixed order
  __syncthreads();
  return t;
}

struct Bits {
  int n;
  int b[kMaxBits];
};

template <int G>
__global__ void __launch_bounds__(kThr) k_scale_sq(const __half* __restrict__ w, int64_t n, int64_t k, Bits bl,
                                                   double* __restrict__ part) {
  __shared__ double red[kThr / 32];
  constexpr int LPG = G / 4;  // lanes per group (4 weights per lane)
  const int lane = threadIdx.x & 31;
  const int64_t chunks = n * (k / 128);  // 128-weight chunks, one per warp per step
  const int64_t wid = (int64_t)blockIdx.x * (kThr / 32) + (threadIdx.x >> 5);
  const int64_t nw = (int64_t)gridDim.x * (kThr / 32);
  double acc[kMaxBits];
#pragma unroll
  for (int i = 0; i < kMaxBits; ++i) acc[i] = 0.0;
  for (int64_t c = wid; c < chunks; c += nw) {
    const int64_t r = c / (k / 128), cc = c % (k / 128);
    const uint2 raw = *reinterpret_cast<const uint2*>(w + r * k + cc * 128 + lane * 4);
    const __half2 a = *reinterpret_cast<const __half2*>(&raw.x), b = *reinterpret_cast<const __half2*>(&raw.y);
    float mn = fminf(fminf(__low2float(a), __high2float(a)), fminf(__low2float(b), __high2float(b)));
    float mx = fmaxf(fmaxf(__low2float(a), __high2float(a)), fmaxf(__low2float(b), __high2float(b)));
#pragma unroll
    for (int o = LPG / 2; o; o >>= 1) {
      mn = fminf(mn, __shfl_xor_sync(0xffffffff, mn, o));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffff, mx, o));
    }
    mn = __fadd_rn(mn, 0.0f);
    mx = __fadd_rn(mx, 0.0f);
    if ((lane % LPG) == 0) {  // one lane per group
#pragma unroll
      for (int i = 0; i < kMaxBits; ++i) {
        if (i < bl.n) {
          const float sf = __fdiv_rn(__fsub_rn(mx, mn), (float)((1 << bl.b[i]) - 1));
          const double s = (double)__half2float(__float2half_rn(sf));
          acc[i] += (double)G * s * s;
        }
      }
    }
  }
  for (int i = 0; i < bl.n; ++i) {
    const double t = block_sum_d(acc[i], red);
    if (threadIdx.x == 0) part[(int64_t)blockIdx.x * kMaxBits + i] = t;
  }
}

// out[i] = sum_c part[c * stride + i] for c < np, fixed order (one CTA, tree over a fixed layout)
__global__ void __launch_bounds__(kThr) k_sum_parts(const double* __restrict__ part, int np, int stride, int nout,
                                                    double* __restrict__ out, double scale) {
  __shared__ double red[kThr / 32];
  for (int i = 0; i < nout; ++i) {
    double v = 0.0;
    for (int c = threadIdx.x; c < np; c += kThr) v += part[(int64_t)c * stride + i];
    const double t = block_sum_d(v, red);
    if (threadIdx.x == 0) out[i] = t * scale;
  }
}

// pass 1 (mean == nullptr): per-CTA sum of x; pass 2: per-CTA sum of (x - mean)^2
__global__ void __launch_bounds__(kThr) k_moment(const __half* __restrict__ x, int64_t count, const double* mean,
                                                 double* __restrict__ part) {
  __shared__ double red[kThr / 32];
  const double mu = mean ? *mean : 0.0;
  double acc = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * kThr + threadIdx.x; i < count; i += (int64_t)gridDim.x * kThr) {
    const double v = (double)__half2float(x[i]);
    acc += mean ? (v - mu) * (v - mu) : v;
  }
  const double t = block_sum_d(acc, red);
  if (threadIdx.x == 0) part[blockIdx.x] = t;
}

int parts_for(int64_t work) {
  const int64_t p = (work + kThr - 1) / kThr;
  const int64_t cap = 4 * (int64_t)num_sms();
  return (int)(p < 1 ? 1 : (p < cap ? p : cap));
}

}  // namespace

size_t scale_sq_workspace_bytes(int64_t n, int64_t k) {
  return (size_t)parts_for(n * (k / 128) * 32) * kMaxBits * sizeof(double);
}

cudaError_t launch_scale_sq(const __half* w, int64_t n, int64_t k, int group, const int32_t* bits, int n_bits,
                            double* out, void* ws, cudaStream_t s) {
  Bits bl{};
  bl.n = n_bits;
  for (int i = 0; i < n_bits; ++i) bl.b[i] = bits[i];
  const int np = parts_for(n * (k / 128) * 32);
  double* part = static_cast<double*>(ws);
  auto t = prof_begin(KC_QUANT, (double)n * k * 2, 0, s);
  switch (group) {
    case 128: k_scale_sq<128><<<np, kThr, 0, s>>>(w, n, k, bl, part); break;
    case 64: k_scale_sq<64><<<np, kThr, 0, s>>>(w, n, k, bl, part); break;
    default: k_scale_sq<32><<<np, kThr, 0, s>>>(w, n, k, bl, part); break;
  }
  k_sum_parts<<<1, kThr, 0, s>>>(part, np, kMaxBits, n_bits, out, 1.0);
  prof_end(t, s);
  count_launch(2);
  return cudaGetLastError();
}

size_t moments_workspace_bytes(int64_t count) { return (size_t)(parts_for(count) + 1) * sizeof(double); }

// out[0] = E[x], out[1] = Var[x] (population)
cudaError_t launch_moments(const __half* x, int64_t count, double* out, void* ws, cudaStream_t s) {
  const int np = parts_for(count);
  double* part = static_cast<double*>(ws);
  auto t = prof_begin(KC_GLUE, (double)count * 4, 0, s);
  k_moment<<<np, kThr, 0, s>>>(x, count, nullptr, part);
  k_sum_parts<<<1, kThr, 0, s>>>(part, np, 1, 1, out, 1.0 / (double)count);
  k_moment<<<np, kThr, 0, s>>>(x, count, out, part);
  k_sum_parts<<<1, kThr, 0, s>>>(part, np, 1, 1, out + 1, 1.0 / (double)count);
  prof_end(t, s);
  count_launch(4);
  return cudaGetLastError();
}

}  // namespace sq

using namespace sq;

extern "C" {

size_t sq_scale_sq_sums_workspace_bytes(int64_t n, int64_t k) {
  if (n <= 0 || k <= 0 || k % 128) return 0;
  return scale_sq_workspace_bytes(n, k);
}

sq_status sq_scale_sq_sums(const void* w_dev, int64_t n, int64_t k, int group, const int32_t* bits_host, int n_bits,
                           double* out_dev, void* ws_dev, size_t ws_bytes, sq_stream_t stream) {
  if (!(group == 32 || group == 64 || group == 128)) return fail(SQ_EINVAL, "sq_scale_sq_sums: group=%d", group);
  if (n <= 0 || k <= 0 || k % 128) return fail(SQ_EINVAL, "sq_scale_sq_sums: need n>0, k%%128==0");
  if (!bits_host || n_bits < 1 || n_bits > kMaxBits) return fail(SQ_EINVAL, "sq_scale_sq_sums: 1..8 bit widths");
  for (int i = 0; i < n_bits; ++i)
    if (bits_host[i] < 2 || bits_host[i] > 8) return fail(SQ_EINVAL, "sq_scale_sq_sums: bits %d not in 2..8", bits_host[i]);
  if (!w_dev || !out_dev || (reinterpret_cast<uintptr_t>(w_dev) & 7u) || (reinterpret_cast<uintptr_t>(out_dev) & 7u))
    return fail(SQ_EINVAL, "sq_scale_sq_sums: null or misaligned pointer");
  if (!ws_dev || ws_bytes < scale_sq_workspace_bytes(n, k) || (reinterpret_cast<uintptr_t>(ws_dev) & 7u))
    return fail(SQ_ENOMEM, "sq_scale_sq_sums: workspace %zu < %zu", ws_bytes, scale_sq_workspace_bytes(n, k));
  return cuda_check(launch_scale_sq((const __half*)w_dev, n, k, group, bits_host, n_bits, out_dev, ws_dev,
                                    (cudaStream_t)stream),
                    "sq_scale_sq_sums");
}

size_t sq_act_moments_workspace_bytes(int64_t count) { return count > 0 ? moments_workspace_bytes(count) : 0; }

sq_status sq_act_moments(const void* x_dev, int64_t count, double* out_dev, void* ws_dev, size_t ws_bytes,
                         sq_stream_t stream) {
  if (count <= 0 || !x_dev || !out_dev || (reinterpret_cast<uintptr_t>(x_dev) & 1u) ||
      (reinterpret_cast<uintptr_t>(out_dev) & 7u))
    return fail(SQ_EINVAL, "sq_act_moments: bad arguments");
  if (!ws_dev || ws_bytes < moments_workspace_bytes(count) || (reinterpret_cast<uintptr_t>(ws_dev) & 7u))
    return fail(SQ_ENOMEM, "sq_act_moments: workspace %zu < %zu", ws_bytes, moments_workspace_bytes(count));
  return cuda_check(launch_moments((const __half*)x_dev, count, out_dev, ws_dev, (cudaStream_t)stream),
                    "sq_act_moments");
}

}  // extern "C"
