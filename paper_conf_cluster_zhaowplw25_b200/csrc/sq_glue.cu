// K5 — stage glue: pre-LN LayerNorm (no affine, eps 1e-5; R11) that
// emits the fp16 linear input AND its per-group sums for the decode GEMV
// (fused, so q/k/v and fc1 need no separate sq_xsum pass), the fp32 LayerNorm
// of the loop-back (R14), and strided row copies.  HBM-bound, one CTA per row.
#include "sq_common.cuh"

namespace sq {
namespace {

// 16 warps per row: the 32-row decode LayerNorm is latency-bound (one CTA per row); 512 threads cut
// the decode phase of the configs[3] bench by 2 % against 256 (same box, two runs each), 1024 also
// but slowed the 4096-row prefill LayerNorms
constexpr int kLnThreads = 512;

__device__ __forceinline__ float block_sum(float v, float* red) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffff, v, o);
  __syncthreads();
  if (lane == 0) red[warp] = v;
  __syncthreads();
  float t = 0.f;
#pragma unroll
  for (int i = 0; i < kLnThreads / 32; ++i) t += red[i];  // fixed order -> deterministic
  return t;
}

// x fp32 [rows, d] -> y = (x - mean) / sqrt(var + eps); d % 1024 == 0 not required, d % 128 == 0.
// Each warp owns groups of 128 consecutive elements (lane: 4 elements), so the
// group sums for the decode GEMV fall out of a warp reduction.
template <bool F16OUT>
__global__ void __launch_bounds__(kLnThreads) k_layernorm(const float* __restrict__ x, int64_t d, void* __restrict__ y,
                                                          float2* __restrict__ xsum, int xsum_rows,
                                                          const float* __restrict__ copy_src, float* __restrict__ copy_dst) {
  constexpr int MAXV = (112 + kLnThreads / 32 - 1) / (kLnThreads / 32);  // up to d = 112 * 128 = 14336 (BLOOM-176B h1)
  __shared__ float red[kLnThreads / 32];
  pdl_trigger();
  pdl_wait();
  const int64_t row = blockIdx.x;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const float* xr = x + row * d;
  const int ng = (int)(d / 128);
  float4 v[MAXV];
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int grp = warp + i * (kLnThreads / 32);
    if (grp < ng) {
      v[i] = *reinterpret_cast<const float4*>(xr + grp * 128 + lane * 4);
      s += (v[i].x + v[i].y) + (v[i].z + v[i].w);
    }
  }
  const float mean = block_sum(s, red) / (float)d;
  float q = 0.f;
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int grp = warp + i * (kLnThreads / 32);
    if (grp < ng) {
      const float a = v[i].x - mean, b = v[i].y - mean, c = v[i].z - mean, e = v[i].w - mean;
      q += (a * a + b * b) + (c * c + e * e);
    }
  }
  const float var = block_sum(q, red) / (float)d;
  const float inv = rsqrtf(var + 1e-5f);
#pragma unroll
  for (int i = 0; i < MAXV; ++i) {
    const int grp = warp + i * (kLnThreads / 32);
    if (grp < ng) {
      const float o0 = (v[i].x - mean) * inv, o1 = (v[i].y - mean) * inv;
      const float o2 = (v[i].z - mean) * inv, o3 = (v[i].w - mean) * inv;
      if constexpr (F16OUT) {
        const __half2 h01 = __floats2half2_rn(o0, o1), h23 = __floats2half2_rn(o2, o3);
        uint2 pk;
        pk.x = *reinterpret_cast<const uint32_t*>(&h01);
        pk.y = *reinterpret_cast<const uint32_t*>(&h23);
        *reinterpret_cast<uint2*>(static_cast<__half*>(y) + row * d + grp * 128 + lane * 4) = pk;
        if (xsum) {  // same definition and order as sq_xsum, on the fp16-rounded values
          float a = __low2float(h01) + __high2float(h01);
          float b = __low2float(h23) + __high2float(h23);
#pragma unroll
          for (int o = 16; o; o >>= 1) {
            a += __shfl_xor_sync(0xffffffff, a, o);
            b += __shfl_xor_sync(0xffffffff, b, o);
          }
          if (lane == 0) xsum[(int64_t)grp * xsum_rows + row] = make_float2(a, b);
        }
      } else {
        *reinterpret_cast<float4*>(static_cast<float*>(y) + row * d + grp * 128 + lane * 4) = make_float4(o0, o1, o2, o3);
      }
      if (copy_dst) {
        *reinterpret_cast<float4*>(copy_dst + row * d + grp * 128 + lane * 4) =
            *reinterpret_cast<const float4*>(copy_src + row * d + grp * 128 + lane * 4);
      }
    }
  }
}

// dst[r, 0:d] = src[r * sstride, 0:d] for r < rows (fp32, d % 4 == 0)
__global__ void k_copy_rows(const float* __restrict__ src, int64_t sstride, int64_t rows, int64_t d,
                            float* __restrict__ dst, int64_t dstride) {
  pdl_trigger();
  pdl_wait();
  const int64_t r = blockIdx.y;
  for (int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) * 4; c < d; c += (int64_t)gridDim.x * blockDim.x * 4)
    *reinterpret_cast<float4*>(dst + r * dstride + c) = *reinterpret_cast<const float4*>(src + r * sstride + c);
}

}  // namespace

cudaError_t launch_layernorm_f16(const float* x, int64_t rows, int64_t d, __half* y, float2* xsum,
                                 const float* copy_src, float* copy_dst, cudaStream_t s) {
  if (d % 128 || d > 14 * 1024) return cudaErrorInvalidValue;
  auto t = prof_begin(KC_GLUE, (double)rows * d * (4 + 2 + (copy_dst ? 8 : 0)), 0, s);
  cudaError_t e = launch_pdl(k_layernorm<true>, dim3((unsigned)rows), dim3(kLnThreads), 0, s, x, d, (void*)y, xsum, 32,
                             copy_src, copy_dst);
  prof_end(t, s);
  count_launch();
  return e;
}

cudaError_t launch_layernorm_f32(const float* x, int64_t rows, int64_t d, float* y, cudaStream_t s) {
  if (d % 128 || d > 14 * 1024) return cudaErrorInvalidValue;
  auto t = prof_begin(KC_GLUE, (double)rows * d * 8, 0, s);
  cudaError_t e = launch_pdl(k_layernorm<false>, dim3((unsigned)rows), dim3(kLnThreads), 0, s, x, d, (void*)y,
                             (float2*)nullptr, 0, (const float*)nullptr, (float*)nullptr);
  prof_end(t, s);
  count_launch();
  return e;
}

cudaError_t launch_copy_rows(const float* src, int64_t sstride, int64_t rows, int64_t d, float* dst, int64_t dstride,
                             cudaStream_t s) {
  if (rows <= 0) return cudaSuccess;
  dim3 grid((unsigned)((d / 4 + 255) / 256), (unsigned)rows);
  auto t = prof_begin(KC_GLUE, (double)rows * d * 8, 0, s);
  cudaError_t e = launch_pdl(k_copy_rows, grid, dim3(256), 0, s, src, sstride, rows, d, dst, dstride);
  prof_end(t, s);
  count_launch();
  return e;
}

}  // namespace sq
