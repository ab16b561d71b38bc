// f3 — causal multi-head self-attention over a per-layer KV cache (DESIGN.md
// R23-R25; KV-cache sizing 2 v (s + n) h1 elements; chunked prefill).
//
//   K6  kv_append   new tokens' k, v (columns [h1, 3 h1) of the fused qkv rows) -> the layer's cache
//                   K / V [n_seq][max_len][h1] fp16 at (seq0 + i, pos0 + j).  HBM-bound copy.
//   K7  attn_prefill  FlashAttention-2 style, one CTA per (sequence, head, 128-query block): Q in
//                   registers, 64-key K / V blocks of the cache double-buffered in shared memory
//                   (cp.async, zero-filled beyond the last visible key), S = Q K^T and O += P V on
//                   mma.sync m16n8k16 (fp16 in, fp32 accumulate), online softmax in fp32 (exp2).
//                   Prefill attention is ~1-2 % of the prefill FLOPs at s = 512 (4 s^2 h1 vs the
//                   linears' 24 s h1^2 per sequence-layer), so the legacy tensor-core path is kept.
//   K8  attn_decode   one CTA (4 warps) per (sequence, head): 8 lanes per key (dh / 8 elements each),
//                   4 keys per warp step, 16-B cache loads issued 4 steps ahead, per-key-group online
//                   softmax, merged across lane groups and warps in a fixed order (deterministic).
//                   HBM-bound: reads 2 (p + 1) dh fp16 per (sequence, head).
// Scores use scale 1/sqrt(dh); the query at position p sees cache positions 0..p (causal).
#include "sq_common.cuh"

namespace sq {
namespace {

constexpr float kLog2e = 1.4426950408889634f;

__global__ void __launch_bounds__(256) k_kv_append(const __half* __restrict__ qkv, int64_t ldq, int nseq, int len,
                                                   int pos0, int64_t seq0, int h1, __half* __restrict__ kc,
                                                   __half* __restrict__ vc, int max_len) {
  // one thread per 16-B chunk of the k and v halves of a row
  const int per_row = 2 * h1 / 8;
  const int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= (int64_t)nseq * len * per_row) return;
  const int64_t row = idx / per_row;
  const int c8 = (int)(idx % per_row) * 8;  // column in [0, 2 h1)
  const int i = (int)(row / len), p = pos0 + (int)(row % len);
  const uint4 v = *reinterpret_cast<const uint4*>(qkv + row * ldq + h1 + c8);
  __half* dst = (c8 < h1 ? kc : vc) + ((seq0 + i) * (int64_t)max_len + p) * h1 + (c8 < h1 ? c8 : c8 - h1);
  *reinterpret_cast<uint4*>(dst) = v;
}

__device__ __forceinline__ void cp_async16(void* smem, const void* g, bool valid) {
  const uint32_t s = smem_u32(smem);
  const int n = valid ? 16 : 0;  // src-size 0 -> zero fill
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(s), "l"(g), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

__device__ __forceinline__ void ldsm_x2_trans(uint32_t& r0, uint32_t& r1, const void* p) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x2.trans.shared.b16 {%0, %1}, [%2];"
               : "=r"(r0), "=r"(r1) : "r"(smem_u32(p)));
}
__device__ __forceinline__ uint32_t pack_h2(float a, float b) {
  __half2 h = __floats2half2_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

template <int DH>
struct PreCfg {
  static constexpr int BQ = 128, BK = 64, LD = DH + 8;  // padded rows: conflict-free fragment loads
  static constexpr int THREADS = 32 * (BQ / 16);        // one warp per 16 query rows
  static constexpr int BLK = BK * LD;                   // halves per K or V block
  static constexpr int SMEM = 2 * 2 * BLK * 2;          // 2 stages x (K + V) x fp16
};

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void ldsm_x4(uint32_t& r0, uint32_t& r1, uint32_t& r2, uint32_t& r3, const void* p) {
  asm volatile("ldmatrix.sync.aligned.m8n8.x4.shared.b16 {%0, %1, %2, %3}, [%4];"
               : "=r"(r0), "=r"(r1), "=r"(r2), "=r"(r3) : "r"(smem_u32(p)));
}

template <int DH>
__global__ void __launch_bounds__(PreCfg<DH>::THREADS) k_attn_prefill(const __half* __restrict__ qkv, int64_t ldq, int len, int pos0,
                                                      int64_t seq0, int h1, const __half* __restrict__ kc,
                                                      const __half* __restrict__ vc, int max_len,
                                                      __half* __restrict__ out, int64_t ldo, float qscale) {
  using C = PreCfg<DH>;
  extern __shared__ __align__(16) __half sm[];
  const int qb = blockIdx.x, h = blockIdx.y, i = blockIdx.z;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  const int q0 = qb * C::BQ;                      // first query row of the block (within the sequence)
  const int qrows = min(C::BQ, len - q0);
  const int last_key = pos0 + q0 + qrows - 1;     // highest visible key of the block
  const int nkb = last_key / C::BK + 1;
  const __half* kbase = kc + (seq0 + i) * (int64_t)max_len * h1 + h * DH;
  const __half* vbase = vc + (seq0 + i) * (int64_t)max_len * h1 + h * DH;
  auto load_block = [&](int kb, int st) {
    __half* ks = sm + st * 2 * C::BLK;
    __half* vs = ks + C::BLK;
    constexpr int CH = DH / 8;  // 16-B chunks per row
    for (int c = threadIdx.x; c < C::BK * CH; c += C::THREADS) {
      const int r = c / CH, cc = (c % CH) * 8, j = kb * C::BK + r;
      const bool ok = j <= last_key;
      const int64_t off = (int64_t)(ok ? j : 0) * h1 + cc;
      cp_async16(ks + r * C::LD + cc, kbase + off, ok);
      cp_async16(vs + r * C::LD + cc, vbase + off, ok);
    }
    cp_async_commit();
  };
  load_block(0, 0);
  // Q fragments (A operand, 16 rows per warp); rows past the block's end are zero
  uint32_t qa[DH / 16][4];
  const int r_lo = q0 + warp * 16 + g, r_hi = r_lo + 8;
  const __half* qlo = qkv + ((int64_t)i * len + r_lo) * ldq + h * DH;
  const __half* qhi = qkv + ((int64_t)i * len + r_hi) * ldq + h * DH;
#pragma unroll
  for (int kk = 0; kk < DH / 16; ++kk) {
    const int c = kk * 16 + 2 * t;
    qa[kk][0] = r_lo < len ? *reinterpret_cast<const uint32_t*>(qlo + c) : 0u;
    qa[kk][1] = r_hi < len ? *reinterpret_cast<const uint32_t*>(qhi + c) : 0u;
    qa[kk][2] = r_lo < len ? *reinterpret_cast<const uint32_t*>(qlo + c + 8) : 0u;
    qa[kk][3] = r_hi < len ? *reinterpret_cast<const uint32_t*>(qhi + c + 8) : 0u;
  }
  const int p_lo = pos0 + r_lo, p_hi = pos0 + r_hi;  // query positions of this thread's two rows
  float o[DH / 8][4];
#pragma unroll
  for (int n = 0; n < DH / 8; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
  float m_lo = -INFINITY, m_hi = -INFINITY, l_lo = 0.f, l_hi = 0.f;
  for (int kb = 0; kb < nkb; ++kb) {
    if (kb + 1 < nkb) {
      load_block(kb + 1, (kb + 1) & 1);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncthreads();
    const __half* ks = sm + (kb & 1) * 2 * C::BLK;
    const __half* vs = ks + C::BLK;
    // S = Q K^T: 16 x 64 per warp (8 n-tiles of 8 keys)
    float s[8][4];
#pragma unroll
    for (int n = 0; n < 8; ++n) s[n][0] = s[n][1] = s[n][2] = s[n][3] = 0.f;
    // B fragments of two 8-key n-tiles per ldmatrix.x4: matrices (keys n0..+7 | k 0-7), (n0 | k 8-15),
    // (n0+8 | k 0-7), (n0+8 | k 8-15) -> b0/b1 of tile n, b0/b1 of tile n+1
    const __half* kbl = ks + ((lane & 7) + ((lane >> 4) & 1) * 8) * C::LD + ((lane >> 3) & 1) * 8;
#pragma unroll
    for (int n = 0; n < 8; n += 2) {
#pragma unroll
      for (int kk = 0; kk < DH / 16; ++kk) {
        uint32_t b0, b1, b2, b3;
        ldsm_x4(b0, b1, b2, b3, kbl + n * 8 * C::LD + kk * 16);
        mma_16816(s[n], qa[kk], b0, b1, s[n]);
        mma_16816(s[n + 1], qa[kk], b2, b3, s[n + 1]);
      }
    }
    // scale (log2 domain), causal mask, online softmax per row
    float mx_lo = m_lo, mx_hi = m_hi;
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      const int j = kb * C::BK + n * 8 + 2 * t;
      s[n][0] = (j <= p_lo) ? s[n][0] * qscale : -INFINITY;
      s[n][1] = (j + 1 <= p_lo) ? s[n][1] * qscale : -INFINITY;
      s[n][2] = (j <= p_hi) ? s[n][2] * qscale : -INFINITY;
      s[n][3] = (j + 1 <= p_hi) ? s[n][3] * qscale : -INFINITY;
      mx_lo = fmaxf(mx_lo, fmaxf(s[n][0], s[n][1]));
      mx_hi = fmaxf(mx_hi, fmaxf(s[n][2], s[n][3]));
    }
    mx_lo = fmaxf(mx_lo, __shfl_xor_sync(0xffffffffu, mx_lo, 1));
    mx_lo = fmaxf(mx_lo, __shfl_xor_sync(0xffffffffu, mx_lo, 2));
    mx_hi = fmaxf(mx_hi, __shfl_xor_sync(0xffffffffu, mx_hi, 1));
    mx_hi = fmaxf(mx_hi, __shfl_xor_sync(0xffffffffu, mx_hi, 2));
    // rows with no visible key yet keep -inf: use 0 as the reference so exp2 gives 0, not NaN
    const float ref_lo = mx_lo == -INFINITY ? 0.f : mx_lo, ref_hi = mx_hi == -INFINITY ? 0.f : mx_hi;
    const float corr_lo = ex2(m_lo - ref_lo), corr_hi = ex2(m_hi - ref_hi);
    m_lo = mx_lo;
    m_hi = mx_hi;
    float sum_lo = 0.f, sum_hi = 0.f;
    uint32_t pa[4][4];  // P as A fragments: keys 16 kk .. 16 kk + 15
#pragma unroll
    for (int n = 0; n < 8; ++n) {
      const float e0 = ex2(s[n][0] - ref_lo), e1 = ex2(s[n][1] - ref_lo);
      const float e2 = ex2(s[n][2] - ref_hi), e3 = ex2(s[n][3] - ref_hi);
      sum_lo += e0 + e1;
      sum_hi += e2 + e3;
      const int kk = n >> 1, hi = n & 1;
      pa[kk][hi ? 2 : 0] = pack_h2(e0, e1);
      pa[kk][hi ? 3 : 1] = pack_h2(e2, e3);
    }
    l_lo = l_lo * corr_lo + sum_lo;
    l_hi = l_hi * corr_hi + sum_hi;
#pragma unroll
    for (int n = 0; n < DH / 8; ++n) {
      o[n][0] *= corr_lo; o[n][1] *= corr_lo;
      o[n][2] *= corr_hi; o[n][3] *= corr_hi;
    }
    // O += P V
#pragma unroll
    for (int kk = 0; kk < 4; ++kk) {
#pragma unroll
      for (int n = 0; n < DH / 8; ++n) {
        uint32_t b0, b1;
        ldsm_x2_trans(b0, b1, vs + (kk * 16 + (lane & 15)) * C::LD + n * 8);
        mma_16816(o[n], pa[kk], b0, b1, o[n]);
      }
    }
    __syncthreads();  // the stage is refilled by the next iteration's prefetch
  }
  // the quad's partial row sums (each lane summed its own 16 keys per block)
  l_lo += __shfl_xor_sync(0xffffffffu, l_lo, 1);
  l_lo += __shfl_xor_sync(0xffffffffu, l_lo, 2);
  l_hi += __shfl_xor_sync(0xffffffffu, l_hi, 1);
  l_hi += __shfl_xor_sync(0xffffffffu, l_hi, 2);
  const float inv_lo = l_lo > 0.f ? 1.f / l_lo : 0.f, inv_hi = l_hi > 0.f ? 1.f / l_hi : 0.f;
#pragma unroll
  for (int n = 0; n < DH / 8; ++n) {
    const int c = h * DH + n * 8 + 2 * t;
    if (r_lo < len)
      *reinterpret_cast<__half2*>(out + ((int64_t)i * len + r_lo) * ldo + c) = __floats2half2_rn(o[n][0] * inv_lo, o[n][1] * inv_lo);
    if (r_hi < len)
      *reinterpret_cast<__half2*>(out + ((int64_t)i * len + r_hi) * ldo + c) = __floats2half2_rn(o[n][2] * inv_hi, o[n][3] * inv_hi);
  }
}

// K8: decode.  Lane group kg = lane / 8 handles key j = 16 q + 4 warp + kg of step q; lane (lane % 8)
// holds dh elements [EPL * (lane % 8), + EPL).
template <int DH>
__global__ void __launch_bounds__(128) k_attn_decode(const __half* __restrict__ qkv, int64_t ldq, int pos, int64_t seq0,
                                                     int h1, const __half* __restrict__ kc, const __half* __restrict__ vc,
                                                     int max_len, __half* __restrict__ out, int64_t ldo, float qscale) {
  constexpr int EPL = DH / 8, V4 = EPL / 8;  // elements per lane, uint4 loads per lane per key
  constexpr int U = 4;                        // steps in flight
  __shared__ float red[4][2 + DH];
  const int h = blockIdx.x, i = blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, kg = lane >> 3, el = lane & 7;
  pdl_wait();
  float q[EPL];
  {
    const __half* qp = qkv + (int64_t)i * ldq + h * DH + el * EPL;
#pragma unroll
    for (int v = 0; v < V4; ++v) {
      const uint4 w = *reinterpret_cast<const uint4*>(qp + 8 * v);
      const __half2* hw = reinterpret_cast<const __half2*>(&w);
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __half22float2(hw[e]);
        q[8 * v + 2 * e] = f.x * qscale;
        q[8 * v + 2 * e + 1] = f.y * qscale;
      }
    }
  }
  const __half* kb = kc + (seq0 + i) * (int64_t)max_len * h1 + h * DH + el * EPL;
  const __half* vb = vc + (seq0 + i) * (int64_t)max_len * h1 + h * DH + el * EPL;
  float m = -INFINITY, l = 0.f, acc[EPL];
#pragma unroll
  for (int e = 0; e < EPL; ++e) acc[e] = 0.f;
  const int nsteps = (pos + 1 + 15) / 16;
  for (int q0 = 0; q0 < nsteps; q0 += U) {
    uint4 kr[U][V4], vr[U][V4];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int j = (q0 + u) * 16 + warp * 4 + kg;
      const bool ok = j <= pos;
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        kr[u][v] = ok ? ldg_nc_v4(kb + (int64_t)j * h1 + 8 * v) : make_uint4(0, 0, 0, 0);
        vr[u][v] = ok ? ldg_nc_v4(vb + (int64_t)j * h1 + 8 * v) : make_uint4(0, 0, 0, 0);
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int j = (q0 + u) * 16 + warp * 4 + kg;
      float sc = 0.f;
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        const __half2* hk = reinterpret_cast<const __half2*>(&kr[u][v]);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __half22float2(hk[e]);
          sc = fmaf(q[8 * v + 2 * e], f.x, sc);
          sc = fmaf(q[8 * v + 2 * e + 1], f.y, sc);
        }
      }
      sc += __shfl_xor_sync(0xffffffffu, sc, 1);
      sc += __shfl_xor_sync(0xffffffffu, sc, 2);
      sc += __shfl_xor_sync(0xffffffffu, sc, 4);
      if (j > pos) continue;  // uniform within the lane group
      const float mn = fmaxf(m, sc);
      const float corr = exp2f(m - mn), pj = exp2f(sc - mn);
      l = l * corr + pj;
#pragma unroll
      for (int v = 0; v < V4; ++v) {
        const __half2* hv = reinterpret_cast<const __half2*>(&vr[u][v]);
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const float2 f = __half22float2(hv[e]);
          acc[8 * v + 2 * e] = fmaf(acc[8 * v + 2 * e], corr, pj * f.x);
          acc[8 * v + 2 * e + 1] = fmaf(acc[8 * v + 2 * e + 1], corr, pj * f.y);
        }
      }
      m = mn;
    }
  }
  // merge the 4 lane groups of the warp (fixed order: xor 8 then 16), then the 4 warps
#pragma unroll
  for (int off = 8; off <= 16; off <<= 1) {
    const float m2 = __shfl_xor_sync(0xffffffffu, m, off), l2 = __shfl_xor_sync(0xffffffffu, l, off);
    const float mn = fmaxf(m, m2);
    const float c1 = mn == -INFINITY ? 0.f : exp2f(m - mn), c2 = mn == -INFINITY ? 0.f : exp2f(m2 - mn);
    l = l * c1 + l2 * c2;
#pragma unroll
    for (int e = 0; e < EPL; ++e) {
      const float a2 = __shfl_xor_sync(0xffffffffu, acc[e], off);
      acc[e] = acc[e] * c1 + a2 * c2;
    }
    m = mn;
  }
  if (kg == 0) {
    if (el == 0) { red[warp][0] = m; red[warp][1] = l; }
#pragma unroll
    for (int e = 0; e < EPL; ++e) red[warp][2 + el * EPL + e] = acc[e];
  }
  __syncthreads();
  if (warp == 0) {
    float M = -INFINITY;
    for (int w = 0; w < 4; ++w) M = fmaxf(M, red[w][0]);
    float L = 0.f;
    float cw[4];
    for (int w = 0; w < 4; ++w) {
      cw[w] = red[w][0] == -INFINITY ? 0.f : exp2f(red[w][0] - M);
      L += red[w][1] * cw[w];
    }
    const float inv = 1.f / L;
    for (int c = lane; c < DH; c += 32) {
      float a = 0.f;
      for (int w = 0; w < 4; ++w) a += red[w][2 + c] * cw[w];
      out[(int64_t)i * ldo + h * DH + c] = __float2half_rn(a * inv);
    }
  }
}

}  // namespace

// kv_append + attention for one layer (see sq.h sq_attention); qkv rows (i, p) = i * len + (p - pos0)
cudaError_t launch_attention(const __half* qkv, int64_t ldq, int nseq, int len, int pos0, int64_t seq0, int h1,
                             int n_heads, __half* kc, __half* vc, int max_len, __half* out, int64_t ldo,
                             cudaStream_t s) {
  const int dh = h1 / n_heads;
  {
    const int64_t n = (int64_t)nseq * len * (2 * h1 / 8);
    k_kv_append<<<(unsigned)((n + 255) / 256), 256, 0, s>>>(qkv, ldq, nseq, len, pos0, seq0, h1, kc, vc, max_len);
    count_launch();
  }
  const float qscale = kLog2e / sqrtf((float)dh);
  // algorithmic work: decode reads the K and V rows 0..p of every (sequence, head); prefill does
  // 2 x 2 dh flops per (query, visible key, head) for S = Q K^T and O = P V
  const double keys = (double)len * pos0 + (double)len * (len + 1) / 2.0;  // sum over queries of (p + 1)
  auto t = prof_begin(len == 1 ? KC_ATTN_DEC : KC_ATTN_PRE, (double)nseq * 2.0 * (pos0 + 1) * h1 * 2,
                      (double)nseq * n_heads * 4.0 * dh * keys, s);
  if (len == 1) {
    dim3 grid(n_heads, nseq);
    if (dh == 128) launch_pdl(k_attn_decode<128>, grid, dim3(128), 0, s, qkv, ldq, pos0, seq0, h1, (const __half*)kc, (const __half*)vc, max_len, out, ldo, qscale);
    else launch_pdl(k_attn_decode<64>, grid, dim3(128), 0, s, qkv, ldq, pos0, seq0, h1, (const __half*)kc, (const __half*)vc, max_len, out, ldo, qscale);
  } else {
    if (dh == 128) {
      using C = PreCfg<128>;
      static bool set = false;
      if (!set) { cudaFuncSetAttribute(k_attn_prefill<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM); set = true; }
      dim3 grid((len + C::BQ - 1) / C::BQ, n_heads, nseq);
      k_attn_prefill<128><<<grid, C::THREADS, C::SMEM, s>>>(qkv, ldq, len, pos0, seq0, h1, kc, vc, max_len, out, ldo, qscale);
    } else {
      using C = PreCfg<64>;
      static bool set = false;
      if (!set) { cudaFuncSetAttribute(k_attn_prefill<64>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM); set = true; }
      dim3 grid((len + C::BQ - 1) / C::BQ, n_heads, nseq);
      k_attn_prefill<64><<<grid, C::THREADS, C::SMEM, s>>>(qkv, ldq, len, pos0, seq0, h1, kc, vc, max_len, out, ldo, qscale);
    }
  }
  prof_end(t, s);
  count_launch();
  return cudaGetLastError();
}

}  // namespace sq

using namespace sq;

extern "C" sq_status sq_attention(const void* qkv_dev, int64_t ld_qkv, int64_t nseq, int64_t len, int64_t pos0,
                                  int64_t seq0, int64_t h1, int n_heads, void* k_cache_dev, void* v_cache_dev,
                                  int64_t max_len, int64_t n_seq_cache, void* out_dev, int64_t ld_out,
                                  sq_stream_t stream) {
  if (!qkv_dev || !k_cache_dev || !v_cache_dev || !out_dev) return fail(SQ_EINVAL, "sq_attention: null pointer");
  if (n_heads <= 0 || h1 % n_heads || (h1 / n_heads != 64 && h1 / n_heads != 128))
    return fail(SQ_EINVAL, "sq_attention: head_dim h1/n_heads must be 64 or 128 (h1=%lld, heads=%d)", (long long)h1, n_heads);
  if (nseq < 1 || len < 1 || pos0 < 0 || pos0 + len > max_len || seq0 < 0 || seq0 + nseq > n_seq_cache)
    return fail(SQ_EINVAL, "sq_attention: positions/sequences out of the cache");
  if (ld_qkv < 3 * h1 || ld_out < h1 || ld_qkv % 8 || ld_out % 8 || h1 % 8 ||
      ((reinterpret_cast<uintptr_t>(qkv_dev) | reinterpret_cast<uintptr_t>(k_cache_dev) |
        reinterpret_cast<uintptr_t>(v_cache_dev) | reinterpret_cast<uintptr_t>(out_dev)) & 15u))
    return fail(SQ_EINVAL, "sq_attention: leading dims / pointers must be 16-B aligned");
  return cuda_check(launch_attention((const __half*)qkv_dev, ld_qkv, (int)nseq, (int)len, (int)pos0, seq0, (int)h1,
                                     n_heads, (__half*)k_cache_dev, (__half*)v_cache_dev, (int)max_len,
                                     (__half*)out_dev, ld_out, (cudaStream_t)stream),
                    "sq_attention");
}
