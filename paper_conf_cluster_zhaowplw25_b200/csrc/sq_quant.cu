// K1 — per-group RTN min/max quantization and bit packing (DESIGN.md
// section 4, layouts L8/L4/L3).  Load-time kernels ("weights are quantized when
// loaded into GPU memory"), HBM-bound: read 2 B/weight, write 1 B/weight
// codes (+ 4 B/group), then packing reads codes and writes bits/8 B/weight.
#include "sq_common.cuh"

namespace sq {
namespace {

// splitmix64 output i of the stream seeded `seed` (finalizer of seed + (i + 1) * golden) and its top 24
// bits as a uniform in [0, 1) -- the counter-based generator of the stochastic-rounding variant (R22).
__device__ __forceinline__ float uniform24(uint64_t seed, uint64_t i) {
  uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  z ^= z >> 31;
  return (float)(uint32_t)(z >> 40) * (1.0f / 16777216.0f);
}

// One warp per (row, group).  IEEE fp32 with one rounding per op, identical op
// sequence to the CPU oracle's definition (R1-R6, R21, R22):
//   mn, mx (canonical +0);
//   asymmetric:  s = fp16(fp32(mx - mn) / (2^b - 1)); z = mn; d = fp32(w - z) / s; c in [0, 2^b - 1]
//   symmetric:  s = fp16(max(|mx|, |mn|) / (2^(b-1) - 1)); z = -2^(b-1) s; d = w / s;
//                       c = clamp(., -(2^(b-1) - 1), 2^(b-1) - 1) + 2^(b-1)
//   rounding: rint_even(d), or stochastic floor(d) + [u < d - floor(d)] (Theorem 1)
//   s == 0 -> d = 0.  A symmetric zero beyond the fp16 range sets *status (the oracle rejects it).
template <int G, int MODE>
__global__ void __launch_bounds__(256) k_quantize(const __half* __restrict__ w, int64_t n, int64_t k, int bits,
                                                  uint8_t* __restrict__ codes, __half* __restrict__ scales,
                                                  __half* __restrict__ zeros, uint64_t seed, int* status) {
  constexpr bool SYM = MODE & SQ_QUANT_SYMMETRIC, STOCH = MODE & SQ_QUANT_STOCHASTIC;
  constexpr int PER = G / 32;  // elements per lane: 4, 2, 1
  const int64_t ng = k / G;
  const int64_t gid = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  if (gid >= n * ng) return;
  const int lane = threadIdx.x & 31;
  const int64_t r = gid / ng, g = gid % ng;
  const __half* p = w + r * k + g * G + lane * PER;
  float v[PER];
  if constexpr (PER == 4) {
    uint2 raw = *reinterpret_cast<const uint2*>(p);
    __half2 a = *reinterpret_cast<__half2*>(&raw.x), b = *reinterpret_cast<__half2*>(&raw.y);
    v[0] = __low2float(a); v[1] = __high2float(a); v[2] = __low2float(b); v[3] = __high2float(b);
  } else if constexpr (PER == 2) {
    __half2 a = *reinterpret_cast<const __half2*>(p);
    v[0] = __low2float(a); v[1] = __high2float(a);
  } else {
    v[0] = __half2float(*p);
  }
  float mn = v[0], mx = v[0];
#pragma unroll
  for (int i = 1; i < PER; ++i) { mn = fminf(mn, v[i]); mx = fmaxf(mx, v[i]); }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    mn = fminf(mn, __shfl_xor_sync(0xffffffff, mn, o));
    mx = fmaxf(mx, __shfl_xor_sync(0xffffffff, mx, o));
  }
  mn = __fadd_rn(mn, 0.0f);  // canonical zeros: -0 -> +0
  mx = __fadd_rn(mx, 0.0f);
  const int half_i = 1 << (bits - 1);
  const float qmax = (float)((1 << bits) - 1);
  const float sf = SYM ? __fdiv_rn(fmaxf(fabsf(mx), fabsf(mn)), (float)(half_i - 1)) : __fdiv_rn(__fsub_rn(mx, mn), qmax);
  const __half s16 = __float2half_rn(sf);
  const float s = __half2float(s16);
  float z = mn;
  if constexpr (SYM) {
    z = __fadd_rn(__fmul_rn(-(float)half_i, s), 0.0f);  // exact; +0 when s == 0
    if (fabsf(z) > 65504.f && lane == 0) atomicOr(status, 1);
  }
  if (lane == 0) {
    scales[r * ng + g] = s16;
    zeros[r * ng + g] = __float2half_rn(z);
  }
  const float cmin = SYM ? -(float)(half_i - 1) : 0.0f, cmax = SYM ? (float)(half_i - 1) : qmax;
  const float off = SYM ? (float)half_i : 0.0f;
  uint32_t packed = 0;
#pragma unroll
  for (int i = 0; i < PER; ++i) {
    float d = 0.0f;
    if (s != 0.0f) d = SYM ? __fdiv_rn(v[i], s) : __fdiv_rn(__fsub_rn(v[i], mn), s);
    float q;
    if constexpr (STOCH) {
      const float fl = floorf(d);
      const float fr = __fsub_rn(d, fl);
      q = fl + (uniform24(seed, (uint64_t)(r * k + g * G + lane * PER + i)) < fr ? 1.0f : 0.0f);
    } else {
      q = rintf(d);
    }
    q = fminf(fmaxf(q, cmin), cmax);
    packed |= (uint32_t)(int)(q + off) << (8 * i);
  }
  uint8_t* cp = codes + r * k + g * G + lane * PER;
  if constexpr (PER == 4) *reinterpret_cast<uint32_t*>(cp) = packed;
  else if constexpr (PER == 2) *reinterpret_cast<uint16_t*>(cp) = (uint16_t)packed;
  else *cp = (uint8_t)packed;
}

// Placement T16: unit u = (tile t, group g) holds the 16 rows'
// group-g bytes contiguously, units tile-major / group-minor; row rr of the unit at
// rr * GB.  Output word i of the packed buffer -> (unit, row-in-tile, word-in-row).
__device__ __forceinline__ int64_t src_row_col(int64_t unit, int rr, int kg, int64_t k, int64_t col_in_group) {
  const int64_t t = unit / kg, g = unit % kg;
  return (t * 16 + rr) * k + g * 128 + col_in_group;
}

// L4: one thread per output word (8 codes): nibble (j%8)/2 + 4*(j%2).
__global__ void k_pack4(const uint8_t* __restrict__ codes, int64_t nwords, int kg, int64_t k, uint32_t* __restrict__ out) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nwords) return;
  const int64_t unit = i / (16 * 16);
  const int rr = (int)((i / 16) % 16), wi = (int)(i % 16);
  uint2 c = *reinterpret_cast<const uint2*>(codes + src_row_col(unit, rr, kg, k, 8 * wi));
  uint32_t b[8] = {c.x & 0xFF, (c.x >> 8) & 0xFF, (c.x >> 16) & 0xFF, c.x >> 24,
                   c.y & 0xFF, (c.y >> 8) & 0xFF, (c.y >> 16) & 0xFF, c.y >> 24};
  uint32_t w = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) w |= (b[j] & 0xF) << (4 * ((j >> 1) + 4 * (j & 1)));
  out[i] = w;
}

// L3: one thread per 32-code block -> words W0..W2; code k' = 2i + e: pairs
// i < 15 at W_{i/5} bits 16e + 3(i%5); pair 15 bit b at W_b bit 15 + 16e.
__global__ void k_pack3(const uint8_t* __restrict__ codes, int64_t nblocks, int kg, int64_t k, uint32_t* __restrict__ out) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nblocks) return;
  const int64_t unit = i / (16 * 4);
  const int rr = (int)((i / 4) % 16), bl = (int)(i % 4);
  const uint4* src = reinterpret_cast<const uint4*>(codes + src_row_col(unit, rr, kg, k, 32 * bl));
  uint4 a = src[0], b = src[1];
  uint32_t wv[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
  uint32_t W[3] = {0, 0, 0};
#pragma unroll
  for (int kp = 0; kp < 30; ++kp) {
    const uint32_t c = (wv[kp >> 2] >> (8 * (kp & 3))) & 0x7;
    const int pi = kp >> 1, e = kp & 1;
    W[pi / 5] |= c << (16 * e + 3 * (pi % 5));
  }
#pragma unroll
  for (int e = 0; e < 2; ++e) {
    const uint32_t c = (wv[7] >> (8 * (2 + e))) & 0x7;  // codes 30 (e = 0) and 31 (e = 1)
#pragma unroll
    for (int bb = 0; bb < 3; ++bb) W[bb] |= ((c >> bb) & 1u) << (15 + 16 * e);
  }
  out[3 * i + 0] = W[0];
  out[3 * i + 1] = W[1];
  out[3 * i + 2] = W[2];
}

// L8: one thread per output word (4 codes).
__global__ void k_pack8(const uint8_t* __restrict__ codes, int64_t nwords, int kg, int64_t k, uint32_t* __restrict__ out) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nwords) return;
  const int64_t unit = i / (16 * 32);
  const int rr = (int)((i / 32) % 16), wi = (int)(i % 32);
  out[i] = *reinterpret_cast<const uint32_t*>(codes + src_row_col(unit, rr, kg, k, 4 * wi));
}

// meta[(t*kg + g)*16 + rr] = scale[r][g] | zero[r][g] << 16
__global__ void k_meta(const __half* __restrict__ s, const __half* __restrict__ z, int64_t n, int kg,
                       uint32_t* __restrict__ meta) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n * kg) return;
  const int64_t unit = i / 16;
  const int rr = (int)(i % 16);
  const int64_t t = unit / kg, g = unit % kg, r = t * 16 + rr;
  uint32_t sv = __half_as_ushort(s[r * kg + g]), zv = __half_as_ushort(z[r * kg + g]);
  meta[i] = sv | (zv << 16);
}

inline unsigned blocks_for(int64_t n, int t) { return (unsigned)((n + t - 1) / t); }

}  // namespace

template <int G>
void launch_quantize_g(dim3 grid, dim3 block, cudaStream_t s, const __half* w, int64_t n, int64_t k, int bits,
                       uint8_t* codes, __half* scales, __half* zeros, int mode, uint64_t seed, int* status) {
  switch (mode) {
    case 0: k_quantize<G, 0><<<grid, block, 0, s>>>(w, n, k, bits, codes, scales, zeros, seed, status); break;
    case 1: k_quantize<G, 1><<<grid, block, 0, s>>>(w, n, k, bits, codes, scales, zeros, seed, status); break;
    case 2: k_quantize<G, 2><<<grid, block, 0, s>>>(w, n, k, bits, codes, scales, zeros, seed, status); break;
    default: k_quantize<G, 3><<<grid, block, 0, s>>>(w, n, k, bits, codes, scales, zeros, seed, status); break;
  }
}

cudaError_t launch_quantize(const __half* w, int64_t n, int64_t k, int bits, int group, uint8_t* codes,
                            __half* scales, __half* zeros, int mode, uint64_t seed, int* status, cudaStream_t s) {
  const int64_t groups = n * (k / group);
  dim3 grid(blocks_for(groups, 8)), block(256);
  auto t = prof_begin(KC_QUANT, (double)n * k * 3 + groups * 4.0, 0, s);
  switch (group) {
    case 128: launch_quantize_g<128>(grid, block, s, w, n, k, bits, codes, scales, zeros, mode, seed, status); break;
    case 64: launch_quantize_g<64>(grid, block, s, w, n, k, bits, codes, scales, zeros, mode, seed, status); break;
    default: launch_quantize_g<32>(grid, block, s, w, n, k, bits, codes, scales, zeros, mode, seed, status); break;
  }
  prof_end(t, s);
  count_launch();
  return cudaGetLastError();
}

cudaError_t launch_pack(const uint8_t* codes, const __half* scales, const __half* zeros, int64_t n, int64_t k,
                        int bits, int group, void* packed, uint32_t* meta, cudaStream_t s) {
  (void)group;  // validated == 128
  const int kg = (int)(k / 128);
  auto t = prof_begin(KC_QUANT, (double)n * k * (1.0 + bits / 8.0), 0, s);
  if (bits == 4) {
    int64_t nw = n * k / 8;
    k_pack4<<<blocks_for(nw, 256), 256, 0, s>>>(codes, nw, kg, k, (uint32_t*)packed);
  } else if (bits == 3) {
    int64_t nb = n * k / 32;
    k_pack3<<<blocks_for(nb, 256), 256, 0, s>>>(codes, nb, kg, k, (uint32_t*)packed);
  } else {
    int64_t nw = n * k / 4;
    k_pack8<<<blocks_for(nw, 256), 256, 0, s>>>(codes, nw, kg, k, (uint32_t*)packed);
  }
  k_meta<<<blocks_for(n * kg, 256), 256, 0, s>>>(scales, zeros, n, kg, meta);
  prof_end(t, s);
  count_launch(2);
  return cudaGetLastError();
}

}  // namespace sq
