// K2 — decode dequant-GEMV (P:57 decode phase; "predominantly memory-bound",
// P:106; decode arithmetic intensity 43-48 on V100).
//
// y[m, n] = epi( sum_k x[m, k] * (s[n,g] * c[n,k] + z[n,g]) ),  m <= 32.
//
// Design (K2):
//  * Work unit = 16 output rows x one group (128 k).  The U units are flattened
//    row-tile-major / group-minor and split evenly over one 16-warp CTA per SM
//    (and evenly over the CTA's warps): every SM streams the same number of
//    bytes whatever the shape.
//  * A lane streams 32 consecutive codes of two rows (g, g+8) per unit with
//    128-bit loads (INT4 2x16 B, INT8 2x32 B, INT3 2x12 B) from a D-deep
//    register ring, plus the group metadata; the activation fragment comes
//    from L1 (re-read by all warps), its group sums from shared memory.
//  * Unpack in registers with the fp16 "magic number" trick: one LOP3 (PRMT
//    for INT8) turns a pair of codes into half2(off + c) exactly (off = 1024,
//    or 64 for the second nibble of each byte in L4) — no per-weight multiply.
//  * Dot products on mma.sync.m16n8k16 with fp32 accumulation (16 weight rows
//    = A operand, up to 8 tokens per n8 tile = B operand).  Per group:
//       sum_k x (off_k + c_k) = sum_k x c_k + xoff   =>
//       y += s * (D - xoff) + z * xs,   xs = sum x,  xoff = sum off_k x
//    with (xs, xoff) from sq_xsum (per-group factorised scale/zero).
//  * Split tiles are reduced in shared memory in fixed warp order; a tile that
//    straddles two CTAs is finished by the last CTA (atomic counter, fixed CTA
//    order).  Deterministic; counters self-reset.
//
// K2s (below, k_gemv_s) is the default for quantized weights at m <= 8 (INT8 up to m = 16): the same
// unpack / mma.sync / factorised scale-zero on STRIPS of RT row tiles x one group, per-warp TMA rings,
// two 8-warp CTAs per SM, group sums on the tensor core.  K2 (k_gemv_q) remains for n not a multiple of
// 32 and for m in 9..32 off the tcgen05 kernel's shapes ("Which decode kernel").
#include <cstdlib>

#include "sq_common.cuh"

namespace sq {
namespace {

constexpr int kWarps = 16;  // one 512-thread CTA per SM
constexpr int kThreads = kWarps * 32;
constexpr int kRows = 16;   // rows per unit (mma M)
constexpr int kXsTok = 32;  // token slots per group in the xsum buffer

struct GemvP {
  const uint8_t* packed;
  const uint32_t* meta;
  const __half* bias;
  const __half* x;
  int ldx;
  int m;
  int n;
  int kg;              // groups per row (k / 128)
  const float2* xsum;  // [kg][32]
  void* y;
  int ldy;
  float* part;  // [CTAs][2][TOK][16] cross-CTA partials
  int* cnt;     // [n / 16]
  int U;        // units
  int W;        // CTAs
};

template <int BITS>
struct Cfg;
template <>
struct Cfg<3> { static constexpr int LU = 3; static constexpr int GB = 48; static constexpr int D = 4; };
template <>
struct Cfg<4> { static constexpr int LU = 4; static constexpr int GB = 64; static constexpr int D = 4; };
template <>
struct Cfg<8> { static constexpr int LU = 8; static constexpr int GB = 128; static constexpr int D = 2; };
template <>
struct Cfg<16> { static constexpr int LU = 16; static constexpr int GB = 256; static constexpr int D = 1; };

// bytes of one row's 32 codes held by a lane (k in [32q, 32q+32) of the group)
template <int BITS>
constexpr int lane_bytes() { return 32 * BITS / 8; }

// this lane's 32 consecutive codes of one row of the current group; p already points at them
template <int BITS>
__device__ __forceinline__ void load_codes(const uint8_t* __restrict__ p, uint32_t* c) {
  if constexpr (BITS == 4) {
    uint4 v = ldg_nc_v4(p);
    c[0] = v.x; c[1] = v.y; c[2] = v.z; c[3] = v.w;
  } else if constexpr (BITS == 8) {
    uint4 v0 = ldg_nc_v4(p), v1 = ldg_nc_v4(p + 16);
    c[0] = v0.x; c[1] = v0.y; c[2] = v0.z; c[3] = v0.w;
    c[4] = v1.x; c[5] = v1.y; c[6] = v1.z; c[7] = v1.w;
  } else if constexpr (BITS == 3) {
    c[0] = ldg_nc_u32(p);
    c[1] = ldg_nc_u32(p + 4);
    c[2] = ldg_nc_u32(p + 8);
  } else {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      uint4 v = ldg_nc_v4(p + 16 * j);
      c[4 * j] = v.x; c[4 * j + 1] = v.y; c[4 * j + 2] = v.z; c[4 * j + 3] = v.w;
    }
  }
}

// Fragment registers of chunk t (k0 = 32q + 4t): lo = codes (k0, k0+1), hi = (k0+2, k0+3), as half2(off + c).
template <int BITS>
__device__ __forceinline__ void frag(const uint32_t* c, int t, uint32_t& lo, uint32_t& hi) {
  if constexpr (BITS == 4) {
    // L4: word w holds k = 8w..8w+7, even k in nibbles 0-3, odd k in nibbles 4-7.
    const uint32_t v = (t & 1) ? (c[t >> 1] >> 8) : c[t >> 1];
    lo = lop3_and_or(v, 0x000F000Fu, 0x64006400u);  // 1024 + c
    hi = lop3_and_or(v, 0x00F000F0u, 0x54005400u);  //   64 + c
  } else if constexpr (BITS == 8) {
    lo = prmt(c[t], 0x64646464u, 0x4140u);
    hi = prmt(c[t], 0x64646464u, 0x4342u);
  } else if constexpr (BITS == 3) {
    // L3: pair i < 15 at word i/5, bits 3(i%5) (+16 for the odd code); pair 15
    // in the spare bits 15 / 31 of the three words.  Each code is moved to mantissa bits 7..9 under
    // exponent 2^3: half2(8 + c), exact; the offset 8 (not 1024) keeps the per-group correction
    // D - xoff free of cancellation (ReLU inputs, measured).
    auto pairv = [&](int i) -> uint32_t {
      if (i < 15) {
        const uint32_t x = c[i / 5];
        const int sh = 7 - 3 * (i % 5);
        return lop3_and_or(sh >= 0 ? (x << sh) : (x >> (-sh)), 0x03800380u, 0x48004800u);
      }
      uint32_t u;
      asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(u) : "r"(0x00010001u), "r"(c[0] >> 15), "r"(c[1] >> 14));
      asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(u) : "r"(0x00030003u), "r"(u), "r"(c[2] >> 13));
      return lop3_and_or(u << 7, 0x03800380u, 0x48004800u);
    };
    lo = pairv(2 * t);
    hi = pairv(2 * t + 1);
  } else {
    lo = c[2 * t];
    hi = c[2 * t + 1];
  }
}

// K2s's INT3 fragments: each 3-bit field read in place under its own magic exponent, one LOP3 per
// code pair (fields at bits 0 / 3 / 6 of a 16-bit half -> 1024 / 128 / 16 + c; fields 9 / 12 via one
// shift per word -> 1024 / 128 + c; pair 15 from the spare bits -> 1024 + c), as K2c's dequant does.
// The per-position offsets are removed by the group correction xoff = sum off_k x_k, which K2s
// computes on the tensor core with the same fragment positions (k3_magic as the A operand).
__device__ __forceinline__ constexpr uint32_t k3_magic(int i) {
  return i == 15 ? 0x64006400u : ((i % 5) % 3 == 0 ? 0x64006400u : ((i % 5) % 3 == 1 ? 0x58005800u : 0x4C004C00u));
}
__device__ __forceinline__ constexpr uint32_t k3_mask(int i) {
  return i == 15 ? 0x00070007u : ((i % 5) % 3 == 0 ? 0x00070007u : ((i % 5) % 3 == 1 ? 0x00380038u : 0x01C001C0u));
}
__device__ __forceinline__ void frag3m(const uint32_t* c, const uint32_t* c9, uint32_t p15, int t, uint32_t& lo,
                                       uint32_t& hi) {
  auto pairv = [&](int i) -> uint32_t {
    if (i == 15) return lop3_and_or(p15, 0x00070007u, 0x64006400u);
    const uint32_t x = (i % 5) < 3 ? c[i / 5] : c9[i / 5];
    return lop3_and_or(x, k3_mask(i), k3_magic(i));
  };
  lo = pairv(2 * t);
  hi = pairv(2 * t + 1);
}
__device__ __forceinline__ uint32_t k3_spare(const uint32_t* c) {
  uint32_t u;
  asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(u) : "r"(0x00010001u), "r"(c[0] >> 15), "r"(c[1] >> 14));
  asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(u) : "r"(0x00030003u), "r"(u), "r"(c[2] >> 13));
  return u;
}

// predicated 16-B load (no divergent branch): dst unchanged when !pred
__device__ __forceinline__ void ldg_v4_pred(uint32_t* d, const void* p, bool pred) {
  asm volatile(
      "{\n\t.reg .pred pp;\n\tsetp.ne.b32 pp, %5, 0;\n\t"
      "@pp ld.global.nc.v4.u32 {%0,%1,%2,%3}, [%4];\n\t}"
      : "+r"(d[0]), "+r"(d[1]), "+r"(d[2]), "+r"(d[3])
      : "l"(p), "r"((int)pred));
}

template <int TOK>
struct NT { static constexpr int v = TOK / 8; };  // token n8 tiles

template <int TOK, int EPI>
__device__ __forceinline__ void store_out(const GemvP& p, int tile, int g, int q, const float (&v)[NT<TOK>::v][4]) {
  const int r0 = tile * kRows + g, r1 = r0 + 8;
  float b0 = 0.f, b1 = 0.f;
  if (p.bias) { b0 = __half2float(p.bias[r0]); b1 = __half2float(p.bias[r1]); }
#pragma unroll
  for (int j = 0; j < NT<TOK>::v; ++j) {
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const int tok = 8 * j + 2 * q + e;
      if (tok >= p.m) continue;
      const float o0 = v[j][e] + b0, o1 = v[j][2 + e] + b1;
      if constexpr (EPI == SQ_EPI_F32_ACCUM) {
        float* yp = static_cast<float*>(p.y) + (int64_t)tok * p.ldy;
        yp[r0] += o0;
        yp[r1] += o1;
      } else {
        __half* yp = static_cast<__half*>(p.y) + (int64_t)tok * p.ldy;
        yp[r0] = __float2half_rn(apply_act<EPI>(o0));
        yp[r1] = __float2half_rn(apply_act<EPI>(o1));
      }
    }
  }
}

__device__ __forceinline__ int range_lo(int i, int total, int parts) {
  return (int)(((long long)i * total) / parts);
}

// CTA-level reduction of split tiles (fixed warp order), then cross-CTA fix-up: a tile that
// straddles two CTAs is finished by the last CTA to arrive (atomic counter), summing the CTA
// partials in fixed CTA order.  Deterministic; counters self-reset.
template <int TOK, int EPI>
__device__ __forceinline__ void reduce_tail(const GemvP& p, const float* part_s, int C0, int C1, int R, int warp,
                                            int lane, int g, int q) {
  constexpr int NJ = NT<TOK>::v;
  const int kg = p.kg;
  if (R <= 0) return;
  const int t_first = C0 / kg, t_last = (C1 - 1) / kg;
  for (int t = t_first + warp; t <= t_last; t += kWarps) {
    const int lo = t * kg > C0 ? t * kg : C0;
    const int hi = (t + 1) * kg < C1 ? (t + 1) * kg : C1;  // exclusive
    const int wa = (int)(((long long)(lo - C0 + 1) * kWarps - 1) / R);
    const int wb = (int)(((long long)(hi - C0) * kWarps - 1) / R);
    if (wa == wb && lo == t * kg && hi == (t + 1) * kg) continue;  // one warp stored it directly
    float v[NJ][4];
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int i = 0; i < 4; ++i) v[j][i] = 0.f;
    for (int wi = wa; wi <= wb; ++wi) {
      const int wlo = C0 + range_lo(wi, R, kWarps), whi = C0 + range_lo(wi + 1, R, kWarps);
      if (whi <= wlo) continue;  // empty warp range
      const int sl = (wlo < t * kg) ? 1 : 0;
      const float* qp = part_s + ((wi * 2 + sl) * TOK) * kRows;
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int tok = 8 * j + 2 * q + e;
          v[j][e] += qp[tok * kRows + g];
          v[j][2 + e] += qp[tok * kRows + g + 8];
        }
    }
    if (lo == t * kg && hi == (t + 1) * kg) {  // tile entirely inside this CTA
      store_out<TOK, EPI>(p, t, g, q, v);
      continue;
    }
    // straddles a CTA boundary: publish this CTA's partial, the last CTA reduces
    const int cslot = (C0 < t * kg) ? 1 : 0;
    float* gp = p.part + (((int64_t)blockIdx.x * 2 + cslot) * TOK) * kRows;
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int e = 0; e < 2; ++e) {
        const int tok = 8 * j + 2 * q + e;
        __stcg(gp + tok * kRows + g, v[j][e]);
        __stcg(gp + tok * kRows + g + 8, v[j][2 + e]);
      }
    __threadfence();
    __syncwarp();
    const int NC = gridDim.x;
    const int ca = (int)(((long long)(t * kg + 1) * NC - 1) / p.U);
    const int cb2 = (int)(((long long)((t + 1) * kg) * NC - 1) / p.U);
    int old = 0;
    if (lane == 0) old = atomicAdd(p.cnt + t, 1);
    old = __shfl_sync(0xffffffff, old, 0);
    if (old != cb2 - ca) continue;
    __threadfence();
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int i = 0; i < 4; ++i) v[j][i] = 0.f;
    for (int c = ca; c <= cb2; ++c) {
      const int sl = (range_lo(c, p.U, NC) < t * kg) ? 1 : 0;
      const float* qp = p.part + (((int64_t)c * 2 + sl) * TOK) * kRows;
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int e = 0; e < 2; ++e) {
          const int tok = 8 * j + 2 * q + e;
          v[j][e] += __ldcg(qp + tok * kRows + g);
          v[j][2 + e] += __ldcg(qp + tok * kRows + g + 8);
        }
    }
    store_out<TOK, EPI>(p, t, g, q, v);
    if (lane == 0) p.cnt[t] = 0;
  }
}

template <int BITS, int TOK, int EPI>
__global__ void __launch_bounds__(kThreads, 1) k_gemv(const GemvP p) {
  constexpr int LU = Cfg<BITS>::LU;
  constexpr int GB = Cfg<BITS>::GB;
  constexpr int D = Cfg<BITS>::D;
  constexpr int NJ = NT<TOK>::v;
  constexpr bool Q = BITS != 16;
  extern __shared__ float4 smem4[];
  float* part_s = reinterpret_cast<float*>(smem4);  // [16 warps][2][TOK][16]
  float2* xs_s = reinterpret_cast<float2*>(part_s + kWarps * 2 * TOK * kRows);  // [kg][32]

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
  const int kg = p.kg, m = p.m;
  const int C0 = range_lo(blockIdx.x, p.U, gridDim.x), C1 = range_lo(blockIdx.x + 1, p.U, gridDim.x);
  const int R = C1 - C0;
  const int u0 = C0 + range_lo(warp, R, kWarps), u1 = C0 + range_lo(warp + 1, R, kWarps);
  const int nunits = u1 - u0;
  const int head_tile = u0 / kg;
  const int grp0 = u0 - head_tile * kg;
  const int64_t pitch = (int64_t)kg * GB;

  // ---- fetch cursor: codes of rows g, g+8 and their meta, D units ahead.
  // Quantized weights use placement T16: unit u is 16 x GB contiguous bytes at u * 16 * GB,
  // row r of the unit at r * GB, so the stream is one pointer bumped by a constant.
  constexpr int UB = 16 * GB;
  const uint8_t* fcp;
  const uint32_t* fmp = nullptr;
  int fgrp = grp0;
  const int64_t cp_wrap = 15 * pitch;  // (fp16 only) end of row g -> start of row g+16
  if constexpr (Q) {
    fcp = p.packed + (int64_t)u0 * UB + g * GB + q * lane_bytes<BITS>();
    fmp = p.meta + (int64_t)u0 * 16 + g;
  } else {
    fcp = p.packed + ((int64_t)head_tile * kRows + g) * pitch + (int64_t)grp0 * GB + q * 64;
  }
  uint32_t cb[D][2][LU];
  uint32_t mb[D][2];
  auto issue = [&](int slot) {
    if constexpr (Q) {
      load_codes<BITS>(fcp, cb[slot][0]);
      load_codes<BITS>(fcp + 8 * GB, cb[slot][1]);
      mb[slot][0] = ldg_nc_u32(fmp);
      mb[slot][1] = ldg_nc_u32(fmp + 8);
      fcp += UB;
      fmp += 16;
    } else {
      load_codes<BITS>(fcp, cb[slot][0]);
      load_codes<BITS>(fcp + 8 * pitch, cb[slot][1]);
      fcp += GB;
      if (++fgrp == kg) { fgrp = 0; fcp += cp_wrap; }
    }
  };
#pragma unroll
  for (int j = 0; j < D; ++j)
    if (j < nunits) issue(j);
  // PDL: the weight fetches above are independent of the previous kernel; everything below is not
  pdl_trigger();
  pdl_wait();

  // ---- stage (xs, xoff) per (group, token) in shared memory (overlaps the weight loads):
  //      xs = sum x, xoff = sum off_k x  (off = 1024 INT8, 1024 / 64 for the two nibble slots of L4, 8 INT3)
  if constexpr (Q) {
    for (int i = threadIdx.x; i < kg * kXsTok; i += kThreads) {
      const float2 v = __ldg(p.xsum + i);
      const float xsv = v.x + v.y;
      const float xov = BITS == 4 ? fmaf(1024.f, v.x, 64.f * v.y) : (BITS == 3 ? 8.f * xsv : 1024.f * xsv);
      xs_s[i] = make_float2(xsv, xov);
    }
  }
  __syncthreads();

  // activation fragment pointers for token n8-tile j: row 8j + g (predicated off beyond m)
  const __half* xrow[NJ];
  bool xon[NJ];
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    xon[j] = (8 * j + g) < m;
    xrow[j] = p.x + (int64_t)(xon[j] ? 8 * j + g : 0) * p.ldx + q * 32;
  }

  // activation fragment (NJ == 1: persistent, lanes beyond m keep zeros under predicated loads)
  uint32_t xt1[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) xt1[i] = 0u;

  int tile = head_tile, grp = grp0;
  bool seg_from_start = (grp0 == 0);
  float acc[NJ][4];
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int i = 0; i < 4; ++i) acc[j][i] = 0.f;

  for (int base = 0; base < nunits; base += D) {
#pragma unroll
    for (int s = 0; s < D; ++s) {
      const int ui = base + s;
      if (ui >= nunits) break;
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        const __half* xp = xrow[j] + grp * 128;
        uint32_t xloc[16];
        uint32_t* xtj = NJ == 1 ? xt1 : xloc;
        if (NJ > 1) {
#pragma unroll
          for (int i = 0; i < 16; ++i) xloc[i] = 0u;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i) ldg_v4_pred(xtj + 4 * i, xp + 8 * i, xon[j]);
        if constexpr (!Q) {
#pragma unroll
          for (int t = 0; t < 8; ++t) {
            uint32_t a[4];
            frag<BITS>(cb[s][0], t, a[0], a[2]);
            frag<BITS>(cb[s][1], t, a[1], a[3]);
            mma_16816(acc[j], a, xtj[2 * t], xtj[2 * t + 1], acc[j]);
          }
        } else {
          float d0[4], d1[4];  // two independent HMMA chains (even / odd chunks)
          {
            uint32_t a[4], b[4];
            frag<BITS>(cb[s][0], 0, a[0], a[2]);
            frag<BITS>(cb[s][1], 0, a[1], a[3]);
            frag<BITS>(cb[s][0], 1, b[0], b[2]);
            frag<BITS>(cb[s][1], 1, b[1], b[3]);
            mma_16816_zc(d0, a, xtj[0], xtj[1]);
            mma_16816_zc(d1, b, xtj[2], xtj[3]);
          }
#pragma unroll
          for (int t = 2; t < 8; t += 2) {
            uint32_t a[4], b[4];
            frag<BITS>(cb[s][0], t, a[0], a[2]);
            frag<BITS>(cb[s][1], t, a[1], a[3]);
            frag<BITS>(cb[s][0], t + 1, b[0], b[2]);
            frag<BITS>(cb[s][1], t + 1, b[1], b[3]);
            mma_16816(d0, a, xtj[2 * t], xtj[2 * t + 1], d0);
            mma_16816(d1, b, xtj[2 * t + 2], xtj[2 * t + 3], d1);
          }
          const float d[4] = {d0[0] + d1[0], d0[1] + d1[1], d0[2] + d1[2], d0[3] + d1[3]};
          const float2 f0 = __half22float2(*reinterpret_cast<const __half2*>(&mb[s][0]));  // (s, z) row g
          const float2 f1 = __half22float2(*reinterpret_cast<const __half2*>(&mb[s][1]));  // row g+8
          const float4 xv = *reinterpret_cast<const float4*>(xs_s + grp * kXsTok + 8 * j + 2 * q);
          // y += s * (D - xoff) + z * xs   (tokens 2q: xv.x/xv.y, 2q+1: xv.z/xv.w)
          acc[j][0] = fmaf(-f0.x, xv.y, fmaf(f0.y, xv.x, fmaf(f0.x, d[0], acc[j][0])));
          acc[j][1] = fmaf(-f0.x, xv.w, fmaf(f0.y, xv.z, fmaf(f0.x, d[1], acc[j][1])));
          acc[j][2] = fmaf(-f1.x, xv.y, fmaf(f1.y, xv.x, fmaf(f1.x, d[2], acc[j][2])));
          acc[j][3] = fmaf(-f1.x, xv.w, fmaf(f1.y, xv.z, fmaf(f1.x, d[3], acc[j][3])));
        }
      }
      if (ui + D < nunits) issue(s);

      // ---- segment end: row tile finished or this warp's run finished
      const bool tile_end = (grp == kg - 1);
      if (tile_end || ui == nunits - 1) {
        if (seg_from_start && tile_end) {
          store_out<TOK, EPI>(p, tile, g, q, acc);
        } else {
          const int slot = (tile == head_tile) ? 0 : 1;  // head / tail tile of this warp
          float* pp = part_s + ((warp * 2 + slot) * TOK) * kRows;
#pragma unroll
          for (int j = 0; j < NJ; ++j)
#pragma unroll
            for (int e = 0; e < 2; ++e) {
              const int tok = 8 * j + 2 * q + e;
              pp[tok * kRows + g] = acc[j][e];
              pp[tok * kRows + g + 8] = acc[j][2 + e];
            }
        }
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int i = 0; i < 4; ++i) acc[j][i] = 0.f;
        seg_from_start = true;
      }
      if (++grp == kg) { grp = 0; ++tile; }
    }
  }
  __syncthreads();

  reduce_tail<TOK, EPI>(p, part_s, C0, C1, R, warp, lane, g, q);
}

// ---------------------------------------------------------------- K2 with a bulk-copy SMEM ring
// Quantized weights (placement T16): a warp's unit range is ONE contiguous byte range (and so is
// its meta), so each warp streams it with cp.async.bulk into its own S-slot shared-memory ring
// (CH units per slot, one mbarrier per slot, lane 0 issues): ~150 KB in flight per SM instead of
// the 4-unit register ring, decoupling HBM latency from the warps.  Unpack, mma.sync, the
// factorised scale/zero and the reductions are those of k_gemv.
template <int BITS, int TOK>
struct QRing {
  static constexpr int UB = 16 * Cfg<BITS>::GB;                   // codes bytes per unit
  static constexpr int UM = 64;                                   // meta bytes per unit
  static constexpr int PART = kWarps * 2 * TOK * kRows * 4;      // split-tile partials
  static constexpr int BARS = kWarps * 8 * 8;                     // <= 8 mbarriers per warp
  static constexpr int CH = BITS == 8 ? 2 : (BITS == 4 ? 3 : 4);  // units per slot (3.3-4.2 KB)
  static constexpr int SLOT = CH * (UB + UM);
  static constexpr int S0 = (227 * 1024 - PART - BARS - 128) / kWarps / SLOT;
  static constexpr int S = S0 > 8 ? 8 : S0;
  static constexpr int BYTES = PART + BARS + kWarps * S * SLOT;
  static_assert(S >= 2, "ring depth");
  static_assert(BYTES <= 227 * 1024, "shared memory budget");
};

// this lane's codes of one row of the unit in shared memory (p = row start + lane offset)
template <int BITS>
__device__ __forceinline__ void lds_codes(const uint8_t* p, uint32_t* c) {
  if constexpr (BITS == 4) {
    const uint4 v = *reinterpret_cast<const uint4*>(p);
    c[0] = v.x; c[1] = v.y; c[2] = v.z; c[3] = v.w;
  } else if constexpr (BITS == 8) {
    // k in [16q, 16q+16) and [64+16q, 64+16q+16): conflict-free 16-B phases
    const uint4 v0 = *reinterpret_cast<const uint4*>(p), v1 = *reinterpret_cast<const uint4*>(p + 64);
    c[0] = v0.x; c[1] = v0.y; c[2] = v0.z; c[3] = v0.w;
    c[4] = v1.x; c[5] = v1.y; c[6] = v1.z; c[7] = v1.w;
  } else {
    const uint32_t* w = reinterpret_cast<const uint32_t*>(p);
    c[0] = w[0]; c[1] = w[1]; c[2] = w[2];
  }
}

template <int BITS, int TOK, int EPI>
__global__ void __launch_bounds__(kThreads, 1) k_gemv_q(const GemvP p) {
  using RC = QRing<BITS, TOK>;
  constexpr int LU = Cfg<BITS>::LU;
  constexpr int GB = Cfg<BITS>::GB;
  constexpr int NJ = NT<TOK>::v;
  constexpr int CH = RC::CH, S = RC::S, UB = RC::UB, SLOT = RC::SLOT;
  extern __shared__ float4 smem4[];
  uint8_t* smem = reinterpret_cast<uint8_t*>(smem4);
  float* part_s = reinterpret_cast<float*>(smem);  // [16 warps][2][TOK][16]
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + RC::PART) + (threadIdx.x >> 5) * 8;

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
  const int kg = p.kg, m = p.m;
  const int C0 = range_lo(blockIdx.x, p.U, gridDim.x), C1 = range_lo(blockIdx.x + 1, p.U, gridDim.x);
  const int R = C1 - C0;
  const int u0 = C0 + range_lo(warp, R, kWarps), u1 = C0 + range_lo(warp + 1, R, kWarps);
  const int nunits = u1 - u0;
  const int head_tile = u0 / kg;
  const int grp0 = u0 - head_tile * kg;
  uint8_t* ring = smem + RC::PART + RC::BARS + warp * S * SLOT;

  // ---- the warp's own ring: lane 0 initialises its barriers and keeps S slots in flight
  const int nch = (nunits + CH - 1) / CH;
  auto issue = [&](int c) {
    const int slot = c % S;
    const int nu = nunits - c * CH < CH ? nunits - c * CH : CH;
    const int64_t u = (int64_t)u0 + (int64_t)c * CH;
    mbar_arrive_expect_tx(&bar[slot], (uint32_t)(nu * (UB + 64)));
    bulk_load(ring + slot * SLOT, p.packed + u * UB, (uint32_t)(nu * UB), &bar[slot]);
    bulk_load(ring + slot * SLOT + CH * UB, p.meta + u * 16, (uint32_t)(nu * 64), &bar[slot]);
  };
  if (lane == 0) {
    for (int i = 0; i < S; ++i) mbar_init(&bar[i], 1);
    fence_barrier_init();
    for (int c = 0; c < S && c < nch; ++c) issue(c);
  }
  __syncwarp();
  // PDL: the weight fetches above are independent of the previous kernel; everything below is not
  pdl_trigger();
  pdl_wait();

  // activation fragment pointers for token n8-tile j: row 8j + g (predicated off beyond m); the
  // lane's k set matches its codes: [32q, 32q+32) (INT3/INT4) or [16q,16q+16) u [64+16q, 80+16q) (INT8)
  const int xq = BITS == 8 ? q * 16 : q * 32;
  const __half* xrow[NJ];
  bool xon[NJ];
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    xon[j] = (8 * j + g) < m;
    xrow[j] = p.x + (int64_t)(xon[j] ? 8 * j + g : 0) * p.ldx + xq;
  }
  uint32_t xt1[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) xt1[i] = 0u;

  int tile = head_tile, grp = grp0;
  bool seg_from_start = (grp0 == 0);
  float acc[NJ][4];
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int i = 0; i < 4; ++i) acc[j][i] = 0.f;
  const int lane_off = BITS == 8 ? q * 16 : q * lane_bytes<BITS>();

  // one unit: codes of rows g / g+8 from the slot, activation fragment from L1, 8 HMMAs, the
  // per-group factorised scale / zero, segment end (row tile finished or end of the warp's run)
  auto unit = [&](const uint8_t* cs, const uint32_t* ms, int s, int ui) {
    uint32_t cw0[LU], cw1[LU];
    lds_codes<BITS>(cs + s * UB + g * GB + lane_off, cw0);
    lds_codes<BITS>(cs + s * UB + (g + 8) * GB + lane_off, cw1);
    const uint32_t mr0 = ms[s * 16 + g], mr1 = ms[s * 16 + g + 8];
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      const uint4* xp = reinterpret_cast<const uint4*>(xrow[j] + grp * 128);
      uint32_t xloc[16];
      uint32_t* xtj = NJ == 1 ? xt1 : xloc;
      if (xon[j]) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int xo = BITS == 8 ? (i < 2 ? i : 8 + (i - 2)) : i;  // 16-B units
          const uint4 v = __ldg(xp + xo);
          xtj[4 * i] = v.x; xtj[4 * i + 1] = v.y; xtj[4 * i + 2] = v.z; xtj[4 * i + 3] = v.w;
        }
      } else if (NJ > 1) {
#pragma unroll
        for (int i = 0; i < 16; ++i) xloc[i] = 0u;
      }
      const float4 xsv = __ldg(reinterpret_cast<const float4*>(p.xsum + grp * kXsTok + 8 * j + 2 * q));
      float d0[4], d1[4];  // two independent HMMA chains (even / odd chunks)
      {
        uint32_t a[4], b[4];
        frag<BITS>(cw0, 0, a[0], a[2]);
        frag<BITS>(cw1, 0, a[1], a[3]);
        frag<BITS>(cw0, 1, b[0], b[2]);
        frag<BITS>(cw1, 1, b[1], b[3]);
        mma_16816_zc(d0, a, xtj[0], xtj[1]);
        mma_16816_zc(d1, b, xtj[2], xtj[3]);
      }
#pragma unroll
      for (int t = 2; t < 8; t += 2) {
        uint32_t a[4], b[4];
        frag<BITS>(cw0, t, a[0], a[2]);
        frag<BITS>(cw1, t, a[1], a[3]);
        frag<BITS>(cw0, t + 1, b[0], b[2]);
        frag<BITS>(cw1, t + 1, b[1], b[3]);
        mma_16816(d0, a, xtj[2 * t], xtj[2 * t + 1], d0);
        mma_16816(d1, b, xtj[2 * t + 2], xtj[2 * t + 3], d1);
      }
      const float d[4] = {d0[0] + d1[0], d0[1] + d1[1], d0[2] + d1[2], d0[3] + d1[3]};
      const float2 f0 = __half22float2(*reinterpret_cast<const __half2*>(&mr0));  // (s, z) row g
      const float2 f1 = __half22float2(*reinterpret_cast<const __half2*>(&mr1));  // row g+8
      // (xs, xoff) of tokens 2q, 2q+1: xs = sum x, xoff = sum off_k x
      const float xs0 = xsv.x + xsv.y, xs1 = xsv.z + xsv.w;
      const float xo0 = BITS == 4 ? fmaf(1024.f, xsv.x, 64.f * xsv.y) : (BITS == 3 ? 8.f * xs0 : 1024.f * xs0);
      const float xo1 = BITS == 4 ? fmaf(1024.f, xsv.z, 64.f * xsv.w) : (BITS == 3 ? 8.f * xs1 : 1024.f * xs1);
      // y += s * (D - xoff) + z * xs
      acc[j][0] = fmaf(-f0.x, xo0, fmaf(f0.y, xs0, fmaf(f0.x, d[0], acc[j][0])));
      acc[j][1] = fmaf(-f0.x, xo1, fmaf(f0.y, xs1, fmaf(f0.x, d[1], acc[j][1])));
      acc[j][2] = fmaf(-f1.x, xo0, fmaf(f1.y, xs0, fmaf(f1.x, d[2], acc[j][2])));
      acc[j][3] = fmaf(-f1.x, xo1, fmaf(f1.y, xs1, fmaf(f1.x, d[3], acc[j][3])));
    }
    const bool tile_end = (grp == kg - 1);
    if (tile_end || ui == nunits - 1) {
      if (seg_from_start && tile_end) {
        store_out<TOK, EPI>(p, tile, g, q, acc);
      } else {
        const int sl = (tile == head_tile) ? 0 : 1;  // head / tail tile of this warp
        float* pp = part_s + ((warp * 2 + sl) * TOK) * kRows;
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int e = 0; e < 2; ++e) {
            const int tok = 8 * j + 2 * q + e;
            pp[tok * kRows + g] = acc[j][e];
            pp[tok * kRows + g + 8] = acc[j][2 + e];
          }
      }
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int i = 0; i < 4; ++i) acc[j][i] = 0.f;
      seg_from_start = true;
    }
    if (++grp == kg) { grp = 0; ++tile; }
  };

  for (int c = 0; c < nch; ++c) {
    const int slot = c % S;
    mbar_wait(&bar[slot], (uint32_t)((c / S) & 1));
    const uint8_t* cs = ring + slot * SLOT;
    const uint32_t* ms = reinterpret_cast<const uint32_t*>(cs + CH * UB);
    if (c * CH + CH <= nunits) {  // full slot (warp-uniform): straight-line body
#pragma unroll
      for (int s = 0; s < CH; ++s) unit(cs, ms, s, c * CH + s);
    } else {
      for (int s = 0; s < nunits - c * CH; ++s) unit(cs, ms, s, c * CH + s);
    }
    __syncwarp();  // every lane's reads of this slot are done (their values fed the MMAs)
    if (lane == 0 && c + S < nch) issue(c + S);
  }
  __syncthreads();
  reduce_tail<TOK, EPI>(p, part_s, C0, C1, R, warp, lane, g, q);
}

// ---------------------------------------------------------------- K2s: strips of RT row tiles (m <= 8;
// INT8 m <= 16 with two token tiles)
// A work item is (strip, group): RT consecutive 16-row tiles x one 128-k group.  The activation
// fragment of a group is loaded once per RT units (K2 re-loads it for every unit), its group sums
// (xs, xoff) are read from the caller's sq_xsum output or computed on the tensor core (HMMA with
// ones / offset A fragments), and the RT units' HMMA chains are independent (ILP).  Items are
// flattened strip-major / group-minor and split evenly over the grid's warps, as K2's units are;
// each warp streams its items into its own S-slot ring, lane 0 issuing one 3-D TMA box of the
// strip's RT units (T16: [tile][group lines][256 B]) and one 2-D box of their meta per item.
// Unpack, mma.sync and the factorised per-group scale / zero are K2's.  Deterministic: the split
// strips are reduced in fixed warp order in shared memory (in the warps' idle rings) and across
// CTAs by the last CTA to arrive, in fixed CTA order.
// K2s CTA: 8 warps, two CTAs per SM (measured against one 16-warp CTA: equal or up to 7 % faster on
// OPT-13B / OPT-66B shapes; tools/gemv_rot.py --graph on variant builds)
constexpr int kSWarps = 8;
constexpr int kSThreads = kSWarps * 32;
constexpr int kSCtasPerSm = 2;
// per-CTA shared memory budget: two-slot rings (a third slot measured 0.9 us slower per launch on
// 20480 x 5120: more bytes requested at kernel start delay the first items)
constexpr int kSSmemKB = 76;

template <int BITS, int RT_>
struct SRing {
  static constexpr int RT = RT_;                                  // tiles per strip
  static constexpr int UB = 16 * Cfg<BITS>::GB;                   // codes bytes per unit
  static constexpr int SLOT = RT * (UB + 64);                     // one item: RT units + their meta
  static constexpr int BAR_BYTES = kSWarps * 8 * 8;                // <= 8 mbarriers per warp
  static constexpr int S0 = (kSSmemKB * 1024 - 128 - BAR_BYTES) / kSWarps / SLOT;
  static constexpr int S = S0 > 8 ? 8 : S0;
  static constexpr int BYTES = 128 + BAR_BYTES + kSWarps * S * SLOT;  // + alignment slack
  static_assert(S >= 2 && BYTES <= 227 * 1024 && SLOT % 128 == 0, "K2s shared memory");
};

template <int EPI, int NJ>
__device__ __forceinline__ void store_strip_tile(const GemvP& p, int tile, int g, int q, const float (&v)[NJ][4]) {
  if (tile < p.n / kRows) store_out<8 * NJ, EPI>(p, tile, g, q, v);
}

// K2's reduce_tail for strips: in-CTA partials live in each warp's ring (stride WS bytes) as
// [2][32 lanes][RT][NJ] float4, the cross-CTA partials in p.part [CTAs][2][32 lanes][RT][NJ] float4.
template <int EPI, int RT, int NJ, int WS>
__device__ __forceinline__ void reduce_tail_s(const GemvP& p, const uint8_t* part_base, int C0, int C1, int R,
                                              int warp, int lane, int g, int q) {
  constexpr int PL = RT * NJ;  // float4 per lane per partial
  const int kg = p.kg;
  if (R <= 0) return;
  const int t_first = C0 / kg, t_last = (C1 - 1) / kg;
  for (int t = t_first + warp; t <= t_last; t += kSWarps) {
    const int lo = t * kg > C0 ? t * kg : C0;
    const int hi = (t + 1) * kg < C1 ? (t + 1) * kg : C1;  // exclusive
    const int wa = (int)(((long long)(lo - C0 + 1) * kSWarps - 1) / R);
    const int wb = (int)(((long long)(hi - C0) * kSWarps - 1) / R);
    const bool whole = lo == t * kg && hi == (t + 1) * kg;
    if (wa == wb && whole) continue;  // one warp stored it directly
    float v[RT][NJ][4];
#pragma unroll
    for (int r = 0; r < RT; ++r)
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int i = 0; i < 4; ++i) v[r][j][i] = 0.f;
    for (int wi = wa; wi <= wb; ++wi) {
      const int wlo = C0 + range_lo(wi, R, kSWarps), whi = C0 + range_lo(wi + 1, R, kSWarps);
      if (whi <= wlo) continue;  // empty warp range
      const int sl = (wlo < t * kg) ? 1 : 0;
      const float4* qp = reinterpret_cast<const float4*>(part_base + (size_t)wi * WS) + (sl * 32 + lane) * PL;
#pragma unroll
      for (int r = 0; r < RT; ++r)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          const float4 u = qp[r * NJ + j];
          v[r][j][0] += u.x; v[r][j][1] += u.y; v[r][j][2] += u.z; v[r][j][3] += u.w;
        }
    }
    if (whole) {
#pragma unroll
      for (int r = 0; r < RT; ++r) store_strip_tile<EPI, NJ>(p, t * RT + r, g, q, v[r]);
      continue;
    }
    // straddles a CTA boundary: publish this CTA's partial, the last CTA to arrive reduces
    const int cslot = (C0 < t * kg) ? 1 : 0;
    float4* gp = reinterpret_cast<float4*>(p.part) + (((int64_t)blockIdx.x * 2 + cslot) * 32 + lane) * PL;
#pragma unroll
    for (int r = 0; r < RT; ++r)
#pragma unroll
      for (int j = 0; j < NJ; ++j) __stcg(gp + r * NJ + j, make_float4(v[r][j][0], v[r][j][1], v[r][j][2], v[r][j][3]));
    const int NC = gridDim.x;
    const int ca = (int)(((long long)(t * kg + 1) * NC - 1) / p.U);
    const int cb2 = (int)(((long long)((t + 1) * kg) * NC - 1) / p.U);
    int old = 0;
    // release (orders this warp's partial stores, __syncwarp + cumulativity) / acquire (the last CTA's
    // reads below) in one atomic: no __threadfence on either side (-0.2-0.7 us per launch)
    __syncwarp();
    if (lane == 0) asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], 1;" : "=r"(old) : "l"(p.cnt + t) : "memory");
    old = __shfl_sync(0xffffffff, old, 0);
    if (old != cb2 - ca) continue;
#pragma unroll
    for (int r = 0; r < RT; ++r)
#pragma unroll
      for (int j = 0; j < NJ; ++j)
#pragma unroll
        for (int i = 0; i < 4; ++i) v[r][j][i] = 0.f;
    for (int c = ca; c <= cb2; ++c) {
      const int sl = (range_lo(c, p.U, NC) < t * kg) ? 1 : 0;
      const float4* qp = reinterpret_cast<const float4*>(p.part) + (((int64_t)c * 2 + sl) * 32 + lane) * PL;
#pragma unroll
      for (int r = 0; r < RT; ++r)
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          const float4 u = __ldcg(qp + r * NJ + j);
          v[r][j][0] += u.x; v[r][j][1] += u.y; v[r][j][2] += u.z; v[r][j][3] += u.w;
        }
    }
#pragma unroll
    for (int r = 0; r < RT; ++r) store_strip_tile<EPI, NJ>(p, t * RT + r, g, q, v[r]);
    if (lane == 0) p.cnt[t] = 0;
  }
}

// NJ = token n8 tiles: 1 (m <= 8) or 2 (m <= 16, RT = 2)
template <int BITS, int RT_, int EPI, bool XS, int NJ>
__global__ void __launch_bounds__(kSThreads, kSCtasPerSm)
    k_gemv_s(const __grid_constant__ CUtensorMap tm_w, const __grid_constant__ CUtensorMap tm_m, const GemvP p) {
  using RC = SRing<BITS, RT_>;
  constexpr int LU = Cfg<BITS>::LU, GB = Cfg<BITS>::GB;
  constexpr int RT = RC::RT, UB = RC::UB, SLOT = RC::SLOT, S = RC::S, PL = RT * NJ;
  static_assert(S * SLOT >= 2 * 32 * PL * 16, "partials fit in the ring");
  extern __shared__ float4 smem4[];
  uint8_t* smem = reinterpret_cast<uint8_t*>(smem4);
  smem += (128 - (smem_u32(smem) & 127)) & 127;  // TMA destinations: 128-B aligned slots
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31, g = lane >> 2, q = lane & 3;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem) + warp * 8;
  uint8_t* ring = smem + RC::BAR_BYTES + warp * S * SLOT;
  const int kg = p.kg, m = p.m;
  const int C0 = range_lo(blockIdx.x, p.U, gridDim.x), C1 = range_lo(blockIdx.x + 1, p.U, gridDim.x);
  const int R = C1 - C0;
  const int u0 = C0 + range_lo(warp, R, kSWarps), u1 = C0 + range_lo(warp + 1, R, kSWarps);
  const int nit = u1 - u0;
  const int head_set = u0 / kg;
  const int grp0 = u0 - head_set * kg;

  // ---- the warp's ring: item c -> slot c % S, filled by lane 0 with two TMA boxes: the strip's RT
  // units of group fgrp ([RT][UB] codes, 3-D map of 256-B lines) and their meta ([RT][16] u32)
  int fset = head_set, fgrp = grp0;
  auto issue = [&](int c) {
    const int slot = c % S;
    mbar_arrive_expect_tx(&bar[slot], (uint32_t)SLOT);
    tma_load_3d(ring + slot * SLOT, &tm_w, &bar[slot], 0, fgrp * (UB / 256), fset * RT);
    tma_load_2d(ring + slot * SLOT + RT * UB, &tm_m, &bar[slot], fgrp * 16, fset * RT);
    if (++fgrp == kg) { fgrp = 0; ++fset; }
  };
  if (lane == 0) {
    if (warp == 0) { prefetch_tmap(&tm_w); prefetch_tmap(&tm_m); }
    for (int i = 0; i < S; ++i) mbar_init(&bar[i], 1);
    fence_barrier_init();
    for (int c = 0; c < S && c < nit; ++c) issue(c);
  }
  __syncwarp();
  // PDL: the weight fetches above are independent of the previous kernel; everything below is not
  pdl_trigger();
  pdl_wait();

  // the lane's activation rows (tokens 8j + g) and k set, matching its codes (see k_gemv_q)
  bool xon[NJ];
  const __half* xrow[NJ];
#pragma unroll
  for (int j = 0; j < NJ; ++j) {
    xon[j] = 8 * j + g < m;
    xrow[j] = p.x + (int64_t)(xon[j] ? 8 * j + g : 0) * p.ldx + (BITS == 8 ? q * 16 : q * 32);
  }
  const int lane_off = BITS == 8 ? q * 16 : q * lane_bytes<BITS>();
  uint32_t xt[NJ][16];
#pragma unroll
  for (int j = 0; j < NJ; ++j)
#pragma unroll
    for (int i = 0; i < 16; ++i) xt[j][i] = 0u;

  int set = head_set, grp = grp0;
  bool seg_from_start = (grp0 == 0);
  float acc[RT][NJ][4], hacc[RT][NJ][4];
#pragma unroll
  for (int r = 0; r < RT; ++r)
#pragma unroll
    for (int j = 0; j < NJ; ++j)
#pragma unroll
      for (int i = 0; i < 4; ++i) { acc[r][j][i] = 0.f; hacc[r][j][i] = 0.f; }
  bool has_head = false;

  for (int c = 0; c < nit; ++c) {
    const int slot = c % S;
    // activation fragments + group sums of this group (independent of the slot)
    float xs0[NJ], xs1[NJ], xo0[NJ], xo1[NJ];
#pragma unroll
    for (int j = 0; j < NJ; ++j) {
      if (xon[j]) {
        const uint4* xp = reinterpret_cast<const uint4*>(xrow[j] + grp * 128);
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int xo = BITS == 8 ? (i < 2 ? i : 8 + (i - 2)) : i;  // 16-B units
          const uint4 v = __ldg(xp + xo);
          xt[j][4 * i] = v.x; xt[j][4 * i + 1] = v.y; xt[j][4 * i + 2] = v.z; xt[j][4 * i + 3] = v.w;
        }
      }
      if constexpr (XS) {
        // the group sums on the tensor core, both from ONE 8-HMMA chain: A rows 0-7 are ones (D rows
        // 0-7 = xs = sum x), rows 8-15 the unpack offsets at each fragment position (D rows 8-15 =
        // xoff = sum off_k x; INT4: lo codes 1024 at k 2q.., hi codes 64 at k 2q+8..) -- the same
        // positions as the codes, so D - xoff cancels the offsets by construction
        constexpr uint32_t H1 = 0x3C003C00u, H1024 = 0x64006400u, H64 = 0x54005400u;
        float ds[4];
#pragma unroll
        for (int t = 0; t < 8; ++t) {
          uint32_t ao[4];
          ao[0] = H1;
          ao[2] = H1;
          if constexpr (BITS == 4) { ao[1] = H1024; ao[3] = H64; }
          else if constexpr (BITS == 3) { ao[1] = k3_magic(2 * t); ao[3] = k3_magic(2 * t + 1); }
          else { ao[1] = H1024; ao[3] = H1024; }
          if (t == 0) mma_16816_zc(ds, ao, xt[j][0], xt[j][1]);
          else mma_16816(ds, ao, xt[j][2 * t], xt[j][2 * t + 1], ds);
        }
        xs0[j] = ds[0];
        xs1[j] = ds[1];
        xo0[j] = ds[2];
        xo1[j] = ds[3];
      } else {
        const float4 xsv = __ldg(reinterpret_cast<const float4*>(p.xsum + grp * kXsTok + 8 * j + 2 * q));
        xs0[j] = xsv.x + xsv.y;
        xs1[j] = xsv.z + xsv.w;
        xo0[j] = BITS == 4 ? fmaf(1024.f, xsv.x, 64.f * xsv.y) : (BITS == 3 ? 8.f * xs0[j] : 1024.f * xs0[j]);
        xo1[j] = BITS == 4 ? fmaf(1024.f, xsv.z, 64.f * xsv.w) : (BITS == 3 ? 8.f * xs1[j] : 1024.f * xs1[j]);
      }
    }
    mbar_wait(&bar[slot], (uint32_t)((c / S) & 1));
    const uint8_t* cs = ring + slot * SLOT;
    const uint32_t* ms = reinterpret_cast<const uint32_t*>(cs + RT * UB);
#pragma unroll
    for (int r = 0; r < RT; ++r) {
      uint32_t cw0[LU], cw1[LU];
      lds_codes<BITS>(cs + r * UB + g * GB + lane_off, cw0);
      lds_codes<BITS>(cs + r * UB + (g + 8) * GB + lane_off, cw1);
      const uint32_t mr0 = ms[r * 16 + g], mr1 = ms[r * 16 + g + 8];
      float d[NJ][4];
      uint32_t c90[3], c91[3], s150 = 0, s151 = 0;
      if constexpr (BITS == 3) {
#pragma unroll
        for (int w = 0; w < 3; ++w) { c90[w] = cw0[w] >> 9; c91[w] = cw1[w] >> 9; }
        s150 = k3_spare(cw0);
        s151 = k3_spare(cw1);
      }
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        uint32_t a[4];
        if constexpr (BITS == 3) {
          frag3m(cw0, c90, s150, t, a[0], a[2]);
          frag3m(cw1, c91, s151, t, a[1], a[3]);
        } else {
          frag<BITS>(cw0, t, a[0], a[2]);
          frag<BITS>(cw1, t, a[1], a[3]);
        }
#pragma unroll
        for (int j = 0; j < NJ; ++j) {
          if (t == 0) mma_16816_zc(d[j], a, xt[j][0], xt[j][1]);
          else mma_16816(d[j], a, xt[j][2 * t], xt[j][2 * t + 1], d[j]);
        }
      }
      const float2 f0 = __half22float2(*reinterpret_cast<const __half2*>(&mr0));  // (s, z) row g
      const float2 f1 = __half22float2(*reinterpret_cast<const __half2*>(&mr1));  // row g+8
      // y += s * (D - xoff) + z * xs
#pragma unroll
      for (int j = 0; j < NJ; ++j) {
        acc[r][j][0] = fmaf(-f0.x, xo0[j], fmaf(f0.y, xs0[j], fmaf(f0.x, d[j][0], acc[r][j][0])));
        acc[r][j][1] = fmaf(-f0.x, xo1[j], fmaf(f0.y, xs1[j], fmaf(f0.x, d[j][1], acc[r][j][1])));
        acc[r][j][2] = fmaf(-f1.x, xo0[j], fmaf(f1.y, xs0[j], fmaf(f1.x, d[j][2], acc[r][j][2])));
        acc[r][j][3] = fmaf(-f1.x, xo1[j], fmaf(f1.y, xs1[j], fmaf(f1.x, d[j][3], acc[r][j][3])));
      }
    }
    __syncwarp();  // every lane's reads of this slot are done
    if (lane == 0 && c + S < nit) issue(c + S);
    if (grp == kg - 1) {  // strip finished
      if (seg_from_start) {
#pragma unroll
        for (int r = 0; r < RT; ++r) store_strip_tile<EPI, NJ>(p, set * RT + r, g, q, acc[r]);
      } else {  // the head strip, entered part-way
#pragma unroll
        for (int r = 0; r < RT; ++r)
#pragma unroll
          for (int j = 0; j < NJ; ++j)
#pragma unroll
            for (int i = 0; i < 4; ++i) hacc[r][j][i] = acc[r][j][i];
        has_head = true;
      }
#pragma unroll
      for (int r = 0; r < RT; ++r)
#pragma unroll
        for (int j = 0; j < NJ; ++j)
#pragma unroll
          for (int i = 0; i < 4; ++i) acc[r][j][i] = 0.f;
      seg_from_start = true;
      grp = 0;
      ++set;
    } else {
      ++grp;
    }
  }
  // partial strips into the warp's idle ring: [2][32 lanes][RT][NJ] float4 (each lane's accumulators
  // contiguous); slot 0 = head strip, 1 = tail strip
  __syncwarp();
  float4* pw = reinterpret_cast<float4*>(ring);
  auto put = [&](int sl, const float (&v)[RT][NJ][4]) {
#pragma unroll
    for (int r = 0; r < RT; ++r)
#pragma unroll
      for (int j = 0; j < NJ; ++j) pw[(sl * 32 + lane) * PL + r * NJ + j] = make_float4(v[r][j][0], v[r][j][1], v[r][j][2], v[r][j][3]);
  };
  if (has_head) put(0, hacc);
  if (nit > 0 && grp != 0) put(set == head_set ? 0 : 1, acc);  // range ended inside a strip
  __syncthreads();
  reduce_tail_s<EPI, RT, NJ, S * SLOT>(p, smem + RC::BAR_BYTES, C0, C1, R, warp, lane, g, q);
}

// xsum[g][t] = (sum_{k%4<2} x[t,k], sum_{k%4>=2} x[t,k]) over group g, t < 32 (0 for t >= m);
// one warp per (g, t), fixed summation order.
__global__ void k_xsum(const __half* __restrict__ x, int64_t ldx, int64_t m, int kg, float2* __restrict__ out) {
  const int64_t id = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  pdl_trigger();
  pdl_wait();
  if (id >= (int64_t)kg * kXsTok) return;
  const int lane = threadIdx.x & 31;
  const int64_t g = id / kXsTok, t = id % kXsTok;
  float a = 0.f, b = 0.f;
  if (t < m) {
    const uint2 raw = *reinterpret_cast<const uint2*>(x + t * ldx + g * 128 + lane * 4);
    const __half2 lo = *reinterpret_cast<const __half2*>(&raw.x), hi = *reinterpret_cast<const __half2*>(&raw.y);
    a = __low2float(lo) + __high2float(lo);  // k%4 in {0,1}
    b = __low2float(hi) + __high2float(hi);  // k%4 in {2,3}
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    a += __shfl_xor_sync(0xffffffff, a, o);
    b += __shfl_xor_sync(0xffffffff, b, o);
  }
  if (lane == 0) out[id] = make_float2(a, b);
}

size_t gemv_smem(int tok, int kg) { return (size_t)kWarps * 2 * tok * kRows * 4 + (size_t)kg * kXsTok * 8; }

template <int BITS, int TOK, int EPI>
cudaError_t launch_e(const GemvP& p, cudaStream_t s) {
  void (*kern)(const GemvP);
  size_t smem;
  if constexpr (BITS == 16) {
    kern = k_gemv<BITS, TOK, EPI>;
    smem = gemv_smem(TOK, p.kg);
  } else {
    kern = k_gemv_q<BITS, TOK, EPI>;
    smem = (size_t)QRing<BITS, TOK>::BYTES;
  }
  static size_t attr = 0;
  if (smem > attr) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = smem;
  }
  return launch_pdl(kern, dim3((unsigned)p.W), dim3(kThreads), smem, s, p);
}

template <int BITS, int RT, int EPI, bool XS, int NJ>
cudaError_t launch_s_x(const CUtensorMap& tw, const CUtensorMap& tm, const GemvP& p, cudaStream_t s) {
  void (*kern)(const CUtensorMap, const CUtensorMap, const GemvP) = k_gemv_s<BITS, RT, EPI, XS, NJ>;
  const size_t smem = (size_t)SRing<BITS, RT>::BYTES;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  return launch_pdl(kern, dim3((unsigned)p.W), dim3(kSThreads), smem, s, tw, tm, p);
}
// XS: group sums computed in the kernel (p.xsum == null) or read from p.xsum
template <int BITS, int RT, int EPI>
cudaError_t launch_s_e(const CUtensorMap& tw, const CUtensorMap& tm, const GemvP& p, cudaStream_t s) {
  // INT3 always computes its own sums (its per-position offsets 1024 / 128 / 16 are not the caller's
  // two-way split)
  // (caller sums, when given, measured 1-5 % faster than the tensor-core chain for INT4 / INT8)
  const bool own = p.xsum == nullptr || BITS == 3;
  if constexpr (RT == 2) {
    if (p.m > 8)
      return own ? launch_s_x<BITS, RT, EPI, true, 2>(tw, tm, p, s) : launch_s_x<BITS, RT, EPI, false, 2>(tw, tm, p, s);
  }
  return own ? launch_s_x<BITS, RT, EPI, true, 1>(tw, tm, p, s) : launch_s_x<BITS, RT, EPI, false, 1>(tw, tm, p, s);
}

template <int BITS, int RT>
cudaError_t launch_s(const sq_qweight& w, const GemvP& p, int epi, cudaStream_t s) {
  // codes: [n/16 tiles][kg * UB/256 lines][256 B], box = RT tiles x one unit; meta: [n/16][kg * 16] u32
  constexpr int UB = SRing<BITS, RT>::UB;
  CUtensorMap tw, tm;
  const uint64_t nt = (uint64_t)w.n / kRows, kg = (uint64_t)p.kg;
  const uint64_t dw[3] = {256, kg * (UB / 256), nt}, sw_[2] = {256, kg * UB};
  const uint32_t bw[3] = {256, (uint32_t)(UB / 256), (uint32_t)RT};
  cudaError_t e = encode_nd(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, w.packed, 3, dw, sw_, bw, CU_TENSOR_MAP_SWIZZLE_NONE);
  if (e != cudaSuccess) return e;
  const uint64_t dm[2] = {kg * 16, nt}, sm_[1] = {kg * 64};
  const uint32_t bm[2] = {16, (uint32_t)RT};
  e = encode_nd(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, w.meta, 2, dm, sm_, bm, CU_TENSOR_MAP_SWIZZLE_NONE);
  if (e != cudaSuccess) return e;
  switch (epi) {
    case SQ_EPI_F16: return launch_s_e<BITS, RT, SQ_EPI_F16>(tw, tm, p, s);
    case SQ_EPI_F16_RELU: return launch_s_e<BITS, RT, SQ_EPI_F16_RELU>(tw, tm, p, s);
    case SQ_EPI_F16_GELU: return launch_s_e<BITS, RT, SQ_EPI_F16_GELU>(tw, tm, p, s);
    default: return launch_s_e<BITS, RT, SQ_EPI_F32_ACCUM>(tw, tm, p, s);
  }
}

template <int BITS, int TOK>
cudaError_t launch_t(const GemvP& p, int epi, cudaStream_t s) {
  switch (epi) {
    case SQ_EPI_F16: return launch_e<BITS, TOK, SQ_EPI_F16>(p, s);
    case SQ_EPI_F16_RELU: return launch_e<BITS, TOK, SQ_EPI_F16_RELU>(p, s);
    case SQ_EPI_F16_GELU: return launch_e<BITS, TOK, SQ_EPI_F16_GELU>(p, s);
    default: return launch_e<BITS, TOK, SQ_EPI_F32_ACCUM>(p, s);
  }
}

template <int BITS>
cudaError_t launch_b(const GemvP& p, int epi, cudaStream_t s) {
  if (p.m <= 8) return launch_t<BITS, 8>(p, epi, s);
  if (p.m <= 16) return launch_t<BITS, 16>(p, epi, s);
  return launch_t<BITS, 32>(p, epi, s);
}

// number of CTAs: one per SM (fewer for tiny problems so every warp gets >= 1 unit)
int64_t gemv_ctas(int64_t U) {
  const int64_t full = (int64_t)num_sms();
  const int64_t need = (U + kWarps - 1) / kWarps;
  return need < full ? need : full;
}

// K2s: two 8-warp CTAs per SM (fewer for tiny problems so every warp gets >= 1 item)
int64_t gemv_s_ctas(int64_t U) {
  const int64_t full = (int64_t)num_sms() * kSCtasPerSm;
  const int64_t need = (U + kSWarps - 1) / kSWarps;
  return need < full ? need : full;
}

int tok_pad(int64_t m) { return m <= 8 ? 8 : (m <= 16 ? 16 : 32); }

// fixed-size counter region (n <= 65536) so linears of different n can share one workspace
constexpr int64_t kMaxN = 65536;
size_t cnt_bytes(int64_t) { return (size_t)(kMaxN / kRows) * sizeof(int); }
// per-CTA boundary partials: K2 [W][2][tok][16], K2s [W][2][8][RT * 16] (RT <= 4)
size_t part_bytes(int64_t W, int64_t m) {
  const int64_t per = tok_pad(m) * kRows > 8 * 4 * kRows ? tok_pad(m) * kRows : 8 * 4 * kRows;
  return (size_t)W * 2 * per * sizeof(float);
}
// K2s (strips) for quantized weights at m <= 8 (SQ_K2S=0: K2)
// Whole strips only (n a multiple of RT * 16, so no TMA box reaches past the matrix).  Measured
// (tools/gemv_rot.py --graph on variant builds, back-to-back graph launches, m = 1 / 8): K2s is as fast as K2 or faster on every
// OPT-125m ... OPT-66B shape, e.g. 36864 x 9216 INT4 34.4 / 37.1 us vs 44.2 / 60.8, 20480 x 5120
// INT4 15.5 / 17.0 vs 17.7 / 23.7, 768 x 3072 5.5 vs 6.0-6.5 (2304 x 768: within 0.2 us), so K2
// remains only for n not a multiple of 32.  SQ_K2S=0 / 1 forces K2 / K2s.
// strip width: 4 tiles (the activation fragment re-used 4x) for INT3 / INT4 linears of more than
// 1280 tiles, else 2 (twice the items per warp; 5120^2 INT4 9.7 -> 8.0 us, 5120 x 20480 17.1 ->
// 16.3 us, but 36864 x 9216 34.2 -> 37.8 us; tools/gemv_rot.py --graph on variant builds); INT8 always 2
// (m in 9..16: two token tiles, RT = 2)
int k2s_rt(int bits, int64_t n, int m) { return (bits != 8 && m <= 8 && n / kRows > 1280) ? 4 : 2; }

// m in 9..16 (two token tiles, tools/gemv_rot.py --graph on variant builds): K2s beats K2c only on INT8 linears up to ~120 MB
// (20480 x 5120: 23.6-23.9 vs 25.3-25.5 us; 5120^2: 10.8-11.2 vs 13.1), and loses up to 1.6x on large or
// INT3 / INT4 ones (HMMA-bound at RT = 2); SQ_K2S16=1 / 0 forces it on / off there.
bool k2s16(int bits, int64_t n, int64_t k) {
  static int forced = -2;
  if (forced == -2) { const char* e = getenv("SQ_K2S16"); forced = !e ? -1 : (e[0] == '1' ? 1 : 0); }
  if (forced >= 0) return forced == 1;
  return bits == 8 && (double)n * k <= 120e6;
}

bool k2s_rule(int bits, int64_t n, int64_t k, int m) {
  static int forced = -2;
  if (forced == -2) { const char* e = getenv("SQ_K2S"); forced = !e ? -1 : (e[0] == '0' ? 0 : 1); }
  if (bits == 16 || m > 16 || (m > 8 && !k2s16(bits, n, k)) || n % (16 * k2s_rt(bits, n, m)) != 0) return false;
  if (forced >= 0) return forced == 1;
  return true;
}

}  // namespace

bool use_k2s(int bits, int64_t n, int64_t k, int m) { return k2s_rule(bits, n, k, m); }

size_t xsum_bytes(int64_t k) { return (size_t)(k / 128) * kXsTok * sizeof(float2); }

size_t gemv_workspace_bytes(int64_t n, int64_t k, int64_t m) {
  const int64_t U = (n / kRows) * (k / 128);
  const int64_t W = gemv_ctas(U) > gemv_s_ctas(U) ? gemv_ctas(U) : gemv_s_ctas(U);
  size_t part = part_bytes(W, m);
  size_t a = cnt_bytes(n) + part + xsum_bytes(k) + 256;
  size_t b = n % 128 == 0 ? gemv_tc_workspace_bytes(n, k) : 0;
  return a > b ? a : b;
}

// K2 (mma.sync, register unpack) for m <= 8; K2c (tcgen05: TMEM dequant, or fp16 weights straight
// from SMEM) for 8 < m <= 32.  K2 takes the activation group sums (xsum; computed here if null).
// SQ_GEMV_PATH=mma|tc overrides (benchmarking).
int gemv_path(int64_t n, int64_t k, int m, int bits) {
  static int forced = -2;
  if (forced == -2) {
    const char* e = getenv("SQ_GEMV_PATH");
    forced = !e ? -1 : (e[0] == 't' ? 1 : (e[0] == 'm' ? 0 : -1));
  }
  if (n % 128) return 0;
  if (forced >= 0) return forced;
  // measured on B200 (tools/gemv_rot.py --graph, back-to-back launches): the tcgen05 kernel's cost
  // does not depend on m; the mma.sync kernel's grows with m (activation fragments from L1) but
  // has the shorter ramp -- it wins on OPT-13B-sized linears at m <= 4 (and m <= 8 off INT4),
  // the tcgen05 kernel everywhere else, and always for fp16 weights
  (void)k;
  // (round 2, INT3 re-laid with a one-LOP3 unpack: the tcgen05 kernel wins INT3 linears from ~80 MB
  // at every m, e.g. 36864 x 9216 at m = 1: 3.34 vs 2.89 TB/s; the mma.sync kernel keeps the OPT-13B
  // sizes at m <= 8, e.g. 20480 x 5120: 2.24 vs 2.05 TB/s)
  // (round 3: the strip kernel K2s streams every quantized linear at m <= 8 at least as fast as the
  // tcgen05 kernel, e.g. 36864 x 9216 INT4 5.1 / 4.6 TB/s at m = 1 / 8 vs 4.4-4.7; tools/gemv_rot.py --graph on variant builds)
  if (bits == 16 || m > 16) return 1;
  if (m > 8) return k2s_rule(bits, n, k, m) ? 0 : 1;
  return 0;
}

cudaError_t launch_xsum(const __half* x, int64_t ldx, int64_t m, int64_t k, float2* xsum, cudaStream_t s) {
  const int64_t items = (k / 128) * kXsTok;
  auto t = prof_begin(KC_GLUE, (double)m * k * 2 + items * 8.0, 0, s);
  cudaError_t e = launch_pdl(k_xsum, dim3((unsigned)((items + 7) / 8)), dim3(256), 0, s, x, ldx, m, (int)(k / 128), xsum);
  prof_end(t, s);
  count_launch();
  return e;
}

cudaError_t launch_gemv(const sq_qweight& w, const __half* x, int64_t ldx, int m, void* y, int64_t ldy, int epi,
                        const float2* xsum, void* ws, cudaStream_t s) {
  if (gemv_path(w.n, w.k, m, w.bits) == 1) return launch_gemv_tc(w, x, ldx, m, y, ldy, epi, ws, s);
  if (w.n > kMaxN || w.n / kRows * (w.k / 128) >= (1ll << 31) / 256) return cudaErrorInvalidValue;  // 32-bit index math
  GemvP p{};
  p.packed = static_cast<const uint8_t*>(w.packed);
  p.meta = static_cast<const uint32_t*>(w.meta);
  p.bias = static_cast<const __half*>(w.bias);
  p.x = x;
  p.ldx = (int)ldx;
  p.m = m;
  p.n = (int)w.n;
  p.kg = (int)(w.k / 128);
  p.y = y;
  p.ldy = (int)ldy;
  p.U = (int)((w.n / kRows) * p.kg);
  p.W = (int)gemv_ctas(p.U);
  const int64_t wmax = gemv_ctas(p.U) > gemv_s_ctas(p.U) ? gemv_ctas(p.U) : gemv_s_ctas(p.U);  // as sized
  uint8_t* base = static_cast<uint8_t*>(ws);
  p.cnt = reinterpret_cast<int*>(base);
  p.part = reinterpret_cast<float*>(base + cnt_bytes(w.n));
  float2* xs_ws = reinterpret_cast<float2*>(base + cnt_bytes(w.n) + part_bytes(wmax, m));
  const bool k2s = use_k2s(w.bits, w.n, w.k, m);
  if (w.bits != 16 && xsum == nullptr && !k2s) {  // K2s computes missing group sums itself
    cudaError_t e = launch_xsum(x, ldx, m, w.k, xs_ws, s);
    if (e != cudaSuccess) return e;
    xsum = xs_ws;
  }
  p.xsum = xsum;
  const double bytes = (double)w.n * w.k * w.bits / 8.0 + (w.bits != 16 ? (double)w.n * (w.k / 128) * 4.0 : 0.0);
  auto t = prof_begin(KC_GEMV, bytes, 2.0 * m * w.n * w.k, s);
  cudaError_t e;
  if (k2s) {
    const int rt = k2s_rt(w.bits, w.n, m);
    p.U = (int)(((w.n / kRows + rt - 1) / rt) * p.kg);
    p.W = (int)gemv_s_ctas(p.U);
    if (rt == 4) e = w.bits == 3 ? launch_s<3, 4>(w, p, epi, s) : launch_s<4, 4>(w, p, epi, s);
    else if (w.bits == 3) e = launch_s<3, 2>(w, p, epi, s);
    else if (w.bits == 4) e = launch_s<4, 2>(w, p, epi, s);
    else e = launch_s<8, 2>(w, p, epi, s);
    prof_end(t, s);
    count_launch();
    return e;
  }
  switch (w.bits) {
    case 3: e = launch_b<3>(p, epi, s); break;
    case 4: e = launch_b<4>(p, epi, s); break;
    case 8: e = launch_b<8>(p, epi, s); break;
    default: e = launch_b<16>(p, epi, s); break;
  }
  prof_end(t, s);
  count_launch();
  return e;
}

}  // namespace sq
