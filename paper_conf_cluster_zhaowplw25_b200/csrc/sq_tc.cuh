// tcgen05 building blocks shared by the prefill GEMM (K3) and the tensor-core
// decode GEMV (K2c): SW128 smem descriptors, the instruction descriptor, and the
// per-row dequantization of one 128-k group straight into tensor memory.
//
// Packed weight stages are [128 rows][GB bytes] fetched by one 3-D TMA box whose rows are
// 128-B lines (INT4: two weight rows per line; INT8: one) under SWIZZLE_128B, or 256-B lines
// without swizzle (INT3: 48-B weight rows are conflict-free) -- the TMA engine moves short box
// rows slowly (64-B rows measured at ~60 % of the 128-B rate), so the box rows are made long;
// fp16 weight stages are two SW128 [128][128 B] tiles.  tcgen05.st is
// .sync.aligned: its TMEM column address must be warp-uniform, so the chunk order is static
// and bank conflicts are avoided by the TMA swizzle, not by per-thread reordering.
#pragma once
#include "sq_common.cuh"

namespace sq {
namespace tc {

template <int BITS>
struct GCfg;
template <>
struct GCfg<3> { static constexpr int GB = 48; static constexpr int S_W = 4; };
template <>
struct GCfg<4> { static constexpr int GB = 64; static constexpr int S_W = 4; };
template <>
struct GCfg<8> { static constexpr int GB = 128; static constexpr int S_W = 4; };
template <>
struct GCfg<16> { static constexpr int GB = 256; static constexpr int S_W = 2; };

// Geometry of the packed-weight tensor map (placement T16 viewed as lines): line bytes, lines per
// (16-row, 1-group) unit, swizzle (0 none, 1 SWIZZLE_128B).  Box = {line, lines_per_unit * UG, 8}.
struct WLines { int line, lpu, sw128; };
inline WLines wlines(int bits) {
  if (bits == 3) return {256, 3, 0};   // 768 B per unit
  if (bits == 4) return {128, 8, 1};   // 1 KB per unit
  return {128, 16, 1};                 // INT8: 2 KB per unit
}

__device__ __forceinline__ uint64_t make_sw128_desc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;              // LBO (ignored for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;    // SBO: 8 rows x 128 B
  d |= (uint64_t)1 << 46;              // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;              // SWIZZLE_128B
  return d;
}

// K-major, no swizzle: core matrices of 8 rows x 16 B stored contiguously (128 B); lbo = byte
// distance between core matrices adjacent in K, sbo = between core matrices adjacent in M/N
__device__ __forceinline__ uint64_t make_noswz_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;  // descriptor version (sm_100); swizzle field 0 = none
  return d;
}

// instruction descriptor: kind::f16, A=B=f16 K-major, D=f32, M x N
constexpr uint32_t make_idesc(int M, int N) {
  return (1u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__device__ __forceinline__ uint32_t hsub_fma(uint32_t h, uint32_t off2, uint32_t s2, uint32_t z2) {
  __half2 c = __hsub2(*reinterpret_cast<__half2*>(&h), *reinterpret_cast<__half2*>(&off2));
  __half2 r = __hfma2(c, *reinterpret_cast<__half2*>(&s2), *reinterpret_cast<__half2*>(&z2));
  return *reinterpret_cast<uint32_t*>(&r);
}

// Dequantize batches [B0, B0 + NB) (32 k each) of this thread's row (r) of one 128-k group into
// half2 columns taddr + 16 b .. + 15 (w~ = s*c + z), one tcgen05.st per batch.  `row_off` = byte
// offset of the row inside the stage (default r * GB); the swizzle pattern only depends on
// r % 16 because every T16 unit starts on a 1-KB boundary.  B0 must be warp-uniform.
template <int BITS, int NB>
__device__ __forceinline__ void dequant_row_batches(const uint8_t* wst, uint32_t meta, int r, uint32_t taddr,
                                                    int row_off, int B0) {
  const uint32_t s2 = (meta & 0xFFFFu) * 0x10001u;
  const uint32_t z2 = (meta >> 16) * 0x10001u;
  constexpr uint32_t K1024 = 0x64006400u, K64 = 0x54005400u;
  if constexpr (BITS == 4) {
    // the stage is a sequence of 128-B lines (two 64-B rows each) under SWIZZLE_128B: logical chunk
    // (row & 1) * 4 + b of line row / 2 sits at physical chunk ^ (line & 7)
    const int lo = row_off >= 0 ? row_off : r * 64;
    const uint8_t* line = wst + (lo & ~127);
    const int h4 = (lo >> 4) & 4, swz = (lo >> 7) & 7;
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int b = B0 + bi;
      const int pc = (h4 | b) ^ swz;
      uint4 v = *reinterpret_cast<const uint4*>(line + pc * 16);
      const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
      uint32_t o[16];
#pragma unroll
      for (int w = 0; w < 4; ++w) {
        const uint32_t x = wv[w], x8 = x >> 8;
        o[4 * w + 0] = hsub_fma(lop3_and_or(x, 0x000F000Fu, K1024), K1024, s2, z2);
        o[4 * w + 1] = hsub_fma(lop3_and_or(x, 0x00F000F0u, K64), K64, s2, z2);
        o[4 * w + 2] = hsub_fma(lop3_and_or(x8, 0x000F000Fu, K1024), K1024, s2, z2);
        o[4 * w + 3] = hsub_fma(lop3_and_or(x8, 0x00F000F0u, K64), K64, s2, z2);
      }
      tmem_st16(taddr + 16 * b, o);
    }
  } else if constexpr (BITS == 8) {
    const uint8_t* row = wst + (row_off >= 0 ? row_off : r * 128);
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int b = B0 + bi;
      uint32_t o[16];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int c = 2 * b + h, pc = c ^ (r & 7);  // SWIZZLE_128B
        uint4 v = *reinterpret_cast<const uint4*>(row + pc * 16);
        const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          o[8 * h + 2 * t] = hsub_fma(prmt(wv[t], 0x64646464u, 0x4140u), K1024, s2, z2);
          o[8 * h + 2 * t + 1] = hsub_fma(prmt(wv[t], 0x64646464u, 0x4342u), K1024, s2, z2);
        }
      }
      tmem_st16(taddr + 16 * b, o);
    }
  } else if constexpr (BITS == 3) {
    const uint32_t* row = reinterpret_cast<const uint32_t*>(wst + (row_off >= 0 ? row_off : r * 48));
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int bl = B0 + bi;
      const uint32_t L0 = row[3 * bl], L1 = row[3 * bl + 1], H = row[3 * bl + 2];
      uint32_t o[16];
#pragma unroll
      for (int a = 0; a < 2; ++a) {
        const uint32_t La = a ? L1 : L0;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const uint32_t lo = La >> (2 * i);
          const int sh = i + 8 * a - 2;
          const uint32_t hs = sh >= 0 ? (H >> sh) : (H << (-sh));
          uint32_t t;
          asm("lop3.b32 %0, %1, %2, %3, 0xD8;" : "=r"(t) : "r"(hs), "r"(lo), "r"(0x00030003u));  // mask ? lo : hs
          o[8 * a + i] = hsub_fma(lop3_and_or(t, 0x00070007u, K1024), K1024, s2, z2);
        }
      }
      tmem_st16(taddr + 16 * bl, o);
    }
  } else {
    // fp16: two SW128 regions (k 0..63, 64..127) of [128 rows x 128 B]
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int b = B0 + bi;
      const uint8_t* region = wst + (b >> 1) * (128 * 128) + r * 128;
      uint32_t o[16];
#pragma unroll
      for (int h = 0; h < 4; ++h) {
        const int c = 4 * (b & 1) + h, pc = c ^ (r & 7);
        uint4 v = *reinterpret_cast<const uint4*>(region + pc * 16);
        o[4 * h] = v.x; o[4 * h + 1] = v.y; o[4 * h + 2] = v.z; o[4 * h + 3] = v.w;
      }
      tmem_st16(taddr + 16 * b, o);
    }
  }
}

// Decode variant (K2c): the A operand holds s*c only -- the zero-point term z * sum(x) of the group
// is added by one extra MMA per unit (z columns x activation group sums, decode kernel).  With the
// magic-number code v = off + c (exact), s*c = v*s + (-off*s) is ONE HFMA2 per pair: -off*s is exact
// in fp16 (power-of-two scaling) and the FMA rounds once, to fp16(s*c).  Rows whose -off*s would
// overflow fp16 (|s| >= 65504/off, pathological outlier groups) take (v - off)*s (HSUB2 + HMUL2).
// Offsets: INT4 1024 / 64 (low / high nibble slot of L4), INT8 1024 (PRMT), INT3 8 (code placed
// under exponent 2^3, as in K2).  Same batch/swizzle conventions as dequant_row_batches.
__device__ __forceinline__ uint32_t hfma2_u(uint32_t a, uint32_t b, uint32_t c) {
  __half2 r = __hfma2(*reinterpret_cast<__half2*>(&a), *reinterpret_cast<__half2*>(&b), *reinterpret_cast<__half2*>(&c));
  return *reinterpret_cast<uint32_t*>(&r);
}
__device__ __forceinline__ uint32_t hsub_mul_u(uint32_t v, uint32_t off2, uint32_t s2) {
  __half2 c = __hsub2(*reinterpret_cast<__half2*>(&v), *reinterpret_cast<__half2*>(&off2));
  __half2 r = __hmul2(c, *reinterpret_cast<__half2*>(&s2));
  return *reinterpret_cast<uint32_t*>(&r);
}
// -off * s as half2 (exact unless it overflows; `ok` false then)
__device__ __forceinline__ uint32_t neg_off_s(uint32_t s_bits, float off, bool& ok) {
  const float nb = -off * __half2float(__ushort_as_half((unsigned short)s_bits));
  ok = fabsf(nb) <= 65504.f;
  const uint32_t h = __half_as_ushort(__float2half_rn(nb));
  return h * 0x10001u;
}

template <int BITS, int NB>
__device__ __forceinline__ void unpack_sc_row_batches(const uint8_t* wst, uint32_t meta, int r, uint32_t taddr,
                                                      int row_off, int B0) {
  const uint32_t sb = meta & 0xFFFFu;
  const uint32_t s2 = sb * 0x10001u;
  constexpr uint32_t K1024 = 0x64006400u, K64 = 0x54005400u, K8 = 0x48004800u;
  bool ok_a, ok_b;
  if constexpr (BITS == 4) {
    const uint32_t nbA = neg_off_s(sb, 1024.f, ok_a), nbB = neg_off_s(sb, 64.f, ok_b);
    const bool fast = ok_a;  // ok_a implies ok_b
    const uint8_t* line = wst + (row_off & ~127);
    const int h4 = (row_off >> 4) & 4, swz = (row_off >> 7) & 7;
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int b = B0 + bi;
      const int pc = (h4 | b) ^ swz;  // 128-B lines under SWIZZLE_128B (see dequant_row_batches)
      uint4 v = *reinterpret_cast<const uint4*>(line + pc * 16);
      const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
      uint32_t o[16];
      if (fast) {
#pragma unroll
        for (int w = 0; w < 4; ++w) {
          const uint32_t x = wv[w], x8 = x >> 8;
          o[4 * w + 0] = hfma2_u(lop3_and_or(x, 0x000F000Fu, K1024), s2, nbA);
          o[4 * w + 1] = hfma2_u(lop3_and_or(x, 0x00F000F0u, K64), s2, nbB);
          o[4 * w + 2] = hfma2_u(lop3_and_or(x8, 0x000F000Fu, K1024), s2, nbA);
          o[4 * w + 3] = hfma2_u(lop3_and_or(x8, 0x00F000F0u, K64), s2, nbB);
        }
      } else {
#pragma unroll
        for (int w = 0; w < 4; ++w) {
          const uint32_t x = wv[w], x8 = x >> 8;
          o[4 * w + 0] = hsub_mul_u(lop3_and_or(x, 0x000F000Fu, K1024), K1024, s2);
          o[4 * w + 1] = hsub_mul_u(lop3_and_or(x, 0x00F000F0u, K64), K64, s2);
          o[4 * w + 2] = hsub_mul_u(lop3_and_or(x8, 0x000F000Fu, K1024), K1024, s2);
          o[4 * w + 3] = hsub_mul_u(lop3_and_or(x8, 0x00F000F0u, K64), K64, s2);
        }
      }
      tmem_st16(taddr + 16 * b, o);
    }
  } else if constexpr (BITS == 8) {
    const uint32_t nbA = neg_off_s(sb, 1024.f, ok_a);
    const uint8_t* row = wst + row_off;
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int b = B0 + bi;
      uint32_t o[16];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int c = 2 * b + h, pc = c ^ (r & 7);  // SWIZZLE_128B
        uint4 v = *reinterpret_cast<const uint4*>(row + pc * 16);
        const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const uint32_t lo = prmt(wv[t], 0x64646464u, 0x4140u), hi = prmt(wv[t], 0x64646464u, 0x4342u);
          o[8 * h + 2 * t] = ok_a ? hfma2_u(lo, s2, nbA) : hsub_mul_u(lo, K1024, s2);
          o[8 * h + 2 * t + 1] = ok_a ? hfma2_u(hi, s2, nbA) : hsub_mul_u(hi, K1024, s2);
        }
      }
      tmem_st16(taddr + 16 * b, o);
    }
  } else {
    static_assert(BITS == 3, "unpack_sc_row_batches: 3/4/8 bits");
    const uint32_t nbA = neg_off_s(sb, 8.f, ok_a);
    const uint32_t* row = reinterpret_cast<const uint32_t*>(wst + row_off);
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int bl = B0 + bi;
      const uint32_t L0 = row[3 * bl], L1 = row[3 * bl + 1], H = row[3 * bl + 2];
      uint32_t o[16];
#pragma unroll
      for (int a = 0; a < 2; ++a) {
        const uint32_t La = a ? L1 : L0;
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          // low two bits -> mantissa bits 7..8, high bit -> bit 9, under exponent 2^3: half2(8 + c)
          const int sl = 7 - 2 * i;
          const uint32_t l = sl >= 0 ? (La << sl) : (La >> (-sl));
          const int sh = i + 8 * a - 9;
          const uint32_t hs = sh >= 0 ? (H >> sh) : (H << (-sh));
          uint32_t t;
          asm("lop3.b32 %0, %1, %2, %3, 0xD8;" : "=r"(t) : "r"(hs), "r"(l), "r"(0x01800180u));  // mask ? l : hs
          const uint32_t v = lop3_and_or(t, 0x03800380u, K8);
          o[8 * a + i] = ok_a ? hfma2_u(v, s2, nbA) : hsub_mul_u(v, K8, s2);
        }
      }
      tmem_st16(taddr + 16 * bl, o);
    }
  }
}

// the whole 128-k group of this thread's row: 64 half2 columns at taddr .. taddr + 63
template <int BITS>
__device__ __forceinline__ void dequant_row_to_tmem(const uint8_t* wst, uint32_t meta, int r, uint32_t taddr,
                                                    int row_off = -1) {
  dequant_row_batches<BITS, 4>(wst, meta, r, taddr, row_off, 0);
}

// Fetch the 128-row x 1-group weight tile (8 T16 units, each 16*GB contiguous bytes at unit
// index t*kg + g) and its meta (8 x 64 B) with 16 bulk copies onto one mbarrier.
template <int BITS>
__device__ __forceinline__ void load_w_tile(uint8_t* wdst, uint8_t* mdst, const uint8_t* packed,
                                            const uint32_t* meta, int64_t tile16, int g, int kg, uint64_t* bar) {
  constexpr int UB = 16 * GCfg<BITS>::GB;
#pragma unroll
  for (int t = 0; t < 8; ++t) {
    const int64_t u = (tile16 + t) * kg + g;
    bulk_load(wdst + t * UB, packed + u * UB, UB, bar);
    bulk_load(mdst + t * 64, meta + u * 16, 64, bar);
  }
}

}  // namespace tc
}  // namespace sq
