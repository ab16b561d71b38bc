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

// w~ = s*c + z in one fp16 FMA (c exact after the magic-number subtraction).  SAT: saturate at the fp16
// maximum (reading R20) -- only a group with s*(2^b - 1) + z >= 65520 can overflow to +inf, and a warp
// holding such a group takes this variant (one extra HMNMX2 per pair; saturation is the identity on
// the other lanes' finite values); q = group min keeps the bottom finite.
template <bool SAT = false>
__device__ __forceinline__ uint32_t hsub_fma(uint32_t h, uint32_t off2, uint32_t s2, uint32_t z2) {
  __half2 c = __hsub2(*reinterpret_cast<__half2*>(&h), *reinterpret_cast<__half2*>(&off2));
  __half2 r = __hfma2(c, *reinterpret_cast<__half2*>(&s2), *reinterpret_cast<__half2*>(&z2));
  if constexpr (SAT) r = __hmin2(r, __half2half2(__ushort_as_half((unsigned short)0x7BFFu)));
  return *reinterpret_cast<uint32_t*>(&r);
}

// true if some code of the group may dequantize beyond the fp16 maximum (conservative: fp32 rounding
// of s*qmax + z is monotone, and overflow needs the exact value >= 65520)
template <int BITS>
__device__ __forceinline__ bool group_may_overflow(uint32_t meta) {
  const float s = __half2float(__ushort_as_half((unsigned short)(meta & 0xFFFFu)));
  const float z = __half2float(__ushort_as_half((unsigned short)(meta >> 16)));
  return fmaf(s, (float)((1 << BITS) - 1), z) >= 65504.f;
}

// Dequantize batches [B0, B0 + NB) (32 k each) of this thread's row (r) of one 128-k group into
// half2 columns taddr + 16 b .. + 15 (w~ = s*c + z), one tcgen05.st per batch.  `row_off` = byte
// offset of the row inside the stage (default r * GB); the swizzle pattern only depends on
// r % 16 because every T16 unit starts on a 1-KB boundary.  B0 must be warp-uniform.
template <int BITS, int NB, bool SAT>
__device__ __forceinline__ void dequant_row_batches_(const uint8_t* wst, uint32_t meta, int r, uint32_t taddr,
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
        o[4 * w + 0] = hsub_fma<SAT>(lop3_and_or(x, 0x000F000Fu, K1024), K1024, s2, z2);
        o[4 * w + 1] = hsub_fma<SAT>(lop3_and_or(x, 0x00F000F0u, K64), K64, s2, z2);
        o[4 * w + 2] = hsub_fma<SAT>(lop3_and_or(x8, 0x000F000Fu, K1024), K1024, s2, z2);
        o[4 * w + 3] = hsub_fma<SAT>(lop3_and_or(x8, 0x00F000F0u, K64), K64, s2, z2);
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
          o[8 * h + 2 * t] = hsub_fma<SAT>(prmt(wv[t], 0x64646464u, 0x4140u), K1024, s2, z2);
          o[8 * h + 2 * t + 1] = hsub_fma<SAT>(prmt(wv[t], 0x64646464u, 0x4342u), K1024, s2, z2);
        }
      }
      tmem_st16(taddr + 16 * b, o);
    }
  } else if constexpr (BITS == 3) {
    // L3: per 32-code block three words; pair q of word w (q < 5) at bits 3q (q >= 3: of w >> 9, bits
    // 3(q-3)); under magic 1024 / 128 / 16 a 3-bit field at bit 0 / 3 / 6 reads as off + c exactly;
    // pair 15 gathered from the spare bits 15 / 31 of the three words
    constexpr uint32_t K128 = 0x58005800u, K16 = 0x4C004C00u;
    const uint32_t* row = reinterpret_cast<const uint32_t*>(wst + (row_off >= 0 ? row_off : r * 48));
#pragma unroll
    for (int bi = 0; bi < NB; ++bi) {
      const int bl = B0 + bi;
      const uint32_t W[3] = {row[3 * bl], row[3 * bl + 1], row[3 * bl + 2]};
      uint32_t o[16];
#pragma unroll
      for (int w = 0; w < 3; ++w) {
        const uint32_t x = W[w], x9 = x >> 9;
        o[5 * w + 0] = hsub_fma<SAT>(lop3_and_or(x, 0x00070007u, K1024), K1024, s2, z2);
        o[5 * w + 1] = hsub_fma<SAT>(lop3_and_or(x, 0x00380038u, K128), K128, s2, z2);
        o[5 * w + 2] = hsub_fma<SAT>(lop3_and_or(x, 0x01C001C0u, K16), K16, s2, z2);
        o[5 * w + 3] = hsub_fma<SAT>(lop3_and_or(x9, 0x00070007u, K1024), K1024, s2, z2);
        o[5 * w + 4] = hsub_fma<SAT>(lop3_and_or(x9, 0x00380038u, K128), K128, s2, z2);
      }
      uint32_t t;
      asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(t) : "r"(0x00010001u), "r"(W[0] >> 15), "r"(W[1] >> 14));  // a ? b : c (bitwise)
      asm("lop3.b32 %0, %1, %2, %3, 0xCA;" : "=r"(t) : "r"(0x00030003u), "r"(t), "r"(W[2] >> 13));
      o[15] = hsub_fma<SAT>(lop3_and_or(t, 0x00070007u, K1024), K1024, s2, z2);
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

template <int BITS, int NB>
__device__ __forceinline__ void dequant_row_batches(const uint8_t* wst, uint32_t meta, int r, uint32_t taddr,
                                                    int row_off, int B0) {
  if constexpr (BITS == 16) {
    dequant_row_batches_<BITS, NB, false>(wst, meta, r, taddr, row_off, B0);
  } else {
    // warp-uniform choice: tcgen05.st is .sync.aligned, so every lane of the warp must take the same path
    if (__builtin_expect(__any_sync(0xffffffffu, group_may_overflow<BITS>(meta)), 0))
      dequant_row_batches_<BITS, NB, true>(wst, meta, r, taddr, row_off, B0);
    else
      dequant_row_batches_<BITS, NB, false>(wst, meta, r, taddr, row_off, B0);
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
