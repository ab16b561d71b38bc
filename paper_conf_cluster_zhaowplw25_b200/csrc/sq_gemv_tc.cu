// K2c — decode dequant-GEMV on tcgen05 for micro-batches of up to 32 tokens
// (the pipeline's decode micro-batch xi = 32).  At 32 tokens a
// decode linear does 64 flop per weight; legacy mma.sync tops out near
// 535 TFLOP/s on B200 (measured), i.e. ~67 % of HBM speed at INT4, so the
// contraction moves to the 5th-generation tensor cores:
//
//  * Work unit = 128 weight rows x one group (128 k).  Units are flattened
//    row-tile-major / group-minor (placement T16 makes a unit 8 consecutive
//    16-row units) and split evenly over one CTA per SM (stream-K): every SM
//    streams the same number of bytes whatever the shape.
//  * Producer warp: TMA 4-D box of packed codes + 3-D box of meta per unit,
//    and the unit's activation slice [32 tokens x 128 k] (2 x SW128 boxes;
//    tokens >= m are zero-filled by TMA).  6-deep weight ring.
//  * 4 dequant warps (one thread per weight row): magic-number unpack,
//    w~ = s*c + z in fp16 (HSUB2 + HFMA2), tcgen05.st into a TMEM A slot.
//  * MMA thread: tcgen05.mma kind::f16, M = 128 rows, N = 32 tokens, K = 16,
//    A from TMEM, B (activations) from SMEM; fp32 accumulator in TMEM,
//    double-buffered per row-tile segment.
//  * 4 epilogue warps: drain each finished segment; a tile fully inside the
//    CTA is written directly (bias / activation / fp32 residual), a tile split
//    across CTAs goes through a workspace and is finished by the last CTA in
//    fixed CTA order (deterministic, counters self-reset).
// Warp roles: 0 producer, 1 MMA (+TMEM alloc), 2..9 dequant (2 groups of 4, alternating
// units so one group's tcgen05.st latency overlaps the other's unpack), 10..13 epilogue.
#include <cuda.h>

#include <cstring>

#include "sq_tc.cuh"

namespace sq {
namespace {
using namespace tc;

constexpr int BN = 128;     // weight rows per unit (TMEM lanes, MMA M)
constexpr int BT = 32;      // token columns (MMA N)
constexpr int XK = 64;
constexpr int X_BLOCK = BT * XK * 2;  // 4 KB: [32 tokens][64 k] SW128 tile
constexpr int DQ_GROUPS = 2;          // dequant warp-groups working on alternating units
// Ring depths are multiples of DQ_GROUPS: unit i uses W slot i % S_W and A slot i % S_A, so
// every slot belongs to ONE group, which consumes its units in order -- an mbarrier parity
// wait can then never be two phases ahead of the slot it waits on.
constexpr int TMEM_COLS = 512;
constexpr int D_COL = 0;              // 2 x 32 columns (double-buffered accumulator)
constexpr int A_COL = 64;             // S_A x (64 * UG) columns
constexpr int NUM_THREADS = 32 * (2 + 4 * DQ_GROUPS + 4);  // producer, MMA, dequant groups, epilogue
constexpr uint32_t kIdescTc = make_idesc(BN, BT);

// UG = 128-k groups per unit (2 when k/128 is even: one TMA box each for codes, meta and
// activations per 256 k, halving the per-byte issue overhead of the single producer thread)
template <int BITS, int UG>
struct DCfg {
  static constexpr int S_W = BITS == 16 ? 4 : (BITS == 8 ? 4 : (UG == 2 ? 6 : 10));
  static constexpr int S_A = UG == 2 ? 2 : 4;  // TMEM A slots of 64*UG columns
  static constexpr int S_X = UG == 2 ? 4 : 8;  // activation ring, in units
};

template <int BITS, int UG>
struct DSmem {
  static constexpr int S_W = DCfg<BITS, UG>::S_W;
  static constexpr int S_X = DCfg<BITS, UG>::S_X;
  static constexpr int X_STAGE = 2 * UG * X_BLOCK;
  static constexpr int W_STAGE = ((BN * GCfg<BITS>::GB * UG + 1023) / 1024) * 1024;
  static constexpr int OFF_X = 0;
  static constexpr int OFF_W = OFF_X + S_X * X_STAGE;
  static constexpr int OFF_META = OFF_W + S_W * W_STAGE;
  static constexpr int OFF_BAR = OFF_META + S_W * BN * 4 * UG;
  static constexpr int NUM_BARS = 2 * S_X + 2 * S_W + 2 * DCfg<BITS, UG>::S_A + 4;
  static constexpr int OFF_MISC = OFF_BAR + NUM_BARS * 8;
  static constexpr int BYTES = OFF_MISC + 64 + 1024;
};

struct TcP {
  const uint8_t* packed;
  const uint32_t* meta;
  const __half* bias;
  void* y;
  int ldy;
  int m;
  int n;
  int kg;
  int U;      // units = (n / 128) * (kg / UG)
  float* part;  // [CTAs][2][32 tokens][128 rows]
  int* cnt;     // [n / 128]
  unsigned long long* trace;  // debug: CTA 0 per-unit clock64 events (sq_debug_trace), or null
};

__device__ __forceinline__ void trace_ev(const TcP& p, int ev, int i) {
  if (p.trace && blockIdx.x == 0 && i < 256) p.trace[ev * 256 + i] = clock64();
}

__device__ __forceinline__ int rlo(int i, int total, int parts) { return (int)(((long long)i * total) / parts); }

template <int EPI>
__device__ __forceinline__ void epi_store(const TcP& p, int64_t row, const float (&v)[BT], float bias) {
#pragma unroll
  for (int t = 0; t < BT; ++t) {
    if (t < p.m) {
      const float o = v[t] + bias;
      if constexpr (EPI == SQ_EPI_F32_ACCUM) {
        float* yp = static_cast<float*>(p.y) + (int64_t)t * p.ldy + row;
        *yp += o;
      } else {
        static_cast<__half*>(p.y)[(int64_t)t * p.ldy + row] = __float2half_rn(apply_act<EPI>(o));
      }
    }
  }
}

template <int BITS, int UG, int EPI>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    k_gemv_tc(const __grid_constant__ CUtensorMap tm_x, const __grid_constant__ CUtensorMap tm_w,
              const __grid_constant__ CUtensorMap tm_m, const TcP p) {
  using SM = DSmem<BITS, UG>;
  constexpr int S_W = SM::S_W;
  constexpr int S_A = DCfg<BITS, UG>::S_A;
  static_assert(S_W % DQ_GROUPS == 0 && S_A % DQ_GROUPS == 0, "slots must not be shared by dequant groups");
  constexpr int S_X = SM::S_X;
  constexpr int X_STAGE = SM::X_STAGE;
  constexpr int GB = GCfg<BITS>::GB;
  constexpr uint32_t W_BYTES = BN * GB * UG;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SM::OFF_BAR);
  uint64_t* full_x = bars;
  uint64_t* empty_x = full_x + S_X;
  uint64_t* full_w = empty_x + S_X;
  uint64_t* empty_w = full_w + S_W;
  uint64_t* full_a = empty_w + S_W;
  uint64_t* empty_a = full_a + S_A;
  uint64_t* d_full = empty_a + S_A;   // [2]
  uint64_t* d_empty = d_full + 2;     // [2]
  uint32_t* misc = reinterpret_cast<uint32_t*>(smem + SM::OFF_MISC);  // [0] tmem base, [1..2] fixup flags

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int kg = p.kg / UG;  // units per row tile
  const int C0 = rlo(blockIdx.x, p.U, gridDim.x), C1 = rlo(blockIdx.x + 1, p.U, gridDim.x);
  const int nunits = C1 - C0;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S_X; ++i) { mbar_init(&full_x[i], 1); mbar_init(&empty_x[i], 1); }
    for (int i = 0; i < S_W; ++i) { mbar_init(&full_w[i], 1); mbar_init(&empty_w[i], 4); }
    for (int i = 0; i < S_A; ++i) { mbar_init(&full_a[i], 4); mbar_init(&empty_a[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&d_full[i], 1); mbar_init(&d_empty[i], 4); }
    fence_barrier_init();
    prefetch_tmap(&tm_x);
    prefetch_tmap(&tm_w);
    if constexpr (BITS != 16) prefetch_tmap(&tm_m);
  }
  if (warp == 1) tmem_alloc(misc, TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = misc[0];

  if (warp == 0) {
    // ---------------- producer: weights (+meta) and the activation slice of every unit
    {  // whole warp runs the loop (warp-uniform operands live in uniform registers); a leader issues
      for (int i = 0; i < nunits; ++i) {
        const int u = C0 + i, rt = u / kg, g = (u - rt * kg) * UG;  // first 128-k group of the unit
        const int sw = i % S_W, rw = i / S_W;
        mbar_wait(&empty_w[sw], (rw & 1) ^ 1);
        trace_ev(p, 0, i);
        uint8_t* wdst = smem + SM::OFF_W + sw * SM::W_STAGE;
        if (elect_one()) mbar_arrive_expect_tx(&full_w[sw], W_BYTES + (BITS != 16 ? BN * 4 * UG : 0));
        if constexpr (BITS == 16) {
          if (elect_one()) tma_load_2d(wdst, &tm_w, &full_w[sw], g * 128, rt * BN);
          if (elect_one()) tma_load_2d(wdst + BN * 128, &tm_w, &full_w[sw], g * 128 + 64, rt * BN);
        } else {
          // placement T16: box {GB bytes, 16 rows, UG groups, 8 row tiles} -> [tile][group][16][GB]
          if (elect_one()) tma_load_4d(wdst, &tm_w, &full_w[sw], 0, 0, g, rt * (BN / 16));
          trace_ev(p, 6, i);
          if (elect_one()) tma_load_3d(smem + SM::OFF_META + sw * BN * 4 * UG, &tm_m, &full_w[sw], 0, g, rt * (BN / 16));
          trace_ev(p, 7, i);
        }
        {
          const int sx = i % S_X, rx = i / S_X;
          mbar_wait(&empty_x[sx], (rx & 1) ^ 1);
          if (elect_one()) mbar_arrive_expect_tx(&full_x[sx], X_STAGE);
          // activations: box {64 k, 32 tokens, 2*UG k-blocks} -> 2*UG SW128 tiles [32][64]
          if (elect_one()) tma_load_3d(smem + SM::OFF_X + sx * X_STAGE, &tm_x, &full_x[sx], 0, 0, g * 2);
          trace_ev(p, 8, i);
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer
    {  // whole warp runs the loop; the elected leader issues tcgen05.mma / commit
      int seg = 0, dbuf = 0;
      for (int i = 0; i < nunits; ++i) {
        const int u = C0 + i, g = u % kg;
        const bool seg_first = (i == 0) || g == 0;
        const bool seg_last = (i == nunits - 1) || g == kg - 1;
        if (seg_first) {
          dbuf = seg & 1;
          mbar_wait(&d_empty[dbuf], ((seg >> 1) & 1) ^ 1);
          tc_fence_after();
        }
        const int sa = i % S_A, ra = i / S_A;
        mbar_wait(&full_a[sa], ra & 1);
        trace_ev(p, 3, i);
        tc_fence_after();
        {
          const int sx = i % S_X, rx = i / S_X;
          mbar_wait(&full_x[sx], rx & 1);
          trace_ev(p, 10, i);
          tc_fence_after();
          const uint32_t xs = smem_u32(smem + SM::OFF_X + sx * X_STAGE);
#pragma unroll
          for (int kk = 0; kk < 8 * UG; ++kk) {
            const uint64_t bdesc = make_sw128_desc(xs + (kk >> 2) * X_BLOCK + (kk & 3) * 32);
            const uint32_t a_tm = tmem + A_COL + sa * 64 * UG + kk * 8;
            if (elect_one()) tc_mma_ts(tmem + D_COL + dbuf * BT, a_tm, bdesc, kIdescTc, (seg_first && kk == 0) ? 0u : 1u);
          }
          trace_ev(p, 11, i);
          if (elect_one()) tc_commit(&empty_x[sx]);
        }
        if (elect_one()) tc_commit(&empty_a[sa]);
        trace_ev(p, 4, i);
        if (seg_last) {
          if (elect_one()) tc_commit(&d_full[dbuf]);
          ++seg;
        }
      }
    }
  } else if (warp < 2 + 4 * DQ_GROUPS) {
    // ---------------- dequant warps: one thread per weight row; group gi takes units i = gi (mod 2)
    const int sp = warp & 3;
    const int gi = (warp - 2) >> 2;
    const int r = sp * 32 + lane;
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    for (int i = gi; i < nunits; i += DQ_GROUPS) {
      const int sw = i % S_W, rw = i / S_W;
      const int sa = i % S_A, ra = i / S_A;
      mbar_wait(&full_w[sw], rw & 1);
      if (threadIdx.x == 64) trace_ev(p, 1, i);
      mbar_wait(&empty_a[sa], (ra & 1) ^ 1);
      if (threadIdx.x == 64) trace_ev(p, 5, i);
      tc_fence_after();
#pragma unroll
      for (int gg = 0; gg < UG; ++gg) {
        // stage layout [tile][group][16 rows]: row r of group gg
        const int ru = ((r >> 4) * UG + gg) * 16 + (r & 15);
        const uint32_t meta = reinterpret_cast<const uint32_t*>(smem + SM::OFF_META + sw * BN * 4 * UG)[ru];
        dequant_row_to_tmem<BITS>(smem + SM::OFF_W + sw * SM::W_STAGE, meta, r,
                                  tmem + lane_base + A_COL + sa * 64 * UG + gg * 64, ru * GB);
      }
      tc_wait_st();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&empty_w[sw]);
        mbar_arrive(&full_a[sa]);
      }
      if (threadIdx.x == 64 || threadIdx.x == 64 + 128) trace_ev(p, 2, i);
    }
  } else {
    // ---------------- epilogue warps: drain finished segments
    const int sp = warp & 3;
    const int r = sp * 32 + lane;
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    int seg = 0;
    int i = 0;
    while (i < nunits) {
      const int u0 = C0 + i, rt = u0 / kg, g0 = u0 - rt * kg;
      const int len = (kg - g0) < (nunits - i) ? (kg - g0) : (nunits - i);
      const bool full = (g0 == 0) && (len == kg);
      const int dbuf = seg & 1;
      mbar_wait_sleepy(&d_full[dbuf], (seg >> 1) & 1);
      tc_fence_after();
      float v[BT];
      {
        uint32_t a[16], b[16];
        tmem_ld16(tmem + lane_base + D_COL + dbuf * BT, a);
        tmem_ld16(tmem + lane_base + D_COL + dbuf * BT + 16, b);
        tc_wait_ld();
#pragma unroll
        for (int t = 0; t < 16; ++t) { v[t] = __uint_as_float(a[t]); v[16 + t] = __uint_as_float(b[t]); }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(&d_empty[dbuf]);
      const int64_t row = (int64_t)rt * BN + r;
      const float bias = p.bias ? __half2float(p.bias[row]) : 0.f;
      if (full) {
        epi_store<EPI>(p, row, v, bias);
      } else {
        // partial tile: publish, the last contributing CTA reduces in fixed CTA order
        const int slot = (C0 < rt * kg) ? 1 : 0;
        float* gp = p.part + (((int64_t)blockIdx.x * 2 + slot) * BT) * BN;
#pragma unroll
        for (int t = 0; t < BT; ++t) __stcg(gp + t * BN + r, v[t]);
        __threadfence();
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (threadIdx.x == (2 + 4 * DQ_GROUPS) * 32) {
          const int NC = gridDim.x;
          const int ca = (int)(((long long)(rt * kg + 1) * NC - 1) / p.U);
          const int cb = (int)(((long long)((rt + 1) * kg) * NC - 1) / p.U);
          const int old = atomicAdd(p.cnt + rt, 1);
          misc[1] = (old == cb - ca) ? 1u : 0u;
          misc[2] = (uint32_t)ca;
          misc[3] = (uint32_t)cb;
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (misc[1]) {
          __threadfence();
          const int ca = (int)misc[2], cb = (int)misc[3];
#pragma unroll
          for (int t = 0; t < BT; ++t) v[t] = 0.f;
          for (int c = ca; c <= cb; ++c) {
            const int sl = (rlo(c, p.U, gridDim.x) < rt * kg) ? 1 : 0;
            const float* qp = p.part + (((int64_t)c * 2 + sl) * BT) * BN;
#pragma unroll
            for (int t = 0; t < BT; ++t) v[t] += __ldcg(qp + t * BN + r);
          }
          epi_store<EPI>(p, row, v, bias);
          if (threadIdx.x == (2 + 4 * DQ_GROUPS) * 32) p.cnt[rt] = 0;
        }
        asm volatile("bar.sync 1, 128;" ::: "memory");  // misc[] reuse
      }
      ++seg;
      i += len;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, TMEM_COLS);
  }
}

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

cudaError_t enc(CUtensorMap* m, CUtensorMapDataType dt, const void* ptr, int rank, const uint64_t* dims,
                const uint64_t* strides, const uint32_t* box, CUtensorMapSwizzle sw) {
  static EncodeFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return cudaErrorNotSupported;
    fn = reinterpret_cast<EncodeFn>(f);
  }
  cuuint64_t d[5], st[4];
  cuuint32_t b[5], es[5];
  for (int i = 0; i < rank; ++i) { d[i] = dims[i]; b[i] = box[i]; es[i] = 1; }
  for (int i = 0; i + 1 < rank; ++i) st[i] = strides[i];
  CUresult r = fn(m, dt, (cuuint32_t)rank, const_cast<void*>(ptr), d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS ? cudaSuccess : cudaErrorInvalidValue;
}

template <int BITS, int UG, int EPI>
cudaError_t launch_tc_be(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const TcP& p, int nc,
                         cudaStream_t s) {
  auto kern = k_gemv_tc<BITS, UG, EPI>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, DSmem<BITS, UG>::BYTES);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  kern<<<nc, NUM_THREADS, DSmem<BITS, UG>::BYTES, s>>>(tx, tw, tm, p);
  return cudaGetLastError();
}

template <int BITS, int UG>
cudaError_t launch_tc_u(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const TcP& p, int epi,
                        int nc, cudaStream_t s) {
  switch (epi) {
    case SQ_EPI_F16: return launch_tc_be<BITS, UG, SQ_EPI_F16>(tx, tw, tm, p, nc, s);
    case SQ_EPI_F16_RELU: return launch_tc_be<BITS, UG, SQ_EPI_F16_RELU>(tx, tw, tm, p, nc, s);
    case SQ_EPI_F16_GELU: return launch_tc_be<BITS, UG, SQ_EPI_F16_GELU>(tx, tw, tm, p, nc, s);
    default: return launch_tc_be<BITS, UG, SQ_EPI_F32_ACCUM>(tx, tw, tm, p, nc, s);
  }
}

template <int BITS>
cudaError_t launch_tc_b(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const TcP& p, int epi,
                        int nc, int ug, cudaStream_t s) {
  if constexpr (BITS != 16) {
    if (ug == 2) return launch_tc_u<BITS, 2>(tx, tw, tm, p, epi, nc, s);
  }
  return launch_tc_u<BITS, 1>(tx, tw, tm, p, epi, nc, s);
}

unsigned long long* g_trace = nullptr;

int tc_ctas(int64_t U) {
  const int64_t full = num_sms();
  return (int)(U < full ? U : full);
}

}  // namespace

// The counter region is the SAME fixed 16-KB region the mma.sync path uses (counters of every
// launch self-reset to 0, so consecutive linears of any n can share one workspace).
constexpr size_t kCntBytes = (65536 / 16) * sizeof(int);

size_t gemv_tc_workspace_bytes(int64_t n, int64_t k) {
  const int64_t U = (n / BN) * (k / 128);
  return kCntBytes + (size_t)tc_ctas(U) * 2 * BT * BN * sizeof(float) + 256;
}

cudaError_t launch_gemv_tc(const sq_qweight& w, const __half* x, int64_t ldx, int m, void* y, int64_t ldy, int epi,
                           void* ws, cudaStream_t s) {
  CUtensorMap tx, tw, tm;
  memset(&tm, 0, sizeof(tm));
  const int kg = (int)(w.k / 128);
  const int ug = (w.bits != 16 && kg % 2 == 0) ? 2 : 1;
  {
    // activations as [k/64][m][64]: one box {64, 32, 2*ug} per unit -> 2*ug SW128 tiles [32 tokens][64 k]
    const uint64_t dx[3] = {64, (uint64_t)m, (uint64_t)w.k / 64}, sx[2] = {(uint64_t)ldx * 2, 128};
    const uint32_t bx[3] = {XK, BT, (uint32_t)(2 * ug)};
    cudaError_t e = enc(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, x, 3, dx, sx, bx, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return e;
  }
  if (w.bits == 16) {
    const uint64_t dw[2] = {(uint64_t)w.k, (uint64_t)w.n}, sw_[1] = {(uint64_t)w.k * 2};
    const uint32_t bw[2] = {64, BN};
    cudaError_t e = enc(&tw, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, w.packed, 2, dw, sw_, bw, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return e;
  } else {
    const uint64_t gb = 128 * w.bits / 8, nt = (uint64_t)w.n / 16;
    CUtensorMapSwizzle sw = w.bits == 8 ? CU_TENSOR_MAP_SWIZZLE_128B
                                        : (w.bits == 4 ? CU_TENSOR_MAP_SWIZZLE_64B : CU_TENSOR_MAP_SWIZZLE_NONE);
    const uint64_t dw[4] = {gb, 16, kg, nt}, sw_[3] = {gb, 16 * gb, kg * 16 * gb};
    const uint32_t bw[4] = {(uint32_t)gb, 16, (uint32_t)ug, BN / 16};
    cudaError_t e = enc(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, w.packed, 4, dw, sw_, bw, sw);
    if (e != cudaSuccess) return e;
    const uint64_t dm[3] = {16, kg, nt}, sm_[2] = {64, kg * 64};
    const uint32_t bm[3] = {16, (uint32_t)ug, BN / 16};
    e = enc(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, w.meta, 3, dm, sm_, bm, CU_TENSOR_MAP_SWIZZLE_NONE);
    if (e != cudaSuccess) return e;
  }
  TcP p{};
  p.packed = static_cast<const uint8_t*>(w.packed);
  p.meta = static_cast<const uint32_t*>(w.meta);
  p.bias = static_cast<const __half*>(w.bias);
  p.y = y;
  p.ldy = (int)ldy;
  p.m = m;
  p.n = (int)w.n;
  p.kg = kg;
  p.U = (int)((w.n / BN) * (kg / ug));
  uint8_t* base = static_cast<uint8_t*>(ws);
  p.cnt = reinterpret_cast<int*>(base);
  p.part = reinterpret_cast<float*>(base + kCntBytes);
  p.trace = g_trace;
  const int nc = tc_ctas(p.U);
  const double bytes = (double)w.n * w.k * w.bits / 8.0 + (w.bits != 16 ? (double)w.n * (w.k / 128) * 4.0 : 0.0);
  auto t = prof_begin(KC_GEMV, bytes, 2.0 * m * w.n * w.k, s);
  cudaError_t e;
  switch (w.bits) {
    case 3: e = launch_tc_b<3>(tx, tw, tm, p, epi, nc, ug, s); break;
    case 4: e = launch_tc_b<4>(tx, tw, tm, p, epi, nc, ug, s); break;
    case 8: e = launch_tc_b<8>(tx, tw, tm, p, epi, nc, ug, s); break;
    default: e = launch_tc_b<16>(tx, tw, tm, p, epi, nc, 1, s); break;
  }
  prof_end(t, s);
  count_launch();
  return e;
}

}  // namespace sq

// debug only (not part of include/sq.h): record CTA 0's per-unit clock64 events of the
// tcgen05 decode kernel into a device buffer of 14 x 256 uint64 (tools/trace_tc.py)
extern "C" void sq_debug_trace(void* dev_buf) { sq::g_trace = static_cast<unsigned long long*>(dev_buf); }
