// K2c — decode dequant-GEMV on tcgen05 for micro-batches of up to 32 tokens
// (the pipeline's decode micro-batch xi = 32).  At 32 tokens a
// decode linear does 64 flop per weight; legacy mma.sync tops out near
// 535 TFLOP/s on B200 (measured), below HBM speed at INT4, so the contraction
// moves to the 5th-generation tensor cores:
//
//  * Unit = 128 weight rows x UG groups (UG*128 k): one MMA M-tile.  Units are
//    grouped in PANELS of P <= 4 row tiles that share every activation slice
//    [32 tokens x UG*128 k] (fetched once per P units): a TMA stream ingests
//    ~45 GB/s per SM whether it hits L2 or HBM (measured, tools/mb_tma.cu), so
//    activation bytes cost as much as weight bytes.
//  * Work item = (panel, k-slice z < Z): the panel's k range is split in Z even
//    slices.  (P, Z) are chosen per shape on the host to minimise the bytes the
//    busiest SM ingests (weights + activations + partial sums) with about one
//    item per SM (tc_plan).
//  * Producer warp: per unit one 4-D TMA box of packed codes and one 3-D box of
//    meta; per k-step one 3-D box of activations (tokens >= m zero-filled),
//    issued one step behind the weights (it is only needed at MMA time).
//  * 16 dequant warps (thread = weight row, warp = a quarter of the unit's k):
//    magic-number unpack, w~ = s*c + z in fp16 (HSUB2 + HFMA2), tcgen05.st into
//    TMEM A slot i % 3 while the MMA reads the others.
//  * MMA warp: tcgen05.mma kind::f16, M = 128 rows, N = 32 tokens, K = 16, A
//    from TMEM, B (activations) from SMEM; fp32 accumulators of the panel's P
//    tiles in TMEM (P x 32 columns).
//  * 4 epilogue warps drain an item: Z = 1 -> bias / activation / fp32 residual
//    straight to y; Z > 1 (one item per CTA) -> the panel's Z CTAs form a
//    thread-block cluster, each leaves its fp32 partial in its own shared memory
//    and CTA z reduces 1/Z of the panel over the cluster through DSMEM in fixed z
//    order.  When the clusters cannot all be resident, the partials go to the
//    workspace instead and the grid is launched cooperatively (co-resident by
//    construction): every CTA waits for its panel's Z partials, then reduces its
//    1/Z share in fixed z order.  Deterministic; counters self-reset.
// Warp roles: 0 producer, 1 MMA (+TMEM alloc), 2..17 dequant, 18..21 epilogue.
#include <cuda.h>

#include <cstdlib>
#include <cstdio>
#include <cstring>

#include "sq_tc.cuh"

namespace sq {
namespace {
using namespace tc;

// barrier waits: try_wait with a suspend-time hint (measured equal to spinning try_wait / test_wait)
__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t parity) { mbar_wait_park(bar, parity); }

constexpr int BN = 128;     // weight rows per unit (TMEM lanes, MMA M)
constexpr int BT = 32;      // token columns (MMA N)
constexpr int PMAX = 4;     // row tiles per panel (activation reuse), at most
constexpr int kCnt2 = 2048;  // second per-panel counter (fix-up done) at cnt + kCnt2
constexpr int XK = 64;
constexpr int X_BLOCK = BT * XK * 2;  // 4 KB: [32 tokens][64 k] SW128 tile
// Dequant warps: 16, in two alternating groups of 8 (4 lane quadrants x 2 k-halves of a unit).
// Measured on OPT-13B/66B shapes (INT3/4/8, m = 32): one group of 16 -> 6-18 % slower, 8 warps
// -> 5-25 % slower, group-granular TMEM A slots with 4 quads of 4 warps -> 5-12 % slower; the
// warps are issue-bound on the unpack, and two units in flight hide the MMA / slot hand-off best.
constexpr int DQ_WARPS = 16;      // dequant warps, in DQ_GROUPS groups of DQ_PER_GROUP
constexpr int DQ_PER_GROUP = 8;   // 4 lane quadrants x KH k-parts of one unit
constexpr int DQ_KH = DQ_PER_GROUP / 4;
constexpr int DQ_GROUPS = DQ_WARPS / DQ_PER_GROUP;  // group q dequantizes units i = q (mod DQ_GROUPS)
constexpr int TMEM_COLS = 512;
constexpr int D_COL = 0;              // P x 32 columns: the panel's accumulators
constexpr int A_COL = PMAX * BT;      // S_A x (64 * UG) columns
constexpr int NUM_THREADS = 32 * (2 + DQ_WARPS + 4);  // producer, MMA, dequant, epilogue
constexpr int EPI_WARP0 = 2 + DQ_WARPS;
constexpr uint32_t kIdescTc = make_idesc(BN, BT);

// UG = 128-k groups per unit, chosen so a weight stage is ~16 KB (INT3/INT4: 2, INT8: 1).
template <int BITS, int UG>
struct DCfg {
  // weight ring: a slot lives TMA latency (~1.8k cycles) + wait for its group + dequant (~2k)
  // (quantized rings are multiples of DQ_GROUPS so each slot is owned by one dequant group)
  static constexpr int S_W0 = UG == 3 ? 6 : (UG == 2 ? 10 : (BITS == 8 ? 10 : (BITS == 4 ? 18 : 24)));
  static constexpr int S_W = BITS == 16 ? 5 : (S_W0 / DQ_GROUPS) * DQ_GROUPS;
  // TMEM A slots of 64*UG columns: the dequant warps fill slot i % S_A while the MMA reads the
  // others (slots are owned by one dequant group: multiples of DQ_GROUPS)
  static constexpr int A_SLOT = 64 * UG;
  static constexpr int S_A = UG == 3 ? 2 : (UG == 2 ? 3 : 6);
  static constexpr int S_X = 3;  // activation ring, in steps
  static_assert(BITS == 16 || A_COL + S_A * A_SLOT <= TMEM_COLS, "TMEM budget");
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
  static constexpr int OFF_BAR = OFF_META + (BITS == 16 ? 0 : S_W * BN * 4 * UG);
  static constexpr int NUM_BARS = 2 * S_X + 2 * S_W + 2 * DCfg<BITS, UG>::S_A + 2;
  static constexpr int OFF_MISC = OFF_BAR + NUM_BARS * 8;
  static constexpr int BYTES = OFF_MISC + 256 + 1024;  // misc: tmem base, pending panels (<= 62)
  static_assert(BYTES <= 227 * 1024, "shared memory budget");

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
  int nt;     // row tiles (n / 128)
  int ks;     // k-steps per row (kg / UG)
  int P;      // row tiles per panel (1..4)
  int Z;      // k slices per panel
  int I;      // work items = panels * Z
  float* part;  // [items][PMAX tiles][32 tokens][128 rows] fp32 partial sums (Z > 1)
  int* cnt;     // [panels]
  unsigned long long* trace;  // debug build (SQ_TC_DEBUG): CTA 0 per-unit clock64 events (sq_debug_trace), or null
  int cl;                     // Z > 1 items of a panel form a thread-block cluster: DSMEM reduction
};

__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// address of the same shared-memory byte in cluster CTA `rank`
__device__ __forceinline__ uint32_t dsmem_addr(uint32_t local, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(local), "r"(rank));
  return r;
}
__device__ __forceinline__ float4 ld_dsmem_f4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr) : "memory");
  return v;
}

#ifndef SQ_TC_DEBUG
#define SQ_TC_DEBUG 0  // 1: clock64 trace (sq_debug_trace) and the SQ_TC_PZ plan override compiled in
#endif
__device__ __forceinline__ void trace_ev(const TcP& p, int ev, int i) {
  if (SQ_TC_DEBUG && p.trace && blockIdx.x == 0 && i < 256) p.trace[ev * 256 + i] = clock64();
}

__device__ __forceinline__ void trace_cta(const TcP& p, int ev) {
  if (SQ_TC_DEBUG && p.trace && blockIdx.x < 256) {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    p.trace[ev * 256 + blockIdx.x] = t;
  }
}


// Segments of this warp's k-part kh of a unit: batches [kh * NBW, (kh + 1) * NBW) of the unit's
// 4 * UG 32-k batches, split at 128-k group boundaries (one meta word per group).  Compile-time segment
// lists (a runtime batch count cost 4-9 % on INT3/INT4), and ONE warp vote per unit for the
// saturating variant (R20) instead of one per segment.
template <int BITS, int UG, int NBW, bool SAT, int KH>
__device__ __forceinline__ void dequant_part(const uint8_t* wst, const uint32_t* mt, int r, uint32_t a_tm) {
  constexpr int GB = GCfg<BITS>::GB;
#pragma unroll
  for (int g = 0; g < UG; ++g) {
    constexpr int b = KH * NBW, e = KH * NBW + NBW;
    const int lo = g * 4 > b ? g * 4 : b, hi = (g + 1) * 4 < e ? (g + 1) * 4 : e;  // constant after unrolling
    if (lo >= hi) continue;
    const int ru = ((r >> 4) * UG + g) * 16 + (r & 15);  // stage layout [tile][group][16 rows]
    const uint32_t m = mt[ru];
    const uint32_t at = a_tm + g * 64;
    if (hi - lo == 4) dequant_row_batches_<BITS, 4, SAT>(wst, m, r, at, ru * GB, lo - g * 4);
    else if (hi - lo == 3) dequant_row_batches_<BITS, 3, SAT>(wst, m, r, at, ru * GB, lo - g * 4);
    else if (hi - lo == 2) dequant_row_batches_<BITS, 2, SAT>(wst, m, r, at, ru * GB, lo - g * 4);
    else dequant_row_batches_<BITS, 1, SAT>(wst, m, r, at, ru * GB, lo - g * 4);
  }
}
template <int BITS, int UG, int NBW, int KH>
__device__ __forceinline__ bool part_may_overflow(const uint32_t* mt, int r) {
  bool any = false;
#pragma unroll
  for (int g = 0; g < UG; ++g) {
    constexpr int b = KH * NBW, e = KH * NBW + NBW;
    if (g * 4 >= e || (g + 1) * 4 <= b) continue;
    any |= group_may_overflow<BITS>(mt[((r >> 4) * UG + g) * 16 + (r & 15)]);
  }
  return any;
}
template <int BITS, int UG, int NBW, int KH>
__device__ __forceinline__ void dequant_part_vote(const uint8_t* wst, const uint32_t* mt, int r, uint32_t a_tm) {
  // warp-uniform choice: tcgen05.st is .sync.aligned, so every lane must take the same variant
  if (__builtin_expect(__any_sync(0xffffffffu, part_may_overflow<BITS, UG, NBW, KH>(mt, r)), 0))
    dequant_part<BITS, UG, NBW, true, KH>(wst, mt, r, a_tm);
  else
    dequant_part<BITS, UG, NBW, false, KH>(wst, mt, r, a_tm);
}
template <int BITS, int UG, int NBW, int KHN>
__device__ __forceinline__ void dequant_warp_range(const uint8_t* wst, const uint32_t* mt, int r, uint32_t a_tm, int kh) {
  static_assert(KHN == 2, "two k-parts per unit");
  if (kh == 0) dequant_part_vote<BITS, UG, NBW, 0>(wst, mt, r, a_tm);
  else dequant_part_vote<BITS, UG, NBW, 1>(wst, mt, r, a_tm);
}

template <int EPI>
__device__ __forceinline__ void epi_store(const TcP& p, int64_t row, const float (&v)[BT], float bias) {
  if constexpr (EPI == SQ_EPI_F32_ACCUM) {
    // residual read-modify-write: every load before any store (no per-token L2 round trip chain)
    float* yb = static_cast<float*>(p.y) + row;
#pragma unroll
    for (int h = 0; h < BT; h += 16) {
      float r[16];
#pragma unroll
      for (int t = 0; t < 16; ++t) r[t] = h + t < p.m ? __ldcg(yb + (int64_t)(h + t) * p.ldy) : 0.f;
#pragma unroll
      for (int t = 0; t < 16; ++t)
        if (h + t < p.m) yb[(int64_t)(h + t) * p.ldy] = r[t] + (v[h + t] + bias);
    }
  } else {
#pragma unroll
    for (int t = 0; t < BT; ++t)
      if (t < p.m) static_cast<__half*>(p.y)[(int64_t)t * p.ldy + row] = __float2half_rn(apply_act<EPI>(v[t] + bias));
  }
}

template <int BITS, int UG, int EPI>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    k_gemv_tc(const __grid_constant__ CUtensorMap tm_x, const __grid_constant__ CUtensorMap tm_w,
              const __grid_constant__ CUtensorMap tm_m, const TcP p) {
  using SM = DSmem<BITS, UG>;
  constexpr int S_W = SM::S_W;
  constexpr int S_A = DCfg<BITS, UG>::S_A;
  constexpr int S_X = SM::S_X;
  constexpr int X_STAGE = SM::X_STAGE;
  constexpr int GB = GCfg<BITS>::GB;
  constexpr uint32_t W_BYTES = BN * GB * UG + (BITS == 16 ? 0 : BN * 4 * UG);  // codes + meta of one unit
  constexpr int LPU = BITS == 3 ? 3 : (BITS == 4 ? 8 : 16);  // TMA lines per T16 unit (wlines)
  extern __shared__ uint8_t smem_raw[];
  // 1-KB aligned (SW128 atoms); pointer arithmetic on smem_raw keeps the shared address space
  // visible to the compiler (LDS, not generic LD)
  uint8_t* smem = smem_raw + ((1024u - (smem_u32(smem_raw) & 1023u)) & 1023u);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + SM::OFF_BAR);
  uint64_t* full_x = bars;
  uint64_t* empty_x = full_x + S_X;
  uint64_t* full_w = empty_x + S_X;
  uint64_t* empty_w = full_w + S_W;
  uint64_t* full_a = empty_w + S_W;
  uint64_t* empty_a = full_a + S_A;
  uint64_t* d_full = empty_a + S_A;
  uint64_t* d_empty = d_full + 1;
  uint32_t* misc = reinterpret_cast<uint32_t*>(smem + SM::OFF_MISC);  // [0] tmem base, [1] #pending, [2..] panels

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int ks = p.ks, C = gridDim.x, P = p.P, Z = p.Z, I = p.I;
  const int last_panel = (p.nt - 1) / P, p_last = p.nt - last_panel * P;  // tiles in the last panel
  auto tiles_of = [&](int pn) { return pn == last_panel ? p_last : P; };
  // item it = (panel it / Z, k-steps [j0, j1) of slice it % Z)
  auto j0_of = [&](int it) { return (int)((long long)(it % Z) * ks / Z); };
  auto j1_of = [&](int it) { return (int)((long long)(it % Z + 1) * ks / Z); };

  if (threadIdx.x == 0) {
    for (int i = 0; i < S_X; ++i) { mbar_init(&full_x[i], 1); mbar_init(&empty_x[i], 1); }
    // fp16 weights are the MMA's A operand straight from SMEM: the MMA commit frees the slot
    for (int i = 0; i < S_W; ++i) { mbar_init(&full_w[i], 1); mbar_init(&empty_w[i], BITS == 16 ? 1 : DQ_PER_GROUP); }
    for (int i = 0; i < S_A; ++i) { mbar_init(&full_a[i], DQ_PER_GROUP); mbar_init(&empty_a[i], 1); }
    mbar_init(d_full, 1);
    mbar_init(d_empty, 4);
    misc[1] = 0;
    fence_barrier_init();
    prefetch_tmap(&tm_x);
    prefetch_tmap(&tm_w);
    if constexpr (BITS != 16) prefetch_tmap(&tm_m);
  }
  pdl_trigger();  // the next kernel may be scheduled as soon as SMs free up
  constexpr int LPU_ = BITS == 3 ? 3 : (BITS == 4 ? 8 : 16);
  // TMA of weight unit i (panel pn, tile t, k-step j) into ring slot i % S_W; one thread
  auto issue_w1 = [&](int i, int pn, int t, int j) {
    const int sw = i % S_W;
    const int tile16 = (pn * P + t) * (BN / 16);
    uint8_t* wdst = smem + SM::OFF_W + sw * SM::W_STAGE;
    mbar_arrive_expect_tx(&full_w[sw], BITS == 16 ? BN * 256u : (uint32_t)(BN * GCfg<BITS>::GB * UG + BN * 4 * UG));
    if constexpr (BITS == 16) {
      // row-major fp16 [n][k]: two SW128 boxes [128 rows][64 k] = the MMA's K-major A tiles
      tma_load_2d(wdst, &tm_w, &full_w[sw], j * 128, (pn * P + t) * BN);
      tma_load_2d(wdst + BN * 128, &tm_w, &full_w[sw], j * 128 + 64, (pn * P + t) * BN);
    } else {
      // placement T16 as lines: box {line, lpu * UG lines, 8 row tiles} -> [tile][group][16][GB]
      tma_load_3d(wdst, &tm_w, &full_w[sw], 0, j * UG * LPU_, tile16);
      tma_load_2d(smem + SM::OFF_META + sw * BN * 4 * UG, &tm_m, &full_w[sw], j * UG * 16, tile16);
    }
  };
  // PDL: weights never depend on the previous kernel -- thread 0 fills the whole weight ring right
  // after the barrier init, before the other warps are released (a producer warp sharing its SMSP
  // with waiting warps issued only ~1 unit per 0.4 us here, measured)
  int pre = 0;
  if (warp == 0) {
    for (int it = blockIdx.x; it < I && pre < S_W; it += C) {
      const int pn = it / Z, j1 = j1_of(it), pp = tiles_of(pn);
      for (int j = j0_of(it); j < j1 && pre < S_W; ++j)
        for (int t = 0; t < pp && pre < S_W; ++t, ++pre)
          if (lane == 0) issue_w1(pre, pn, t, j);
    }
  }
  if (warp == 1) tmem_alloc(misc, TMEM_COLS);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (misc[0] != 0) __trap();  // a 512-column allocation owns all of TMEM: base is lane 0, column 0
  constexpr uint32_t tmem = 0;
  if (threadIdx.x == 0) { trace_cta(p, 14); trace_ev(p, 13, 0); }

  if (warp == 0) {
    // ---------------- producer.  The warp runs the loop and the waits; one elected lane issues.
    int i = 0, qx = 0;  // units issued, k-steps issued (activations)
    auto issue_x = [&](int j) {
      const int sx = qx % S_X, rx = qx / S_X;
      wait_bar(&empty_x[sx], (rx & 1) ^ 1);
      if (elect_one()) {
        // box {64 k, 32 tokens, 2*UG k-blocks} -> 2*UG SW128 tiles [32][64]
        mbar_arrive_expect_tx(&full_x[sx], X_STAGE);
        tma_load_3d(smem + SM::OFF_X + sx * X_STAGE, &tm_x, &full_x[sx], 0, 0, j * UG * 2);
      }
      __syncwarp();
      ++qx;
    };
    auto issue_w = [&](int i, int pn, int t, int j) {
      if (elect_one()) issue_w1(i, pn, t, j);
      __syncwarp();
    };
    pdl_wait();
    trace_ev(p, 7, 0);
    for (int it = blockIdx.x; it < I; it += C) {
      const int pn = it / Z, j1 = j1_of(it), pp = tiles_of(pn);
      for (int j = j0_of(it); j < j1; ++j) {
        issue_x(j);  // the step's activation slice, just before its weights
        for (int t = 0; t < pp; ++t, ++i) {
          if (i < pre) continue;
          const int sw = i % S_W, rw = i / S_W;
          wait_bar(&empty_w[sw], (rw & 1) ^ 1);
          trace_ev(p, 0, i);
          issue_w(i, pn, t, j);
          trace_ev(p, 8, i);
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer: the warp waits, one elected lane issues a unit's 8*UG MMAs and
    // commits.  TMEM base is 0, so every operand is warp-uniform.
    int i = 0, q = 0, n_item = 0;
    for (int it = blockIdx.x; it < I; it += C, ++n_item) {
      const int pn = it / Z, j0 = j0_of(it), j1 = j1_of(it), pp = tiles_of(pn);
      wait_bar(d_empty, (n_item & 1) ^ 1);  // the epilogue drained the previous item
      for (int j = j0; j < j1; ++j, ++q) {
        const int sx = q % S_X, rx = q / S_X;
        wait_bar(&full_x[sx], rx & 1);
        trace_ev(p, 6, q);
        const uint64_t bdesc0 = make_sw128_desc(smem_u32(smem + SM::OFF_X + sx * X_STAGE));
        for (int t = 0; t < pp; ++t, ++i) {
          if constexpr (BITS == 16) {
            // A (fp16 weights) straight from the W stage: two SW128 [128 x 64] tiles
            const int sw = i % S_W, rw = i / S_W;
            wait_bar(&full_w[sw], rw & 1);
            tc_fence_after();
            trace_ev(p, 3, i);
            if (elect_one()) {
              const uint32_t d_tm = tmem + D_COL + t * BT;
              const uint64_t adesc0 = make_sw128_desc(smem_u32(smem + SM::OFF_W + sw * SM::W_STAGE));
#pragma unroll
              for (int kk = 0; kk < 8; ++kk) {
                const uint64_t off = (uint64_t)(((kk >> 2) * BN * 128 + (kk & 3) * 32) >> 4);
                const uint64_t boff = (uint64_t)(((kk >> 2) * X_BLOCK + (kk & 3) * 32) >> 4);
                tc_mma_ss(d_tm, adesc0 + off, bdesc0 + boff, kIdescTc, (j == j0 && kk == 0) ? 0u : 1u);
              }
              tc_commit(&empty_w[sw]);
              if (t == pp - 1) {
                tc_commit(&empty_x[sx]);
                if (j == j1 - 1) tc_commit(d_full);
              }
            }
            __syncwarp();
            trace_ev(p, 4, i);
            continue;
          }
          const int sa = i % S_A, ra = i / S_A;
          wait_bar(&full_a[sa], ra & 1);
          tc_fence_after();
          trace_ev(p, 3, i);
          if (elect_one()) {
            const uint32_t d_tm = tmem + D_COL + t * BT;
            const uint32_t a_tm = tmem + A_COL + sa * DCfg<BITS, UG>::A_SLOT;
            // B descriptor as two words: the per-k-step offsets are 32-bit adds on the address word (fewer
            // R2UR moves into the uniform registers UTCHMMA reads; 0-7 % faster, tools/gemv_rot.py --graph on variant builds)
            const uint32_t blo = (uint32_t)bdesc0, bhi = (uint32_t)(bdesc0 >> 32);
#pragma unroll
            for (int kk = 0; kk < 8 * UG; ++kk)
              tc_mma_ts_w(d_tm, a_tm + kk * 8, blo + (uint32_t)(((kk >> 2) * X_BLOCK + (kk & 3) * 32) >> 4), bhi,
                          kIdescTc, (j == j0 && kk == 0) ? 0u : 1u);
            tc_commit(&empty_a[sa]);
            if (t == pp - 1) {
              tc_commit(&empty_x[sx]);
              if (j == j1 - 1) tc_commit(d_full);
            }
          }
          __syncwarp();
          trace_ev(p, 4, i);
        }
      }
    }
  } else if (warp < EPI_WARP0) {
    // ---------------- dequant warps: DQ_GROUPS groups of 8; group dg takes units i = dg (mod
    // DQ_GROUPS).  Thread = weight row (lane quadrant warp % 4); warp kh of the group takes batches
    // [kh*2*UG, kh*2*UG + 2*UG) of the unit's 4*UG 32-k batches.  Slots of both rings are owned by
    // one group (ring depths are multiples of DQ_GROUPS), so phases follow from i alone.
    // (A slots alternate between the groups; in-order MMA completion keeps every waiter within one
    // phase of the slot's barrier)
    static_assert(BITS == 16 || S_W % DQ_GROUPS == 0, "weight ring slots owned by one dequant group");
    int nunits = 0;
    if constexpr (BITS != 16)
      for (int it = blockIdx.x; it < I; it += C) nunits += (j1_of(it) - j0_of(it)) * tiles_of(it / Z);
    constexpr int NBW = 4 * UG / DQ_KH;                      // 32-k batches per warp (may straddle groups)
    static_assert(4 * UG % DQ_KH == 0, "a unit's batches split evenly over the k-parts");
    const int sp = warp & 3;
    const int dg = (warp - 2) / DQ_PER_GROUP;
    const int kh = ((warp - 2) >> 2) % DQ_KH;
    const int r = sp * 32 + lane;
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    const bool tr = (warp == 2 && lane == 0);
    for (int i = dg; i < nunits; i += DQ_GROUPS) {
      const int sw = i % S_W, sa = i % S_A;
      wait_bar(&full_w[sw], (uint32_t)((i / S_W) & 1));
      if (tr) trace_ev(p, 1, i);
      wait_bar(&empty_a[sa], (uint32_t)(((i / S_A) & 1) ^ 1));
      if (tr) trace_ev(p, 5, i);
      tc_fence_after();
      const uint32_t* mt = reinterpret_cast<const uint32_t*>(smem + SM::OFF_META + sw * BN * 4 * UG);
      const uint32_t a_tm = tmem + lane_base + A_COL + sa * DCfg<BITS, UG>::A_SLOT;
      const uint8_t* wst = smem + SM::OFF_W + sw * SM::W_STAGE;
      if constexpr (BITS != 16) dequant_warp_range<BITS, UG, NBW, DQ_KH>(wst, mt, r, a_tm, kh);
      if (tr) trace_ev(p, 12, i);
      tc_wait_st();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&empty_w[sw]);
        mbar_arrive(&full_a[sa]);
      }
      if (tr) trace_ev(p, 2, i);
    }
    // split panels keep their partials in the weight ring: an explicit CTA barrier with the epilogue
    // (on top of the mbarrier chain dequant -> MMA -> d_full) orders this warp's last stage reads first
    if (Z > 1 && p.cl) asm volatile("bar.arrive 2, %0;" :: "r"((DQ_WARPS + 4) * 32) : "memory");
  } else {
    // ---------------- epilogue warps: drain each item's accumulators
    const int sp = warp & 3;
    const int r = sp * 32 + lane;
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    const bool leader = threadIdx.x == EPI_WARP0 * 32;
    int n_item = 0;
    for (int it = blockIdx.x; it < I; it += C, ++n_item) {
      const int pn = it / Z, pp = tiles_of(pn);
      wait_bar(d_full, n_item & 1);
      tc_fence_after();
      if (Z > 1 && p.cl) asm volatile("bar.sync 2, %0;" :: "r"((DQ_WARPS + 4) * 32) : "memory");
      for (int t = 0; t < pp; ++t) {
        float v[BT];
        {
          uint32_t a[16], b[16];
          tmem_ld16(tmem + lane_base + D_COL + t * BT, a);
          tmem_ld16(tmem + lane_base + D_COL + t * BT + 16, b);
          tc_wait_ld();
#pragma unroll
          for (int c = 0; c < 16; ++c) { v[c] = __uint_as_float(a[c]); v[16 + c] = __uint_as_float(b[c]); }
        }
        if (Z == 1) {
          const int64_t row = (int64_t)(pn * P + t) * BN + r;
          epi_store<EPI>(p, row, v, p.bias ? __half2float(p.bias[row]) : 0.f);
        } else if (p.cl) {
          // the weight ring is idle once the item's MMAs completed (one item per CTA when Z > 1)
          float* sp_ = reinterpret_cast<float*>(smem + SM::OFF_W) + (t * BT) * BN + r;  // [tile][tok][row]
#pragma unroll
          for (int c = 0; c < BT; ++c) sp_[c * BN] = v[c];
        } else {
          float* gp = p.part + (((int64_t)it * PMAX + t) * BT) * BN + r;  // [tok][row]: coalesced
#pragma unroll
          for (int c = 0; c < BT; ++c) __stcg(gp + c * BN, v[c]);
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive(d_empty);  // accumulators drained: the MMA may start the next item
      if (Z > 1 && !p.cl) {  // publish this slice's partial (one item per CTA when Z > 1)
        __threadfence();
        asm volatile("bar.sync 1, 128;" ::: "memory");
        if (leader) atomicAdd(p.cnt + pn, 1);
      }
    }
  }
  // ---------------- split-k fix-up (Z > 1: one item per CTA, all Z items of a panel resident):
  // wait until the panel's Z partials are published, then this CTA reduces its 1/Z share of the
  // panel's outputs, summing the partials in fixed z order (deterministic).  The last CTA to finish
  // resets the panel's two counters for the next launch.
  __syncthreads();
  if (threadIdx.x == 0) trace_cta(p, 11);
  // (no griddepcontrol.wait here: everything below is ordered after the producer's wait by the
  // CTA barrier, and a redundant wait by all 704 threads measured ~2 us)
  if (Z > 1 && p.cl) {
    // cluster of the panel's Z items: partials stay in each CTA's shared memory; CTA z sums its
    // 1/Z share over the Z CTAs in fixed order through DSMEM (deterministic), then a second cluster
    // barrier keeps every partial alive until all peers have read it
    static_assert(PMAX * BT * BN * 4 <= SM::S_W * SM::W_STAGE, "partials fit the weight ring");
    const int it = blockIdx.x, pn = it / Z, z = it % Z, pp = tiles_of(pn);
    cluster_sync_all();
    const uint32_t base = smem_u32(smem + SM::OFF_W);
    const int nel = pp * BT * (BN / 4);
    const int e0 = (int)((long long)z * nel / Z), e1 = (int)((long long)(z + 1) * nel / Z);
    for (int idx = e0 + threadIdx.x; idx < e1; idx += NUM_THREADS) {
      const int t = idx / (BT * (BN / 4)), rem = idx - t * (BT * (BN / 4));
      const int tok = rem / (BN / 4), r4 = (rem % (BN / 4)) * 4;
      if (tok >= p.m) continue;
      const uint32_t off = (uint32_t)(((t * BT + tok) * BN + r4) * 4);
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int zz = 0; zz < Z; ++zz) {
        const float4 v = ld_dsmem_f4(dsmem_addr(base + off, (uint32_t)zz));
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
      const int64_t row0 = (int64_t)(pn * P + t) * BN + r4;
      float o[4] = {acc.x, acc.y, acc.z, acc.w};
      if (p.bias) {
#pragma unroll
        for (int c = 0; c < 4; ++c) o[c] += __half2float(p.bias[row0 + c]);
      }
      if constexpr (EPI == SQ_EPI_F32_ACCUM) {
        float* yp = static_cast<float*>(p.y) + (int64_t)tok * p.ldy + row0;
        const float4 y0 = __ldcg(reinterpret_cast<const float4*>(yp));
        *reinterpret_cast<float4*>(yp) = make_float4(y0.x + o[0], y0.y + o[1], y0.z + o[2], y0.w + o[3]);
      } else {
        __half* yp = static_cast<__half*>(p.y) + (int64_t)tok * p.ldy + row0;
        const __half2 h01 = __floats2half2_rn(apply_act<EPI>(o[0]), apply_act<EPI>(o[1]));
        const __half2 h23 = __floats2half2_rn(apply_act<EPI>(o[2]), apply_act<EPI>(o[3]));
        uint2 pk;
        pk.x = *reinterpret_cast<const uint32_t*>(&h01);
        pk.y = *reinterpret_cast<const uint32_t*>(&h23);
        *reinterpret_cast<uint2*>(yp) = pk;
      }
    }
    cluster_sync_all();
  } else if (Z > 1 && (int)blockIdx.x < I) {
    const int it = blockIdx.x, pn = it / Z, z = it % Z, pp = tiles_of(pn);
    if (threadIdx.x == 0) {
      volatile int* c = p.cnt + pn;
      while (*c < Z) __nanosleep(64);
      __threadfence();
    }
    __syncthreads();
    const int nel = pp * BT * (BN / 4);  // (tile, token, 4 rows)
    const int e0 = (int)((long long)z * nel / Z), e1 = (int)((long long)(z + 1) * nel / Z);
    for (int idx = e0 + threadIdx.x; idx < e1; idx += NUM_THREADS) {
      const int t = idx / (BT * (BN / 4)), rem = idx - t * (BT * (BN / 4));
      const int tok = rem / (BN / 4), r4 = (rem % (BN / 4)) * 4;
      if (tok >= p.m) continue;
      float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
      for (int zz = 0; zz < Z; ++zz) {
        const float4 v = __ldcg(reinterpret_cast<const float4*>(
            p.part + (((int64_t)(pn * Z + zz) * PMAX + t) * BT + tok) * BN + r4));
        acc.x += v.x; acc.y += v.y; acc.z += v.z; acc.w += v.w;
      }
      const int64_t row0 = (int64_t)(pn * P + t) * BN + r4;
      float o[4] = {acc.x, acc.y, acc.z, acc.w};
      if (p.bias) {
#pragma unroll
        for (int c = 0; c < 4; ++c) o[c] += __half2float(p.bias[row0 + c]);
      }
      if constexpr (EPI == SQ_EPI_F32_ACCUM) {
        float* yp = static_cast<float*>(p.y) + (int64_t)tok * p.ldy + row0;
#pragma unroll
        for (int c = 0; c < 4; ++c) yp[c] += o[c];
      } else {
        __half* yp = static_cast<__half*>(p.y) + (int64_t)tok * p.ldy + row0;
#pragma unroll
        for (int c = 0; c < 4; ++c) yp[c] = __float2half_rn(apply_act<EPI>(o[c]));
      }
    }
    __syncthreads();
    if (threadIdx.x == 0 && atomicAdd(p.cnt + kCnt2 + pn, 1) == Z - 1) {
      p.cnt[pn] = 0;
      p.cnt[kCnt2 + pn] = 0;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x == 0) trace_cta(p, 15);
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc(tmem, TMEM_COLS);
  }
}

template <int BITS, int UG, int EPI>
cudaError_t launch_tc_be(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const TcP& p0, int nc,
                         cudaStream_t s) {
  auto kern = k_gemv_tc<BITS, UG, EPI>;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, DSmem<BITS, UG>::BYTES);
    if (e != cudaSuccess) return e;
    cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    attr = true;
  }
  TcP p = p0;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(nc);
  cfg.blockDim = dim3(NUM_THREADS);
  cfg.dynamicSmemBytes = DSmem<BITS, UG>::BYTES;
  cfg.stream = s;
  cudaLaunchAttribute at[3];
  int na = 0;
  at[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[na++].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = at;
  if (p.cl) {
    // the panel's Z items as one cluster, only if every cluster of the grid can be resident at once
    // (the DSMEM reduction waits for all Z CTAs); the occupancy answer is cached per Z
    static int ncl_of_z[33];
    static bool init = false;
    if (!init) { for (int& v : ncl_of_z) v = -1; init = true; }
    at[na].id = cudaLaunchAttributeClusterDimension;
    at[na].val.clusterDim.x = p.Z;
    at[na].val.clusterDim.y = 1;
    at[na].val.clusterDim.z = 1;
    cfg.numAttrs = na + 1;
    int& ncl = ncl_of_z[p.Z];
    if (ncl < 0) {
      int v = 0;
      if (cudaOccupancyMaxActiveClusters(&v, kern, &cfg) != cudaSuccess) { cudaGetLastError(); v = 0; }
      ncl = v;
    }
    if (ncl * p.Z >= nc) ++na;
    else p.cl = 0;
  }
  if (!p.cl && p.Z > 1) {
    // global-memory split-k fix-up: a panel's CTAs wait for each other's partials, so the grid (one
    // item per SM) is launched cooperatively -- co-residency is guaranteed even when other kernels
    // (NCCL on the pipeline's comm streams) hold SMs
    at[na].id = cudaLaunchAttributeCooperative;
    at[na++].val.cooperative = 1;
  }
  cfg.numAttrs = na;
  cudaError_t e = cudaLaunchKernelEx(&cfg, kern, tx, tw, tm, p);
  if (e != cudaSuccess && na > 1 && pdl_enabled()) {
    // a driver that rejects PDL together with a cluster / cooperative launch: plain stream order
    cudaGetLastError();
    at[0].val.programmaticStreamSerializationAllowed = 0;
    e = cudaLaunchKernelEx(&cfg, kern, tx, tw, tm, p);
  }
  return e;
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
  if constexpr (BITS == 3 || BITS == 4) {
    if (ug == 2) return launch_tc_u<BITS, 2>(tx, tw, tm, p, epi, nc, s);
    if (ug == 3) return launch_tc_u<BITS, 3>(tx, tw, tm, p, epi, nc, s);
  }
  return launch_tc_u<BITS, 1>(tx, tw, tm, p, epi, nc, s);
}

// UG: groups per unit -- a ~16-KB weight stage (INT3/INT4 two groups when k/128 is even)
// INT3/INT4 take three groups per unit when 3 | k/128 (a ~24 KB INT4 stage, 2 TMEM A slots): one
// hand-off chain per 1.5x the bytes; measured +5-8 % INT4 GB/s on OPT-66B shapes.
int tc_ug(int bits, int kg) {
  if (bits <= 4 && kg % 3 == 0) return 3;
  return (bits <= 4 && kg % 2 == 0) ? 2 : 1;
}

struct TcPlan { int P, Z, I, ctas; };

// Panel width P and k split Z: minimise the bytes the busiest SM ingests -- weights + meta and the
// activation slice of every panel k-step (activation bytes cost as much as weight bytes in the
// per-SM TMA pipeline, ~45-50 GB/s per SM, tools/mb_tma.cu) -- plus, for Z > 1, the split-k fix-up
// (partials written and re-read, the panel-wide wait).  Z > 1 requires a single round (every item
// resident: the fix-up waits for the panel's other items).
TcPlan tc_plan(int64_t n, int64_t k, int bits) {
  const int64_t nt = n / BN, kg = k / 128;
  const int ug = tc_ug(bits, (int)kg);
  const int64_t ks = kg / ug, C = num_sms();
  const double unit_w = BN * ug * 128.0 * bits / 8 + (bits == 16 ? 0.0 : BN * 4.0 * ug), unit_x = ug * 128.0 * BT * 2;
  TcPlan best{1, 1, 0, 0};
  double best_cost = 1e300;
  constexpr int zmax = 32;
  for (int P = 1; P <= PMAX; ++P) {
    for (int Z = 1; Z <= zmax && Z <= ks; ++Z) {
      const int64_t I = ((nt + P - 1) / P) * Z, rounds = (I + C - 1) / C;
      if (Z > 1 && rounds > 1) continue;
      // (split panels run as resident clusters when they fit -- cluster residency on B200: z = 2 -> 148 CTAs, 3 -> 135, 4 -> 132, 8 -> 120 --
      // else with the cooperative global fix-up; restricting the plan to fitting clusters measured
      // 5-15 % slower on the o-proj / fc2 shapes, which need P = 4 with Z = 8 for activation reuse)
      const int64_t steps = (ks + Z - 1) / Z;
      const double fix = Z > 1 ? 2.0 * P * BT * BN * 4 + 131072.0 : 0.0;
      const double cost = rounds * steps * (P * unit_w + unit_x) + fix;
      if (cost < best_cost * 0.999) { best_cost = cost; best = {P, Z, (int)I, (int)(I < C ? I : C)}; }
    }
  }
  return best;
}
unsigned long long* g_trace = nullptr;


}  // namespace

// The counter region is the SAME fixed 16-KB region the mma.sync path uses (counters of every
// launch self-reset to 0, so consecutive linears of any n can share one workspace).
constexpr size_t kCntBytes = (65536 / 16) * sizeof(int);

size_t gemv_tc_xsum_offset(int64_t n, int64_t k);

// [counters][partials: [items][PMAX tiles][32 x 128] fp32, worst case over the bit widths][xsum]
size_t gemv_tc_workspace_bytes(int64_t n, int64_t k) {
  return gemv_tc_xsum_offset(n, k) + xsum_bytes(k) + 256;
}

// the activation group sums (when the caller passes none) follow the partials
size_t gemv_tc_xsum_offset(int64_t n, int64_t k) {
  // partials of the global-memory fix-up (the fallback when a split launch's clusters cannot all be
  // resident): at most one item per SM; sized without asking the device, so host-only callers agree
  int64_t items = SQ_TC_DEBUG && getenv("SQ_TC_PZ") ? 2 * num_sms() : num_sms();
  return (kCntBytes + (size_t)items * PMAX * BT * BN * sizeof(float) + 255) / 256 * 256;
}

cudaError_t launch_gemv_tc(const sq_qweight& w, const __half* x, int64_t ldx, int m, void* y, int64_t ldy, int epi,
                           void* ws, cudaStream_t s) {
  CUtensorMap tx, tw, tm;
  memset(&tm, 0, sizeof(tm));
  const int kg = (int)(w.k / 128);
  const int ug = tc_ug(w.bits, kg);
  {
    // activations as [k/64][m][64]: one box {64, 32, 2*ug} per unit -> 2*ug SW128 tiles [32 tokens][64 k]
    const uint64_t dx[3] = {64, (uint64_t)m, (uint64_t)w.k / 64}, sx[2] = {(uint64_t)ldx * 2, 128};
    const uint32_t bx[3] = {XK, BT, (uint32_t)(2 * ug)};
    cudaError_t e = encode_nd(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, x, 3, dx, sx, bx, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return e;
  }
  if (w.bits == 16) {
    const uint64_t dw[2] = {(uint64_t)w.k, (uint64_t)w.n}, sw_[1] = {(uint64_t)w.k * 2};
    const uint32_t bw[2] = {64, BN};
    cudaError_t e = encode_nd(&tw, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, w.packed, 2, dw, sw_, bw, CU_TENSOR_MAP_SWIZZLE_128B);
    if (e != cudaSuccess) return e;
  } else {
    // T16 units as lines: [n/16 tiles][kg * lpu lines][line bytes]; box = UG units of 8 tiles
    const uint64_t gb = 128 * w.bits / 8, nt = (uint64_t)w.n / 16;
    const WLines wl = wlines(w.bits);
    const uint64_t dw[3] = {(uint64_t)wl.line, (uint64_t)kg * wl.lpu, nt}, sw_[2] = {(uint64_t)wl.line, kg * 16 * gb};
    const uint32_t bw[3] = {(uint32_t)wl.line, (uint32_t)(wl.lpu * ug), BN / 16};
    cudaError_t e = encode_nd(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, w.packed, 3, dw, sw_, bw,
                        wl.sw128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE);
    if (e != cudaSuccess) return e;
    // meta as [n/16 tiles][kg * 16] u32: one box row = the UG groups of a tile (64 * UG contiguous
    // bytes), 8 rows per unit (a 3-D {16, UG, 8} box would move 16 rows of 64 B)
    const uint64_t dm[2] = {(uint64_t)kg * 16, nt}, sm_[1] = {(uint64_t)kg * 64};
    const uint32_t bm[2] = {(uint32_t)(16 * ug), BN / 16};
    e = encode_nd(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, w.meta, 2, dm, sm_, bm, CU_TENSOR_MAP_SWIZZLE_NONE);
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
  p.nt = (int)(w.n / BN);
  p.ks = kg / ug;
  TcPlan pl = tc_plan(w.n, w.k, w.bits);
  {
    // debug build only: SQ_TC_PZ="P,Z" forces the panel width and k split
    static int fp = -1, fz = -1;
    if (SQ_TC_DEBUG && fp < 0) {
      const char* e = getenv("SQ_TC_PZ");
      fp = 0;
      if (e && sscanf(e, "%d,%d", &fp, &fz) != 2) fp = 0;
    }
    if (fp > 0 && fp <= PMAX && fz >= 1 && fz <= p.ks) {
      const int64_t I = ((p.nt + fp - 1) / fp) * (int64_t)fz;
      if (fz == 1 || I <= num_sms()) pl = {fp, fz, (int)I, (int)(I < num_sms() ? I : num_sms())};
    }
  }
  p.P = pl.P;
  p.Z = pl.Z;
  p.I = pl.I;
  uint8_t* base = static_cast<uint8_t*>(ws);
  p.cnt = reinterpret_cast<int*>(base);
  p.part = reinterpret_cast<float*>(base + kCntBytes);
  p.trace = g_trace;
  {
    static int cl = -1;  // SQ_TC_CLUSTER=0 disables the cluster/DSMEM split-k reduction
    if (cl < 0) { const char* e = getenv("SQ_TC_CLUSTER"); cl = (e && e[0] == '0') ? 0 : 1; }
    p.cl = (cl && pl.Z > 1 && pl.Z <= 8 && pl.I == pl.ctas && pl.I % pl.Z == 0) ? 1 : 0;
  }
  const int nc = pl.ctas;
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
// tcgen05 decode kernel into a device buffer of 16 x 256 uint64 (rows 14/15: per-CTA globaltimer start/end) (tools/trace_tc.py)
extern "C" void sq_debug_trace(void* dev_buf) { sq::g_trace = static_cast<unsigned long long*>(dev_buf); }
