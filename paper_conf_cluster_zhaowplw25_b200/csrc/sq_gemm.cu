// K3 — prefill dequant-GEMM on tcgen05 (P:57 prefill phase; compute-bound,
// arithmetic intensity 6354-9553 on V100; dequant overhead made FP16
// faster than 3/4-bit in prefill on the paper's GPUs, P:108 — here it is
// hidden behind the tensor cores).
//
// Y^T tile [128 weight rows x 256 tokens] = W~[128 x K] . X[256 x K]^T
//
//  * A operand = dequantized weights in TENSOR MEMORY (tcgen05.mma ... [a_tmem]):
//    packed codes + meta of a 128-row x 128-k group are staged into shared memory
//    by TMA (swizzled so each thread's row is bank-conflict free), four "dequant"
//    warps (one per TMEM sub-partition, one thread per weight row) turn them into
//    fp16 w~ = s*c + z (magic-number unpack, HSUB2 + HFMA2) and tcgen05.st them
//    into a 2-slot TMEM ring.  Keeping A out of shared memory leaves the SMEM
//    port to the activation stream (K3).
//  * B operand = activation tile [256 tokens x 64 k] fp16 by TMA, 128B swizzle,
//    K-major; 4-stage ring.
//  * D = fp32 accumulator in TMEM (256 columns); one thread issues
//    tcgen05.mma.cta_group::1.kind::f16 (M=128, N=256, K=16).
//  * Epilogue: the dequant warps tcgen05.ld the accumulator (lane = weight row,
//    column = token), add bias / activation / residual, store y.
// Warp roles: 0 = TMA producer, 1 = MMA issuer (+TMEM alloc), 2..9 = dequant (2 groups) + epilogue.
//
// CTA-pair variant (CG = 2, the default when n / 128 is even and m >= 512): the two CTAs of a (2, 1, 1) cluster
// hold adjacent 128-row weight tiles of the same 256-token tile; each loads HALF the activation tile
// (128 tokens) by TMA with .cta_group::2 (both halves complete on the leader's barrier) and
// dequantizes its own rows into its own TMEM; the leader issues tcgen05.mma.cta_group::2 (M = 256,
// N = 256, A from both CTAs' TMEM, B from both CTAs' shared memory) and commits to both CTAs'
// barriers (multicast); the peer's dequant warps signal the leader's "A ready" barrier remotely.
// Each SM then streams and reads half the activation bytes per MMA (the 1-CTA tile's activation
// traffic -- TMA writes + MMA reads of B -- saturated the shared-memory port), and the pair reads the
// activation tile from L2 once instead of twice.
#include <cuda.h>

#include <cstring>
#include <mutex>

#include "sq_tc.cuh"

#ifndef SQ_GEMM_SX2
#define SQ_GEMM_SX2 8
#endif

namespace sq {
namespace {
using namespace tc;

constexpr int BN = 128;   // weight rows per tile (TMEM lanes, MMA M)
constexpr int BT = 256;   // tokens per tile (MMA N)
constexpr int XK = 64;    // k per activation stage (one 128-B swizzle row)
constexpr int S_A = 4;
constexpr int DQ_GROUPS = 2;  // dequant warp-groups on alternating groups of k
// ring depths S_A and S_W are multiples of DQ_GROUPS so that every slot belongs to one group
// (consumed in order): an mbarrier parity wait can never run two phases ahead of its slot
template <int CG>
constexpr int x_stage_bytes() { return BT / CG * XK * 2; }  // 32 KB (one CTA) / 16 KB (per CTA of a pair)
// activation ring depth: the pair's half-size stages buy twice the stages for the same shared memory
template <int CG>
constexpr int x_stages() { return CG == 2 ? SQ_GEMM_SX2 : 4; }
constexpr int TMEM_COLS = 512;
constexpr int D_COL = 0;
constexpr int A_COL = 256;
constexpr int NUM_THREADS = 32 * (2 + 4 * DQ_GROUPS);

template <int BITS, int CG>
struct Smem {
  static constexpr int X_STAGE_BYTES = x_stage_bytes<CG>();
  static constexpr int S_X = x_stages<CG>();
  static constexpr int W_STAGE = ((BN * GCfg<BITS>::GB + 1023) / 1024) * 1024;
  static constexpr int OFF_X = 0;
  static constexpr int OFF_W = OFF_X + S_X * X_STAGE_BYTES;
  static constexpr int OFF_META = OFF_W + GCfg<BITS>::S_W * W_STAGE;
  static constexpr int OFF_BAR = OFF_META + GCfg<BITS>::S_W * BN * 4;
  static constexpr int NUM_BARS = 2 * S_X + 2 * GCfg<BITS>::S_W + 2 * S_A + 1;
  static constexpr int OFF_TMEM = OFF_BAR + NUM_BARS * 8;
  static constexpr int BYTES = OFF_TMEM + 16 + 1024;  // + alignment slack
};

struct GemmP {
  const uint8_t* packed;
  const uint32_t* meta;   // T16 [N/16][K/128][16]
  const __half* bias;
  void* y;
  int64_t ldy;
  int64_t m;
  int64_t n;
  int kg;
};

// ---- CTA-pair (cta_group::2) primitives
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// shared::cluster address of the same byte in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa_u32(uint32_t local, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(local), "r"(rank));
  return r;
}
// arrive on a barrier of either CTA of the pair (cluster address).  Default .release.cta semantics,
// as CUTLASS's cluster barrier: the TMEM stores it publishes are ordered by tcgen05.wait::st +
// tcgen05.fence::before_thread_sync, and a cluster-scope release (plus cluster-scope acquire polls
// on the leader) put a memory barrier on every arrival and poll: measured 15-30 % slower GEMMs.
__device__ __forceinline__ void mbar_arrive_cl(uint32_t cl_addr) {
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cl_addr) : "memory");
}
// TMA load by either CTA of a pair, completing on the barrier at cluster address mbar_cl (the leader's)
__device__ __forceinline__ void tma_load_2d_cg2(void* smem_dst, const void* tmap, uint32_t mbar_cl, int32_t c0,
                                                int32_t c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];"
      ::"r"(smem_u32(smem_dst)), "l"(tmap), "r"(mbar_cl), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void tc_mma_ts_cg2(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// commit the leader's MMAs to the barrier at the same offset in both CTAs of the pair
__device__ __forceinline__ void tc_commit_cg2(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
               ::"r"(smem_u32(bar)), "h"((uint16_t)0x3)
               : "memory");
}

template <int BITS, int EPI, int CG>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    k_gemm(const __grid_constant__ CUtensorMap tm_x, const __grid_constant__ CUtensorMap tm_w,
           const __grid_constant__ CUtensorMap tm_m, const GemmP p) {
  using SM = Smem<BITS, CG>;
  constexpr int X_STAGE_BYTES = SM::X_STAGE_BYTES;
  constexpr int S_X = SM::S_X;
  // instruction descriptor: kind::f16, A=B=f16 K-major, D=f32, M = 128 per CTA, N = 256
  constexpr uint32_t kIdesc = make_idesc(BN * CG, BT);
  constexpr int S_W = GCfg<BITS>::S_W;
  static_assert(S_W % DQ_GROUPS == 0 && S_A % DQ_GROUPS == 0, "slots must not be shared by dequant groups");
  constexpr int GB = GCfg<BITS>::GB;
  constexpr uint32_t W_BYTES = BN * GB;
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
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(smem + SM::OFF_TMEM);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // weight-row tile, token tile.  Pairs (cluster (2, 1, 1): tcgen05 pairs CTAs along x) take
  // blockIdx.x = 2 x token tile + rank, blockIdx.y = row-tile pair, so consecutive CTAs still share a
  // weight panel as in the one-CTA grid (x = token tile, y = row tile)
  const int64_t n0 = CG == 2 ? ((int64_t)blockIdx.y * 2 + (blockIdx.x & 1)) * BN : (int64_t)blockIdx.y * BN;
  const int64_t t0 = CG == 2 ? (int64_t)(blockIdx.x >> 1) * BT : (int64_t)blockIdx.x * BT;
  const int kg = p.kg;
  const uint32_t rank = CG == 2 ? cluster_rank() : 0;  // CTA of the pair (0 = leader, issues the MMAs)

  if (threadIdx.x == 0) {
    for (int i = 0; i < S_X; ++i) { mbar_init(&full_x[i], 1); mbar_init(&empty_x[i], 1); }
    for (int i = 0; i < S_W; ++i) { mbar_init(&full_w[i], 1); mbar_init(&empty_w[i], 4); }
    for (int i = 0; i < S_A; ++i) { mbar_init(&full_a[i], 4 * CG); mbar_init(&empty_a[i], 1); }
    mbar_init(d_full, 1);
    fence_barrier_init();
    prefetch_tmap(&tm_x);
    prefetch_tmap(&tm_w);
    if constexpr (BITS != 16) prefetch_tmap(&tm_m);
  }
  if (warp == 1) {
    if constexpr (CG == 2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                   "r"(TMEM_COLS) : "memory");
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
    } else {
      tmem_alloc(tmem_slot, TMEM_COLS);
    }
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync_all();  // the peer's barriers are initialised before any remote arrive
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    // ---------------- TMA producer
    {  // whole warp runs the loop (warp-uniform operands live in uniform registers); a leader issues
      int it_x = 0;
      for (int g = 0; g < kg; ++g) {
        const int sw = g % S_W, rw = g / S_W;
        mbar_wait(&empty_w[sw], (rw & 1) ^ 1);
        uint8_t* wdst = smem + SM::OFF_W + sw * SM::W_STAGE;
        if (elect_one()) mbar_arrive_expect_tx(&full_w[sw], W_BYTES + (BITS != 16 ? BN * 4 : 0));
        if constexpr (BITS == 16) {
          if (elect_one()) tma_load_2d(wdst, &tm_w, &full_w[sw], g * 128, (int32_t)n0);
          if (elect_one()) tma_load_2d(wdst + BN * 128, &tm_w, &full_w[sw], g * 128 + 64, (int32_t)n0);
        } else {
          // placement T16: 4-D box {GB bytes, 16 rows, 1 group, 8 row tiles} -> [128 rows][GB]
          if (elect_one()) tma_load_3d(wdst, &tm_w, &full_w[sw], 0, g * (BITS == 3 ? 3 : (BITS == 4 ? 8 : 16)), (int32_t)(n0 / 16));
          if (elect_one()) tma_load_3d(smem + SM::OFF_META + sw * BN * 4, &tm_m, &full_w[sw], 0, g, (int32_t)(n0 / 16));
        }
        for (int h = 0; h < 2; ++h, ++it_x) {
          const int sx = it_x % S_X, rx = it_x / S_X;
          mbar_wait(&empty_x[sx], (rx & 1) ^ 1);
          if constexpr (CG == 2) {
            // this CTA's half of the token tile; both halves complete on the leader's barrier
            if (rank == 0 && elect_one()) mbar_arrive_expect_tx(&full_x[sx], 2 * X_STAGE_BYTES);
            if (elect_one())
              tma_load_2d_cg2(smem + SM::OFF_X + sx * X_STAGE_BYTES, &tm_x, mapa_u32(smem_u32(&full_x[sx]), 0),
                              g * 128 + h * XK, (int32_t)(t0 + rank * (BT / 2)));
          } else {
            if (elect_one()) mbar_arrive_expect_tx(&full_x[sx], X_STAGE_BYTES);
            if (elect_one()) tma_load_2d(smem + SM::OFF_X + sx * X_STAGE_BYTES, &tm_x, &full_x[sx], g * 128 + h * XK, (int32_t)t0);
          }
        }
      }
    }
  } else if (warp == 1) {
    // ---------------- MMA issuer (single thread; the pair's leader only)
    if (CG == 1 || rank == 0) {  // whole warp runs the loop; the elected leader issues tcgen05.mma / commit
      int it_x = 0;
      for (int g = 0; g < kg; ++g) {
        const int sa = g % S_A, ra = g / S_A;
        mbar_wait(&full_a[sa], ra & 1);
        tc_fence_after();
        for (int h = 0; h < 2; ++h, ++it_x) {
          const int sx = it_x % S_X, rx = it_x / S_X;
          mbar_wait(&full_x[sx], rx & 1);
          tc_fence_after();
          const uint32_t xs = smem_u32(smem + SM::OFF_X + sx * X_STAGE_BYTES);
#pragma unroll
          for (int kk = 0; kk < XK / 16; ++kk) {
            const uint64_t bdesc = make_sw128_desc(xs + kk * 32);
            const uint32_t a_tm = tmem + A_COL + sa * 64 + h * 32 + kk * 8;
            if constexpr (CG == 2) {
              if (elect_one()) tc_mma_ts_cg2(tmem + D_COL, a_tm, bdesc, kIdesc, (g | h | kk) != 0);
            } else {
              if (elect_one()) tc_mma_ts(tmem + D_COL, a_tm, bdesc, kIdesc, (g | h | kk) != 0);
            }
          }
          if (elect_one()) { if constexpr (CG == 2) tc_commit_cg2(&empty_x[sx]); else tc_commit(&empty_x[sx]); }
        }
        if (elect_one()) { if constexpr (CG == 2) tc_commit_cg2(&empty_a[sa]); else tc_commit(&empty_a[sa]); }
      }
      if (elect_one()) { if constexpr (CG == 2) tc_commit_cg2(d_full); else tc_commit(d_full); }
    }
  } else {
    // ---------------- dequant warps (one thread per weight row; group gi takes k-groups
    // g = gi (mod 2) so one group's tcgen05.st latency overlaps the other's unpack), then epilogue
    const int sp = warp & 3;            // TMEM sub-partition this warp may access
    const int gi = (warp - 2) >> 2;
    const int r = sp * 32 + lane;       // row within the tile
    const uint32_t lane_base = (uint32_t)(sp * 32) << 16;
    for (int g = gi; g < kg; g += DQ_GROUPS) {
      const int sw = g % S_W, rw = g / S_W;
      const int sa = g % S_A, ra = g / S_A;
      mbar_wait(&full_w[sw], rw & 1);
      mbar_wait(&empty_a[sa], (ra & 1) ^ 1);
      tc_fence_after();
      const uint32_t meta = reinterpret_cast<const uint32_t*>(smem + SM::OFF_META + sw * BN * 4)[r];
      dequant_row_to_tmem<BITS>(smem + SM::OFF_W + sw * SM::W_STAGE, meta, r, tmem + lane_base + A_COL + sa * 64);
      tc_wait_st();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&empty_w[sw]);
        // (pair: the leader's barrier, from either CTA)
        if constexpr (CG == 2) mbar_arrive_cl(mapa_u32(smem_u32(&full_a[sa]), 0)); else mbar_arrive(&full_a[sa]);
      }
    }
    // ---------------- epilogue (each dequant group drains half of the 256 token columns)
    mbar_wait_sleepy(d_full, 0);
    tc_fence_after();
    const int64_t nrow = n0 + r;
    float bias = 0.f;
    if (p.bias) bias = __half2float(p.bias[nrow]);
    if constexpr (EPI == SQ_EPI_F32_ACCUM) {
      // residual read-modify-write: all 32 loads of a 32-token batch are issued before any store
      // (a load -> add -> store chain per token serialised on the L2 round trip: measured 1.7x
      // slower o-proj GEMMs)
      float* yb = static_cast<float*>(p.y) + nrow;
#pragma unroll 1
      for (int c = gi * (BT / 32); c < (gi + 1) * (BT / 32); c += 2) {
        uint32_t v[32];
        tmem_ld16(tmem + lane_base + D_COL + c * 16, *reinterpret_cast<uint32_t(*)[16]>(v));
        tmem_ld16(tmem + lane_base + D_COL + c * 16 + 16, *reinterpret_cast<uint32_t(*)[16]>(v + 16));
        float r[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const int64_t tok = t0 + c * 16 + i;
          r[i] = tok < p.m ? __ldcg(yb + tok * p.ldy) : 0.f;
        }
        tc_wait_ld();
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const int64_t tok = t0 + c * 16 + i;
          if (tok < p.m) yb[tok * p.ldy] = r[i] + (__uint_as_float(v[i]) + bias);
        }
      }
    } else {
#pragma unroll 1
      for (int c = gi * (BT / 32); c < (gi + 1) * (BT / 32); ++c) {
        uint32_t v[16];
        tmem_ld16(tmem + lane_base + D_COL + c * 16, v);
        tc_wait_ld();
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const int64_t tok = t0 + c * 16 + i;
          if (tok < p.m) {
            const float o = __uint_as_float(v[i]) + bias;
            static_cast<__half*>(p.y)[tok * p.ldy + nrow] = __float2half_rn(apply_act<EPI>(o));
          }
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG == 2) cluster_sync_all();  // neither CTA frees TMEM / shared memory the pair still reads
  if (warp == 1) {
    tc_fence_after();
    if constexpr (CG == 2)
      asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TMEM_COLS) : "memory");
    else
      tmem_dealloc(tmem, TMEM_COLS);
  }
}

// ---------------------------------------------------------------- host side
cudaError_t encode_2d(CUtensorMap* m, CUtensorMapDataType dt, const void* ptr, uint64_t inner, uint64_t outer,
                      uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer, CUtensorMapSwizzle sw) {
  const uint64_t dims[2] = {inner, outer}, st[1] = {row_bytes};
  const uint32_t box[2] = {box_inner, box_outer};
  return encode_nd(m, dt, ptr, 2, dims, st, box, sw);
}

template <int BITS, int EPI, int CG>
cudaError_t launch_be(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const GemmP& p, cudaStream_t s) {
  auto kern = k_gemm<BITS, EPI, CG>;
  static bool attr_set = false;
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, Smem<BITS, CG>::BYTES);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  dim3 grid((unsigned)((p.m + BT - 1) / BT), (unsigned)(p.n / BN));
  if constexpr (CG == 2) grid = dim3(2 * grid.x, grid.y / 2);
  if constexpr (CG == 1) {
    kern<<<grid, NUM_THREADS, Smem<BITS, CG>::BYTES, s>>>(tx, tw, tm, p);
    return cudaGetLastError();
  } else {
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = grid;
    cfg.blockDim = dim3(NUM_THREADS);
    cfg.dynamicSmemBytes = Smem<BITS, CG>::BYTES;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;  // the pair: adjacent 128-row weight tiles of one token tile
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, kern, tx, tw, tm, p);
  }
}

template <int BITS, int CG>
cudaError_t launch_bc(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const GemmP& p, int epi,
                      cudaStream_t s) {
  switch (epi) {
    case SQ_EPI_F16: return launch_be<BITS, SQ_EPI_F16, CG>(tx, tw, tm, p, s);
    case SQ_EPI_F16_RELU: return launch_be<BITS, SQ_EPI_F16_RELU, CG>(tx, tw, tm, p, s);
    case SQ_EPI_F16_GELU: return launch_be<BITS, SQ_EPI_F16_GELU, CG>(tx, tw, tm, p, s);
    default: return launch_be<BITS, SQ_EPI_F32_ACCUM, CG>(tx, tw, tm, p, s);
  }
}

// CTA pairs when the row tiles pair up (n / 128 even) and the GEMM has at least two token tiles' worth
// of tokens (a 32-token OPT-125m prefill linear took ~9 us longer as a pair: cluster launch and
// barriers for a few CTAs); SQ_GEMM_CG=1 forces the one-CTA tile, SQ_GEMM_CG=2 pairs at any m
int gemm_cg(int64_t n, int64_t m) {
  static int forced = -1;
  if (forced < 0) { const char* e = getenv("SQ_GEMM_CG"); forced = !e ? 0 : (e[0] == '1' ? 1 : (e[0] == '2' ? 2 : 0)); }
  if (forced == 1 || (n / BN) % 2) return 1;
  return (forced == 2 || m >= 2 * BT) ? 2 : 1;
}

template <int BITS>
cudaError_t launch_b(const CUtensorMap& tx, const CUtensorMap& tw, const CUtensorMap& tm, const GemmP& p, int epi,
                     cudaStream_t s) {
  return gemm_cg(p.n, p.m) == 2 ? launch_bc<BITS, 2>(tx, tw, tm, p, epi, s) : launch_bc<BITS, 1>(tx, tw, tm, p, epi, s);
}

}  // namespace

cudaError_t launch_gemm(const sq_qweight& w, const __half* x, int64_t ldx, int64_t m, void* y, int64_t ldy, int epi,
                        cudaStream_t s) {
  CUtensorMap tx, tw, tm;
  memset(&tm, 0, sizeof(tm));
  cudaError_t e = encode_2d(&tx, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, x, (uint64_t)w.k, (uint64_t)m, (uint64_t)ldx * 2,
                            XK, BT / gemm_cg(w.n, m), CU_TENSOR_MAP_SWIZZLE_128B);
  if (e != cudaSuccess) return e;
  if (w.bits == 16) {
    e = encode_2d(&tw, CU_TENSOR_MAP_DATA_TYPE_FLOAT16, w.packed, (uint64_t)w.k, (uint64_t)w.n, (uint64_t)w.k * 2, 64,
                  BN, CU_TENSOR_MAP_SWIZZLE_128B);
  } else {
    // placement T16: [n/16 tiles][kg groups][16 rows][GB bytes]
    const uint64_t gb = 128 * w.bits / 8, kg = (uint64_t)w.k / 128, nt = (uint64_t)w.n / 16;
    const WLines wl = wlines(w.bits);  // T16 units as long TMA lines (sq_tc.cuh)
    const uint64_t dw[3] = {(uint64_t)wl.line, kg * wl.lpu, nt}, sw_[2] = {(uint64_t)wl.line, kg * 16 * gb};
    const uint32_t bw[3] = {(uint32_t)wl.line, (uint32_t)wl.lpu, BN / 16};
    e = encode_nd(&tw, CU_TENSOR_MAP_DATA_TYPE_UINT8, w.packed, 3, dw, sw_, bw,
                  wl.sw128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE);
    if (e == cudaSuccess) {
      const uint64_t dm[3] = {16, kg, nt}, sm_[2] = {64, kg * 64};
      const uint32_t bm[3] = {16, 1, BN / 16};
      e = encode_nd(&tm, CU_TENSOR_MAP_DATA_TYPE_UINT32, w.meta, 3, dm, sm_, bm, CU_TENSOR_MAP_SWIZZLE_NONE);
    }
  }
  if (e != cudaSuccess) return e;
  GemmP p{};
  p.packed = static_cast<const uint8_t*>(w.packed);
  p.meta = static_cast<const uint32_t*>(w.meta);
  p.bias = static_cast<const __half*>(w.bias);
  p.y = y;
  p.ldy = ldy;
  p.m = m;
  p.n = w.n;
  p.kg = (int)(w.k / 128);
  auto t = prof_begin(KC_GEMM, (double)w.n * w.k * w.bits / 8.0 + 2.0 * m * w.k, 2.0 * m * w.n * w.k, s);
  switch (w.bits) {
    case 3: e = launch_b<3>(tx, tw, tm, p, epi, s); break;
    case 4: e = launch_b<4>(tx, tw, tm, p, epi, s); break;
    case 8: e = launch_b<8>(tx, tw, tm, p, epi, s); break;
    default: e = launch_b<16>(tx, tw, tm, p, epi, s); break;
  }
  prof_end(t, s);
  count_launch();
  return e;
}

}  // namespace sq
