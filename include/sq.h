/*
 * sq.h — C-ABI of the SplitQuant hot path on B200 (libsq.so, sm_100a).
 *
 * Paper: Zhao et al., "SplitQuant" (PAPER.md in /root/reference; "P:<line>"
 * below are its line numbers).  The library executes a plan (per-layer
 * bit-widths, layer->stage partition, micro-batch sizes) produced host-side
 * (P:133); it does not plan.
 *
 * Conventions for every entry point
 *  - Pointers named *_dev are DEVICE pointers (any CUDA allocation on the
 *    current device); *_host are host pointers.  The caller owns all memory;
 *    the library never allocates in a hot call (only sq_comm_* and the
 *    per-thread TMA-descriptor cache -- one entry per distinct (pointer, shape,
 *    box) the first time it is seen -- allocate host memory).
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).  Kernels are
 *    enqueued asynchronously; device faults surface at the next sync.
 *  - Every call returns sq_status and never throws.  All validation happens
 *    before any launch: SQ_EINVAL has no side effects.  The message of the last
 *    non-OK status of the calling thread is in sq_last_error().
 *  - Inputs must be finite (NaN/Inf behaviour of the quantizer is unspecified).
 *  - Matrices are row-major.  A linear weight W is [n, k] (n = out_features,
 *    k = in_features); y[m, n] = x[m, k] . W~^T.
 */
#ifndef SQ_H_
#define SQ_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct CUstream_st* sq_stream_t; /* == cudaStream_t */

typedef enum {
  SQ_OK = 0,
  SQ_EINVAL = 1,    /* bad argument (null, misaligned, unsupported bits/shape, bad plan) */
  SQ_ENOTSUP = 2,   /* valid but not implemented (e.g. group != 128 in a linear) */
  SQ_ENOMEM = 3,    /* workspace too small / host allocation failed */
  SQ_ECUDA = 4,     /* CUDA runtime/driver error (message in sq_last_error) */
  SQ_ENCCL = 5,     /* NCCL error */
  SQ_EINTERNAL = 6
} sq_status;

const char* sq_last_error(void);
const char* sq_version(void);
int sq_abi_version(void); /* bumped on any incompatible change of this header (2: sq_plan.n_heads/kappa; 3: sq_plan.tp) */

/* ------------------------------------------------------------------------
 * Sizes.  P:160: a decoder layer with precision `bit` stores
 * (4 h1^2 + 2 h1 h2) * bit/8 bytes of weights; sq_packed_bytes is that count
 * for one [n,k] linear (codes only).  Group metadata is separate.
 * Returns 0 on invalid input.
 * ------------------------------------------------------------------------ */
size_t sq_packed_bytes(int64_t n, int64_t k, int bits);        /* n*k*bits/8; bits in {3,4,8,16} */
size_t sq_meta_bytes(int64_t n, int64_t k, int group);         /* n*(k/group)*4 */

/* ------------------------------------------------------------------------
 * a1 — per-group round-to-nearest min/max quantization (S_W of P:184).
 *   For row r, group g (k in [g*group, (g+1)*group)), IEEE fp32, one rounding/op:
 *     mn = min w, mx = max w (canonical +0);  s = fp16((mx - mn) / (2^bits - 1));
 *     z = mn;  c = s == 0 ? 0 : clamp(rint_half_even((w - z) / s), 0, 2^bits - 1)
 *   (readings R1-R6).
 *   w_dev     fp16 [n, k], 16-B aligned.       codes_dev  u8 [n, k]
 *   scales_dev, zeros_dev  fp16 [n, k/group]
 *   bits in {3,4,8}; group in {32,64,128}; k % group == 0; n >= 1.
 *   Result is bit-exact with the CPU oracle.
 * ------------------------------------------------------------------------ */
sq_status sq_quantize_groups(const void* w_dev, int64_t n, int64_t k, int bits, int group,
                             uint8_t* codes_dev, void* scales_dev, void* zeros_dev,
                             sq_stream_t stream);

/* a1 variants.  mode = OR of:
 *   SQ_QUANT_SYMMETRIC  P:184's symmetric scale (R21):
 *       s = fp16(max(|mx|, |mn|) / (2^(bits-1) - 1)), z = -2^(bits-1) * s (exact),
 *       c = clamp(round(w / s), -(2^(bits-1) - 1), 2^(bits-1) - 1) + 2^(bits-1)  (in [1, 2^bits - 1]),
 *       stored in the same (codes, scales, zeros) form, so sq_pack and every linear take it as is
 *       (w~ = s c + z = s c^).  A group whose z overflows fp16 (max|w| close to 65504) sets bit 0 of
 *       *status_dev (device int32 the caller zeroes and reads after a sync); its outputs are undefined.
 *   SQ_QUANT_STOCHASTIC Theorem 1's stochastic rounding (R22):
 *       c = floor(d) + [u_i < d - floor(d)] (then clamped), d the scaled value, u_i the top 24 bits
 *       of splitmix64 output i (state seed + (i + 1) * 0x9E3779B97F4A7C15, finalizer) / 2^24 for the
 *       weight's row-major index i = row * k + col.  Bit-exact with the oracle for a given seed.
 * mode 0 is sq_quantize_groups.  status_dev may be NULL unless SQ_QUANT_SYMMETRIC. */
enum { SQ_QUANT_SYMMETRIC = 1, SQ_QUANT_STOCHASTIC = 2 };
sq_status sq_quantize_groups_ex(const void* w_dev, int64_t n, int64_t k, int bits, int group, int mode,
                                uint64_t seed, uint8_t* codes_dev, void* scales_dev, void* zeros_dev,
                                int32_t* status_dev, sq_stream_t stream);

/* ------------------------------------------------------------------------
 * a2 — bit packing (layouts L8/L4/L3 + tile placement T16 of DESIGN.md
 *   section 4; the paper is silent on packing; P:160 fixes bits/8 bytes
 *   per weight).  codes_dev u8 [n,k]; scales/zeros fp16 [n, k/128] ->
 *   packed_dev n*k*bits/8 bytes (16-B aligned): unit (tile t = rows 16t..16t+15,
 *   group g) is a contiguous chunk of 16 x (128*bits/8) bytes at unit index
 *   t*(k/128) + g; meta_dev u32 [n/16][k/128][16] (low half = scale, high half =
 *   zero).  bits in {3,4,8}; group == 128; n % 16 == 0; k % 128 == 0.
 *   Bit-exact with the CPU oracle.
 * ------------------------------------------------------------------------ */
sq_status sq_pack(const uint8_t* codes_dev, const void* scales_dev, const void* zeros_dev,
                  int64_t n, int64_t k, int bits, int group, void* packed_dev, void* meta_dev,
                  sq_stream_t stream);

/* ------------------------------------------------------------------------
 * f2 — inputs of the variance indicator (Proposition 1, eq. 3, P:186-192;
 *   Theorem 1):  omega_{i,b} = sum_{o in layer i} D_{W_o} S_{W_o}(b)^2 G(X_o),
 *   G(X) = Var[X] / 4 for round-to-nearest (deterministic) quantization.
 *   sq_scale_sq_sums: W fp16 [n,k] (8-B aligned), groups of `group` (32/64/128) along k;
 *     for each b = bits_host[i] (2..8, n_bits <= 8) out_dev[i] = sum_g group * s_g(b)^2 (fp64)
 *     with s_g(b) = fp16(fp32(mx - mn) / (2^b - 1)) -- exactly the scale sq_quantize_groups
 *     stores (R5), i.e. D_W * S_W(b)^2 with per-group scales (R17).  k % 128 == 0.
 *     ws_dev: sq_scale_sq_sums_workspace_bytes(n, k) bytes, 8-B aligned.  Deterministic.
 *   sq_act_moments: x fp16 [count] (calibration activations X_o, any shape flattened) ->
 *     out_dev[0] = E[X], out_dev[1] = Var[X] (population), fp64.  Deterministic.
 *   omega is assembled on the host from these (paper_conf_cluster_zhaowplw25_b200.indicator).
 * ------------------------------------------------------------------------ */
size_t sq_scale_sq_sums_workspace_bytes(int64_t n, int64_t k);
sq_status sq_scale_sq_sums(const void* w_dev, int64_t n, int64_t k, int group, const int32_t* bits_host,
                           int n_bits, double* out_dev, void* ws_dev, size_t ws_bytes, sq_stream_t stream);
size_t sq_act_moments_workspace_bytes(int64_t count);
sq_status sq_act_moments(const void* x_dev, int64_t count, double* out_dev, void* ws_dev, size_t ws_bytes,
                         sq_stream_t stream);

/* One quantized linear: non-owning view of device memory. */
typedef struct {
  int32_t bits;          /* 3, 4, 8, or 16 (16 = fp16 weight, not quantized, R7) */
  int32_t group;         /* 128 (only value the linear kernels implement) */
  int64_t n, k;          /* n % 16 == 0, k % 128 == 0 */
  const void* packed;    /* bits<16: packed codes (sq_pack, T16); bits==16: fp16 W [n,k] row-major */
  const void* meta;      /* bits<16: u32 [n/16][k/128][16] (sq_pack); NULL when bits == 16 */
  const void* bias;      /* fp16 [n] or NULL */
} sq_qweight;

/* Epilogue of a linear (fused into the kernel). */
typedef enum {
  SQ_EPI_F16 = 0,       /* y fp16 [m, ldy] = x W~^T (+bias) */
  SQ_EPI_F16_RELU = 1,  /* y fp16 = relu(x W~^T + bias)        (OPT fc1, R11) */
  SQ_EPI_F16_GELU = 2,  /* y fp16 = gelu_tanh(x W~^T + bias)   (BLOOM fc1, R11) */
  SQ_EPI_F32_ACCUM = 3  /* y fp32 [m, ldy] += x W~^T (+bias)  (fused residual add, R9) */
} sq_epilogue;

/* ------------------------------------------------------------------------
 * a4 — decode linear (P:57 decode phase, memory-bound per P:106/P:164):
 *   y = epi(x . W~^T), m in [1, 32] tokens (one per sequence of the decode
 *   micro-batch xi).  Streams the packed weights once (TMA / bulk copies into
 *   shared-memory rings), unpacks in registers, fp32 accumulation: mma.sync
 *   strips for quantized weights at m <= 8 (INT8 m <= 16; K2s, K2
 *   when n % 32 != 0), tcgen05 with the dequantized weights in tensor memory
 *   otherwise (K2c).
 *   x_dev fp16 [m, ldx] (ldx % 8 == 0, 16-B aligned).  y_dev per epi.
 *   xsum_dev: optional float2 [k/128][32] group sums of x produced by
 *     sq_xsum (NULL: computed by the kernel on the tensor core (K2s) or into
 *     the workspace by sq_xsum (K2); ignored by K2c).
 *   ws_dev/ws_bytes: >= sq_linear_workspace_bytes(w, m); must be ZEROED once
 *     before first use (holds self-resetting counters); one workspace per
 *     concurrently running call.
 *   Deterministic: identical inputs give bit-identical outputs.
 * ------------------------------------------------------------------------ */
size_t sq_linear_workspace_bytes(const sq_qweight* w, int64_t m);
sq_status sq_linear_decode(const sq_qweight* w, const void* x_dev, int64_t ldx, int64_t m,
                           void* y_dev, int64_t ldy, int epi, const void* xsum_dev,
                           void* ws_dev, size_t ws_bytes, sq_stream_t stream);

/* Group sums used by sq_linear_decode: xsum[g][t] = (sum of x[t,k] over k%4<2 ; over k%4>=2)
 * for the 128 k of group g, fp32, fixed summation order.  float2 [k/128][32]; slots t >= m
 * are written as 0.  m <= 32. */
sq_status sq_xsum(const void* x_dev, int64_t ldx, int64_t m, int64_t k, void* xsum_dev,
                  sq_stream_t stream);

/* ------------------------------------------------------------------------
 * a3 — prefill linear (P:57 prefill phase, compute-bound per P:164): the same
 *   function for m >= 1 prompt tokens (m = eta * s).  tcgen05 tensor cores:
 *   packed weight tiles staged by TMA into shared memory, dequantized
 *   (w~ = s*c + z in fp16) into tensor memory as the A operand, activation
 *   tiles by TMA (128B swizzle) as the B operand, fp32 accumulation in TMEM.
 *   x_dev fp16 [m, ldx] (ldx % 8 == 0).  n % 128 == 0.
 * ------------------------------------------------------------------------ */
sq_status sq_linear_prefill(const sq_qweight* w, const void* x_dev, int64_t ldx, int64_t m,
                            void* y_dev, int64_t ldy, int epi, sq_stream_t stream);

/* ------------------------------------------------------------------------
 * a5 — stage forward (one pipeline stage = consecutive decoder layers, each
 *   with its own bit-width, P:152/P:160/P:198; glue R11, attention stub R12):
 *     a = LN(x); [q k v] = a Wqkv^T (+b); h = x + v Wo^T (+b);
 *     u = act(LN(h) W1^T + b1); x = h + u W2^T (+b2)
 *   phase SQ_PREFILL uses sq_linear_prefill kernels, SQ_DECODE (tokens <= 32)
 *   the decode kernels.  x_in/x_out fp32 [tokens, h1] (may alias).
 *   qkv_dbg_dev: optional fp16 [tokens, 3*h1] receiving the LAST layer's q,k,v.
 *   ws: >= sq_stage_workspace_bytes(...), zeroed once before first use.
 * ------------------------------------------------------------------------ */
typedef struct {
  int32_t bits;          /* this layer's precision (all four linears share it) */
  int32_t act;           /* 0 = ReLU (OPT), 1 = tanh-GeLU (BLOOM) */
  sq_qweight qkv;        /* [3*h1, h1] (q, k, v stacked along n) */
  sq_qweight o;          /* [h1, h1] */
  sq_qweight fc1;        /* [h2, h1] */
  sq_qweight fc2;        /* [h1, h2] */
} sq_layer;

typedef enum { SQ_PREFILL = 0, SQ_DECODE = 1 } sq_phase;

size_t sq_stage_workspace_bytes(const sq_layer* layers, int n_layers, int64_t max_tokens);
sq_status sq_stage_forward(const sq_layer* layers, int n_layers, int phase, const float* x_in_dev,
                           int64_t tokens, float* x_out_dev, void* qkv_dbg_dev, void* ws_dev,
                           size_t ws_bytes, sq_stream_t stream);

/* ------------------------------------------------------------------------
 * f3 — causal multi-head self-attention over a per-layer KV cache (DESIGN.md
 *   R23-R25; cache sized 2 v (s + n) h1 elements per layer; chunked prefill kappa).
 *   Head j uses columns [j*dh, (j+1)*dh) of q = qkv[:, 0:h1], k = qkv[:, h1:2h1], v = qkv[:, 2h1:3h1]
 *   (dh = h1 / n_heads in {64, 128}); scores q.k / sqrt(dh); the query at position p attends over
 *   cache positions 0..p of its own sequence; no positional term inside the layer (R24).
 *   The KV cache of one layer is K, V fp16 [n_seq_cache][max_len][h1] each (caller-owned, device).
 * ------------------------------------------------------------------------ */

/* One layer, one micro-batch: nseq sequences (cache rows seq0..seq0+nseq-1), each with `len` new
 * tokens at positions pos0..pos0+len-1; qkv row i*len + (p - pos0) is (sequence i, position p).
 * Appends the new k, v rows to the cache, then writes the attention output fp16 [nseq*len, h1]
 * (row stride ld_out) -- len == 1: the HBM-bound decode kernel, else the prefill kernel.
 * qkv_dev / caches / out_dev 16-B aligned, ld_qkv >= 3*h1 and ld_out >= h1 multiples of 8. */
sq_status sq_attention(const void* qkv_dev, int64_t ld_qkv, int64_t nseq, int64_t len, int64_t pos0,
                       int64_t seq0, int64_t h1, int n_heads, void* k_cache_dev, void* v_cache_dev,
                       int64_t max_len, int64_t n_seq_cache, void* out_dev, int64_t ld_out,
                       sq_stream_t stream);

typedef struct {            /* attention context of one stage call (host memory) */
  int32_t n_heads;          /* h1 / head_dim, head_dim in {64, 128} */
  int32_t max_len;          /* cache positions per sequence (>= s + n_decode) */
  int64_t n_seq_cache;      /* sequences each layer's cache holds */
  void* const* k_cache;     /* [n_layers] device pointers: layer l's K cache fp16 [n_seq_cache][max_len][h1] */
  void* const* v_cache;     /* [n_layers] device pointers: layer l's V cache */
  int64_t seq0;             /* cache row of the micro-batch's first sequence */
  int32_t nseq, seq_len;    /* tokens = nseq * seq_len (decode: seq_len = 1) */
  int32_t pos0;             /* position of each sequence's first token in this call */
} sq_attn;

/* a5 with real attention in place of the R12 stub:
 *   a = LN(x); [q k v] = a Wqkv^T (+b); att = attention(q, k, v; cache) (sq_attention);
 *   h = x + att Wo^T (+b); u = act(LN(h) W1^T + b1); x = h + u W2^T (+b2).
 * Same workspace rules as sq_stage_forward (sq_stage_workspace_bytes covers both). */
sq_status sq_stage_forward_attn(const sq_layer* layers, int n_layers, int phase, const sq_attn* attn,
                                const float* x_in_dev, int64_t tokens, float* x_out_dev, void* ws_dev,
                                size_t ws_bytes, sq_stream_t stream);

/* ------------------------------------------------------------------------
 * f4 — W8A8 linear (weight-activation INT8, P:93 SmoothQuant / bitsandbytes; R26):
 *   weights symmetric per output channel: s_w[n] = fp16(max_k |W[n,k]| / 127),
 *     q_w = clamp(rint(W / s_w), -127, 127) int8;
 *   activations symmetric per token (dynamic): s_x[t] = max_k |x[t,k]| / 127 (fp32),
 *     q_x = clamp(rint(x / s_x), -127, 127) int8;     (fp32 single-rounded ops, ties to even)
 *   acc = sum_k q_x q_w (exact int32 on tcgen05 kind::i8),  y = acc * s_x[t] * s_w[n] (+ bias).
 * Codes and scales are bit-exact with the oracle; acc is exact (mode SQ_W8A8_I32 returns it).
 * ------------------------------------------------------------------------ */
enum { SQ_W8A8_I32 = 4 };   /* mode: raw int32 accumulator y_dev [m][n] (epilogue modes 0..3 as SQ_EPI_*) */
sq_status sq_quantize_w8(const void* w_dev /* fp16 [n,k] */, int64_t n, int64_t k, int8_t* codes_dev /* [n,k] */,
                         void* scales_f16_dev /* [n] */, sq_stream_t stream);
sq_status sq_quantize_act8(const void* x_dev /* fp16 [m, ldx] */, int64_t m, int64_t k, int64_t ldx,
                           int8_t* codes_dev /* [m,k] */, float* scales_dev /* [m] */, sq_stream_t stream);
size_t sq_linear_w8a8_workspace_bytes(int64_t n, int64_t k, int64_t m);   /* split-k int32 partials (0: none) */
/* n, k multiples of 128; codes 16-B aligned; y fp16 / fp32 [m, ldy] by mode (SQ_EPI_F16, _RELU, _GELU,
 * _F32_ACCUM) or int32 [m, n] (SQ_W8A8_I32).  Narrow grids (decode) split k over Z CTAs whose exact int32
 * partials a second kernel sums (order-independent: deterministic). */
sq_status sq_linear_w8a8(const int8_t* wq_dev, const void* sw_f16_dev, const void* bias_f16_dev, int64_t n, int64_t k,
                         const int8_t* xq_dev, const float* sx_dev, int64_t m, void* y_dev, int64_t ldy, int mode,
                         void* ws_dev, size_t ws_bytes, sq_stream_t stream);

/* Loop-back glue (R14): out_row = x (fp32 copy) and e = LN(x) for the next decode step. */
sq_status sq_layernorm_f32(const float* x_dev, int64_t rows, int64_t d, float* y_dev,
                           sq_stream_t stream);

/* ------------------------------------------------------------------------
 * a6 — uneven layer-wise pipeline with phase-specific micro-batches
 *   (eq. (4), eqs. (5)-(8), (15)-(16) P:210-232).
 * ------------------------------------------------------------------------ */
typedef struct sq_comm sq_comm;   /* owns NCCL link communicators + comm streams + events */

size_t sq_comm_unique_id_bytes(void);                         /* 128 */
sq_status sq_comm_get_unique_id(uint8_t* id_host);            /* rank 0; broadcast by caller */
/* One process per GPU; id_host from sq_comm_get_unique_id on rank 0 (world comm),
 * nranks = number of pipeline stages (any P >= 1: one 2-rank NCCL communicator per link
 * r -> r+1 mod P, built with up to three ncclCommSplit calls).  Collective over all ranks. */
sq_status sq_comm_init(sq_comm** out, const uint8_t* id_host, int nranks, int rank);
/* Single-process "virtual pipeline": every stage on the current device, transfers
 * are device copies.  Bitwise reference for the multi-GPU run. */
sq_status sq_comm_init_local(sq_comm** out, int nstages);
/* P x T mesh (f4: TP inside every pipeline stage): nranks = n_stages * tp, global rank
 * g = stage * tp + j.  Builds the T independent stage rings (link (p, j) -> (p+1 mod P, j), the same
 * three-split scheme as sq_comm_init per ring) plus one tp-rank communicator per stage (ncclCommSplit
 * colour = stage, key = j) that carries sq_stage_forward_tp's all-reduce.  Collective over all ranks. */
sq_status sq_comm_init_mesh(sq_comm** out, const uint8_t* id_host, int n_stages, int tp, int rank);
sq_status sq_comm_destroy(sq_comm* comm);

typedef struct {            /* host memory, identical on every rank */
  int32_t n_layers, n_stages;
  int32_t hidden, ffn;      /* h1, h2 */
  int32_t group;            /* 128 */
  const int32_t* bits;            /* [n_layers], in {3,4,8,16}            (y_{i,b}) */
  const int32_t* stage_of_layer;  /* [n_layers] non-decreasing 0..n_stages-1, every stage
                                     non-empty (u_{i,j}, eqs. 15-16) */
  int32_t B;                /* global batch (sequences) */
  int32_t eta, xi;          /* prefill / decode micro-batch sizes (sequences) */
  int32_t prompt_len;       /* s */
  int32_t n_decode;         /* decode steps after the prefill token (R14) */
  int32_t n_heads;          /* 0: attention stub out = v (R12); > 0: real attention (f3) with a KV
                               cache of 2 x B x (s + n_decode) x h1 fp16 per layer inside the
                               pipeline workspace */
  int32_t kappa;            /* prefill chunks per prompt (0 or 1 = whole prompt); s % kappa == 0;
                               needs n_heads > 0 when > 1 */
  int32_t tp;               /* intra-node tensor parallelism per stage (f4, P:63 / P:236; 0 or 1 = none):
                               every stage spans tp ranks (a P x tp mesh, e.g. TP2+PP2 of P:318), each
                               holding the sq_stage_forward_tp shard of its stage's layers; hidden and
                               ffn multiples of 128 tp, n_heads % tp == 0 */
} sq_plan;

typedef struct {
  double t_total_ms, t_prefill_ms, t_decode_ms;  /* device time (events) on this rank */
  double tokens_per_s;      /* B*(1+n_decode) / t_total */
  int64_t bytes_sent;       /* inter-stage bytes sent by this rank */
  int64_t gpu_launches;     /* kernels launched by this rank (graph replays count their kernels) */
  double host_enqueue_ms;   /* host time spent issuing the run's work (before the final sync) */
  int64_t graph_replays;    /* decode micro-batches replayed from a cached CUDA graph */
} sq_run_stats;

size_t sq_pipeline_workspace_bytes(const sq_plan* plan, const sq_layer* layers, int rank);
/* rank >= 0: this process's stage (layers = its layers, in order); rank == -1 with a
 * local comm: all stages (layers = all n_layers).  x0_dev: embeddings fp32 [B, s, h1]
 * (needed on stage 0); out_dev: fp32 [B, 1+n_decode, h1] (written on the last stage).
 * With plan.tp = T > 1 the global rank is g = stage * T + j (j = TP index), comm comes from
 * sq_comm_init_mesh, layers = this rank's TP shards of its stage's layers (n_layers = the stage's
 * layer count), and hidden states travel (stage p, j) -> (stage p+1, j), loop-back (P-1, j) -> (0, j)
 * (the residual is replicated over a TP group).  rank == -1 runs the whole mesh on one device:
 * layers = [T][n_layers] (TP index major), n_layers = plan.n_layers.
 * Blocking: returns after the run completed on this rank.
 * Decode micro-batches of the attention-stub path (plan.n_heads == 0) are captured once per
 * (layers, input / output buffer, rows, workspace) into a CUDA graph and replayed (a process-wide
 * cache of instantiated graphs; SQ_GRAPH=0 disables it, and it is bypassed while sq_profile is on and
 * around a real TP rank's NCCL all-reduce). */
sq_status sq_pipeline_run(const sq_plan* plan, int rank, const sq_layer* layers, int n_layers,
                          sq_comm* comm, const float* x0_dev, float* out_dev, void* ws_dev,
                          size_t ws_bytes, sq_run_stats* stats, sq_stream_t stream);

/* Validate a plan (contiguity eqs. 15-16, non-empty stages, bits set, micro-batches). */
sq_status sq_plan_check(const sq_plan* plan);

/* Host-only: the exact op sequence `rank` executes inside sq_pipeline_run (rank -1, or a
 * 1-stage plan: the single-process order).  Items: prefill (m, c) for m = 0..mu_pre-1 and chunk
 * c = 0..kappa-1 (only the last chunk produces OUT / loop-back ops), then decode
 * t = 1..n_decode, m = 0..mu_dec-1 (R13/R14).  Send/recv ops name the peer's global rank;
 * the sequence of SEND ops of rank j to j+1 equals, op for op and size for size, the
 * sequence of RECV ops of rank j+1 from j (tests/test_pipeline_schedule.py).  Returns the
 * number of ops (writes at most max_ops; ops may be NULL to query), or -1 on a bad plan. */
typedef enum {
  SQ_OP_RECV_LB = 0,       /* stage 0: loop-back rows LN(hidden) from the last stage -> decode input */
  SQ_OP_RECV_ACT = 1,      /* hidden [rows, h1] fp32 from the previous stage */
  SQ_OP_COMPUTE = 2,       /* this stage's layers on the item (phase, rows tokens) */
  SQ_OP_SEND_ACT = 3,      /* hidden to the next stage */
  SQ_OP_OUT = 4,           /* last stage: write out[b, t] (prefill: last prompt position) */
  SQ_OP_SEND_LB = 5,       /* last stage: LN(out rows) to stage 0 */
  SQ_OP_LOOPBACK_LOCAL = 6 /* single process: LN(out rows) -> decode input in place */
} sq_op_kind;
typedef struct {
  int32_t kind, item, phase, t;   /* t: decode step (0 = prefill) */
  int32_t slot, peer;             /* activation buffer slot; peer global rank (-1 none) */
  int64_t seq0, nseq;             /* sequences of the item / loop-back rows */
  int64_t rows;                   /* tokens moved or computed */
} sq_sched_op;
int64_t sq_pipeline_schedule(const sq_plan* plan, int rank, sq_sched_op* ops, int64_t max_ops);

/* ------------------------------------------------------------------------
 * f4 — intra-node tensor-parallel (TP) stage ("we force intra-node TP", P:236 2-D device
 *   meshes such as TP2+PP2, P:318 TP4 / TP2+PP2 winning on homogeneous clusters).
 * The TP split of one decoder layer over T ranks (R27):
 *   qkv, fc1  column-parallel: shard r holds output rows [r n/T, (r+1) n/T) of each of q, k, v
 *             (resp. of fc1) with that bias slice -> qkv [3 h1/T, h1], fc1 [h2/T, h1];
 *   o, fc2    row-parallel: shard r holds input columns [r k/T, (r+1) k/T) -> o [h1, h1/T],
 *             fc2 [h1, h2/T]; the bias sits in tp rank 0's shard only (other ranks: bias NULL);
 *   attention (attn != NULL) head-parallel: rank r owns heads [r H/T, (r+1) H/T) and a KV cache of
 *             width h1/T (its sq_attn.n_heads = H/T).
 * Every shard is quantized on its own; groups run along k and h1/T, h2/T are multiples of 128, so the
 * shard codes are exactly the matching codes of the unsharded weight.
 * Per layer on each rank: a = LN(x) (x replicated), the q/k/v and u shards, then the partial o / fc2
 * products summed over the T ranks in place on the fp32 residual: rank 0 accumulates x + p_0 (the
 * fused residual epilogue), ranks r > 0 write p_r into a zeroed x, and one NCCL all-reduce (sum)
 * returns x + sum_r p_r on every rank, so the residual add costs no extra pass.
 *   tp_rank >= 0: one rank of a T-rank NCCL group; comm from sq_comm_init(nranks = T, rank = tp_rank)
 *                 (its world communicator carries the all-reduce) or from sq_comm_init_mesh (its
 *                 stage's TP communicator); shards = this rank's n_layers
 *                 layers; attn NULL or one context.
 *   tp_rank == -1: virtual TP on the current device (tests, single-GPU runs of a TP plan): comm
 *                 ignored (may be NULL); shards = [T][n_layers] rank-major; attn NULL or [T]
 *                 contexts; the partial products accumulate into x in rank order 0..T-1
 *                 (deterministic).
 * x_in, x_out fp32 [tokens, h1] device (may alias); decode: tokens <= 32.  Workspace (256-B aligned)
 * from sq_stage_tp_workspace_bytes over all the shard layers passed (n_layers * T for virtual TP).
 * Errors: SQ_EINVAL (shard shapes inconsistent, h1 or h2 not a multiple of 128 T, heads % T, bad
 * phase / tokens / pointers), SQ_ENOMEM (workspace), SQ_ENCCL, SQ_ECUDA. */
size_t sq_stage_tp_workspace_bytes(const sq_layer* shards, int n_shard_layers, int64_t max_tokens);
sq_status sq_stage_forward_tp(const sq_layer* shards, int n_layers, int tp, int tp_rank, sq_comm* comm,
                              int phase, const sq_attn* attn, const float* x_in_dev, int64_t tokens,
                              float* x_out_dev, void* ws_dev, size_t ws_bytes, sq_stream_t stream);

/* ------------------------------------------------------------------------
 * Measurement hooks (bench.py): per-kernel-class CUDA-event timing of every
 * launch made by the library while enabled, on the launching stream.
 * class 0 = decode GEMV, 1 = prefill GEMM, 2 = glue (LN/xsum), 3 = quantize/pack,
 * 4 = decode attention (KV-cache bytes), 5 = prefill attention (causal flops).
 * ------------------------------------------------------------------------ */
#define SQ_PROFILE_CLASSES 6
typedef struct {
  int64_t launches[SQ_PROFILE_CLASSES];
  double ms[SQ_PROFILE_CLASSES];      /* summed event durations */
  double bytes[SQ_PROFILE_CLASSES];   /* algorithmic bytes */
  double flops[SQ_PROFILE_CLASSES];   /* algorithmic flops */
} sq_profile;
sq_status sq_profile_enable(int on);
sq_status sq_profile_read(sq_profile* out);   /* synchronizes the device */
int64_t sq_launch_count(void);                /* kernels launched by the library so far */

#ifdef __cplusplus
}
#endif
#endif /* SQ_H_ */
