// a5 — stage forward: the consecutive decoder layers of one pipeline stage, each
// with its own bit-width from the plan.  Per layer
// (R11/R12, pre-LN block, attention stub = V; with an sq_attn context the
// stub is replaced by causal attention over the layer's KV cache, f3 / sq_attn.cu):
//   a = LN(x) -> fp16 (+ group sums)     [K5]
//   qkv = a Wqkv^T (+b)                  [K2 decode | K3 prefill]   fp16
//   x  += v Wo^T (+b)                    [K2 | K3, fused fp32 residual add]
//   a = LN(x)                            [K5]
//   u = act(a W1^T + b1)                 [K2 | K3, fused activation] fp16
//   x += u W2^T (+b2)                    [K2 | K3, fused fp32 residual add]
// The residual stream stays fp32 in HBM (R9); every linear reads fp16.
#include <cstring>

#include "sq_common.cuh"

namespace sq {
namespace {

struct WsLayout {
  size_t a16, qkv16, u16, att16, xs, gemv, total;
};

int64_t align_up(int64_t v, int64_t a) { return (v + a - 1) / a * a; }

WsLayout layout(const sq_layer* layers, int n_layers, int64_t T) {
  // The decode GEMV region (self-resetting counters first) sits at a FIXED offset 0 and is
  // sized for the largest decode micro-batch (32 tokens), so its zero-initialised counters
  // are never overwritten by activations when the token count changes between calls.
  const int64_t h1 = layers[0].o.n, h2 = layers[0].fc1.n;
  WsLayout L{};
  size_t g = 0;
  for (int l = 0; l < n_layers; ++l) {
    const sq_qweight* ws[4] = {&layers[l].qkv, &layers[l].o, &layers[l].fc1, &layers[l].fc2};
    for (auto* w : ws) {
      size_t b = gemv_workspace_bytes(w->n, w->k, 32);
      if (b > g) g = b;
    }
  }
  size_t off = 0;
  L.gemv = off;  off += align_up((int64_t)g, 256);
  L.a16 = off;   off += align_up(T * h1 * 2, 256);
  L.qkv16 = off; off += align_up(T * 3 * h1 * 2, 256);
  L.u16 = off;   off += align_up(T * h2 * 2, 256);
  L.att16 = off; off += align_up(T * h1 * 2, 256);
  L.xs = off;    off += align_up((int64_t)xsum_bytes(h2 > h1 ? h2 : h1), 256);
  L.total = off;
  return L;
}

sq_status check_w(const sq_qweight& w, int64_t n, int64_t k, int bits, const char* who, int l, const char* name) {
  if (w.n != n || w.k != k) return fail(SQ_EINVAL, "%s: layer %d %s shape [%lld,%lld] != [%lld,%lld]", who, l, name, (long long)w.n, (long long)w.k, (long long)n, (long long)k);
  if (w.bits != bits) return fail(SQ_EINVAL, "%s: layer %d %s bits %d != layer bits %d", who, l, name, w.bits, bits);
  if (w.bits != 3 && w.bits != 4 && w.bits != 8 && w.bits != 16) return fail(SQ_EINVAL, "%s: bad bits", who);
  if (w.bits != 16 && (w.group != 128 || !w.meta)) return fail(SQ_ENOTSUP, "%s: layer %d %s needs group 128 + meta", who, l, name);
  if (!w.packed) return fail(SQ_EINVAL, "%s: layer %d %s null packed", who, l, name);
  return SQ_OK;
}

}  // namespace

// h1: the width this context's heads and cache cover (the hidden size, or h1/T for a TP rank)
sq_status check_attn(const sq_attn* a, int64_t h1, int n_layers, int phase, int64_t tokens, const char* who) {
  if (!a || !a->k_cache || !a->v_cache) return fail(SQ_EINVAL, "%s: null attention context / cache arrays", who);
  if (a->n_heads <= 0 || h1 % a->n_heads || (h1 / a->n_heads != 64 && h1 / a->n_heads != 128))
    return fail(SQ_EINVAL, "%s: head_dim h1/n_heads must be 64 or 128", who);
  if (a->nseq < 1 || a->seq_len < 1 || (int64_t)a->nseq * a->seq_len != tokens || (phase == SQ_DECODE && a->seq_len != 1))
    return fail(SQ_EINVAL, "%s: tokens %lld != nseq %d x seq_len %d (decode: seq_len 1)", who, (long long)tokens, a->nseq, a->seq_len);
  if (a->pos0 < 0 || a->pos0 + a->seq_len > a->max_len || a->seq0 < 0 || a->seq0 + a->nseq > a->n_seq_cache)
    return fail(SQ_EINVAL, "%s: positions / sequences outside the cache", who);
  for (int l = 0; l < n_layers; ++l)
    if (!a->k_cache[l] || !a->v_cache[l] || ((reinterpret_cast<uintptr_t>(a->k_cache[l]) | reinterpret_cast<uintptr_t>(a->v_cache[l])) & 15u))
      return fail(SQ_EINVAL, "%s: layer %d cache null or not 16-B aligned", who, l);
  return SQ_OK;
}

sq_status check_layers(const sq_layer* layers, int n_layers, const char* who) {
  if (!layers || n_layers <= 0) return fail(SQ_EINVAL, "%s: no layers", who);
  const int64_t h1 = layers[0].o.n, h2 = layers[0].fc1.n;
  if (h1 <= 0 || h1 % 128 || h1 > 14336 || h2 <= 0 || h2 % 128)
    return fail(SQ_EINVAL, "%s: hidden %lld must be a multiple of 128 <= 14336; ffn %lld multiple of 128", who, (long long)h1, (long long)h2);
  for (int l = 0; l < n_layers; ++l) {
    const sq_layer& L = layers[l];
    if (L.act != 0 && L.act != 1) return fail(SQ_EINVAL, "%s: layer %d act %d", who, l, L.act);
    sq_status st;
    if ((st = check_w(L.qkv, 3 * h1, h1, L.bits, who, l, "qkv"))) return st;
    if ((st = check_w(L.o, h1, h1, L.bits, who, l, "o"))) return st;
    if ((st = check_w(L.fc1, h2, h1, L.bits, who, l, "fc1"))) return st;
    if ((st = check_w(L.fc2, h1, h2, L.bits, who, l, "fc2"))) return st;
  }
  return SQ_OK;
}

size_t stage_workspace_bytes(const sq_layer* layers, int n_layers, int64_t max_tokens) {
  return layout(layers, n_layers, max_tokens).total;
}

sq_status stage_forward(const sq_layer* layers, int n_layers, int phase, const float* x_in, int64_t T, float* x_out,
                        void* qkv_dbg, void* ws, size_t ws_bytes, cudaStream_t s, const sq_attn* att) {
  const int64_t h1 = layers[0].o.n, h2 = layers[0].fc1.n;
  const WsLayout W = layout(layers, n_layers, T);
  uint8_t* base = static_cast<uint8_t*>(ws);
  __half* a16 = reinterpret_cast<__half*>(base + W.a16);
  __half* qkv16 = reinterpret_cast<__half*>(base + W.qkv16);
  __half* u16 = reinterpret_cast<__half*>(base + W.u16);
  float2* xs = reinterpret_cast<float2*>(base + W.xs);
  __half* att16 = reinterpret_cast<__half*>(base + W.att16);
  void* gws = base + W.gemv;
  const bool dec = phase == SQ_DECODE;
  // linears of a decode step, and of a prefill micro-batch of <= 32 tokens (configs[0]'s 32-token
  // prompt, small chunks), run on the decode kernels: the prefill GEMM's 256-token tile would be at
  // most 1/8 full and every launch pays its TMEM / pipeline prologue (same function)
  const bool gv = dec || T <= 32;
  auto lin = [&](const sq_qweight& w, const __half* x, int64_t ldx, void* y, int64_t ldy, int epi,
                 const float2* xsum) -> cudaError_t {
    if (gv) return launch_gemv(w, x, ldx, (int)T, y, ldy, epi, xsum, gws, s);
    return launch_gemm(w, x, ldx, T, y, ldy, epi, s);
  };
  cudaError_t e = cudaSuccess;
  for (int l = 0; l < n_layers && e == cudaSuccess; ++l) {
    const sq_layer& L = layers[l];
    // per-group activation sums only for linears on the round-1 mma.sync decode kernel (K2); the strip
    // kernel K2s computes its own on the tensor core, the tcgen05 decode (K2c) dequantizes and needs none
    const bool q = L.bits != 16;
    auto k2 = [&](const sq_qweight& w) { return gv && q && gemv_path(w.n, w.k, (int)T, w.bits) == 0 &&
                                                   !use_k2s(w.bits, w.n, w.k, (int)T); };
    // LayerNorm's group sums (free: it holds the row) feed K2 and K2s alike
    auto lnxs = [&](const sq_qweight& w) { return gv && q && gemv_path(w.n, w.k, (int)T, w.bits) == 0; };
    const float* xr = (l == 0) ? x_in : x_out;
    const bool copy = (l == 0 && x_in != x_out);
    // a = LN(x) (layer 0 also initialises the residual buffer x_out = x_in)
    e = launch_layernorm_f16(xr, T, h1, a16, lnxs(L.qkv) ? xs : nullptr, copy ? x_in : nullptr, copy ? x_out : nullptr, s);
    if (e) break;
    e = lin(L.qkv, a16, h1, qkv16, 3 * h1, SQ_EPI_F16, lnxs(L.qkv) ? xs : nullptr);
    if (e) break;
    // attention: the R12 stub attn = v = qkv[:, 2h1:3h1], or causal attention over the KV cache (f3)
    const __half* v = qkv16 + 2 * h1;
    int64_t ldv = 3 * h1;
    if (att) {
      e = launch_attention(qkv16, 3 * h1, att->nseq, att->seq_len, att->pos0, att->seq0, (int)h1, att->n_heads,
                           static_cast<__half*>(att->k_cache[l]), static_cast<__half*>(att->v_cache[l]), att->max_len,
                           att16, h1, s);
      if (e) break;
      v = att16;
      ldv = h1;
    }
    if (k2(L.o)) {
      e = launch_xsum(v, ldv, T, h1, xs, s);
      if (e) break;
    }
    e = lin(L.o, v, ldv, x_out, h1, SQ_EPI_F32_ACCUM, k2(L.o) ? xs : nullptr);
    if (e) break;
    e = launch_layernorm_f16(x_out, T, h1, a16, lnxs(L.fc1) ? xs : nullptr, nullptr, nullptr, s);
    if (e) break;
    e = lin(L.fc1, a16, h1, u16, h2, L.act == 0 ? SQ_EPI_F16_RELU : SQ_EPI_F16_GELU, lnxs(L.fc1) ? xs : nullptr);
    if (e) break;
    if (k2(L.fc2)) {
      e = launch_xsum(u16, h2, T, h2, xs, s);
      if (e) break;
    }
    e = lin(L.fc2, u16, h2, x_out, h1, SQ_EPI_F32_ACCUM, k2(L.fc2) ? xs : nullptr);
    if (e) break;
    if (qkv_dbg && l == n_layers - 1)
      e = cudaMemcpyAsync(qkv_dbg, qkv16, (size_t)T * 3 * h1 * 2, cudaMemcpyDeviceToDevice, s);
  }
  return cuda_check(e, "sq_stage_forward");
}

// ---------------------------------------------------------------- f4: tensor-parallel stage (R27)
namespace {

struct TpLayout {
  size_t gemv, a16, qkv16, u16, att16, xsa, xsb, total;
};

// shard shapes: o [h1, h1s], qkv [3 h1s, h1], fc1 [h2s, h1], fc2 [h1, h2s]
TpLayout tp_layout(const sq_layer* sh, int n, int64_t T) {
  const int64_t h1 = sh[0].o.n, h1s = sh[0].o.k, h2s = sh[0].fc1.n;
  size_t g = 0;
  for (int l = 0; l < n; ++l) {
    const sq_qweight* ws[4] = {&sh[l].qkv, &sh[l].o, &sh[l].fc1, &sh[l].fc2};
    for (auto* w : ws) {
      size_t b = gemv_workspace_bytes(w->n, w->k, 32);
      if (b > g) g = b;
    }
  }
  TpLayout L{};
  size_t off = 0;
  L.gemv = off;  off += align_up((int64_t)g, 256);  // fixed offset 0: self-resetting counters (see layout())
  L.a16 = off;   off += align_up(T * h1 * 2, 256);
  L.qkv16 = off; off += align_up(T * 3 * h1s * 2, 256);
  L.u16 = off;   off += align_up(T * h2s * 2, 256);
  L.att16 = off; off += align_up(T * h1s * 2, 256);
  L.xsa = off;   off += align_up((int64_t)xsum_bytes(h1), 256);                     // LN(x) group sums
  L.xsb = off;   off += align_up((int64_t)xsum_bytes(h2s > h1s ? h2s : h1s), 256);  // v / u group sums
  L.total = off;
  return L;
}

}  // namespace

sq_status check_tp(const sq_layer* sh, int n_layers, int tp, int n_sets, const char* who) {
  if (!sh || n_layers <= 0 || tp < 1) return fail(SQ_EINVAL, "%s: no shards / tp < 1", who);
  const int64_t h1 = sh[0].o.n, h1s = sh[0].o.k, h2s = sh[0].fc1.n;
  if (h1 <= 0 || h1 > 14336 || h1s * tp != h1 || h1s % 128 || h2s <= 0 || h2s % 128)
    return fail(SQ_EINVAL, "%s: hidden %lld must equal tp %d x shard width %lld, both multiples of 128 (ffn shard %lld)",
                who, (long long)h1, tp, (long long)h1s, (long long)h2s);
  for (int i = 0; i < n_layers * n_sets; ++i) {
    const sq_layer& L = sh[i];
    const int l = i % n_layers;
    if (L.act != 0 && L.act != 1) return fail(SQ_EINVAL, "%s: layer %d act %d", who, l, L.act);
    if (L.bits != sh[l].bits || L.act != sh[l].act)
      return fail(SQ_EINVAL, "%s: layer %d bits / act differ between tp ranks", who, l);
    sq_status st;
    if ((st = check_w(L.qkv, 3 * h1s, h1, L.bits, who, l, "qkv"))) return st;
    if ((st = check_w(L.o, h1, h1s, L.bits, who, l, "o"))) return st;
    if ((st = check_w(L.fc1, h2s, h1, L.bits, who, l, "fc1"))) return st;
    if ((st = check_w(L.fc2, h1, h2s, L.bits, who, l, "fc2"))) return st;
  }
  return SQ_OK;
}

size_t stage_tp_workspace_bytes(const sq_layer* sh, int n_shard_layers, int64_t max_tokens) {
  return tp_layout(sh, n_shard_layers, max_tokens).total;
}

// The n_sets shard sets in `sh` ([set][n_layers], rank-major) run on this device one after the other
// (virtual TP); `comm` != NULL means one real TP rank (n_sets = 1) whose partial sums go through the
// in-place all-reduce.
sq_status stage_forward_tp(const sq_layer* sh, int n_layers, int n_sets, sq_comm* comm, int tp_rank, int phase,
                           const sq_attn* att, const float* x_in, int64_t T, float* x_out, void* ws, cudaStream_t s) {
  const int64_t h1 = sh[0].o.n, h1s = sh[0].o.k, h2s = sh[0].fc1.n;
  const TpLayout W = tp_layout(sh, n_layers * n_sets, T);
  uint8_t* base = static_cast<uint8_t*>(ws);
  __half* a16 = reinterpret_cast<__half*>(base + W.a16);
  __half* qkv16 = reinterpret_cast<__half*>(base + W.qkv16);
  __half* u16 = reinterpret_cast<__half*>(base + W.u16);
  __half* att16 = reinterpret_cast<__half*>(base + W.att16);
  float2* xsa = reinterpret_cast<float2*>(base + W.xsa);
  float2* xsb = reinterpret_cast<float2*>(base + W.xsb);
  void* gws = base + W.gemv;
  const bool dec = phase == SQ_DECODE;
  // linears of a decode step, and of a prefill micro-batch of <= 32 tokens (configs[0]'s 32-token
  // prompt, small chunks), run on the decode kernels: the prefill GEMM's 256-token tile would be at
  // most 1/8 full and every launch pays its TMEM / pipeline prologue (same function)
  const bool gv = dec || T <= 32;
  const bool zero_first = comm && tp_rank > 0;  // ranks r > 0 contribute p_r only (x comes from rank 0)
  auto lin = [&](const sq_qweight& w, const __half* x, int64_t ldx, void* y, int64_t ldy, int epi,
                 const float2* xsum) -> cudaError_t {
    if (gv) return launch_gemv(w, x, ldx, (int)T, y, ldy, epi, xsum, gws, s);
    return launch_gemm(w, x, ldx, T, y, ldy, epi, s);
  };
  auto reduce = [&]() -> sq_status {
    if (!comm) return SQ_OK;
    return comm_allreduce_sum_f32(comm, x_out, (size_t)T * h1, s);
  };
  cudaError_t e = cudaSuccess;
  sq_status st = SQ_OK;
  for (int l = 0; l < n_layers && e == cudaSuccess && st == SQ_OK; ++l) {
    const sq_layer& L0 = sh[l];
    const bool q = L0.bits != 16;
    auto k2 = [&](const sq_qweight& w) { return gv && q && gemv_path(w.n, w.k, (int)T, w.bits) == 0 &&
                                                   !use_k2s(w.bits, w.n, w.k, (int)T); };
    // LayerNorm's group sums (free: it holds the row) feed K2 and K2s alike
    auto lnxs = [&](const sq_qweight& w) { return gv && q && gemv_path(w.n, w.k, (int)T, w.bits) == 0; };
    const float* xr = (l == 0) ? x_in : x_out;
    const bool copy = (l == 0 && x_in != x_out);
    e = launch_layernorm_f16(xr, T, h1, a16, lnxs(L0.qkv) ? xsa : nullptr, copy ? x_in : nullptr, copy ? x_out : nullptr, s);
    if (e) break;
    for (int r = 0; r < n_sets && !e; ++r) {
      const sq_layer& L = sh[r * n_layers + l];
      e = lin(L.qkv, a16, h1, qkv16, 3 * h1s, SQ_EPI_F16, lnxs(L.qkv) ? xsa : nullptr);
      if (e) break;
      const __half* v = qkv16 + 2 * h1s;
      int64_t ldv = 3 * h1s;
      if (att) {
        const sq_attn& A = att[r];
        e = launch_attention(qkv16, 3 * h1s, A.nseq, A.seq_len, A.pos0, A.seq0, (int)h1s, A.n_heads,
                             static_cast<__half*>(A.k_cache[l]), static_cast<__half*>(A.v_cache[l]), A.max_len,
                             att16, h1s, s);
        if (e) break;
        v = att16;
        ldv = h1s;
      }
      if (k2(L.o) && (e = launch_xsum(v, ldv, T, h1s, xsb, s))) break;
      if (zero_first && (e = cudaMemsetAsync(x_out, 0, (size_t)T * h1 * sizeof(float), s))) break;
      e = lin(L.o, v, ldv, x_out, h1, SQ_EPI_F32_ACCUM, k2(L.o) ? xsb : nullptr);
    }
    if (e || (st = reduce())) break;
    e = launch_layernorm_f16(x_out, T, h1, a16, lnxs(L0.fc1) ? xsa : nullptr, nullptr, nullptr, s);
    if (e) break;
    for (int r = 0; r < n_sets && !e; ++r) {
      const sq_layer& L = sh[r * n_layers + l];
      e = lin(L.fc1, a16, h1, u16, h2s, L.act == 0 ? SQ_EPI_F16_RELU : SQ_EPI_F16_GELU, lnxs(L.fc1) ? xsa : nullptr);
      if (e) break;
      if (k2(L.fc2) && (e = launch_xsum(u16, h2s, T, h2s, xsb, s))) break;
      if (zero_first && (e = cudaMemsetAsync(x_out, 0, (size_t)T * h1 * sizeof(float), s))) break;
      e = lin(L.fc2, u16, h2s, x_out, h1, SQ_EPI_F32_ACCUM, k2(L.fc2) ? xsb : nullptr);
    }
    if (e) break;
    st = reduce();
  }
  if (st) return st;
  return cuda_check(e, "sq_stage_forward_tp");
}

}  // namespace sq

using namespace sq;

extern "C" {

size_t sq_stage_workspace_bytes(const sq_layer* layers, int n_layers, int64_t max_tokens) {
  if (!layers || n_layers <= 0 || max_tokens <= 0) return 0;
  return stage_workspace_bytes(layers, n_layers, max_tokens);
}

sq_status sq_stage_forward(const sq_layer* layers, int n_layers, int phase, const float* x_in_dev, int64_t tokens,
                           float* x_out_dev, void* qkv_dbg_dev, void* ws_dev, size_t ws_bytes, sq_stream_t stream) {
  sq_status st = check_layers(layers, n_layers, "sq_stage_forward");
  if (st) return st;
  if (phase != SQ_PREFILL && phase != SQ_DECODE) return fail(SQ_EINVAL, "sq_stage_forward: bad phase %d", phase);
  if (tokens < 1 || (phase == SQ_DECODE && tokens > 32))
    return fail(SQ_EINVAL, "sq_stage_forward: tokens=%lld (decode needs 1..32)", (long long)tokens);
  if (phase == SQ_PREFILL) {
    for (int l = 0; l < n_layers; ++l)
      if (layers[l].o.n % 128 || layers[l].fc1.n % 128) return fail(SQ_EINVAL, "sq_stage_forward: prefill needs n%%128==0");
  }
  if (!x_in_dev || !x_out_dev || (reinterpret_cast<uintptr_t>(x_in_dev) & 15u) || (reinterpret_cast<uintptr_t>(x_out_dev) & 15u))
    return fail(SQ_EINVAL, "sq_stage_forward: x_in/x_out null or not 16-B aligned");
  const size_t need = stage_workspace_bytes(layers, n_layers, tokens);
  if (!ws_dev || ws_bytes < need || (reinterpret_cast<uintptr_t>(ws_dev) & 255u))
    return fail(SQ_ENOMEM, "sq_stage_forward: workspace %zu < %zu (or null / not 256-B aligned)", ws_bytes, need);
  return stage_forward(layers, n_layers, phase, x_in_dev, tokens, x_out_dev, qkv_dbg_dev, ws_dev, ws_bytes,
                       (cudaStream_t)stream, nullptr);
}

sq_status sq_stage_forward_attn(const sq_layer* layers, int n_layers, int phase, const sq_attn* attn,
                                const float* x_in_dev, int64_t tokens, float* x_out_dev, void* ws_dev, size_t ws_bytes,
                                sq_stream_t stream) {
  sq_status st = check_layers(layers, n_layers, "sq_stage_forward_attn");
  if (st) return st;
  if ((st = check_attn(attn, layers[0].o.n, n_layers, phase, tokens, "sq_stage_forward_attn"))) return st;
  if (!x_in_dev || !x_out_dev || (reinterpret_cast<uintptr_t>(x_in_dev) & 15u) || (reinterpret_cast<uintptr_t>(x_out_dev) & 15u))
    return fail(SQ_EINVAL, "sq_stage_forward_attn: x_in/x_out null or not 16-B aligned");
  const size_t need = stage_workspace_bytes(layers, n_layers, tokens);
  if (!ws_dev || ws_bytes < need || (reinterpret_cast<uintptr_t>(ws_dev) & 255u))
    return fail(SQ_ENOMEM, "sq_stage_forward_attn: workspace %zu < %zu (or null / not 256-B aligned)", ws_bytes, need);
  return stage_forward(layers, n_layers, phase, x_in_dev, tokens, x_out_dev, nullptr, ws_dev, ws_bytes,
                       (cudaStream_t)stream, attn);
}

size_t sq_stage_tp_workspace_bytes(const sq_layer* shards, int n_shard_layers, int64_t max_tokens) {
  if (!shards || n_shard_layers <= 0 || max_tokens <= 0) return 0;
  return tp_layout(shards, n_shard_layers, max_tokens).total;
}

sq_status sq_stage_forward_tp(const sq_layer* shards, int n_layers, int tp, int tp_rank, sq_comm* comm, int phase,
                              const sq_attn* attn, const float* x_in_dev, int64_t tokens, float* x_out_dev,
                              void* ws_dev, size_t ws_bytes, sq_stream_t stream) {
  const char* who = "sq_stage_forward_tp";
  if (tp < 1 || tp_rank < -1 || tp_rank >= tp) return fail(SQ_EINVAL, "%s: tp %d, tp_rank %d", who, tp, tp_rank);
  const int n_sets = tp_rank < 0 ? tp : 1;
  sq_status st = check_tp(shards, n_layers, tp, n_sets, who);
  if (st) return st;
  if (tp_rank >= 0 && tp > 1) {
    if (!comm || comm_is_local(comm) || comm_size(comm) != tp || comm_rank(comm) != tp_rank)
      return fail(SQ_EINVAL, "%s: tp_rank %d needs an NCCL comm of %d ranks with that rank", who, tp_rank, tp);
  }
  if (phase != SQ_PREFILL && phase != SQ_DECODE) return fail(SQ_EINVAL, "%s: bad phase %d", who, phase);
  if (tokens < 1 || (phase == SQ_DECODE && tokens > 32))
    return fail(SQ_EINVAL, "%s: tokens=%lld (decode needs 1..32)", who, (long long)tokens);
  if (attn) {
    for (int r = 0; r < n_sets; ++r)
      if ((st = check_attn(&attn[r], shards[0].o.k, n_layers, phase, tokens, who))) return st;
  }
  if (!x_in_dev || !x_out_dev || (reinterpret_cast<uintptr_t>(x_in_dev) & 15u) || (reinterpret_cast<uintptr_t>(x_out_dev) & 15u))
    return fail(SQ_EINVAL, "%s: x_in/x_out null or not 16-B aligned", who);
  const size_t need = tp_layout(shards, n_layers * n_sets, tokens).total;
  if (!ws_dev || ws_bytes < need || (reinterpret_cast<uintptr_t>(ws_dev) & 255u))
    return fail(SQ_ENOMEM, "%s: workspace %zu < %zu (or null / not 256-B aligned)", who, ws_bytes, need);
  return stage_forward_tp(shards, n_layers, n_sets, (tp_rank >= 0 && tp > 1) ? comm : nullptr, tp_rank, phase,
                          attn, x_in_dev, tokens, x_out_dev, ws_dev, (cudaStream_t)stream);
}

sq_status sq_layernorm_f32(const float* x_dev, int64_t rows, int64_t d, float* y_dev, sq_stream_t stream) {
  if (!x_dev || !y_dev || rows <= 0 || d <= 0 || d % 128 || d > 14336) return fail(SQ_EINVAL, "sq_layernorm_f32: bad args");
  return cuda_check(launch_layernorm_f32(x_dev, rows, d, y_dev, (cudaStream_t)stream), "sq_layernorm_f32");
}

}  // extern "C"
