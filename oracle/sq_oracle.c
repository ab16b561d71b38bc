/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.  Plain, slow, obviously-correct CPU
 * reference for the SplitQuant hot path (DESIGN.md
 * "Oracle").  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load it.  It shares no code with
 * the CUDA path (paper_conf_cluster_zhaowplw25_b200/csrc); neither side
 * includes or calls the other.
 *
 * Build: gcc -O2 -fopenmp -ffp-contract=off -fno-fast-math -shared -fPIC
 * (no FMA contraction: the quantizer is defined by single-rounded IEEE fp32
 * operations, one rounding per operation).
 *
 * Citations are PAPER.md line numbers ("P:<line>") in /root/reference.
 *
 * Functions and what pins them (tests/test_oracle_pins.py):
 *   oq_quantize_groups  P:91 (x^ = round((x - q_x)/s_x), s_x = (x_max - x_min)/(2^b - 1)),
 *                       asymmetric S_W of P:184; readings R1-R6 of DESIGN.md.
 *                       Pinned by brute-force argmin, exact ties, |w - w~| <= s/2, grid-aligned
 *                       recovery, constant groups, closed-form scale bound.
 *   oq_quantize_groups_ex  + symmetric S_W (R21) and stochastic rounding (Theorem 1,
 *                       P:176-180, R22).  Pinned by the published splitmix64 vectors, brute
 *                       force (symmetric), sign symmetry, unbiasedness, the floor/ceil
 *                       frequencies and Theorem 1's stochastic variance (tests/test_quant_variants.py).
 *   oq_pack/oq_unpack   Layouts L3/L4/L8 + tiling T16 of DESIGN.md (paper silent).  Pinned by
 *                       hand-derived golden words (tests/golden/pack_words.txt),
 *                       round trip, and the P:160 byte count.
 *   oq_dequant_row      x~ = s_x x^ + q_x, exact in fp64, saturated at 65504 (R20).
 *                       Pinned by the hand-computed +-65504 group (tests/test_oracle_pins.py).
 *   oq_linear           y = x W~^T (+ bias) in fp64 (weight-only W.A16).  Pinned by
 *                       numpy fp64 matmul at bits = 16 and on grid-aligned weights,
 *                       Theorem 1 variance bound.
 *   oq_layernorm        pre-LN block glue (R11), pinned by mean 0 / var 1.
 *   oq_stage            one pipeline stage = layers of P:160's linear set with the
 *                       attention stub (R12); pinned by composition checks.
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------- fp16 <-> fp32 (IEEE binary16, round-to-nearest-even) ---------------- */
static float h2f(uint16_t h) {
  _Float16 v;
  memcpy(&v, &h, 2);
  return (float)v;
}
static uint16_t f2h(float f) {
  _Float16 v = (_Float16)f; /* RNE */
  uint16_t h;
  memcpy(&h, &v, 2);
  return h;
}

float oq_h2f(uint16_t h) { return h2f(h); }

/* host threads of the parallel loops (timing the oracle at 1 thread and at all cores; no arithmetic) */
void oq_set_threads(int n) { omp_set_num_threads(n > 0 ? n : 1); }
int oq_max_threads(void) { return omp_get_max_threads(); }
uint16_t oq_f2h(float f) { return f2h(f); }

/* ---------------- O1: per-group quantization (S_W variants of P:184; rounding of P:176-180) ----
 * x^ = round((x - q_x) / s_x),  s_x = (x_max - x_min) / (2^b - 1),  x~ = s_x x^ + q_x.
 * Group = `group` contiguous weights of one output row (reading R4).  All arithmetic is
 * IEEE binary32 with one rounding per operation; the code is computed against the
 * fp16-ROUNDED scale that is stored (R5).
 *
 * mode bit 0 (OQ_SYMMETRIC, reading R21): P:184's symmetric scale
 *   S = max(|W_max|, |W_min|) / (2^(b-1) - 1), signed code c^ = clamp(round(w / S), -(2^(b-1)-1), 2^(b-1)-1),
 *   stored in the same unsigned (code, scale, zero) form as the asymmetric quantizer:
 *   c = c^ + 2^(b-1) in [1, 2^b - 1], zero q = -2^(b-1) S (so x~ = S c + q = S c^).  S == 0 -> c^ = 0, q = +0.
 *   A group whose q overflows fp16 is rejected (return 3).
 * otherwise (asymmetric, readings R2/R3): q_x = group minimum (fp16 exact, -0 -> +0), c in [0, 2^b - 1].
 *
 * mode bit 1 (OQ_STOCHASTIC, reading R22): the stochastic rounding of Theorem 1: with
 *   d the scaled value, c = floor(d) + [u < d - floor(d)], u = uniform24(seed, i) the i-th output of
 *   the counter-based generator below for the weight's row-major index i = r*k + col.
 *   Otherwise round to nearest, ties to even (R1).  s == 0 (constant group / underflow) -> d = 0.
 */
#define OQ_SYMMETRIC 1
#define OQ_STOCHASTIC 2

/* splitmix64 (Steele, Lea, Flood 2014): output i of the stream seeded `seed`, i.e. the finalizer of
 * state seed + (i + 1) * 0x9E3779B97F4A7C15.  uniform24 = top 24 bits / 2^24, exact in fp32. */
uint64_t oq_splitmix64(uint64_t seed, uint64_t i) {
  uint64_t z = seed + (i + 1) * 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
float oq_uniform24(uint64_t seed, uint64_t i) { return (float)(oq_splitmix64(seed, i) >> 40) * (1.0f / 16777216.0f); }

int oq_quantize_groups_ex(const uint16_t* w, int64_t n, int64_t k, int bits, int group, int mode, uint64_t seed,
                          uint8_t* codes, uint16_t* scales, uint16_t* zeros) {
  if (!(bits == 3 || bits == 4 || bits == 8) || group <= 0 || k % group || mode < 0 || mode > 3) return 1;
  const int64_t ng = k / group;
  const int sym = mode & OQ_SYMMETRIC, stoch = mode & OQ_STOCHASTIC;
  const int half_i = 1 << (bits - 1);
  const float qmax = (float)((1 << bits) - 1);
  const float cmin = sym ? -(float)(half_i - 1) : 0.0f;   /* clamp range of the (signed) code */
  const float cmax = sym ? (float)(half_i - 1) : qmax;
  const float off = sym ? (float)half_i : 0.0f;           /* stored code = code + off */
  for (int64_t r = 0; r < n; ++r) {
    for (int64_t g = 0; g < ng; ++g) {
      const uint16_t* p = w + r * k + g * group;
      float mn = h2f(p[0]), mx = mn;
      for (int j = 1; j < group; ++j) {
        float v = h2f(p[j]);
        if (v < mn) mn = v;
        if (v > mx) mx = v;
      }
      mn = mn + 0.0f;                       /* canonical zeros: -0 -> +0 */
      mx = mx + 0.0f;
      float sf, z;
      if (sym) {
        const float amax = fabsf(mx) > fabsf(mn) ? fabsf(mx) : fabsf(mn);
        sf = amax / (float)(half_i - 1);
      } else {
        sf = (mx - mn) / qmax;              /* two single-rounded fp32 ops */
      }
      const uint16_t s16 = f2h(sf);
      const float s = h2f(s16);
      if (sym) {
        z = -(float)half_i * s + 0.0f;      /* exact (power-of-two multiple); +0 when s == 0 */
        if (fabsf(z) > 65504.0f) return 3;
      } else {
        z = mn;
      }
      scales[r * ng + g] = s16;
      zeros[r * ng + g] = f2h(z);           /* exact */
      for (int j = 0; j < group; ++j) {
        float d = 0.0f;
        if (s != 0.0f) d = sym ? h2f(p[j]) / s : (h2f(p[j]) - mn) / s;  /* fp32 (sub), fp32 div */
        float q;
        if (stoch) {
          const float fl = floorf(d);
          const float fr = d - fl;          /* fp32 sub */
          q = fl + (oq_uniform24(seed, (uint64_t)(r * k + g * group + j)) < fr ? 1.0f : 0.0f);
        } else {
          q = rintf(d);                     /* round half to even */
        }
        if (q < cmin) q = cmin;
        if (q > cmax) q = cmax;
        codes[r * k + g * group + j] = (uint8_t)(int)(q + off);
      }
    }
  }
  return 0;
}

int oq_quantize_groups(const uint16_t* w, int64_t n, int64_t k, int bits, int group,
                       uint8_t* codes, uint16_t* scales, uint16_t* zeros) {
  return oq_quantize_groups_ex(w, n, k, bits, group, 0, 0, codes, scales, zeros);
}

/* ---------------- O2/O3: bit packing (DESIGN.md layouts L8, L4, L3 + tiling T16) ----------------
 * Within one row and one group of 128 codes (GB = 128*bits/8 bytes):
 * L8: byte j = c_j.
 * L4: 32-bit little-endian word j/8, nibble (j%8)/2 + 4*(j%2)   (even j in the low
 *     four nibbles, odd j in the high four).
 * L3 (reading R8, round 2): blocks of 32 codes = 3 words W0..W2; for j' = j%32: pair i = j'/2,
 *     half e = j'%2 (even k in the low 16 bits, odd k in the high 16 bits).  Pairs i < 15: word
 *     W_{i/5}, bits 16e + 3(i%5) .. +2 (five 3-bit codes per half).  Pair 15 (j' = 30, 31): code
 *     bit b at bit 15 + 16e of word W_b (the three spare bits of each half).
 * T16 (placement): rows are grouped in tiles of 16; the 16 rows' bytes of group g of
 *     tile t form one contiguous chunk ("unit") at byte ((t*kg + g)*16 + r%16)*GB,
 *     kg = k/128, units ordered tile-major / group-minor.
 * meta: uint32 at ((t*kg + g)*16 + r%16), low half = scale, high half = zero.
 * Requires n % 16 == 0, k % 128 == 0, group == 128.
 */
size_t oq_packed_bytes(int64_t n, int64_t k, int bits) { return (size_t)(n * k * bits / 8); }

static int64_t unit_off(int64_t r, int64_t g, int64_t kg) { return ((r / 16) * kg + g) * 16 + r % 16; }

int oq_pack(const uint8_t* codes, const uint16_t* scales, const uint16_t* zeros, int64_t n,
            int64_t k, int bits, int group, uint8_t* packed, uint32_t* meta) {
  if (!(bits == 3 || bits == 4 || bits == 8) || k % 128 || group != 128 || n % 16) return 1;
  const int64_t kg = k / 128, GB = 128 * bits / 8;
  memset(packed, 0, (size_t)(n * k * bits / 8));
  for (int64_t r = 0; r < n; ++r) {
    for (int64_t kk = 0; kk < k; ++kk) {
      uint32_t c = codes[r * k + kk];
      const int64_t g = kk / 128, j = kk % 128;
      uint8_t* grp = packed + unit_off(r, g, kg) * GB;
      if (bits == 8) {
        grp[j] = (uint8_t)c;
      } else if (bits == 4) {
        uint32_t word;
        int64_t wi = j / 8;
        int nib = (int)((j % 8) / 2 + 4 * (j % 2));
        memcpy(&word, grp + 4 * wi, 4);
        word |= (c & 0xF) << (4 * nib);
        memcpy(grp + 4 * wi, &word, 4);
      } else {
        int64_t blk = j / 32;
        int kp = (int)(j % 32), i = kp / 2, e = kp % 2;
        for (int b = 0; b < 3; ++b) {
          int wi, bit;
          if (i < 15) { wi = i / 5; bit = 16 * e + 3 * (i % 5) + b; }
          else { wi = b; bit = 15 + 16 * e; }
          uint32_t word;
          memcpy(&word, grp + 4 * (3 * blk + wi), 4);
          word |= ((c >> b) & 1u) << bit;
          memcpy(grp + 4 * (3 * blk + wi), &word, 4);
        }
      }
    }
  }
  for (int64_t r = 0; r < n; ++r)
    for (int64_t g = 0; g < kg; ++g)
      meta[unit_off(r, g, kg)] = (uint32_t)scales[r * kg + g] | ((uint32_t)zeros[r * kg + g] << 16);
  return 0;
}

/* O3: code of row r, column kk (inverse of oq_pack's placement and bit layout) */
static uint32_t code_at(const uint8_t* packed, int64_t r, int64_t kk, int64_t kg, int bits) {
  const int64_t GB = 128 * bits / 8, g = kk / 128, j = kk % 128;
  const uint8_t* grp = packed + unit_off(r, g, kg) * GB;
  if (bits == 8) return grp[j];
  if (bits == 4) {
    uint32_t word;
    memcpy(&word, grp + 4 * (j / 8), 4);
    int nib = (int)((j % 8) / 2 + 4 * (j % 2));
    return (word >> (4 * nib)) & 0xF;
  }
  int64_t blk = j / 32;
  int kp = (int)(j % 32), i = kp / 2, e = kp % 2;
  uint32_t c = 0;
  for (int b = 0; b < 3; ++b) {
    int wi, bit;
    if (i < 15) { wi = i / 5; bit = 16 * e + 3 * (i % 5) + b; }
    else { wi = b; bit = 15 + 16 * e; }
    uint32_t word;
    memcpy(&word, grp + 4 * (3 * blk + wi), 4);
    c |= ((word >> bit) & 1u) << b;
  }
  return c;
}

int oq_unpack(const uint8_t* packed, int64_t n, int64_t k, int bits, uint8_t* codes) {
  if (!(bits == 3 || bits == 4 || bits == 8) || k % 128 || n % 16) return 1;
  for (int64_t r = 0; r < n; ++r)
    for (int64_t kk = 0; kk < k; ++kk) codes[r * k + kk] = (uint8_t)code_at(packed, r, kk, k / 128, bits);
  return 0;
}

/* ---------------- O4: dequantize one row of a packed weight into fp64 ----------------
 * x~ = s x^ + q, exact in fp64 (s, q fp16; x^ < 256), then saturated to the fp16
 * finite range (reading R20: the dequantized weight is an fp16 operand of the W.A16 product,
 * P:93; only the top can overflow, since q = group min >= -65504 and s x^ >= 0, and the
 * saturation never moves x~ away from x, because every x <= 65504).  bits == 16: the fp16
 * weight itself (reading R7: FP16 layers are not quantized).
 */
#define OQ_F16_MAX 65504.0
static void dequant_row(const uint8_t* packed, const uint32_t* meta, int64_t n, int64_t k,
                        int bits, int group, int64_t r, double* out, uint8_t* tmp_codes) {
  (void)group; (void)n; (void)tmp_codes;
  if (bits == 16) {
    const uint16_t* wrow = (const uint16_t*)packed + r * k;
    for (int64_t kk = 0; kk < k; ++kk) out[kk] = (double)h2f(wrow[kk]);
    return;
  }
  const int64_t kg = k / 128;
  for (int64_t kk = 0; kk < k; ++kk) {
    uint32_t m = meta[unit_off(r, kk / 128, kg)];
    double s = (double)h2f((uint16_t)(m & 0xFFFF));
    double z = (double)h2f((uint16_t)(m >> 16));
    const double wt = s * (double)code_at(packed, r, kk, kg, bits) + z;
    out[kk] = wt > OQ_F16_MAX ? OQ_F16_MAX : wt;
  }
}

int oq_dequant(const uint8_t* packed, const uint32_t* meta, int64_t n, int64_t k, int bits,
               int group, double* w_out) {
  uint8_t* tmp = (uint8_t*)malloc((size_t)k);
  if (!tmp) return 2;
  for (int64_t r = 0; r < n; ++r) dequant_row(packed, meta, n, k, bits, group, r, w_out + r * k, tmp);
  free(tmp);
  return 0;
}

/* ---------------- O5: weight-only linear, fp64 ----------------
 * y[i][j] = sum_k x[i][k] * w~[j][k] (+ bias[j]);  x given in fp64 (fp16 values when the
 * caller passes fp16 activations).  Plain loops, parallel over output rows only.
 */
int oq_linear(const double* x, int64_t m, int64_t k, const uint8_t* packed, const uint32_t* meta,
              int64_t n, int bits, int group, const uint16_t* bias_f16, double* y) {
  int err = 0;
#pragma omp parallel
  {
    double* wrow = (double*)malloc((size_t)k * sizeof(double));
    uint8_t* tmp = (uint8_t*)malloc((size_t)k);
    if (!wrow || !tmp) err = 2;
#pragma omp for schedule(static)
    for (int64_t j = 0; j < n; ++j) {
      if (!wrow || !tmp) continue;
      dequant_row(packed, meta, n, k, bits, group, j, wrow, tmp);
      double b = bias_f16 ? (double)h2f(bias_f16[j]) : 0.0;
      for (int64_t i = 0; i < m; ++i) {
        double acc = 0.0;
        for (int64_t kk = 0; kk < k; ++kk) acc += x[i * k + kk] * wrow[kk];
        y[i * n + j] = acc + b;
      }
    }
    free(wrow);
    free(tmp);
  }
  return err;
}

/* ---------------- glue (R11/R12) ---------------- */
void oq_layernorm(const double* x, int64_t t, int64_t d, double eps, double* out) {
  for (int64_t i = 0; i < t; ++i) {
    const double* r = x + i * d;
    double mean = 0.0, var = 0.0;
    for (int64_t j = 0; j < d; ++j) mean += r[j];
    mean /= (double)d;
    for (int64_t j = 0; j < d; ++j) var += (r[j] - mean) * (r[j] - mean);
    var /= (double)d;
    double inv = 1.0 / sqrt(var + eps);
    for (int64_t j = 0; j < d; ++j) out[i * d + j] = (r[j] - mean) * inv;
  }
}

static double act_fn(double v, int act) {
  if (act == 0) return v > 0.0 ? v : 0.0;                         /* ReLU (OPT) */
  const double c = 0.7978845608028654;                             /* sqrt(2/pi) */
  return 0.5 * v * (1.0 + tanh(c * (v + 0.044715 * v * v * v)));  /* tanh-GeLU (BLOOM) */
}

typedef struct {
  int32_t bits, group;
  int64_t n, k;
  const uint8_t* packed; /* bits<16: packed codes; bits==16: fp16 W [n,k] */
  const uint32_t* meta;  /* NULL iff bits == 16 */
  const uint16_t* bias;  /* fp16 [n] or NULL */
} oq_weight;

typedef struct {
  int32_t bits, act;
  oq_weight qkv, o, fc1, fc2; /* qkv: [3*h1, h1]; o: [h1, h1]; fc1: [h2, h1]; fc2: [h1, h2] */
} oq_layer;

/* One stage = consecutive layers of a pre-LN decoder block with the attention stub
 * (attention output = V, R12).  For each layer (bits b):
 *   a = LN(x); [q k v] = a Wqkv^T (+b); h = x + v Wo^T (+b);
 *   u = act(LN(h) W1^T + b1); x = h + u W2^T (+b2)
 * x: fp64 [t, h1], updated in place.  qkv_dbg (optional): last layer's [t, 3*h1].
 */
int oq_stage(const oq_layer* layers, int n_layers, double* x, int64_t t, int64_t h1,
             double* qkv_dbg) {
  const int64_t h2 = layers[0].fc1.n;
  double* a = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* qkv = (double*)malloc((size_t)(t * 3 * h1) * sizeof(double));
  double* v = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* o = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* u = (double*)malloc((size_t)(t * h2) * sizeof(double));
  int err = (!a || !qkv || !v || !o || !u) ? 2 : 0;
  for (int l = 0; l < n_layers && !err; ++l) {
    const oq_layer* L = &layers[l];
    oq_layernorm(x, t, h1, 1e-5, a);
    err |= oq_linear(a, t, h1, L->qkv.packed, L->qkv.meta, 3 * h1, L->qkv.bits, L->qkv.group, L->qkv.bias, qkv);
    for (int64_t i = 0; i < t; ++i)
      for (int64_t j = 0; j < h1; ++j) v[i * h1 + j] = qkv[i * 3 * h1 + 2 * h1 + j];
    err |= oq_linear(v, t, h1, L->o.packed, L->o.meta, h1, L->o.bits, L->o.group, L->o.bias, o);
    for (int64_t i = 0; i < t * h1; ++i) x[i] += o[i];
    oq_layernorm(x, t, h1, 1e-5, a);
    err |= oq_linear(a, t, h1, L->fc1.packed, L->fc1.meta, h2, L->fc1.bits, L->fc1.group, L->fc1.bias, u);
    for (int64_t i = 0; i < t * h2; ++i) u[i] = act_fn(u[i], L->act);
    err |= oq_linear(u, t, h2, L->fc2.packed, L->fc2.meta, h1, L->fc2.bits, L->fc2.group, L->fc2.bias, o);
    for (int64_t i = 0; i < t * h1; ++i) x[i] += o[i];
    if (qkv_dbg && l == n_layers - 1) memcpy(qkv_dbg, qkv, (size_t)(t * 3 * h1) * sizeof(double));
  }
  free(a);
  free(qkv);
  free(v);
  free(o);
  free(u);
  return err;
}

/* ---------------- O8: causal multi-head self-attention with a KV cache ----------------
 * Readings R23-R25: h1 = n_heads * dh; the fused qkv row holds q = [0, h1), k = [h1, 2h1),
 * v = [2h1, 3h1) (R11), head j = columns j*dh .. (j+1)*dh - 1; scores q.k / sqrt(dh), causal within
 * a sequence (query at position p sees cache positions 0..p), softmax, no positional term inside the
 * layer; the KV cache of a layer holds k, v per (sequence, position): [B][max_len][h1] (P:162 sizes it
 * 2 v (s + n) h1 elements).
 * One call = one micro-batch of nseq sequences (cache rows seq0 .. seq0 + nseq - 1), each with `len`
 * new tokens at positions pos0 .. pos0 + len - 1 (prefill chunk: pos0 = chunk start; decode: len = 1,
 * pos0 = s + t - 1).  Row i*len + (p - pos0) of qkv/out is (sequence i, position p).  The new k, v rows
 * are written into the cache first, then every query attends over cache positions 0..p.  fp64.
 */
int oq_attention(const double* qkv, int64_t nseq, int64_t len, int64_t pos0, int64_t seq0, int64_t h1,
                 int n_heads, double* kc, double* vc, int64_t max_len, double* out) {
  if (n_heads <= 0 || h1 % n_heads || pos0 < 0 || pos0 + len > max_len) return 1;
  const int64_t dh = h1 / n_heads;
  const double scale = 1.0 / sqrt((double)dh);
  for (int64_t i = 0; i < nseq; ++i)
    for (int64_t p = pos0; p < pos0 + len; ++p) {
      const double* row = qkv + (i * len + (p - pos0)) * 3 * h1;
      double* kd = kc + ((seq0 + i) * max_len + p) * h1;
      double* vd = vc + ((seq0 + i) * max_len + p) * h1;
      for (int64_t c = 0; c < h1; ++c) { kd[c] = row[h1 + c]; vd[c] = row[2 * h1 + c]; }
    }
  double* w = (double*)malloc((size_t)max_len * sizeof(double));
  if (!w) return 2;
  for (int64_t i = 0; i < nseq; ++i)
    for (int64_t p = pos0; p < pos0 + len; ++p) {
      const double* q = qkv + (i * len + (p - pos0)) * 3 * h1;
      double* o = out + (i * len + (p - pos0)) * h1;
      for (int hd = 0; hd < n_heads; ++hd) {
        double mx = -INFINITY;
        for (int64_t j = 0; j <= p; ++j) {
          const double* kj = kc + ((seq0 + i) * max_len + j) * h1 + hd * dh;
          double sc = 0.0;
          for (int64_t c = 0; c < dh; ++c) sc += q[hd * dh + c] * kj[c];
          w[j] = sc * scale;
          if (w[j] > mx) mx = w[j];
        }
        double den = 0.0;
        for (int64_t j = 0; j <= p; ++j) { w[j] = exp(w[j] - mx); den += w[j]; }
        for (int64_t c = 0; c < dh; ++c) {
          double acc = 0.0;
          for (int64_t j = 0; j <= p; ++j) acc += w[j] * vc[((seq0 + i) * max_len + j) * h1 + hd * dh + c];
          o[hd * dh + c] = acc / den;
        }
      }
    }
  free(w);
  return 0;
}

/* One stage with real attention (O6 with O8 in place of the R12 stub): for each layer l,
 *   a = LN(x); [q k v] = a Wqkv^T (+b); att = O8(q, k, v; cache of layer l); h = x + att Wo^T (+b);
 *   u = act(LN(h) W1^T + b1); x = h + u W2^T (+b2).
 * kc_all / vc_all: [n_layers][B][max_len][h1] fp64 (this stage's layers). */
int oq_stage_attn(const oq_layer* layers, int n_layers, double* x, int64_t nseq, int64_t len, int64_t pos0,
                  int64_t seq0, int64_t h1, int n_heads, int64_t B, int64_t max_len, double* kc_all,
                  double* vc_all) {
  const int64_t t = nseq * len;
  const int64_t h2 = layers[0].fc1.n;
  double* a = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* qkv = (double*)malloc((size_t)(t * 3 * h1) * sizeof(double));
  double* att = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* o = (double*)malloc((size_t)(t * h1) * sizeof(double));
  double* u = (double*)malloc((size_t)(t * h2) * sizeof(double));
  int err = (!a || !qkv || !att || !o || !u) ? 2 : 0;
  const size_t cl = (size_t)(B * max_len * h1);
  for (int l = 0; l < n_layers && !err; ++l) {
    const oq_layer* L = &layers[l];
    oq_layernorm(x, t, h1, 1e-5, a);
    err |= oq_linear(a, t, h1, L->qkv.packed, L->qkv.meta, 3 * h1, L->qkv.bits, L->qkv.group, L->qkv.bias, qkv);
    err |= oq_attention(qkv, nseq, len, pos0, seq0, h1, n_heads, kc_all + l * cl, vc_all + l * cl, max_len, att);
    err |= oq_linear(att, t, h1, L->o.packed, L->o.meta, h1, L->o.bits, L->o.group, L->o.bias, o);
    for (int64_t i = 0; i < t * h1; ++i) x[i] += o[i];
    oq_layernorm(x, t, h1, 1e-5, a);
    err |= oq_linear(a, t, h1, L->fc1.packed, L->fc1.meta, h2, L->fc1.bits, L->fc1.group, L->fc1.bias, u);
    for (int64_t i = 0; i < t * h2; ++i) u[i] = act_fn(u[i], L->act);
    err |= oq_linear(u, t, h2, L->fc2.packed, L->fc2.meta, h1, L->fc2.bits, L->fc2.group, L->fc2.bias, o);
    for (int64_t i = 0; i < t * h1; ++i) x[i] += o[i];
  }
  free(a);
  free(qkv);
  free(att);
  free(o);
  free(u);
  return err;
}

/* ---------------- O9: W8A8 (weight-activation INT8; P:93 SmoothQuant / bitsandbytes) ------------
 * Reading R26: weights symmetric per output channel, activations symmetric per token (dynamic),
 * no smoothing factor; codes against the stored scale, fp32 single-rounded ops, ties to even:
 *   s_w[n] = fp16(fp32(max_k |W[n,k]|) / 127),  q_w = clamp(rint(fp32(W) / s_w), -127, 127)   (s_w == 0 -> 0)
 *   s_x[t] = fp32(max_k |x[t,k]|) / 127 (kept fp32),  q_x = clamp(rint(fp32(x) / s_x), -127, 127)
 *   acc[t,n] = sum_k q_x q_w (exact integer),  y = acc * s_x[t] * s_w[n] (+ bias) in fp64.
 */
static float rint_clamp127(float d) {
  float q = rintf(d);
  if (q < -127.0f) q = -127.0f;
  if (q > 127.0f) q = 127.0f;
  return q;
}

int oq_quantize_w8_channel(const uint16_t* w, int64_t n, int64_t k, int8_t* codes, uint16_t* scales) {
  for (int64_t r = 0; r < n; ++r) {
    float amax = 0.0f;
    for (int64_t j = 0; j < k; ++j) {
      const float a = fabsf(h2f(w[r * k + j]));
      if (a > amax) amax = a;
    }
    const uint16_t s16 = f2h(amax / 127.0f);
    const float s = h2f(s16);
    scales[r] = s16;
    for (int64_t j = 0; j < k; ++j) codes[r * k + j] = (int8_t)(s == 0.0f ? 0 : (int)rint_clamp127(h2f(w[r * k + j]) / s));
  }
  return 0;
}

int oq_quantize_act8(const uint16_t* x, int64_t m, int64_t k, int8_t* codes, float* scales) {
  for (int64_t t = 0; t < m; ++t) {
    float amax = 0.0f;
    for (int64_t j = 0; j < k; ++j) {
      const float a = fabsf(h2f(x[t * k + j]));
      if (a > amax) amax = a;
    }
    const float s = amax / 127.0f;
    scales[t] = s;
    for (int64_t j = 0; j < k; ++j) codes[t * k + j] = (int8_t)(s == 0.0f ? 0 : (int)rint_clamp127(h2f(x[t * k + j]) / s));
  }
  return 0;
}

int oq_linear_w8a8(const int8_t* xq, const float* sx, int64_t m, int64_t k, const int8_t* wq, const uint16_t* sw,
                   int64_t n, const uint16_t* bias, int64_t* acc_out, double* y) {
#pragma omp parallel for schedule(static)
  for (int64_t j = 0; j < n; ++j) {
    for (int64_t t = 0; t < m; ++t) {
      int64_t acc = 0;
      for (int64_t kk = 0; kk < k; ++kk) acc += (int64_t)xq[t * k + kk] * (int64_t)wq[j * k + kk];
      if (acc_out) acc_out[t * n + j] = acc;
      y[t * n + j] = (double)acc * (double)sx[t] * (double)h2f(sw[j]) + (bias ? (double)h2f(bias[j]) : 0.0);
    }
  }
  return 0;
}
