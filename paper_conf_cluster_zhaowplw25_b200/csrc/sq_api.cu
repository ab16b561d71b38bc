// C-ABI entry points of libsq (include/sq.h): argument validation (before any
// launch), error state, launch accounting and the event-based profiler.
#include <atomic>
#include <cstdlib>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <vector>

#include "sq_common.cuh"

namespace sq {

static thread_local char g_err[512] = "";

sq_status fail(sq_status st, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return st;
}

sq_status cuda_check(cudaError_t e, const char* what) {
  if (e == cudaSuccess) return SQ_OK;
  return fail(SQ_ECUDA, "%s: %s", what, cudaGetErrorString(e));
}

bool pdl_enabled() {
  static int on = -1;
  if (on < 0) {
    const char* e = getenv("SQ_PDL");
    on = (e && e[0] == '0') ? 0 : 1;
  }
  return on == 1;
}

int num_sms() {
  static int cached = 0;
  if (!cached) {
    int dev = 0, v = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev);
    cached = v > 0 ? v : 148;
  }
  return cached;
}

// ---------------------------------------------------------------- profiling
static std::atomic<int64_t> g_launches{0};
static std::atomic<int> g_prof_on{0};
struct ProfRec {
  int kclass;
  double bytes, flops;
  cudaEvent_t e0, e1;
};
static std::mutex g_prof_mu;
static std::vector<ProfRec> g_prof;
static std::vector<cudaEvent_t> g_event_pool;

void count_launch(int n) { g_launches.fetch_add(n, std::memory_order_relaxed); }

static cudaEvent_t get_event() {
  if (!g_event_pool.empty()) {
    cudaEvent_t e = g_event_pool.back();
    g_event_pool.pop_back();
    return e;
  }
  cudaEvent_t e;
  cudaEventCreate(&e);
  return e;
}

ProfTicket prof_begin(int kclass, double bytes, double flops, cudaStream_t s) {
  ProfTicket t;
  if (!g_prof_on.load(std::memory_order_relaxed)) return t;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  ProfRec r{kclass, bytes, flops, get_event(), get_event()};
  cudaEventRecord(r.e0, s);
  g_prof.push_back(r);
  t.slot = (int)g_prof.size() - 1;
  return t;
}

void prof_end(ProfTicket t, cudaStream_t s) {
  if (t.slot < 0) return;
  std::lock_guard<std::mutex> lk(g_prof_mu);
  cudaEventRecord(g_prof[t.slot].e1, s);
}

bool prof_enabled() { return g_prof_on.load(std::memory_order_relaxed) != 0; }

}  // namespace sq

using namespace sq;

namespace {

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }
bool valid_bits(int b) { return b == 3 || b == 4 || b == 8 || b == 16; }

sq_status check_qweight(const sq_qweight* w, const char* who) {
  if (!w) return fail(SQ_EINVAL, "%s: null weight", who);
  if (!valid_bits(w->bits)) return fail(SQ_EINVAL, "%s: bits=%d not in {3,4,8,16}", who, w->bits);
  if (w->n <= 0 || w->k <= 0 || w->n % 16 || w->k % 128)
    return fail(SQ_EINVAL, "%s: need n%%16==0, k%%128==0 (n=%lld k=%lld)", who, (long long)w->n, (long long)w->k);
  if (w->bits != 16 && w->group != 128)
    return fail(SQ_ENOTSUP, "%s: linear kernels implement group=128 only (got %d)", who, w->group);
  if (!w->packed || !aligned16(w->packed)) return fail(SQ_EINVAL, "%s: packed null or not 16-B aligned", who);
  if (w->bits != 16 && (!w->meta || !aligned16(w->meta)))
    return fail(SQ_EINVAL, "%s: meta null or not 16-B aligned", who);
  if (w->bias && (reinterpret_cast<uintptr_t>(w->bias) & 3u))
    return fail(SQ_EINVAL, "%s: bias must be 4-B aligned", who);
  return SQ_OK;
}

sq_status check_x(const void* x, int64_t ldx, int64_t k, const char* who) {
  if (!x || !aligned16(x)) return fail(SQ_EINVAL, "%s: x null or not 16-B aligned", who);
  if (ldx < k || ldx % 8) return fail(SQ_EINVAL, "%s: ldx=%lld must be >= k and a multiple of 8", who, (long long)ldx);
  return SQ_OK;
}

sq_status check_y(const void* y, int64_t ldy, int64_t n, int epi, const char* who) {
  if (!y || !aligned16(y)) return fail(SQ_EINVAL, "%s: y null or not 16-B aligned", who);
  if (epi < SQ_EPI_F16 || epi > SQ_EPI_F32_ACCUM) return fail(SQ_EINVAL, "%s: bad epilogue %d", who, epi);
  if (ldy < n || ldy % 8) return fail(SQ_EINVAL, "%s: ldy=%lld must be >= n and a multiple of 8", who, (long long)ldy);
  return SQ_OK;
}

}  // namespace

extern "C" {

const char* sq_last_error(void) { return g_err; }
const char* sq_version(void) { return "libsq 0.1 (sm_100a)"; }
int sq_abi_version(void) { return 3; }

size_t sq_packed_bytes(int64_t n, int64_t k, int bits) {
  if (n <= 0 || k <= 0 || !valid_bits(bits) || (n * k * bits) % 8) return 0;
  return (size_t)(n * k * bits / 8);
}

size_t sq_meta_bytes(int64_t n, int64_t k, int group) {
  if (n <= 0 || k <= 0 || group <= 0 || k % group) return 0;
  return (size_t)(n * (k / group) * 4);
}

sq_status sq_quantize_groups_ex(const void* w_dev, int64_t n, int64_t k, int bits, int group, int mode,
                                uint64_t seed, uint8_t* codes_dev, void* scales_dev, void* zeros_dev,
                                int32_t* status_dev, sq_stream_t stream) {
  if (!(bits == 3 || bits == 4 || bits == 8)) return fail(SQ_EINVAL, "sq_quantize_groups: bits=%d not in {3,4,8}", bits);
  if (!(group == 32 || group == 64 || group == 128))
    return fail(SQ_EINVAL, "sq_quantize_groups: group=%d not in {32,64,128}", group);
  if (n <= 0 || k <= 0 || k % group) return fail(SQ_EINVAL, "sq_quantize_groups: bad shape n=%lld k=%lld", (long long)n, (long long)k);
  if (mode < 0 || mode > (SQ_QUANT_SYMMETRIC | SQ_QUANT_STOCHASTIC))
    return fail(SQ_EINVAL, "sq_quantize_groups_ex: mode=%d", mode);
  if (!w_dev || !codes_dev || !scales_dev || !zeros_dev) return fail(SQ_EINVAL, "sq_quantize_groups: null pointer");
  if ((mode & SQ_QUANT_SYMMETRIC) && !status_dev)
    return fail(SQ_EINVAL, "sq_quantize_groups_ex: the symmetric mode needs status_dev");
  if ((reinterpret_cast<uintptr_t>(w_dev) & 7u) || (reinterpret_cast<uintptr_t>(codes_dev) & 3u))
    return fail(SQ_EINVAL, "sq_quantize_groups: w must be 8-B and codes 4-B aligned");
  return cuda_check(launch_quantize((const __half*)w_dev, n, k, bits, group, codes_dev, (__half*)scales_dev,
                                    (__half*)zeros_dev, mode, seed, (int*)status_dev, (cudaStream_t)stream),
                    "sq_quantize_groups");
}

sq_status sq_quantize_groups(const void* w_dev, int64_t n, int64_t k, int bits, int group, uint8_t* codes_dev,
                             void* scales_dev, void* zeros_dev, sq_stream_t stream) {
  return sq_quantize_groups_ex(w_dev, n, k, bits, group, 0, 0, codes_dev, scales_dev, zeros_dev, nullptr, stream);
}

sq_status sq_pack(const uint8_t* codes_dev, const void* scales_dev, const void* zeros_dev, int64_t n, int64_t k,
                  int bits, int group, void* packed_dev, void* meta_dev, sq_stream_t stream) {
  if (!(bits == 3 || bits == 4 || bits == 8)) return fail(SQ_EINVAL, "sq_pack: bits=%d not in {3,4,8}", bits);
  if (group != 128) return fail(SQ_ENOTSUP, "sq_pack: packed layout T16 implements group=128 only (got %d)", group);
  if (n <= 0 || k <= 0 || k % 128 || n % 16) return fail(SQ_EINVAL, "sq_pack: need n%%16==0, k%%128==0");
  if (!codes_dev || !scales_dev || !zeros_dev || !packed_dev || !meta_dev) return fail(SQ_EINVAL, "sq_pack: null pointer");
  if (!aligned16(codes_dev) || !aligned16(packed_dev) || (reinterpret_cast<uintptr_t>(meta_dev) & 3u))
    return fail(SQ_EINVAL, "sq_pack: codes/packed must be 16-B aligned, meta 4-B aligned");
  return cuda_check(launch_pack(codes_dev, (const __half*)scales_dev, (const __half*)zeros_dev, n, k, bits, group,
                                packed_dev, (uint32_t*)meta_dev, (cudaStream_t)stream),
                    "sq_pack");
}

size_t sq_linear_workspace_bytes(const sq_qweight* w, int64_t m) {
  if (!w || w->n <= 0 || w->k <= 0 || m <= 0) return 0;
  return gemv_workspace_bytes(w->n, w->k, m < 32 ? m : 32);
}

sq_status sq_xsum(const void* x_dev, int64_t ldx, int64_t m, int64_t k, void* xsum_dev, sq_stream_t stream) {
  if (m <= 0 || k <= 0 || k % 128) return fail(SQ_EINVAL, "sq_xsum: bad shape");
  sq_status st = check_x(x_dev, ldx, k, "sq_xsum");
  if (st) return st;
  if (!xsum_dev || (reinterpret_cast<uintptr_t>(xsum_dev) & 7u)) return fail(SQ_EINVAL, "sq_xsum: xsum null/misaligned");
  return cuda_check(launch_xsum((const __half*)x_dev, ldx, m, k, (float2*)xsum_dev, (cudaStream_t)stream), "sq_xsum");
}

sq_status sq_linear_decode(const sq_qweight* w, const void* x_dev, int64_t ldx, int64_t m, void* y_dev, int64_t ldy,
                           int epi, const void* xsum_dev, void* ws_dev, size_t ws_bytes, sq_stream_t stream) {
  sq_status st = check_qweight(w, "sq_linear_decode");
  if (st) return st;
  if (m < 1 || m > 32) return fail(SQ_EINVAL, "sq_linear_decode: m=%lld not in [1,32]", (long long)m);
  if (w->n > 65536) return fail(SQ_ENOTSUP, "sq_linear_decode: n=%lld > 65536", (long long)w->n);
  if ((st = check_x(x_dev, ldx, w->k, "sq_linear_decode"))) return st;
  if ((st = check_y(y_dev, ldy, w->n, epi, "sq_linear_decode"))) return st;
  if (xsum_dev && (reinterpret_cast<uintptr_t>(xsum_dev) & 7u)) return fail(SQ_EINVAL, "sq_linear_decode: xsum misaligned");
  const size_t need = sq_linear_workspace_bytes(w, m);
  if (!ws_dev || ws_bytes < need || !aligned16(ws_dev))
    return fail(SQ_ENOMEM, "sq_linear_decode: workspace %zu < %zu bytes (or null/misaligned)", ws_bytes, need);
  return cuda_check(launch_gemv(*w, (const __half*)x_dev, ldx, (int)m, y_dev, ldy, epi, (const float2*)xsum_dev,
                                ws_dev, (cudaStream_t)stream),
                    "sq_linear_decode");
}

sq_status sq_linear_prefill(const sq_qweight* w, const void* x_dev, int64_t ldx, int64_t m, void* y_dev, int64_t ldy,
                            int epi, sq_stream_t stream) {
  sq_status st = check_qweight(w, "sq_linear_prefill");
  if (st) return st;
  if (w->n % 128) return fail(SQ_EINVAL, "sq_linear_prefill: n=%lld must be a multiple of 128", (long long)w->n);
  if (m < 1 || m > (1ll << 31)) return fail(SQ_EINVAL, "sq_linear_prefill: bad m=%lld", (long long)m);
  if ((st = check_x(x_dev, ldx, w->k, "sq_linear_prefill"))) return st;
  if ((st = check_y(y_dev, ldy, w->n, epi, "sq_linear_prefill"))) return st;
  return cuda_check(launch_gemm(*w, (const __half*)x_dev, ldx, m, y_dev, ldy, epi, (cudaStream_t)stream),
                    "sq_linear_prefill");
}

sq_status sq_profile_enable(int on) {
  std::lock_guard<std::mutex> lk(g_prof_mu);
  g_prof_on.store(on ? 1 : 0);
  return SQ_OK;
}

sq_status sq_profile_read(sq_profile* out) {
  if (!out) return fail(SQ_EINVAL, "sq_profile_read: null");
  std::lock_guard<std::mutex> lk(g_prof_mu);
  memset(out, 0, sizeof(*out));
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) return cuda_check(e, "sq_profile_read");
  for (auto& r : g_prof) {
    float ms = 0.f;
    cudaEventElapsedTime(&ms, r.e0, r.e1);
    out->launches[r.kclass] += 1;
    out->ms[r.kclass] += ms;
    out->bytes[r.kclass] += r.bytes;
    out->flops[r.kclass] += r.flops;
    g_event_pool.push_back(r.e0);
    g_event_pool.push_back(r.e1);
  }
  g_prof.clear();
  return SQ_OK;
}

int64_t sq_launch_count(void) { return g_launches.load(); }

}  // extern "C"
