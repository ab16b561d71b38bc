// Tensor-map (TMA descriptor) encoding with a per-thread cache.
//
// cuTensorMapEncodeTiled is a pure function of its arguments, so a descriptor encoded once for a
// given (dtype, base pointer, dims, strides, box, swizzle) is reused by every later launch with the
// same arguments: the decode step's ~6 linears per layer re-use their weight and activation maps
// instead of re-encoding 2-3 descriptors per launch (include/sq.h, "TMA-descriptor cache").  The
// cache is thread-local (no locking on the launch path) and bounded: it is cleared when it reaches
// kMaxEntries.
#include <cuda.h>

#include <cstring>
#include <mutex>
#include <unordered_map>

#include "sq_internal.h"

namespace sq {
namespace {

typedef CUresult (*EncodeFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                             const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                             CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

EncodeFn get_encode() {
  static EncodeFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeFn>(f);
  });
  return fn;
}

struct Key {
  uint64_t v[16];  // dtype | rank | swizzle, ptr, dims[5], strides[4], box[5] packed
  bool operator==(const Key& o) const { return memcmp(v, o.v, sizeof(v)) == 0; }
};
struct KeyHash {
  size_t operator()(const Key& k) const {
    uint64_t h = 1469598103934665603ull;
    for (uint64_t x : k.v) { h ^= x + 0x9E3779B97F4A7C15ull + (h << 6) + (h >> 2); }
    return (size_t)h;
  }
};
constexpr size_t kMaxEntries = 8192;
thread_local std::unordered_map<Key, CUtensorMap, KeyHash>* t_cache = nullptr;
thread_local int64_t t_hits = 0, t_misses = 0;

}  // namespace

cudaError_t encode_nd(CUtensorMap* m, CUtensorMapDataType dt, const void* ptr, int rank, const uint64_t* dims,
                      const uint64_t* strides_bytes, const uint32_t* box, CUtensorMapSwizzle sw) {
  if (rank < 1 || rank > 5) return cudaErrorInvalidValue;
  Key key;
  memset(&key, 0, sizeof(key));
  key.v[0] = (uint64_t)dt | ((uint64_t)rank << 8) | ((uint64_t)sw << 16);
  key.v[1] = reinterpret_cast<uint64_t>(ptr);
  for (int i = 0; i < rank; ++i) key.v[2 + i] = dims[i];
  for (int i = 0; i + 1 < rank; ++i) key.v[7 + i] = strides_bytes[i];
  for (int i = 0; i < rank; ++i) key.v[11 + i] = box[i];
  if (!t_cache) t_cache = new std::unordered_map<Key, CUtensorMap, KeyHash>();
  auto it = t_cache->find(key);
  if (it != t_cache->end()) {
    ++t_hits;
    *m = it->second;
    return cudaSuccess;
  }
  ++t_misses;
  EncodeFn fn = get_encode();
  if (!fn) return cudaErrorNotSupported;
  cuuint64_t d[5], st[4];
  cuuint32_t b[5], es[5];
  for (int i = 0; i < rank; ++i) { d[i] = dims[i]; b[i] = box[i]; es[i] = 1; }
  for (int i = 0; i + 1 < rank; ++i) st[i] = strides_bytes[i];
  CUresult r = fn(m, dt, (cuuint32_t)rank, const_cast<void*>(ptr), d, st, b, es, CU_TENSOR_MAP_INTERLEAVE_NONE, sw,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return cudaErrorInvalidValue;
  if (t_cache->size() >= kMaxEntries) t_cache->clear();
  t_cache->emplace(key, *m);
  return cudaSuccess;
}

void tmap_cache_stats(int64_t* hits, int64_t* misses) {
  *hits = t_hits;
  *misses = t_misses;
}

}  // namespace sq

// debug/diagnostics (not part of include/sq.h): this thread's tensor-map cache hits / misses
extern "C" void sq_debug_tmap_stats(int64_t* hits, int64_t* misses) { sq::tmap_cache_stats(hits, misses); }
