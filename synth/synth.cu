// Device-side twin of synth/synth.py: the same counter-based, integer-exact
// generator, so multi-GB synthetic weight sets can be created directly in HBM
// with values bit-identical to the host generator.  Holds no SplitQuant
// arithmetic; the product library does not link it.
#include <cstdint>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

namespace {

__host__ __device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__device__ __forceinline__ float synth_value(uint64_t base, uint64_t i, float scale,
                                             float scale_out, int outliers) {
  uint64_t h1 = splitmix64(base + i);
  uint64_t h2 = splitmix64(h1);
  int64_t n = (int64_t)((h1 & 0xFFFF) + ((h1 >> 16) & 0xFFFF) + ((h1 >> 32) & 0xFFFF) + (h1 >> 48)) - 131070;
  float m = scale;
  if (outliers && ((h2 >> 32) % 1000ull) == 0) m = scale_out;
  return __fmul_rn((float)n, m);
}

__global__ void k_fill_f16(__half* out, uint64_t base, uint64_t start, uint64_t count,
                           float scale, float scale_out, int outliers) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
    out[i] = __float2half_rn(synth_value(base, start + i, scale, scale_out, outliers));
}

__global__ void k_fill_f32(float* out, uint64_t base, uint64_t start, uint64_t count,
                           float scale, float scale_out, int outliers) {
  uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < count; i += stride)
    out[i] = synth_value(base, start + i, scale, scale_out, outliers);
}

int grid_for(uint64_t count) {
  uint64_t b = (count + 255) / 256;
  return (int)(b < 148ull * 64 ? (b ? b : 1) : 148ull * 64);
}

}  // namespace

extern "C" {

// Fill out[0..count) with generator elements start..start+count (fp16, RNE).
int synth_fill_f16(void* out, uint64_t seed, uint64_t start, uint64_t count, float scale,
                   float scale_out, int outliers, void* stream) {
  if (count == 0) return 0;
  k_fill_f16<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(
      (__half*)out, splitmix64(seed), start, count, scale, scale_out, outliers);
  return (int)cudaGetLastError();
}

int synth_fill_f32(void* out, uint64_t seed, uint64_t start, uint64_t count, float scale,
                   float scale_out, int outliers, void* stream) {
  if (count == 0) return 0;
  k_fill_f32<<<grid_for(count), 256, 0, (cudaStream_t)stream>>>(
      (float*)out, splitmix64(seed), start, count, scale, scale_out, outliers);
  return (int)cudaGetLastError();
}

// Host C implementation (used by tests to check numpy == C == device).
void synth_fill_f32_host(float* out, uint64_t seed, uint64_t start, uint64_t count, float scale,
                         float scale_out, int outliers) {
  uint64_t base = splitmix64(seed);
  for (uint64_t j = 0; j < count; ++j) {
    uint64_t h1 = splitmix64(base + start + j);
    uint64_t h2 = splitmix64(h1);
    int64_t n = (int64_t)((h1 & 0xFFFF) + ((h1 >> 16) & 0xFFFF) + ((h1 >> 32) & 0xFFFF) + (h1 >> 48)) - 131070;
    float m = scale;
    if (outliers && ((h2 >> 32) % 1000ull) == 0) m = scale_out;
    volatile float v = (float)n * m;
    out[j] = v;
  }
}

}  // extern "C"
