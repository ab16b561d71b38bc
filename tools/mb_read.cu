// Microbenchmark: what a plain streaming read of S bytes costs on this B200, per launch, when
// launched back to back from a CUDA graph over R rotating copies (> 2 x L2, so every launch
// streams from HBM) -- the floor a decode GEMV of the same bytes can reach, launch gaps,
// ramp-up and tail included.  Also: an empty kernel (the per-launch floor).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/mb_read tools/mb_read.cu
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__global__ void k_empty() {}

// grid-stride 16-B loads, 4 in flight per thread, one store per CTA
__global__ void __launch_bounds__(512) k_read(const uint4* __restrict__ p, size_t n16, float* out) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 3 * stride < n16; i += 4 * stride) {
    uint4 a = __ldg(p + i), b = __ldg(p + i + stride), c = __ldg(p + i + 2 * stride), d = __ldg(p + i + 3 * stride);
    acc ^= a.x ^ a.y ^ a.z ^ a.w ^ b.x ^ b.y ^ b.z ^ b.w ^ c.x ^ c.y ^ c.z ^ c.w ^ d.x ^ d.y ^ d.z ^ d.w;
  }
  for (; i < n16; i += stride) { uint4 a = __ldg(p + i); acc ^= a.x ^ a.y ^ a.z ^ a.w; }
  if (acc == 0x12345678u) out[blockIdx.x] = 1.f;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaStream_t s;
  cudaStreamCreate(&s);
  float* out;
  cudaMalloc(&out, 1 << 20);
  const int NL = 60;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto time_graph = [&](auto&& body) {
    cudaGraph_t g;
    cudaGraphExec_t ge;
    cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal);
    body();
    cudaStreamEndCapture(s, &g);
    cudaGraphInstantiate(&ge, g, 0);
    cudaGraphLaunch(ge, s);
    cudaStreamSynchronize(s);
    float best = 1e30f;
    for (int r = 0; r < 5; ++r) {
      cudaEventRecord(e0, s);
      cudaGraphLaunch(ge, s);
      cudaEventRecord(e1, s);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (ms < best) best = ms;
    }
    cudaGraphExecDestroy(ge);
    cudaGraphDestroy(g);
    return best * 1e3f / NL;  // us per launch
  };
  printf("{\"empty_us\": %.3f}\n", time_graph([&] { for (int i = 0; i < NL; ++i) k_empty<<<sms, 512, 0, s>>>(); }));
  for (double mb : {3.5, 7.0, 14.0, 28.0, 56.0, 112.0, 185.0, 400.0}) {
    const size_t bytes = (size_t)(mb * 1e6) / 16 * 16;
    int R = (int)(600e6 / bytes) + 1;
    if (R < 2) R = 2;
    std::vector<uint4*> bufs(R);
    for (auto& b : bufs) { cudaMalloc(&b, bytes); cudaMemset(b, 1, bytes); }
    for (int cpb : {1, 2, 4}) {
      const float us = time_graph([&] {
        for (int i = 0; i < NL; ++i) k_read<<<sms * cpb, 512, 0, s>>>(bufs[i % R], bytes / 16, out);
      });
      printf("{\"MB\": %.1f, \"ctas_per_sm\": %d, \"us\": %.2f, \"GBps\": %.1f}\n", mb, cpb, us, bytes / us / 1e3);
    }
    for (auto& b : bufs) cudaFree(b);
  }
  return 0;
}
