// Internal declarations shared by the libsq translation units (not installed).
#pragma once
#include <cstdarg>
#include <cstdint>
#include <cuda.h>
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include "sq.h"

namespace sq {

// ---- error state (thread-local message, sq_last_error) ----
sq_status fail(sq_status st, const char* fmt, ...);
sq_status cuda_check(cudaError_t e, const char* what);

// ---- launch accounting / profiling (sq_profile_*) ----
enum KClass { KC_GEMV = 0, KC_GEMM = 1, KC_GLUE = 2, KC_QUANT = 3, KC_ATTN_DEC = 4, KC_ATTN_PRE = 5 };
struct ProfTicket {
  int slot = -1;
};
ProfTicket prof_begin(int kclass, double bytes, double flops, cudaStream_t s);
void prof_end(ProfTicket t, cudaStream_t s);
void count_launch(int n = 1);
bool prof_enabled();

// ---- kernel launchers (validated arguments) ----
cudaError_t launch_quantize(const __half* w, int64_t n, int64_t k, int bits, int group, uint8_t* codes,
                            __half* scales, __half* zeros, int mode, uint64_t seed, int* status, cudaStream_t s);
cudaError_t launch_pack(const uint8_t* codes, const __half* scales, const __half* zeros, int64_t n, int64_t k,
                        int bits, int group, void* packed, uint32_t* meta, cudaStream_t s);
cudaError_t launch_xsum(const __half* x, int64_t ldx, int64_t m, int64_t k, float2* xsum, cudaStream_t s);

size_t gemv_workspace_bytes(int64_t n, int64_t k, int64_t m);
size_t xsum_bytes(int64_t k);
cudaError_t launch_gemv(const sq_qweight& w, const __half* x, int64_t ldx, int m, void* y, int64_t ldy, int epi,
                        const float2* xsum, void* ws, cudaStream_t s);

size_t gemv_tc_workspace_bytes(int64_t n, int64_t k);
size_t gemv_tc_xsum_offset(int64_t n, int64_t k);
cudaError_t launch_gemv_tc(const sq_qweight& w, const __half* x, int64_t ldx, int m, void* y, int64_t ldy, int epi,
                           void* ws, cudaStream_t s);
int gemv_path(int64_t n, int64_t k, int m, int bits);  // 0 = mma.sync (K2 / K2s), 1 = tcgen05 (K2c)
bool use_k2s(int bits, int64_t n, int64_t k, int m);   // within path 0: the strip kernel (own group sums)

cudaError_t launch_gemm(const sq_qweight& w, const __half* x, int64_t ldx, int64_t m, void* y, int64_t ldy,
                        int epi, cudaStream_t s);

cudaError_t launch_layernorm_f16(const float* x, int64_t rows, int64_t d, __half* y, float2* xsum,
                                 const float* copy_src, float* copy_dst, cudaStream_t s);
cudaError_t launch_layernorm_f32(const float* x, int64_t rows, int64_t d, float* y, cudaStream_t s);
cudaError_t launch_copy_rows(const float* src, int64_t sstride, int64_t rows, int64_t d, float* dst, int64_t dstride,
                             cudaStream_t s);

// ---- stage forward (sq_stage.cu), used by the pipeline runner ----
size_t stage_workspace_bytes(const sq_layer* layers, int n_layers, int64_t max_tokens);
sq_status stage_forward(const sq_layer* layers, int n_layers, int phase, const float* x_in, int64_t tokens,
                        float* x_out, void* qkv_dbg, void* ws, size_t ws_bytes, cudaStream_t s,
                        const sq_attn* att = nullptr);
sq_status check_layers(const sq_layer* layers, int n_layers, const char* who);
sq_status check_attn(const sq_attn* a, int64_t h1, int n_layers, int phase, int64_t tokens, const char* who);

// ---- tensor-parallel stage (sq_stage.cu, f4)
size_t stage_tp_workspace_bytes(const sq_layer* sh, int n_shard_layers, int64_t max_tokens);
sq_status check_tp(const sq_layer* sh, int n_layers, int tp, int n_sets, const char* who);
sq_status stage_forward_tp(const sq_layer* sh, int n_layers, int n_sets, sq_comm* comm, int tp_rank, int phase,
                           const sq_attn* att, const float* x_in, int64_t T, float* x_out, void* ws, cudaStream_t s);

// ---- TP all-reduce (sq_pipeline.cu): in-place fp32 sum over the comm's world communicator
sq_status comm_allreduce_sum_f32(sq_comm* c, float* buf, size_t count, cudaStream_t s);
int comm_size(const sq_comm* c);
int comm_rank(const sq_comm* c);
bool comm_is_local(const sq_comm* c);

// ---- attention (sq_attn.cu): kv_append + prefill / decode attention for one layer
cudaError_t launch_attention(const __half* qkv, int64_t ldq, int nseq, int len, int pos0, int64_t seq0, int h1,
                             int n_heads, __half* kc, __half* vc, int max_len, __half* out, int64_t ldo,
                             cudaStream_t s);

int num_sms();

// ---- TMA descriptors (sq_tmap.cu): cuTensorMapEncodeTiled behind a per-thread cache
cudaError_t encode_nd(CUtensorMap* m, CUtensorMapDataType dt, const void* ptr, int rank, const uint64_t* dims,
                      const uint64_t* strides_bytes, const uint32_t* box, CUtensorMapSwizzle sw);

// ---- programmatic dependent launch (PDL) ----
// Decode kernels are launched with programmatic stream serialization: the next kernel of the
// stream may be scheduled while this one drains, runs its prologue (barriers, TMEM, and the
// first weight fetches -- weights never depend on the previous kernel), and blocks in
// griddepcontrol.wait (pdl_wait) before it touches anything the previous kernel produces or
// consumes.  Every kernel launched this way calls pdl_wait before its first dependent access.
// SQ_PDL=0 disables the attribute (plain stream order).
bool pdl_enabled();
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, static_cast<Args&&>(args)...);
}

}  // namespace sq
