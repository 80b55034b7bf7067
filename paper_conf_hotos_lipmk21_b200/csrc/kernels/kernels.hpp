// kernels.hpp — host launchers of the step's kernels (all asynchronous on `st`).
#pragma once
#include <cmath>
#include <algorithm>
#include <utility>

#include "../common.hpp"
#include "harmony_kernels.h"

namespace hm {

// Programmatic dependent launch: every kernel of the step is launched with programmatic stream
// serialisation, so the next kernel on the stream is launched (and, for the persistent tcgen05
// kernels, runs its setup: barriers, tensor-map prefetch, TMEM allocation) while the previous one
// drains; each kernel executes griddepcontrol.wait (pdl_wait) before it touches global memory, which
// returns once the previous grid has completed and its writes are visible — the results are the
// same as with plain stream order.  HARMONY_PDL=0 launches without the attribute (A/B).
bool pdl_enabled();
template <typename... KArgs, typename... Args>
inline void launch_k(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl_enabled() ? 1 : 0;
  HM_CUDA(cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...));
}
#ifdef __CUDACC__
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
#endif

void gemm(const hk_gemm_args& a, cudaStream_t st);
// gemm() with a bf16 output C (nz0 = nz1 = 1) that also writes partial[rb][c] = sum of the STORED
// (bf16-rounded) C[r][c] over the rows r of block rb = r / 32, rows in increasing order (fp32);
// partial is [ceil(M/32)][N].  The ACT_BWD CTA-pair kernel sums its staged output boxes in its
// epilogue; any other path runs a separate pass with the same order (identical partials).
void gemm_colsum(const hk_gemm_args& a, float* partial, cudaStream_t st);
inline size_t colsum32_partial_bytes(int64_t rows, int n) { return (size_t)((rows + 31) / 32) * n * sizeof(float); }
void colsum32_partial(int64_t rows, int n, const void* X, int64_t ld, float* partial, cudaStream_t st);
// out[c] (+)= sum over the ceil(rows/32) partials of gemm_colsum, in a fixed tree (deterministic)
void colsum32_reduce(int64_t rows, int n, const float* partial, float* out, int accumulate, cudaStream_t st);

void layernorm_fwd(int dtype, int64_t rows, int d, const float* X, const void* g, const void* b, void* U, float* mean,
                   float* rstd, cudaStream_t st, float* Xcopy = nullptr);
size_t layernorm_bwd_scratch_bytes(int64_t rows, int d);
// register-resident variants (d % 4 == 0, d <= 2048); return false when not applicable
bool layernorm_fwd_vec(int dtype, int64_t rows, int d, const float* X, const void* g, const void* b, void* U,
                       float* mean, float* rstd, cudaStream_t st, float* Xcopy = nullptr);
size_t layernorm_bwd_vec_scratch_bytes(int64_t rows, int d);
bool layernorm_bwd_vec(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                       const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db,
                       int accumulate, void* dXt, float* dsum, int dsum_acc, float* scratch, cudaStream_t st);
// LN backward that also writes dX cast to T (dXt, nullable) and (+)= its column sums (dsum, nullable):
// the residual gradient's bf16 GEMM operand and the bias gradient of the branch it feeds, in one pass
void layernorm_bwd_ex(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                      const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db,
                      int accumulate, void* dXt, float* dsum, int dsum_acc, float* scratch, cudaStream_t st);
void layernorm_bwd(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                   const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db, int accumulate,
                   float* scratch, cudaStream_t st);
size_t colsum_scratch_bytes(int64_t rows, int n);
// C (+)= sum of S fp32 split-K partials ws[z][n] in z order (deterministic)
void splitk_sum(int S, int64_t n, const float* ws, float* C, int accumulate, cudaStream_t st);
void colsum(int in_dtype, int64_t rows, int n, const void* X, int64_t ld, float* out, int accumulate, float* scratch,
            cudaStream_t st);
// Xt = (T) X and out (+)= column sums of X, one pass over the fp32 [rows, n] X (n % 4 == 0)
void cast_colsum(int dtype, int64_t rows, int n, const float* X, void* Xt, float* out, int accumulate, float* scratch,
                 cudaStream_t st);
void softmax_fwd(int dtype, int64_t rows, int S, int causal, float scale, const float* Z, void* P, cudaStream_t st);
void softmax_bwd(int dtype, int64_t rows, int S, float alpha, const float* dP, const void* P, void* dZ,
                 cudaStream_t st);
// t_dev (nullable): device int holding the step t (read at execution time; CUDA-graph friendly)
void adam(int dtype, int64_t n, float* W, float* m, float* v, const float* g, void* Wc, double lr, double b1, double b2,
          double eps, int t, const int* t_dev, cudaStream_t st);
size_t mse_scratch_bytes();
void mse(int64_t n, const float* Y, const float* Tg, float inv_batch, float* dY, double* loss_out, double* scratch,
         cudaStream_t st);
void cast(int dtype, int64_t n, const float* in, void* out, cudaStream_t st);
void act_bwd(int dtype, int act, int64_t n, const float* dY, const void* Z, void* dZ, cudaStream_t st);
void copy_f32(int64_t n, const float* src, float* dst, cudaStream_t st);
// fused attention forward (attention.cu); false when the shape does not qualify
bool attention_fwd_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, void* C, float* lse,
                         cudaStream_t st);
// two-query-tile forward (attention_fwd2.cu): dh = 64, S % 256 == 0; false otherwise
bool attention_fwd2_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, void* C, float* lse,
                          cudaStream_t st);
// fused attention backward: dQKV from QKV, O, dO, lse (scratch: attention_bwd_scratch_bytes)
size_t attention_bwd_scratch_bytes(int64_t b, int S, int H);
bool attention_bwd_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, const void* O, const void* dO,
                         const float* lse, void* dQKV, void* scratch, cudaStream_t st);

// The library's own collectives (collective.cu; harmony_init_group): dst = sum of nsrc fp32
// buffers in source order (sources may live on peer GPUs).
constexpr int HM_MAX_GROUP = 16;
void rank_sum(int nsrc, const float* const* src, int64_t n, float* dst, cudaStream_t st);

// Convenience: a GEMM descriptor with defaults (batch 1, alpha 1, no bias/aux).
inline hk_gemm_args gemm_args(int dtype, int M, int N, int K) {
  hk_gemm_args a{};
  a.dtype = dtype; a.M = M; a.N = N; a.K = K; a.nz0 = 1; a.nz1 = 1; a.alpha = 1.f;
  return a;
}

}  // namespace hm
