// kapi.cu — kernel-level C ABI (include/harmony_kernels.h): the step's kernels on caller buffers.
#include <mutex>

#include "common.hpp"
#include "kernels/kernels.hpp"

using namespace hm;

namespace {
// Scratch for the two-stage reductions when called outside a step (tests / benchmarks only).
struct Scratch {
  void* p = nullptr;
  size_t n = 0;
  std::mutex mu;
  void* get(size_t bytes) {
    if (bytes > n) {
      if (p) cudaFree(p);
      p = nullptr;
      HM_CUDA(cudaMalloc(&p, bytes));
      n = bytes;
    }
    return p;
  }
};
Scratch& scratch() {
  static Scratch s;
  return s;
}
harmony_status kfail(const Error& e) {
  set_global_error(e.msg);
  return e.code;
}
}  // namespace

#define K_BEGIN try {
#define K_END                                 \
  }                                           \
  catch (const Error& e) { return kfail(e); } \
  return HARMONY_OK;

extern "C" {

harmony_status hk_gemm(const hk_gemm_args* a, void* stream) {
  K_BEGIN
  HM_CHECK(a != nullptr, HARMONY_E_INVALID_ARG, "args NULL");
  gemm(*a, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_layernorm_fwd(int32_t dtype, int64_t rows, int32_t d, const float* X, const void* g, const void* b,
                                void* U, float* mean, float* rstd, void* stream) {
  K_BEGIN
  layernorm_fwd(dtype, rows, d, X, g, b, U, mean, rstd, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_layernorm_bwd(int32_t dtype, int64_t rows, int32_t d, const float* dU, const float* X,
                                const float* mean, const float* rstd, const void* g, const float* dres, float* dX,
                                float* dg, float* db, int32_t accumulate, void* stream) {
  K_BEGIN
  std::lock_guard<std::mutex> lk(scratch().mu);
  float* sc = static_cast<float*>(scratch().get(layernorm_bwd_scratch_bytes(rows, d) + 256));
  layernorm_bwd(dtype, rows, d, dU, X, mean, rstd, g, dres, dX, dg, db, accumulate, sc,
                static_cast<cudaStream_t>(stream));
  HM_CUDA(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  K_END
}

harmony_status hk_softmax_fwd(int32_t dtype, int64_t rows, int32_t S, int32_t causal, float scale, const float* Z,
                              void* P, void* stream) {
  K_BEGIN
  softmax_fwd(dtype, rows, S, causal, scale, Z, P, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_softmax_bwd(int32_t dtype, int64_t rows, int32_t S, float alpha, const float* dP, const void* P,
                              void* dZ, void* stream) {
  K_BEGIN
  softmax_bwd(dtype, rows, S, alpha, dP, P, dZ, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_colsum(int32_t in_dtype, int64_t rows, int32_t n, const void* X, int64_t ld, float* out,
                         int32_t accumulate, void* stream) {
  K_BEGIN
  std::lock_guard<std::mutex> lk(scratch().mu);
  float* sc = static_cast<float*>(scratch().get(colsum_scratch_bytes(rows, n) + 256));
  colsum(in_dtype, rows, n, X, ld, out, accumulate, sc, static_cast<cudaStream_t>(stream));
  HM_CUDA(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  K_END
}

harmony_status hk_adam(int32_t dtype, int64_t n, float* W, float* m, float* v, const float* g, void* Wc, double lr,
                       double beta1, double beta2, double eps, int32_t t, void* stream) {
  K_BEGIN
  HM_CHECK(t >= 1, HARMONY_E_INVALID_ARG, "Adam step t starts at 1");
  adam(dtype, n, W, m, v, g, Wc, lr, beta1, beta2, eps, t, nullptr, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_mse(int64_t n, const float* Y, const float* T, float inv_batch, float* dY, double* loss_out,
                      void* stream) {
  K_BEGIN
  std::lock_guard<std::mutex> lk(scratch().mu);
  double* sc = static_cast<double*>(scratch().get(mse_scratch_bytes()));
  mse(n, Y, T, inv_batch, dY, loss_out, sc, static_cast<cudaStream_t>(stream));
  HM_CUDA(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  K_END
}

harmony_status hk_cast(int32_t dtype, int64_t n, const float* in, void* out, void* stream) {
  K_BEGIN
  cast(dtype, n, in, out, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_act_bwd(int32_t dtype, int32_t act, int64_t n, const float* dY, const void* Z, void* dZ,
                          void* stream) {
  K_BEGIN
  act_bwd(dtype, act, n, dY, Z, dZ, static_cast<cudaStream_t>(stream));
  K_END
}

harmony_status hk_attention_fwd(int64_t b, int32_t S, int32_t H, int32_t dh, int32_t causal, const void* QKV, void* C,
                                float* lse, void* stream) {
  K_BEGIN
  HM_CHECK(attention_fwd_fused(b, S, H, dh, causal, QKV, C, lse, static_cast<cudaStream_t>(stream)),
           HARMONY_E_UNSUPPORTED, "fused attention needs S % 128 == 0 and dh in {64, 128}");
  K_END
}

harmony_status hk_attention_bwd(int64_t b, int32_t S, int32_t H, int32_t dh, int32_t causal, const void* QKV,
                                const void* O, const void* dO, const float* lse, void* dQKV, void* stream) {
  K_BEGIN
  std::lock_guard<std::mutex> lk(scratch().mu);
  void* sc = scratch().get(attention_bwd_scratch_bytes(b, S, H));
  HM_CHECK(attention_bwd_fused(b, S, H, dh, causal, QKV, O, dO, lse, dQKV, sc, static_cast<cudaStream_t>(stream)),
           HARMONY_E_UNSUPPORTED, "fused attention needs S % 128 == 0 and dh in {64, 128}");
  HM_CUDA(cudaStreamSynchronize(static_cast<cudaStream_t>(stream)));
  K_END
}

harmony_status hk_sync(void) {
  K_BEGIN
  HM_CUDA(cudaDeviceSynchronize());
  HM_CUDA(cudaGetLastError());
  K_END
}

}  // extern "C"
