/*
 * harmony_kernels.h — kernel-level C ABI of libharmony.so (test and benchmark
 * entry points).  These launch exactly the kernels the training step uses,
 * on caller-provided DEVICE buffers, so parity tests can compare each op with
 * the fp64 oracle (tests/test_gpu_kernels.py).  All pointers are device
 * pointers owned by the caller; `stream` is a cudaStream_t (NULL = legacy
 * default stream).  Calls are asynchronous unless noted; errors are returned
 * as harmony_status and the message is in harmony_last_error(NULL).
 *
 * dtype: 0 = fp32 (SIMT FFMA path, the fp32 precision of the step),
 *        1 = bf16 operands / bf16 activations with fp32 accumulation
 *            (tcgen05.mma kind::f16, accumulators in TMEM, TMA-fed).
 * "T" below means the activation type selected by dtype (float or bf16).
 */
#ifndef HARMONY_KERNELS_H_
#define HARMONY_KERNELS_H_

#include <stdint.h>
#include "harmony.h"

#ifdef __cplusplus
extern "C" {
#endif

/* GEMM epilogues (what happens to the fp32 accumulator acc[m][n]). */
typedef enum {
  HK_EPI_STORE_T = 0,     /* C(T)   = alpha*acc + bias[n]                                  */
  HK_EPI_STORE_F32 = 1,   /* C(f32) = alpha*acc + bias[n]                                  */
  HK_EPI_RESID_F32 = 2,   /* C(f32) = aux_f32[m][n] + acc + bias[n]  (residual add, c23)   */
  HK_EPI_ACC_F32 = 3,     /* C(f32) = (accumulate ? C : 0) + alpha*acc  (wgrad, dW += .)   */
  HK_EPI_BIAS_ACT = 4,    /* C(T) = z = acc + bias[n];  aux_out(T) = act(z)   (FC1: H, G)  */
  HK_EPI_ACT_BWD = 5,     /* C(T) = acc * act'(aux_T[m][n])                  (dG -> dH)   */
  HK_EPI_BIAS_ACT_F32 = 6, /* C(T) = z = acc + bias[n]; aux_out(f32) = act(z)  (MLP layer)  */
  HK_EPI_ACT_T = 7        /* C(T) = act(RN_T(acc + bias[n]))   (FC1 when only G is needed;
                             bit-identical to the aux_out of HK_EPI_BIAS_ACT)             */
} hk_epilogue;

/* C[z0,z1][m][n] = epilogue( sum_k A[z0,z1](m,k) * B[z0,z1](n,k) )
 * Operand X in {A,B} with logical index (r,k) (r = m for A, n for B) lives at
 *   X + z0*x_sz0 + z1*x_sz1 + (x_mn_major ? k*ldx + r : r*ldx + k)        (elements)
 * i.e. K-major = K contiguous; MN-major = M (or N) contiguous.
 * C and every aux tensor:  C + z0*c_sz0 + z1*c_sz1 + m*ldc + n.
 * bf16 path requirements (TMA): 16-byte aligned base pointers, ld and batch strides
 * multiples of 8 elements. */
typedef struct {
  int32_t dtype;
  int32_t M, N, K;
  int32_t nz0, nz1;
  const void* A; int32_t a_mn_major; int64_t lda, a_sz0, a_sz1;
  const void* B; int32_t b_mn_major; int64_t ldb, b_sz0, b_sz1;
  void* C; int64_t ldc, c_sz0, c_sz1;
  int32_t epilogue;    /* hk_epilogue */
  int32_t act;         /* harmony_act for BIAS_ACT / ACT_BWD */
  int32_t accumulate;  /* HK_EPI_ACC_F32: 1 = add into C; 2 = CONTINUE C's reduction: the K sum starts
                          from C instead of 0 (alpha 1; fp32 SIMT GEMM only), so a K-split into
                          slices run in order is bit-identical to one GEMM over the whole K */
  float alpha;
  const void* bias;    /* [N] of T, nullable */
  const void* aux;     /* RESID_F32: f32 residual; ACT_BWD: T pre-activation */
  void* aux_out;       /* BIAS_ACT(_F32): activation output */
} hk_gemm_args;

harmony_status hk_gemm(const hk_gemm_args* args, void* stream);

/* LayerNorm over the last axis of X (fp32 [rows][d]); biased variance, eps = 1e-5 (c10).
 * U(T) = (X - mean)*rstd*g + b; mean, rstd: fp32 [rows].  g, b: T [d]. */
harmony_status hk_layernorm_fwd(int32_t dtype, int64_t rows, int32_t d, const float* X, const void* g, const void* b,
                                void* U, float* mean, float* rstd, void* stream);

/* dX = (dres ? dres : 0) + rstd*(dxh - mean(dxh) - xh*mean(dxh*xh)), dxh = dU*g;
 * dg (+)= sum_rows dU*xh, db (+)= sum_rows dU   (fp32 [d], deterministic two-stage
 * column reduction; accumulate = 1 adds into dg/db).  dU is fp32 [rows][d]. */
harmony_status hk_layernorm_bwd(int32_t dtype, int64_t rows, int32_t d, const float* dU, const float* X,
                                const float* mean, const float* rstd, const void* g, const float* dres, float* dX,
                                float* dg, float* db, int32_t accumulate, void* stream);

/* P(T)[r][:] = softmax(scale * Z[r][:]) with the causal mask of row (r % S) when causal.
 * Z fp32 [rows][S]. */
harmony_status hk_softmax_fwd(int32_t dtype, int64_t rows, int32_t S, int32_t causal, float scale, const float* Z,
                              void* P, void* stream);

/* dZ(T) = alpha * P.(dP - rowsum(dP.P));  dP fp32 [rows][S], P (T). */
harmony_status hk_softmax_bwd(int32_t dtype, int64_t rows, int32_t S, float alpha, const float* dP, const void* P,
                              void* dZ, void* stream);

/* out[n] (+)= sum_r X[r][n] (X of type in_dtype: 0 fp32, 1 bf16; row stride ld). */
harmony_status hk_colsum(int32_t in_dtype, int64_t rows, int32_t n, const void* X, int64_t ld, float* out,
                         int32_t accumulate, void* stream);

/* Fused Adam on n elements (reading c3): m = b1 m + (1-b1) g; v = b2 v + (1-b2) g^2;
 * W -= lr * (m/bc1) / (sqrt(v/bc2) + eps); Wc(T) = round(W).  bc1 = 1-b1^t, bc2 = 1-b2^t. */
harmony_status hk_adam(int32_t dtype, int64_t n, float* W, float* m, float* v, const float* g, void* Wc, double lr,
                       double beta1, double beta2, double eps, int32_t t, void* stream);

/* MSE (reading c2): dY = (Y - T) * inv_batch; loss_out[0] (double) = 0.5*inv_batch*sum (Y-T)^2,
 * reduced in a fixed order.  Y, T, dY fp32 [n]. */
harmony_status hk_mse(int64_t n, const float* Y, const float* T, float inv_batch, float* dY, double* loss_out,
                      void* stream);

/* out(T)[i] = in[i] (fp32 -> T, round to nearest even). */
harmony_status hk_cast(int32_t dtype, int64_t n, const float* in, void* out, void* stream);

/* dZ(T) = dY(f32) * act'(Z(T)). */
harmony_status hk_act_bwd(int32_t dtype, int32_t act, int64_t n, const float* dY, const void* Z, void* dZ,
                          void* stream);

/* Fused multi-head attention forward (bf16, tcgen05; S % 128 == 0, dh in {64, 128}) on the packed
 * QKV [b*S][3*H*dh] layout: C[b*S][H*dh] (bf16, heads interleaved) = softmax(scale Q K^T (+causal)) V
 * per head, lse[b][H][S] = log-sum-exp of the scaled scores (natural log).  HARMONY_E_UNSUPPORTED
 * when the shape does not qualify. */
harmony_status hk_attention_fwd(int64_t b, int32_t S, int32_t H, int32_t dh, int32_t causal, const void* QKV, void* C,
                                float* lse, void* stream);

/* Fused attention backward: dQKV[b*S][3d] (bf16: dQ, dK, dV column blocks) from QKV, O = C of the
 * forward, dO = dC (bf16 [b*S][d]) and lse; deterministic (dS^T materialised, dQ by GEMM).
 * Synchronous.  Same shape conditions as hk_attention_fwd. */
harmony_status hk_attention_bwd(int64_t b, int32_t S, int32_t H, int32_t dh, int32_t causal, const void* QKV,
                                const void* O, const void* dO, const float* lse, void* dQKV, void* stream);

/* Blocks until the device is idle; returns HARMONY_E_CUDA with the message on error. */
harmony_status hk_sync(void);

#ifdef __cplusplus
}
#endif
#endif /* HARMONY_KERNELS_H_ */
