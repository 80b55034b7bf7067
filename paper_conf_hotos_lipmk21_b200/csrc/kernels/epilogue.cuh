// epilogue.cuh — GEMM epilogues shared by the SIMT (fp32) and tcgen05 (bf16) GEMMs.
// What each epilogue computes is specified in include/harmony_kernels.h (hk_epilogue).
#pragma once
#include "../common.hpp"
#include "harmony_kernels.h"

namespace hm {

struct EpiParams {
  void* C;
  int64_t ldc, c_sz0, c_sz1;
  int epi, act, accumulate;
  float alpha;
  const void* bias;
  const void* aux;
  void* aux_out;
  int M, N;
  float* colsum = nullptr;  // optional: per-32-row-block column sums of the bf16 output (gemm_colsum)
};

// Apply the epilogue to one accumulator element.  T = activation type.
template <typename T>
__device__ __forceinline__ void epi_scalar(const EpiParams& e, int64_t off, int n, float acc) {
  float b = e.bias ? to_f32(reinterpret_cast<const T*>(e.bias)[n]) : 0.f;
  switch (e.epi) {
    case HK_EPI_STORE_T:
      reinterpret_cast<T*>(e.C)[off] = from_f32<T>(e.alpha * acc + b);
      break;
    case HK_EPI_STORE_F32:
      reinterpret_cast<float*>(e.C)[off] = e.alpha * acc + b;
      break;
    case HK_EPI_RESID_F32:
      reinterpret_cast<float*>(e.C)[off] = reinterpret_cast<const float*>(e.aux)[off] + (acc + b);
      break;
    case HK_EPI_ACC_F32: {
      float* c = reinterpret_cast<float*>(e.C) + off;
      float v = e.alpha * acc;
      *c = e.accumulate ? (*c + v) : v;
      break;
    }
    case HK_EPI_BIAS_ACT: {
      // act is applied to the STORED pre-activation, so a backward that recomputes act(H) from
      // the stashed H (stash policies 1, 2) reproduces G bit for bit
      const T zt = from_f32<T>(acc + b);
      reinterpret_cast<T*>(e.C)[off] = zt;
      reinterpret_cast<T*>(e.aux_out)[off] = from_f32<T>(act_T<T>(e.act, to_f32(zt)));
      break;
    }
    case HK_EPI_ACT_T: {
      const T zt = from_f32<T>(acc + b);
      reinterpret_cast<T*>(e.C)[off] = from_f32<T>(act_T<T>(e.act, to_f32(zt)));
      break;
    }
    case HK_EPI_ACT_BWD: {
      float z = to_f32(reinterpret_cast<const T*>(e.aux)[off]);
      reinterpret_cast<T*>(e.C)[off] = from_f32<T>(acc * act_grad_T<T>(e.act, z));
      break;
    }
    case HK_EPI_BIAS_ACT_F32: {
      float z = acc + b;
      reinterpret_cast<T*>(e.C)[off] = from_f32<T>(z);
      reinterpret_cast<float*>(e.aux_out)[off] = act_T<T>(e.act, z);
      break;
    }
    default:
      break;
  }
}

// bias[n0 .. n0+31] (bf16) as fp32, zeros without a bias and past N; vector loads when aligned
__device__ __forceinline__ void load_bias32(const EpiParams& e, int n0, float* bb) {
  if (!e.bias) {
#pragma unroll
    for (int j = 0; j < 32; ++j) bb[j] = 0.f;
    return;
  }
  const __nv_bfloat16* b = reinterpret_cast<const __nv_bfloat16*>(e.bias) + n0;
  if (n0 + 32 > e.N) {
#pragma unroll
    for (int j = 0; j < 32; ++j) bb[j] = n0 + j < e.N ? __bfloat162float(b[j]) : 0.f;
  } else if ((reinterpret_cast<uintptr_t>(b) & 15) == 0) {
    const uint4* b4 = reinterpret_cast<const uint4*>(b);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 u = b4[q];
      const __nv_bfloat16* h = reinterpret_cast<const __nv_bfloat16*>(&u);
#pragma unroll
      for (int j = 0; j < 8; ++j) bb[8 * q + j] = __bfloat162float(h[j]);
    }
  } else {
#pragma unroll
    for (int j = 0; j < 32; ++j) bb[j] = __bfloat162float(b[j]);
  }
}

// 16 contiguous columns n0..n0+15 of one row (vectorised when aligned and in range).
template <typename T>
__device__ __forceinline__ void epi_row16(const EpiParams& e, int64_t row_off, int n0, const float* acc) {
  const int64_t off = row_off + n0;
  bool full = (n0 + 16 <= e.N);
  if (full && e.epi != HK_EPI_ACC_F32 && e.epi != HK_EPI_RESID_F32 && sizeof(T) == 2) {
    // bf16 outputs: 32-byte vector stores when 16-byte aligned
    const bool al = ((reinterpret_cast<uintptr_t>(reinterpret_cast<T*>(e.C) + off) & 15) == 0) &&
                    (e.aux == nullptr || (reinterpret_cast<uintptr_t>(reinterpret_cast<const T*>(e.aux) + off) & 15) == 0) &&
                    (e.aux_out == nullptr || (reinterpret_cast<uintptr_t>(reinterpret_cast<T*>(e.aux_out) + off) & 15) == 0);
    if (al && (e.epi == HK_EPI_STORE_T || e.epi == HK_EPI_BIAS_ACT || e.epi == HK_EPI_ACT_BWD)) {
      float v[16];
      float bb[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) bb[j] = 0.f;
      if (e.bias) {
        const uint4* bp = reinterpret_cast<const uint4*>(reinterpret_cast<const T*>(e.bias) + n0);
        if ((reinterpret_cast<uintptr_t>(bp) & 15) == 0) {
          uint4 q0 = bp[0], q1 = bp[1];
          const __nv_bfloat16* h0 = reinterpret_cast<const __nv_bfloat16*>(&q0);
          const __nv_bfloat16* h1 = reinterpret_cast<const __nv_bfloat16*>(&q1);
#pragma unroll
          for (int j = 0; j < 8; ++j) { bb[j] = __bfloat162float(h0[j]); bb[8 + j] = __bfloat162float(h1[j]); }
        } else {
#pragma unroll
          for (int j = 0; j < 16; ++j) bb[j] = to_f32(reinterpret_cast<const T*>(e.bias)[n0 + j]);
        }
      }
      if (e.epi == HK_EPI_STORE_T) {
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] = e.alpha * acc[j] + bb[j];
      } else if (e.epi == HK_EPI_BIAS_ACT) {
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] = acc[j] + bb[j];
      } else {  // ACT_BWD
        const uint4* ap = reinterpret_cast<const uint4*>(reinterpret_cast<const T*>(e.aux) + off);
        uint4 q0 = ap[0], q1 = ap[1];
        const __nv_bfloat16* h0 = reinterpret_cast<const __nv_bfloat16*>(&q0);
        const __nv_bfloat16* h1 = reinterpret_cast<const __nv_bfloat16*>(&q1);
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          v[j] = acc[j] * act_grad_T<T>(e.act, __bfloat162float(h0[j]));
          v[8 + j] = acc[8 + j] * act_grad_T<T>(e.act, __bfloat162float(h1[j]));
        }
      }
      uint4 o[2];
      __nv_bfloat162* op = reinterpret_cast<__nv_bfloat162*>(o);
#pragma unroll
      for (int j = 0; j < 8; ++j) op[j] = __floats2bfloat162_rn(v[2 * j], v[2 * j + 1]);
      uint4* cp = reinterpret_cast<uint4*>(reinterpret_cast<T*>(e.C) + off);
      cp[0] = o[0];
      cp[1] = o[1];
      if (e.epi == HK_EPI_BIAS_ACT) {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const float2 zr = __bfloat1622float2(op[j]);  // the stored (rounded) pre-activation
          op[j] = __floats2bfloat162_rn(act_T<T>(e.act, zr.x), act_T<T>(e.act, zr.y));
        }
        uint4* gp = reinterpret_cast<uint4*>(reinterpret_cast<T*>(e.aux_out) + off);
        gp[0] = o[0];
        gp[1] = o[1];
      }
      return;
    }
  }
  if (full && (e.epi == HK_EPI_ACC_F32 || e.epi == HK_EPI_RESID_F32 || e.epi == HK_EPI_STORE_F32)) {
    float* cp = reinterpret_cast<float*>(e.C) + off;
    if ((reinterpret_cast<uintptr_t>(cp) & 15) == 0 &&
        (e.epi != HK_EPI_RESID_F32 || (reinterpret_cast<uintptr_t>(reinterpret_cast<const float*>(e.aux) + off) & 15) == 0)) {
      float bb[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) bb[j] = e.bias ? to_f32(reinterpret_cast<const T*>(e.bias)[n0 + j]) : 0.f;
      float4* c4 = reinterpret_cast<float4*>(cp);
      if (e.epi == HK_EPI_ACC_F32) {
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          float4 o = make_float4(e.alpha * acc[4 * q], e.alpha * acc[4 * q + 1], e.alpha * acc[4 * q + 2],
                                 e.alpha * acc[4 * q + 3]);
          if (e.accumulate) {
            float4 c = c4[q];
            o.x = c.x + o.x; o.y = c.y + o.y; o.z = c.z + o.z; o.w = c.w + o.w;
          }
          c4[q] = o;
        }
      } else if (e.epi == HK_EPI_RESID_F32) {
        const float4* a4 = reinterpret_cast<const float4*>(reinterpret_cast<const float*>(e.aux) + off);
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          float4 a = a4[q];
          c4[q] = make_float4(a.x + (acc[4 * q] + bb[4 * q]), a.y + (acc[4 * q + 1] + bb[4 * q + 1]),
                              a.z + (acc[4 * q + 2] + bb[4 * q + 2]), a.w + (acc[4 * q + 3] + bb[4 * q + 3]));
        }
      } else {
#pragma unroll
        for (int q = 0; q < 4; ++q)
          c4[q] = make_float4(e.alpha * acc[4 * q] + bb[4 * q], e.alpha * acc[4 * q + 1] + bb[4 * q + 1],
                              e.alpha * acc[4 * q + 2] + bb[4 * q + 2], e.alpha * acc[4 * q + 3] + bb[4 * q + 3]);
      }
      return;
    }
  }
#pragma unroll
  for (int j = 0; j < 16; ++j)
    if (n0 + j < e.N) epi_scalar<T>(e, off + j, n0 + j, acc[j]);
}

}  // namespace hm
