// common.hpp — shared helpers of libharmony (error plumbing, bf16 conversion, launch helpers).
#pragma once

#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdio.h>
#include <cmath>
#include <string>
#include <vector>

#include "harmony.h"

namespace hm {

// Thread-local message of the last failure of a context-less call (kernel ABI).
void set_global_error(const std::string& msg);
const char* global_error();

struct Error {
  harmony_status code;
  std::string msg;
};

#define HM_CUDA(expr)                                                                                   \
  do {                                                                                                  \
    cudaError_t _e = (expr);                                                                            \
    if (_e != cudaSuccess) {                                                                            \
      throw ::hm::Error{HARMONY_E_CUDA, std::string(#expr) + " -> " + cudaGetErrorString(_e) + " at " + \
                                           __FILE__ + ":" + std::to_string(__LINE__)};                  \
    }                                                                                                   \
  } while (0)

#define HM_CHECK(cond, code, msg)                                  \
  do {                                                             \
    if (!(cond)) throw ::hm::Error{(code), std::string(msg)};      \
  } while (0)

// Kernel launch accounting (the ledger counts the kernels a step launches).
extern thread_local uint64_t g_kernel_launches;

// Optional per-launch timing (harmony_set_profiling): CUDA events recorded on the launching
// stream around each kernel of a class, with the launch's algorithmic work (FLOPs or bytes).
enum ProfCat { PROF_GEMM = 0, PROF_ADAM = 1, PROF_LN = 2, PROF_SOFTMAX = 3, PROF_OTHER = 4, PROF_ATTN = 5, PROF_NUM = 6 };
struct KProf {
  bool on = false;
  bool external = false;  // inside a stream capture: record event nodes into the graph
  std::vector<cudaEvent_t> pool;
  size_t used = 0;
  struct Rec { int cat, e0, e1; double work; cudaStream_t st; };
  std::vector<Rec> recs;
  struct OpRec { int op, e0, e1; };  // the step timeline: events around every op of the program
  std::vector<OpRec> oprecs;
  int begin(cudaStream_t st) {
    if (!on) return -1;
    if (used == pool.size()) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) != cudaSuccess) return -1;
      pool.push_back(e);
    }
    if (external) cudaEventRecordWithFlags(pool[used], st, cudaEventRecordExternal);
    else cudaEventRecord(pool[used], st);
    return (int)used++;
  }
  void end(int cat, int e0, cudaStream_t st, double work) {
    if (e0 < 0) return;
    int e1 = begin(st);
    if (e1 >= 0) recs.push_back({cat, e0, e1, work, st});
  }
};
extern thread_local KProf g_prof;
inline void count_launch() { ++g_kernel_launches; }

inline void check_launch(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) throw Error{HARMONY_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e)};
  count_launch();
}

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }

// Activation types of the step: fp32 path stores T = float, bf16 path T = __nv_bfloat16.
template <typename T> struct TypeTag;
template <> struct TypeTag<float> { static constexpr int id = 0; };
template <> struct TypeTag<__nv_bfloat16> { static constexpr int id = 1; };

__device__ __forceinline__ float to_f32(float x) { return x; }
__device__ __forceinline__ float to_f32(__nv_bfloat16 x) { return __bfloat162float(x); }
template <typename T> __device__ __forceinline__ T from_f32(float x);
template <> __device__ __forceinline__ float from_f32<float>(float x) { return x; }
template <> __device__ __forceinline__ __nv_bfloat16 from_f32<__nv_bfloat16>(float x) { return __float2bfloat16_rn(x); }

// GeLU (tanh approximation, reading c12) and its derivative.
// FAST (the bf16 path): tanh u by the hardware tanh.approx.f32 (one MUFU op; relative error
// ~2^-11, an order below the bf16 rounding of every value it feeds — reading c12a).
// Exact (the fp32 path, 1e-5 budget): 0.5(1 + tanh u) written as the logistic
// s = 1/(1 + e^{-2u}) (an identity) with ex2.approx and a fast divide, a few fp32 ulp;
// tanh u = 2s - 1 and 1 - tanh^2 u = 4 s (1 - s).  Forward and recompute use the same
// instance for a dtype, so a recomputed activation matches the stored one bit for bit.
__device__ __forceinline__ float tanh_approx(float x) {
  float y;
  asm("tanh.approx.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ float gelu_sigmoid_f(float x) {
  const float c2 = 2.0f * 0.7978845608028654f, a = 0.044715f;
  const float u2 = c2 * (x + a * x * x * x);
  return __fdividef(1.0f, 1.0f + __expf(-u2));
}
template <bool FAST>
__device__ __forceinline__ float gelu_tanh_f(float x) {
  if (FAST) {
    const float c = 0.7978845608028654f, a = 0.044715f;
    const float hx = 0.5f * x;
    return fmaf(hx, tanh_approx(c * (x + a * x * x * x)), hx);
  }
  return x * gelu_sigmoid_f(x);
}
template <bool FAST>
__device__ __forceinline__ float gelu_tanh_grad_f(float x) {
  const float c = 0.7978845608028654f, a = 0.044715f;
  if (FAST) {
    const float t = tanh_approx(c * (x + a * x * x * x));
    return 0.5f * (1.0f + t) + 0.5f * x * (1.0f - t * t) * c * (1.0f + 3.0f * a * x * x);
  }
  const float s = gelu_sigmoid_f(x);
  return s + 2.0f * x * s * (1.0f - s) * c * (1.0f + 3.0f * a * x * x);
}
template <bool FAST = false>
__device__ __forceinline__ float act_f(int act, float z) {
  if (act == HARMONY_ACT_RELU) return z > 0.f ? z : 0.f;
  if (act == HARMONY_ACT_GELU_TANH) return gelu_tanh_f<FAST>(z);
  return z;
}
template <bool FAST = false>
__device__ __forceinline__ float act_grad_f(int act, float z) {
  if (act == HARMONY_ACT_RELU) return z > 0.f ? 1.f : 0.f;
  if (act == HARMONY_ACT_GELU_TANH) return gelu_tanh_grad_f<FAST>(z);
  return 1.f;
}
// the instance a layer of activation type T uses (bf16: FAST)
template <typename T>
__device__ __forceinline__ float act_T(int act, float z) { return act_f<sizeof(T) == 2>(act, z); }
template <typename T>
__device__ __forceinline__ float act_grad_T(int act, float z) { return act_grad_f<sizeof(T) == 2>(act, z); }

}  // namespace hm
