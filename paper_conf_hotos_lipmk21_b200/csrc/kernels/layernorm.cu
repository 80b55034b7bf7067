// layernorm.cu — register-resident LayerNorm forward/backward (K8).
//
// One warp per row; the row is read ONCE with float4 loads and kept in registers (VPT float4 per
// lane, d <= 128*VPT), so the kernel moves the algorithmic bytes only: fwd reads X (4d) and
// writes U (ts*d) + 8 B of statistics per row; bwd reads dU, X, dres (12d) and writes dX (4d).
// Statistics are two-pass on the registers (mean, then centred sum of squares; reading c10).
// The backward also accumulates this warp's dgamma/dbeta column partials in registers (each lane
// owns fixed columns), the 8 warps of a block are combined in warp order through shared memory
// and the block partial is written for the fixed-order column reduction — no atomics.
#include "../common.hpp"
#include "kernels.hpp"

namespace hm {

constexpr int LNV_ROWS = 16;  // rows per block in the backward (2 per warp)

__device__ __forceinline__ float wsum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

template <typename T>
__device__ __forceinline__ float4 ld4(const T* p);
template <>
__device__ __forceinline__ float4 ld4<float>(const float* p) { return *reinterpret_cast<const float4*>(p); }
template <>
__device__ __forceinline__ float4 ld4<__nv_bfloat16>(const __nv_bfloat16* p) {
  uint2 u = *reinterpret_cast<const uint2*>(p);
  __nv_bfloat162 a = *reinterpret_cast<__nv_bfloat162*>(&u.x), b = *reinterpret_cast<__nv_bfloat162*>(&u.y);
  float2 fa = __bfloat1622float2(a), fb = __bfloat1622float2(b);
  return make_float4(fa.x, fa.y, fb.x, fb.y);
}
template <typename T>
__device__ __forceinline__ void st4(T* p, float4 v);
template <>
__device__ __forceinline__ void st4<float>(float* p, float4 v) { *reinterpret_cast<float4*>(p) = v; }
template <>
__device__ __forceinline__ void st4<__nv_bfloat16>(__nv_bfloat16* p, float4 v) {
  __nv_bfloat162 a = __floats2bfloat162_rn(v.x, v.y), b = __floats2bfloat162_rn(v.z, v.w);
  uint2 u;
  u.x = *reinterpret_cast<uint32_t*>(&a);
  u.y = *reinterpret_cast<uint32_t*>(&b);
  *reinterpret_cast<uint2*>(p) = u;
}

template <typename T, int VPT>
__global__ void __launch_bounds__(256) ln_fwd_v(int64_t rows, int d, const float* __restrict__ X,
                                               const T* __restrict__ g, const T* __restrict__ b, T* __restrict__ U,
                                               float* __restrict__ mean, float* __restrict__ rstd,
                                               float* __restrict__ Xcopy) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int lane = threadIdx.x & 31;
  const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (row >= rows) return;
  const float* x = X + row * d;
  float4 v[VPT];
  float s = 0.f;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int c = (j * 32 + lane) * 4;
    v[j] = c < d ? *reinterpret_cast<const float4*>(x + c) : make_float4(0.f, 0.f, 0.f, 0.f);
    s += (v[j].x + v[j].y) + (v[j].z + v[j].w);
  }
  if (Xcopy) {  // the block input stashed by the same pass that normalises it (block recompute)
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int c = (j * 32 + lane) * 4;
      if (c < d) *reinterpret_cast<float4*>(Xcopy + row * d + c) = v[j];
    }
  }
  const float mu = wsum(s) / (float)d;
  float q = 0.f;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int c = (j * 32 + lane) * 4;
    if (c < d) {
      float a0 = v[j].x - mu, a1 = v[j].y - mu, a2 = v[j].z - mu, a3 = v[j].w - mu;
      q += (a0 * a0 + a1 * a1) + (a2 * a2 + a3 * a3);
    }
  }
  const float rs = rsqrtf(wsum(q) / (float)d + 1e-5f);
  T* u = U + row * d;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int c = (j * 32 + lane) * 4;
    if (c < d) {
      float4 gg = ld4<T>(g + c), bb = ld4<T>(b + c);
      st4<T>(u + c, make_float4((v[j].x - mu) * rs * gg.x + bb.x, (v[j].y - mu) * rs * gg.y + bb.y,
                                (v[j].z - mu) * rs * gg.z + bb.z, (v[j].w - mu) * rs * gg.w + bb.w));
    }
  }
  if (lane == 0) { mean[row] = mu; rstd[row] = rs; }
}

template <typename T, int VPT>
// __launch_bounds__(256, 2): two blocks per SM, i.e. at most 128 registers per thread
__global__ void __launch_bounds__(256, 2) ln_bwd_v(int64_t rows, int d, const float* __restrict__ dU,
                                               const float* __restrict__ X, const float* __restrict__ mean,
                                               const float* __restrict__ rstd, const T* __restrict__ g,
                                               const float* __restrict__ dres, float* __restrict__ dX,
                                               T* __restrict__ dXt, int np, float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  // per-warp column partials of dgamma / dbeta (/ sum dX when np == 3) live in shared memory
  // ([8][np][d]); each lane owns
  // fixed columns, so a warp accumulates its rows without races; the 8 warps are then summed in
  // warp order per column (deterministic)
  extern __shared__ float sred[];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t r0 = (int64_t)blockIdx.x * LNV_ROWS;
  float* sg = sred + (size_t)warp * np * d;
  float* sb = sg + d;
  float* ss = np == 3 ? sb + d : nullptr;
#pragma unroll
  for (int j = 0; j < VPT; ++j) {
    const int c = (j * 32 + lane) * 4;
    if (c < d) {
      *reinterpret_cast<float4*>(sg + c) = make_float4(0.f, 0.f, 0.f, 0.f);
      *reinterpret_cast<float4*>(sb + c) = make_float4(0.f, 0.f, 0.f, 0.f);
      if (ss) *reinterpret_cast<float4*>(ss + c) = make_float4(0.f, 0.f, 0.f, 0.f);
    }
  }
  for (int i = warp; i < LNV_ROWS; i += 8) {
    const int64_t row = r0 + i;
    if (row >= rows) break;
    const float* x = X + row * d;
    const float* du = dU + row * d;
    const float* dr = dres ? dres + row * d : nullptr;
    // all of the row's global loads first (x, dU and the residual gradient), so the warp waits for
    // one memory round trip per row; the shared-memory partials are touched only afterwards
    // (wide rows, VPT > 8: the residual gradient is loaded in the second pass, to stay in registers)
    constexpr bool PRE = VPT <= 8;
    float4 xv[VPT], dv[VPT], rv[PRE ? VPT : 1];
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int c = (j * 32 + lane) * 4;
      const bool in = c < d;
      xv[j] = in ? __ldg(reinterpret_cast<const float4*>(x + c)) : make_float4(0.f, 0.f, 0.f, 0.f);
      dv[j] = in ? __ldg(reinterpret_cast<const float4*>(du + c)) : make_float4(0.f, 0.f, 0.f, 0.f);
      if (PRE) rv[PRE ? j : 0] = in && dr ? __ldg(reinterpret_cast<const float4*>(dr + c)) : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    const float mu = mean[row], rs = rstd[row];
    float s1 = 0.f, s2 = 0.f;
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int c = (j * 32 + lane) * 4;
      if (c < d) {
        const float4 gv = ld4<T>(g + c);  // gamma re-read per row (L1-resident): keeps registers < 128
        const float4 xh = make_float4((xv[j].x - mu) * rs, (xv[j].y - mu) * rs, (xv[j].z - mu) * rs, (xv[j].w - mu) * rs);
        const float4 dx = make_float4(dv[j].x * gv.x, dv[j].y * gv.y, dv[j].z * gv.z, dv[j].w * gv.w);
        s1 += (dx.x + dx.y) + (dx.z + dx.w);
        s2 += (dx.x * xh.x + dx.y * xh.y) + (dx.z * xh.z + dx.w * xh.w);
      }
    }
    s1 = wsum(s1) / (float)d;
    s2 = wsum(s2) / (float)d;
    float* dxr = dX + row * d;
#pragma unroll
    for (int j = 0; j < VPT; ++j) {
      const int c = (j * 32 + lane) * 4;
      if (c < d) {
        const float4 xh = make_float4((xv[j].x - mu) * rs, (xv[j].y - mu) * rs, (xv[j].z - mu) * rs, (xv[j].w - mu) * rs);
        const float4 gv = ld4<T>(g + c);
        float4 o = make_float4(rs * (dv[j].x * gv.x - s1 - xh.x * s2), rs * (dv[j].y * gv.y - s1 - xh.y * s2),
                               rs * (dv[j].z * gv.z - s1 - xh.z * s2), rs * (dv[j].w * gv.w - s1 - xh.w * s2));
        if (dr) {
          const float4 rr = PRE ? rv[PRE ? j : 0] : __ldg(reinterpret_cast<const float4*>(dr + c));
          o.x = rr.x + o.x; o.y = rr.y + o.y; o.z = rr.z + o.z; o.w = rr.w + o.w;
        }
        *reinterpret_cast<float4*>(dxr + c) = o;
        if (dXt) st4<T>(dXt + row * d + c, o);  // the bf16 GEMM operand copy of dX
        float4 a = *reinterpret_cast<float4*>(sg + c), bq = *reinterpret_cast<float4*>(sb + c);
        *reinterpret_cast<float4*>(sg + c) =
            make_float4(a.x + dv[j].x * xh.x, a.y + dv[j].y * xh.y, a.z + dv[j].z * xh.z, a.w + dv[j].w * xh.w);
        *reinterpret_cast<float4*>(sb + c) = make_float4(bq.x + dv[j].x, bq.y + dv[j].y, bq.z + dv[j].z, bq.w + dv[j].w);
        if (ss) {
          float4 q = *reinterpret_cast<float4*>(ss + c);
          *reinterpret_cast<float4*>(ss + c) = make_float4(q.x + o.x, q.y + o.y, q.z + o.z, q.w + o.w);
        }
      }
    }
  }
  __syncthreads();
  float* pg = partial + (int64_t)blockIdx.x * np * d;
  for (int c = threadIdx.x; c < np * d; c += 256) {
    float t = sred[c];
#pragma unroll
    for (int w = 1; w < 8; ++w) t += sred[(size_t)w * np * d + c];
    pg[c] = t;
  }
}

// fixed-order tree column reduction (as colreduce_kernel in ops.cu): 32 columns x 32 warps per block,
// blockIdx.y selects which of the np interleaved partial sets (dgamma, dbeta[, sum dX]) -> one launch
struct ColOuts {
  float* out[3];
  int acc[3];
};
__global__ void __launch_bounds__(1024) colreduce2_kernel(int nchunks, int n, const float* __restrict__ partial,
                                                          int64_t stride, ColOuts outs) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  __shared__ float sh[32][33];
  const int cl = threadIdx.x & 31, g = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + cl;
  const float* pp = partial + (int64_t)blockIdx.y * n;
  float s = 0.f;
  if (c < n) {
#pragma unroll 8
    for (int j = g; j < nchunks; j += 32) s += pp[(int64_t)j * stride + c];  // loads hoisted, adds in order
  }
  sh[g][cl] = s;
  __syncthreads();
  if (g == 0 && c < n) {
    float t = sh[0][cl];
#pragma unroll
    for (int k = 1; k < 32; ++k) t += sh[k][cl];
    float* out = outs.out[blockIdx.y];
    out[c] = outs.acc[blockIdx.y] ? out[c] + t : t;
  }
}

static int ln_vpt(int d) {
  if (d % 4) return 0;
  int v = (int)ceil_div(d, 128);
  if (v <= 1) return 1;
  if (v <= 2) return 2;
  if (v <= 4) return 4;
  if (v <= 8) return 8;
  if (v <= 13) return 13;
  if (v <= 16) return 16;
  return 0;  // wider rows: the streaming kernels in ops.cu
}

bool layernorm_fwd_vec(int dtype, int64_t rows, int d, const float* X, const void* g, const void* b, void* U,
                       float* mean, float* rstd, cudaStream_t st, float* Xcopy) {
  const int v = ln_vpt(d);
  if (!v) return false;
  const unsigned grid = (unsigned)ceil_div(rows, 8);
#define HM_LNF(T, V) launch_k(ln_fwd_v<T, V>, dim3(grid), dim3(256), 0, st, rows, d, X, (const T*)g, (const T*)b, (T*)U, mean, rstd, Xcopy)
#define HM_LNF_ALL(T)                   \
  switch (v) {                          \
    case 1: HM_LNF(T, 1); break;        \
    case 2: HM_LNF(T, 2); break;        \
    case 4: HM_LNF(T, 4); break;        \
    case 8: HM_LNF(T, 8); break;        \
    case 13: HM_LNF(T, 13); break;      \
    default: HM_LNF(T, 16); break;      \
  }
  if (dtype == 1) { HM_LNF_ALL(__nv_bfloat16) } else { HM_LNF_ALL(float) }
#undef HM_LNF_ALL
#undef HM_LNF
  check_launch("layernorm_fwd_vec");
  return true;
}

size_t layernorm_bwd_vec_scratch_bytes(int64_t rows, int d) {
  return (size_t)ceil_div(rows, LNV_ROWS) * 3 * d * sizeof(float);
}

bool layernorm_bwd_vec(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                       const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db,
                       int accumulate, void* dXt, float* dsum, int dsum_acc, float* scratch, cudaStream_t st) {
  const int v = ln_vpt(d);
  if (!v) return false;
  const int nblk = (int)ceil_div(rows, LNV_ROWS);
  const int np = dsum ? 3 : 2;
  const size_t smem = 8 * (size_t)np * d * sizeof(float);  // per-warp column partials
  if (smem > 200 * 1024) return false;
#define HM_LNB(T, V)                                                                                   \
  do {                                                                                                 \
    if (smem > 48 * 1024)                                                                              \
      HM_CUDA(cudaFuncSetAttribute(ln_bwd_v<T, V>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem)); \
    launch_k(ln_bwd_v<T, V>, dim3(nblk), dim3(256), smem, st, rows, d, dU, X, mean, rstd, (const T*)g, dres, dX, (T*)dXt, np, scratch); \
  } while (0)
#define HM_LNB_ALL(T)                   \
  switch (v) {                          \
    case 1: HM_LNB(T, 1); break;        \
    case 2: HM_LNB(T, 2); break;        \
    case 4: HM_LNB(T, 4); break;        \
    case 8: HM_LNB(T, 8); break;        \
    case 13: HM_LNB(T, 13); break;      \
    default: HM_LNB(T, 16); break;      \
  }
  if (dtype == 1) { HM_LNB_ALL(__nv_bfloat16) } else { HM_LNB_ALL(float) }
#undef HM_LNB_ALL
#undef HM_LNB
  check_launch("layernorm_bwd_vec");
  ColOuts outs{{dg, db, dsum}, {accumulate, accumulate, dsum_acc}};
  launch_k(colreduce2_kernel, dim3(dim3((unsigned)ceil_div(d, 32), (unsigned)np)), dim3(1024), 0, st, nblk, d, scratch, np * (int64_t)d,
                                                                                 outs);
  check_launch("colreduce(dgamma, dbeta[, sum dX])");
  return true;
}

}  // namespace hm
