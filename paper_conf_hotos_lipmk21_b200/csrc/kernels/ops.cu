// ops.cu — the step's HBM-bound kernels (kernels K6-K12).
//
// LayerNorm fwd/bwd and softmax fwd/bwd use one warp per row with warp-shuffle reductions
// (fixed butterfly order).  Column reductions (LN dgamma/dbeta, bias grads) are two-stage
// and deterministic: fixed row chunks write partials, a second kernel sums them in chunk
// order — no floating-point atomics anywhere (bit-exact capped == uncapped).
// Adam, cast and the activation backward are vectorised grid-stride elementwise kernels.
#include "../common.hpp"
#include "kernels.hpp"

namespace hm {

bool pdl_enabled() {
  static const bool on = [] {
    const char* v = getenv("HARMONY_PDL");
    return !(v && *v == '0');
  }();
  return on;
}

__device__ __forceinline__ float warp_sum(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}
__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
  return v;
}

static int grid_for(int64_t n, int per_block) {
  int64_t g = ceil_div(n, per_block);
  int64_t cap = 148 * 16;
  return (int)(g < 1 ? 1 : (g > cap ? cap : g));
}

// ------------------------------------------------------------------------------------- LayerNorm fwd
// Two-pass statistics (mean, then centred sum of squares; reading c10), eps = 1e-5.
template <typename T>
__global__ void __launch_bounds__(256) layernorm_fwd_kernel(int64_t rows, int d, const float* __restrict__ X,
                                                            const T* __restrict__ g, const T* __restrict__ b,
                                                            T* __restrict__ U, float* __restrict__ mean,
                                                            float* __restrict__ rstd) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int lane = threadIdx.x & 31;
  const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (row >= rows) return;
  const float* x = X + row * d;
  float s = 0.f;
  for (int c = lane; c < d; c += 32) s += x[c];
  const float mu = warp_sum(s) / (float)d;
  float q = 0.f;
  for (int c = lane; c < d; c += 32) {
    float t = x[c] - mu;
    q += t * t;
  }
  const float var = warp_sum(q) / (float)d;
  const float rs = rsqrtf(var + 1e-5f);
  T* u = U + row * d;
  for (int c = lane; c < d; c += 32) u[c] = from_f32<T>((x[c] - mu) * rs * to_f32(g[c]) + to_f32(b[c]));
  if (lane == 0) { mean[row] = mu; rstd[row] = rs; }
}

// ------------------------------------------------------------------------------------- LayerNorm bwd
constexpr int LN_ROWS_PER_BLOCK = 32;

template <typename T>
__global__ void __launch_bounds__(256) layernorm_bwd_kernel(int64_t rows, int d, const float* __restrict__ dU,
                                                            const float* __restrict__ X, const float* __restrict__ mean,
                                                            const float* __restrict__ rstd, const T* __restrict__ g,
                                                            const float* __restrict__ dres, float* __restrict__ dX,
                                                            float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t r0 = (int64_t)blockIdx.x * LN_ROWS_PER_BLOCK;
  // phase 1: dX per row (one warp per row)
  for (int i = warp; i < LN_ROWS_PER_BLOCK; i += 8) {
    const int64_t row = r0 + i;
    if (row >= rows) break;
    const float mu = mean[row], rs = rstd[row];
    const float* x = X + row * d;
    const float* du = dU + row * d;
    float s1 = 0.f, s2 = 0.f;
    for (int c = lane; c < d; c += 32) {
      float xh = (x[c] - mu) * rs;
      float dxh = du[c] * to_f32(g[c]);
      s1 += dxh;
      s2 += dxh * xh;
    }
    s1 = warp_sum(s1) / (float)d;
    s2 = warp_sum(s2) / (float)d;
    float* dx = dX + row * d;
    const float* dr = dres ? dres + row * d : nullptr;
    for (int c = lane; c < d; c += 32) {
      float xh = (x[c] - mu) * rs;
      float dxh = du[c] * to_f32(g[c]);
      float v = rs * (dxh - s1 - xh * s2);
      dx[c] = dr ? dr[c] + v : v;
    }
  }
  // phase 2: this block's column partials of dgamma = sum dU*xh and dbeta = sum dU (rows in order)
  const int64_t rend = min(rows, r0 + LN_ROWS_PER_BLOCK);
  float* pg = partial + (int64_t)blockIdx.x * 2 * d;
  for (int c = threadIdx.x; c < d; c += 256) {
    float ag = 0.f, ab = 0.f;
    for (int64_t row = r0; row < rend; ++row) {
      float du = dU[row * d + c];
      ag += du * ((X[row * d + c] - mean[row]) * rstd[row]);
      ab += du;
    }
    pg[c] = ag;
    pg[d + c] = ab;
  }
}

// out[c] (+)= sum over chunks of partial[j][c] (row stride `stride`): 32 columns per block, 32 warps
// each summing every 32nd chunk, then the 32 warp sums in warp order — a fixed tree (deterministic),
// coalesced along the columns, every load of a warp in flight at once.
__global__ void __launch_bounds__(1024) colreduce_kernel(int nchunks, int n, const float* __restrict__ partial,
                                                         int64_t stride, float* __restrict__ out, int accumulate) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  // 32 columns x 32 warps per block: warp g sums chunks g, g+32, ... in order (a handful of loads,
  // all in flight at once), then the 32 warp sums are added in warp order — a fixed tree
  __shared__ float sh[32][33];
  const int cl = threadIdx.x & 31, g = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + cl;
  float s = 0.f;
  if (c < n) {
#pragma unroll 8
    for (int j = g; j < nchunks; j += 32) s += partial[(int64_t)j * stride + c];
  }
  sh[g][cl] = s;
  __syncthreads();
  if (g == 0 && c < n) {
    float t = sh[0][cl];
#pragma unroll
    for (int k = 1; k < 32; ++k) t += sh[k][cl];
    out[c] = accumulate ? out[c] + t : t;
  }
}
// Split-K reduction: C[i] (+)= sum_{z < S} ws[z * n + i], the S partial products added in z order
// (a fixed order: deterministic), four elements per thread with 16-byte loads.
__global__ void __launch_bounds__(256) splitk_sum_kernel(int S, int64_t n4, const float4* __restrict__ ws,
                                                        float4* __restrict__ C, int accumulate) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n4) return;
  float4 t = ws[i];
  for (int z = 1; z < S; ++z) {
    const float4 u = ws[(int64_t)z * n4 + i];
    t.x += u.x; t.y += u.y; t.z += u.z; t.w += u.w;
  }
  if (accumulate) {
    const float4 c = C[i];
    t = make_float4(c.x + t.x, c.y + t.y, c.z + t.z, c.w + t.w);
  }
  C[i] = t;
}
void splitk_sum(int S, int64_t n, const float* ws, float* C, int accumulate, cudaStream_t st) {
  HM_CHECK(n % 4 == 0, HARMONY_E_INVALID_ARG, "splitk_sum: n % 4 != 0");
  const int e0 = g_prof.begin(st);
  launch_k(splitk_sum_kernel, dim3((unsigned)ceil_div(n / 4, 256)), dim3(256), 0, st, S, n / 4, reinterpret_cast<const float4*>(ws),
                                                                   reinterpret_cast<float4*>(C), accumulate);
  check_launch("splitk_sum");
  g_prof.end(PROF_OTHER, e0, st, (double)n * 4 * (S + 1 + (accumulate ? 1 : 0)));
}

static void colreduce(int nchunks, int n, const float* partial, int64_t stride, float* out, int accumulate,
                      cudaStream_t st) {
  launch_k(colreduce_kernel, dim3((unsigned)ceil_div(n, 32)), dim3(1024), 0, st, nchunks, n, partial, stride, out, accumulate);
  check_launch("colreduce");
}

// gemm_colsum's 32-row-block partials when the GEMM did not produce them: one thread per column, the
// block's rows in increasing order — the order of the fused epilogue, so the partials are identical
__global__ void colsum32_partial_kernel(int64_t rows, int n, const __nv_bfloat16* __restrict__ X, int64_t ld,
                                        float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t rb = blockIdx.y;
  if (c >= n) return;
  float s = 0.f;
  for (int r = 0; r < 32 && rb * 32 + r < rows; ++r) s += __bfloat162float(X[(rb * 32 + r) * ld + c]);
  partial[rb * n + c] = s;
}
void colsum32_partial(int64_t rows, int n, const void* X, int64_t ld, float* partial, cudaStream_t st) {
  if (rows <= 0 || n <= 0) return;
  dim3 grid((unsigned)ceil_div(n, 128), (unsigned)ceil_div(rows, 32));
  launch_k(colsum32_partial_kernel, dim3(grid), dim3(128), 0, st, rows, n, static_cast<const __nv_bfloat16*>(X), ld, partial);
  check_launch("colsum32_partial");
}
void colsum32_reduce(int64_t rows, int n, const float* partial, float* out, int accumulate, cudaStream_t st) {
  const int nch = (int)ceil_div(rows, 32);
  if (nch == 0) {
    if (!accumulate) HM_CUDA(cudaMemsetAsync(out, 0, sizeof(float) * n, st));
    return;
  }
  const int e0 = g_prof.begin(st);
  colreduce(nch, n, partial, n, out, accumulate, st);
  g_prof.end(PROF_OTHER, e0, st, (double)nch * n * 4);
}

// ------------------------------------------------------------------------------------- column sums
// partial[chunk][c] = sum of rows [chunk*CS_ROWS, ...) of column c, rows in increasing order; each
// thread owns VEC adjacent columns (16-byte loads) and keeps CS_ROWS independent loads in flight.
constexpr int CS_ROWS = 16;
template <typename Tin>
__global__ void colsum_partial_kernel(int64_t rows, int n, const Tin* __restrict__ X, int64_t ld,
                                      float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  int64_t r0 = (int64_t)blockIdx.y * CS_ROWS, r1 = min(rows, r0 + CS_ROWS);
  float s = 0.f;
  for (int64_t r = r0; r < r1; ++r) s += to_f32(X[r * ld + c]);
  partial[(int64_t)blockIdx.y * n + c] = s;
}
template <typename Tin>
__global__ void __launch_bounds__(128) colsum_partial_vec_kernel(int64_t rows, int n, const Tin* __restrict__ X,
                                                                 int64_t ld, float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  constexpr int VEC = 16 / sizeof(Tin);
  const int c0 = (blockIdx.x * blockDim.x + threadIdx.x) * VEC;
  if (c0 >= n) return;
  const int64_t r0 = (int64_t)blockIdx.y * CS_ROWS, r1 = min(rows, r0 + CS_ROWS);
  float s[VEC];
#pragma unroll
  for (int v = 0; v < VEC; ++v) s[v] = 0.f;
  uint4 u[CS_ROWS];  // every load in flight before the first add (one memory round trip per thread)
#pragma unroll
  for (int i = 0; i < CS_ROWS; ++i)
    u[i] = r0 + i < r1 ? __ldg(reinterpret_cast<const uint4*>(X + (r0 + i) * ld + c0)) : make_uint4(0, 0, 0, 0);
#pragma unroll
  for (int i = 0; i < CS_ROWS; ++i) {
    const Tin* e = reinterpret_cast<const Tin*>(&u[i]);
#pragma unroll
    for (int v = 0; v < VEC; ++v) s[v] += to_f32(e[v]);
  }
  float* p = partial + (int64_t)blockIdx.y * n + c0;
#pragma unroll
  for (int v = 0; v < VEC; v += 4) *reinterpret_cast<float4*>(p + v) = make_float4(s[v], s[v + 1], s[v + 2], s[v + 3]);
}

// One pass over an fp32 [rows, n] array: its T copy (the GEMM operand) and the column partials of
// the column sum (the bias gradient of the branch it feeds), rows in increasing order per chunk.
template <typename T>
__global__ void __launch_bounds__(128) cast_colsum_partial_kernel(int64_t rows, int n, const float* __restrict__ X,
                                                                  T* __restrict__ Xt, float* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int c0 = (blockIdx.x * blockDim.x + threadIdx.x) * 4;
  if (c0 >= n) return;
  const int64_t r0 = (int64_t)blockIdx.y * CS_ROWS, r1 = min(rows, r0 + CS_ROWS);
  float4 u[CS_ROWS];
#pragma unroll
  for (int i = 0; i < CS_ROWS; ++i)
    u[i] = r0 + i < r1 ? __ldg(reinterpret_cast<const float4*>(X + (r0 + i) * n + c0)) : make_float4(0.f, 0.f, 0.f, 0.f);
  float4 s = make_float4(0.f, 0.f, 0.f, 0.f);
#pragma unroll
  for (int i = 0; i < CS_ROWS; ++i) {
    s.x += u[i].x; s.y += u[i].y; s.z += u[i].z; s.w += u[i].w;
    if (r0 + i < r1) {
      T* o = Xt + (r0 + i) * n + c0;
      o[0] = from_f32<T>(u[i].x); o[1] = from_f32<T>(u[i].y); o[2] = from_f32<T>(u[i].z); o[3] = from_f32<T>(u[i].w);
    }
  }
  *reinterpret_cast<float4*>(partial + (int64_t)blockIdx.y * n + c0) = s;
}

// ------------------------------------------------------------------------------------- softmax
// P = softmax(scale * Z) over each row; causal rows mask keys j > (row % S) to exactly 0 (c11).
template <typename T>
__global__ void __launch_bounds__(256) softmax_fwd_kernel(int64_t rows, int S, int causal, float scale,
                                                          const float* __restrict__ Z, T* __restrict__ P) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int lane = threadIdx.x & 31;
  const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (row >= rows) return;
  const int lim = causal ? (int)(row % S) + 1 : S;
  const float* z = Z + row * S;
  float mx = -INFINITY;
  for (int c = lane; c < lim; c += 32) mx = fmaxf(mx, scale * z[c]);
  mx = warp_max(mx);
  float s = 0.f;
  for (int c = lane; c < lim; c += 32) s += __expf(scale * z[c] - mx);
  s = warp_sum(s);
  const float inv = 1.f / s;
  T* p = P + row * S;
  for (int c = lane; c < S; c += 32) p[c] = from_f32<T>(c < lim ? __expf(scale * z[c] - mx) * inv : 0.f);
}

template <typename T>
__global__ void __launch_bounds__(256) softmax_bwd_kernel(int64_t rows, int S, float alpha,
                                                          const float* __restrict__ dP, const T* __restrict__ P,
                                                          T* __restrict__ dZ) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int lane = threadIdx.x & 31;
  const int64_t row = (int64_t)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (row >= rows) return;
  const float* dp = dP + row * S;
  const T* p = P + row * S;
  float s = 0.f;
  for (int c = lane; c < S; c += 32) s += dp[c] * to_f32(p[c]);
  s = warp_sum(s);
  T* dz = dZ + row * S;
  for (int c = lane; c < S; c += 32) dz[c] = from_f32<T>(alpha * to_f32(p[c]) * (dp[c] - s));
}

// ------------------------------------------------------------------------------------- Adam
// Kingma & Ba [30], Algorithm 1 with bias correction; fp32 master state (reading c3).
template <typename T>
__global__ void adam_kernel(int64_t n, float* __restrict__ W, float* __restrict__ m, float* __restrict__ v,
                            const float* __restrict__ g, T* __restrict__ Wc, float lr, float b1, float omb1, float b2,
                            float omb2, float eps, double b1d, double b2d, const int* __restrict__ t_dev, int t_host) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  // bias corrections 1/(1-b^t) in double, once per block; t from device memory when given
  // (a CUDA-graph replay updates it without re-launching)
  __shared__ float s_bc[2];
  if (threadIdx.x == 0) {
    const double t = (double)(t_dev ? *t_dev : t_host);
    s_bc[0] = (float)(1.0 / (1.0 - pow(b1d, t)));
    s_bc[1] = (float)(1.0 / (1.0 - pow(b2d, t)));
  }
  __syncthreads();
  const float inv_bc1 = s_bc[0], inv_bc2 = s_bc[1];
  const int64_t n4 = n / 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) {
    float4 w = reinterpret_cast<float4*>(W)[i];
    float4 mm = reinterpret_cast<float4*>(m)[i];
    float4 vv = reinterpret_cast<float4*>(v)[i];
    float4 gg = reinterpret_cast<const float4*>(g)[i];
    float* wp = &w.x; float* mp = &mm.x; float* vp = &vv.x; const float* gp = &gg.x;
    float out[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      mp[j] = b1 * mp[j] + omb1 * gp[j];
      vp[j] = b2 * vp[j] + omb2 * gp[j] * gp[j];
      wp[j] = wp[j] - lr * (mp[j] * inv_bc1) / (sqrtf(vp[j] * inv_bc2) + eps);
      out[j] = wp[j];
    }
    reinterpret_cast<float4*>(W)[i] = w;
    reinterpret_cast<float4*>(m)[i] = mm;
    reinterpret_cast<float4*>(v)[i] = vv;
    if (sizeof(T) == 2) {
      __nv_bfloat162 lo = __floats2bfloat162_rn(out[0], out[1]);
      __nv_bfloat162 hi = __floats2bfloat162_rn(out[2], out[3]);
      uint2 pk;
      pk.x = *reinterpret_cast<uint32_t*>(&lo);
      pk.y = *reinterpret_cast<uint32_t*>(&hi);
      reinterpret_cast<uint2*>(Wc)[i] = pk;
    } else {
      reinterpret_cast<float4*>(Wc)[i] = make_float4(out[0], out[1], out[2], out[3]);
    }
  }
  for (int64_t i = n4 * 4 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    float mi = b1 * m[i] + omb1 * g[i];
    float vi = b2 * v[i] + omb2 * g[i] * g[i];
    float wi = W[i] - lr * (mi * inv_bc1) / (sqrtf(vi * inv_bc2) + eps);
    m[i] = mi; v[i] = vi; W[i] = wi;
    Wc[i] = from_f32<T>(wi);
  }
}

// ------------------------------------------------------------------------------------- MSE loss
constexpr int MSE_BLOCK = 256;
__global__ void mse_kernel(int64_t n, const float* __restrict__ Y, const float* __restrict__ Tg, float inv_batch,
                           float* __restrict__ dY, double* __restrict__ partial) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  __shared__ double sh[MSE_BLOCK / 32];
  double acc = 0.0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    float dlt = Y[i] - Tg[i];
    dY[i] = dlt * inv_batch;
    acc += (double)dlt * (double)dlt;
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if ((threadIdx.x & 31) == 0) sh[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double s = 0.0;
    for (int w = 0; w < MSE_BLOCK / 32; ++w) s += sh[w];
    partial[blockIdx.x] = s;
  }
}
// fixed-order tree over the block partials: thread t sums t, t+256, ...; then a smem tree
__global__ void __launch_bounds__(256) mse_final_kernel(int nblk, const double* __restrict__ partial,
                                                        double half_inv_batch, double* __restrict__ out) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  __shared__ double sh[256];
  double s = 0.0;
  for (int j = threadIdx.x; j < nblk; j += 256) s += partial[j];
  sh[threadIdx.x] = s;
  __syncthreads();
  for (int w = 128; w > 0; w >>= 1) {
    if (threadIdx.x < w) sh[threadIdx.x] += sh[threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x == 0) *out = sh[0] * half_inv_batch;
}

// ------------------------------------------------------------------------------------- elementwise
template <typename T>
__global__ void cast_kernel(int64_t n, const float* __restrict__ in, T* __restrict__ out) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) out[i] = from_f32<T>(in[i]);
}
template <typename T>
__global__ void act_bwd_kernel(int act, int64_t n, const float* __restrict__ dY, const T* __restrict__ Z,
                               T* __restrict__ dZ) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
    dZ[i] = from_f32<T>(dY[i] * act_grad_T<T>(act, to_f32(Z[i])));
}
template <typename T>
__global__ void act_fwd_kernel(int act, int64_t n, const T* __restrict__ Z, T* __restrict__ out) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
    out[i] = from_f32<T>(act_T<T>(act, to_f32(Z[i])));
}
__global__ void copy_rows_kernel(int64_t n4, const float4* __restrict__ src, float4* __restrict__ dst) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride) dst[i] = src[i];
}

// ===================================================================================== launchers
#define HM_DISPATCH_T(dtype, ...)                                 \
  do {                                                            \
    if ((dtype) == 1) {                                           \
      using T = __nv_bfloat16;                                    \
      __VA_ARGS__;                                                \
    } else {                                                      \
      using T = float;                                            \
      __VA_ARGS__;                                                \
    }                                                             \
  } while (0)

void layernorm_fwd(int dtype, int64_t rows, int d, const float* X, const void* g, const void* b, void* U, float* mean,
                   float* rstd, cudaStream_t st, float* Xcopy) {
  if (rows == 0) return;
  const int e0 = g_prof.begin(st);
  if (layernorm_fwd_vec(dtype, rows, d, X, g, b, U, mean, rstd, st, Xcopy)) {
    g_prof.end(PROF_LN, e0, st, (double)rows * d * (4 + (dtype ? 2 : 4) + (Xcopy ? 4 : 0)) + rows * 8.0);
    return;
  }
  if (Xcopy) copy_f32(rows * d, X, Xcopy, st);
  HM_DISPATCH_T(dtype, (launch_k(layernorm_fwd_kernel<T>, dim3((unsigned)ceil_div(rows, 8)), dim3(256), 0, st, 
                           rows, d, X, (const T*)g, (const T*)b, (T*)U, mean, rstd)));
  check_launch("layernorm_fwd");
  g_prof.end(PROF_LN, e0, st, (double)rows * d * (4 + (dtype ? 2 : 4)) + rows * 8.0);
}

size_t layernorm_bwd_scratch_bytes(int64_t rows, int d) {
  return std::max((size_t)ceil_div(rows, LN_ROWS_PER_BLOCK) * 2 * d * sizeof(float),
                  layernorm_bwd_vec_scratch_bytes(rows, d));
}

void layernorm_bwd(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                   const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db, int accumulate,
                   float* scratch, cudaStream_t st) {
  layernorm_bwd_ex(dtype, rows, d, dU, X, mean, rstd, g, dres, dX, dg, db, accumulate, nullptr, nullptr, 0, scratch, st);
}

void layernorm_bwd_ex(int dtype, int64_t rows, int d, const float* dU, const float* X, const float* mean,
                      const float* rstd, const void* g, const float* dres, float* dX, float* dg, float* db,
                      int accumulate, void* dXt, float* dsum, int dsum_acc, float* scratch, cudaStream_t st) {
  if (rows == 0) {
    return;
  }
  const int e0 = g_prof.begin(st);
  if (layernorm_bwd_vec(dtype, rows, d, dU, X, mean, rstd, g, dres, dX, dg, db, accumulate, dXt, dsum, dsum_acc,
                        scratch, st)) {
    g_prof.end(PROF_LN, e0, st, (double)rows * d * (4 * (dres ? 4 : 3) + (dXt ? (dtype ? 2 : 4) : 0)) + rows * 8.0);
    return;
  }
  int nblk = (int)ceil_div(rows, LN_ROWS_PER_BLOCK);
  HM_DISPATCH_T(dtype, (launch_k(layernorm_bwd_kernel<T>, dim3(nblk), dim3(256), 0, st, rows, d, dU, X, mean, rstd, (const T*)g, dres,
                                                                      dX, scratch)));
  check_launch("layernorm_bwd");
  colreduce(nblk, d, scratch, 2 * (int64_t)d, dg, accumulate, st);
  colreduce(nblk, d, scratch + d, 2 * (int64_t)d, db, accumulate, st);
  if (dXt) cast(dtype, rows * d, dX, dXt, st);
  if (dsum) colsum(0, rows, d, dX, d, dsum, dsum_acc, scratch, st);
  g_prof.end(PROF_LN, e0, st, (double)rows * d * 4 * (dres ? 4 : 3) + rows * 8.0);
}

size_t colsum_scratch_bytes(int64_t rows, int n) { return (size_t)ceil_div(rows, CS_ROWS) * n * sizeof(float); }

void colsum(int in_dtype, int64_t rows, int n, const void* X, int64_t ld, float* out, int accumulate, float* scratch,
            cudaStream_t st) {
  int nch = (int)ceil_div(rows, CS_ROWS);
  if (nch == 0) {
    if (!accumulate) HM_CUDA(cudaMemsetAsync(out, 0, sizeof(float) * n, st));
    return;
  }
  const int vec = 16 / (in_dtype ? 2 : 4);
  const bool vok = n % vec == 0 && ld % vec == 0 && (reinterpret_cast<uintptr_t>(X) & 15) == 0;
  const int e0 = g_prof.begin(st);
  if (vok) {
    dim3 grid((unsigned)ceil_div(n / vec, 128), (unsigned)nch);
    HM_DISPATCH_T(in_dtype, (launch_k(colsum_partial_vec_kernel<T>, dim3(grid), dim3(128), 0, st, rows, n, (const T*)X, ld, scratch)));
  } else {
    dim3 grid((unsigned)ceil_div(n, 128), (unsigned)nch);
    HM_DISPATCH_T(in_dtype, (launch_k(colsum_partial_kernel<T>, dim3(grid), dim3(128), 0, st, rows, n, (const T*)X, ld, scratch)));
  }
  check_launch("colsum_partial");
  colreduce(nch, n, scratch, n, out, accumulate, st);
  g_prof.end(PROF_OTHER, e0, st, (double)rows * n * (in_dtype ? 2 : 4));
}

void cast_colsum(int dtype, int64_t rows, int n, const float* X, void* Xt, float* out, int accumulate, float* scratch,
                 cudaStream_t st) {
  const int nch = (int)ceil_div(rows, CS_ROWS);
  if (n % 4 || (reinterpret_cast<uintptr_t>(X) & 15) || nch == 0) {  // unaligned: the two separate passes
    cast(dtype, rows * n, X, Xt, st);
    colsum(0, rows, n, X, n, out, accumulate, scratch, st);
    return;
  }
  const int e0 = g_prof.begin(st);
  dim3 grid((unsigned)ceil_div(n / 4, 128), (unsigned)nch);
  HM_DISPATCH_T(dtype, (launch_k(cast_colsum_partial_kernel<T>, dim3(grid), dim3(128), 0, st, rows, n, X, (T*)Xt, scratch)));
  check_launch("cast_colsum_partial");
  colreduce(nch, n, scratch, n, out, accumulate, st);
  g_prof.end(PROF_OTHER, e0, st, (double)rows * n * (4 + (dtype ? 2 : 4)));
}

void softmax_fwd(int dtype, int64_t rows, int S, int causal, float scale, const float* Z, void* P, cudaStream_t st) {
  if (rows == 0) return;
  const int e0 = g_prof.begin(st);
  HM_DISPATCH_T(dtype, (launch_k(softmax_fwd_kernel<T>, dim3((unsigned)ceil_div(rows, 8)), dim3(256), 0, st, rows, S, causal, scale, Z,
                                                                                          (T*)P)));
  check_launch("softmax_fwd");
  g_prof.end(PROF_SOFTMAX, e0, st, (double)rows * S * (4 + (dtype ? 2 : 4)));
}

void softmax_bwd(int dtype, int64_t rows, int S, float alpha, const float* dP, const void* P, void* dZ,
                 cudaStream_t st) {
  if (rows == 0) return;
  const int e0 = g_prof.begin(st);
  HM_DISPATCH_T(dtype, (launch_k(softmax_bwd_kernel<T>, dim3((unsigned)ceil_div(rows, 8)), dim3(256), 0, st, rows, S, alpha, dP,
                                                                                          (const T*)P, (T*)dZ)));
  check_launch("softmax_bwd");
  g_prof.end(PROF_SOFTMAX, e0, st, (double)rows * S * (4 + 2 * (dtype ? 2 : 4)));
}

void adam(int dtype, int64_t n, float* W, float* m, float* v, const float* g, void* Wc, double lr, double b1, double b2,
          double eps, int t, const int* t_dev, cudaStream_t st) {
  if (n == 0) return;
  HM_CHECK(((uintptr_t)W | (uintptr_t)m | (uintptr_t)v | (uintptr_t)g) % 16 == 0, HARMONY_E_INVALID_ARG,
           "adam: fp32 state must be 16-byte aligned");
  const int e0 = g_prof.begin(st);
  HM_DISPATCH_T(dtype, (launch_k(adam_kernel<T>, dim3(grid_for(ceil_div(n, 4), 256)), dim3(256), 0, st, 
                           n, W, m, v, g, (T*)Wc, (float)lr, (float)b1, (float)(1.0 - b1), (float)b2, (float)(1.0 - b2), (float)eps,
                           b1, b2, t_dev, t)));
  check_launch("adam");
  g_prof.end(PROF_ADAM, e0, st, (double)n * (16 + 12 + (dtype ? 2 : 4)));  // read W,m,v,g; write W,m,v,Wc
}

size_t mse_scratch_bytes() { return 1024 * sizeof(double); }

void mse(int64_t n, const float* Y, const float* Tg, float inv_batch, float* dY, double* loss_out, double* scratch,
         cudaStream_t st) {
  int nblk = (int)std::min<int64_t>(1024, std::max<int64_t>(1, ceil_div(n, MSE_BLOCK * 8)));
  launch_k(mse_kernel, dim3(nblk), dim3(MSE_BLOCK), 0, st, n, Y, Tg, inv_batch, dY, scratch);
  check_launch("mse");
  launch_k(mse_final_kernel, dim3(1), dim3(256), 0, st, nblk, scratch, 0.5 * (double)inv_batch, loss_out);
  check_launch("mse_final");
}

void cast(int dtype, int64_t n, const float* in, void* out, cudaStream_t st) {
  if (n == 0) return;
  const int e0 = g_prof.begin(st);
  HM_DISPATCH_T(dtype, (launch_k(cast_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, n, in, (T*)out)));
  check_launch("cast");
  g_prof.end(PROF_OTHER, e0, st, (double)n * (4 + (dtype ? 2 : 4)));
}

void act_bwd(int dtype, int act, int64_t n, const float* dY, const void* Z, void* dZ, cudaStream_t st) {
  if (n == 0) return;
  const int e0 = g_prof.begin(st);
  HM_DISPATCH_T(dtype, (launch_k(act_bwd_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, act, n, dY, (const T*)Z, (T*)dZ)));
  check_launch("act_bwd");
  g_prof.end(PROF_OTHER, e0, st, (double)n * (4 + 2 * (dtype ? 2 : 4)));
}

void act_fwd_T(int dtype, int act, int64_t n, const void* Z, void* out, cudaStream_t st) {
  if (n == 0) return;
  HM_DISPATCH_T(dtype, (launch_k(act_fwd_kernel<T>, dim3(grid_for(n, 256)), dim3(256), 0, st, act, n, (const T*)Z, (T*)out)));
  check_launch("act_fwd");
}

void copy_f32(int64_t n, const float* src, float* dst, cudaStream_t st) {
  if (n == 0) return;
  if (n % 4 == 0 && ((uintptr_t)src | (uintptr_t)dst) % 16 == 0) {
    const int e0 = g_prof.begin(st);
    launch_k(copy_rows_kernel, dim3(grid_for(n / 4, 256)), dim3(256), 0, st, n / 4, (const float4*)src, (float4*)dst);
    check_launch("copy_f32");
    g_prof.end(PROF_OTHER, e0, st, (double)n * 8);
  } else {
    HM_CUDA(cudaMemcpyAsync(dst, src, n * sizeof(float), cudaMemcpyDeviceToDevice, st));
  }
}

}  // namespace hm
