// gemm.cu — the step's dense contractions (kernels K1-K5).
//
//  * bf16 path: a warp-specialised tcgen05 GEMM for sm_100a.  TMA (cp.async.bulk.tensor,
//    128-byte swizzle, OOB zero fill for M/N/K tails) feeds a STAGES-deep mbarrier ring in
//    shared memory; one elected thread issues tcgen05.mma.cta_group::1.kind::f16
//    (bf16 x bf16 -> fp32) with the accumulator in TMEM; four epilogue warps drain TMEM
//    with tcgen05.ld and apply the fused epilogue (bias / residual / GeLU / dW accumulate).
//    K-major and MN-major operands are both native (UMMA descriptor major bits), so
//    fwd (X.W: W is N-contiguous), dgrad (dY.W^T: K-major) and wgrad (X^T.dY: both
//    MN-major) read the stored tensors directly - no transposes.  Batched (two batch
//    dims) for the attention contractions.
//  * fp32 path (precision HARMONY_FP32): a tiled SIMT FFMA GEMM with the same operand
//    and epilogue conventions (true fp32; kind::tf32 would miss the 1e-5 budget).
// Determinism: the K reduction order is fixed per (shape, tile config), the tile config
// never depends on the memory cap, and each output element has exactly one writer.
#include <cuda.h>
#include <cudaTypedefs.h>
#include <mutex>

#include "epilogue.cuh"
#include "kernels.hpp"
#include "tc_common.cuh"

namespace hm {

// ----------------------------------------------------------------------------------------- SIMT fp32
struct SimtParams {
  int M, N, K, nz0;
  const float* A; int a_mn; int64_t lda, a_sz0, a_sz1;
  const float* B; int b_mn; int64_t ldb, b_sz0, b_sz1;
  EpiParams e;
};

constexpr int SBM = 64, SBN = 64, SBK = 16;

__global__ void __launch_bounds__(256) gemm_simt_kernel(SimtParams p) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  __shared__ float As[SBK][SBM + 4];
  __shared__ float Bs[SBK][SBN + 4];
  const int tid = threadIdx.x;
  const int z = blockIdx.z, z0 = z % p.nz0, z1 = z / p.nz0;
  const int m0 = blockIdx.y * SBM, n0 = blockIdx.x * SBN;
  const float* A = p.A + z0 * p.a_sz0 + z1 * p.a_sz1;
  const float* B = p.B + z0 * p.b_sz0 + z1 * p.b_sz1;
  const int tx = tid % 16, ty = tid / 16;
  float acc[4][4] = {};
  const bool cont = p.e.epi == HK_EPI_ACC_F32 && p.e.accumulate == 2;  // continue C's K reduction
  if (cont) {
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int m = m0 + ty + 16 * i, n = n0 + tx + 16 * j;
        if (m < p.M && n < p.N)
          acc[i][j] = reinterpret_cast<const float*>(p.e.C)[z0 * p.e.c_sz0 + z1 * p.e.c_sz1 + (int64_t)m * p.e.ldc + n];
      }
  }
  for (int k0 = 0; k0 < p.K; k0 += SBK) {
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      int idx = tid + i * 256;
      int r, kk;
      if (p.a_mn) { kk = idx / SBM; r = idx % SBM; } else { r = idx / SBK; kk = idx % SBK; }
      int gm = m0 + r, gk = k0 + kk;
      As[kk][r] = (gm < p.M && gk < p.K) ? (p.a_mn ? A[(int64_t)gk * p.lda + gm] : A[(int64_t)gm * p.lda + gk]) : 0.f;
      if (p.b_mn) { kk = idx / SBN; r = idx % SBN; } else { r = idx / SBK; kk = idx % SBK; }
      int gn = n0 + r;
      gk = k0 + kk;
      Bs[kk][r] = (gn < p.N && gk < p.K) ? (p.b_mn ? B[(int64_t)gk * p.ldb + gn] : B[(int64_t)gn * p.ldb + gk]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < SBK; ++kk) {
      float a[4], b[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { a[i] = As[kk][ty + 16 * i]; b[i] = Bs[kk][tx + 16 * i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
  const EpiParams& e = p.e;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int m = m0 + ty + 16 * i;
    if (m >= p.M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx + 16 * j;
      if (n >= p.N) continue;
      int64_t off = z0 * e.c_sz0 + z1 * e.c_sz1 + (int64_t)m * e.ldc + n;
      if (cont) reinterpret_cast<float*>(e.C)[off] = acc[i][j];
      else epi_scalar<float>(e, off, n, acc[i][j]);
    }
  }
}

// ----------------------------------------------------------------------------------------- tcgen05
namespace tc {

constexpr int BM = 128;
constexpr int BK = 64;                 // 64 bf16 = 128 bytes = one 128B swizzle row
constexpr int EPI_WARPS = 8;           // two epilogue warps per TMEM lane quadrant (column halves)
constexpr int NUM_THREADS = 64 + 32 * EPI_WARPS;  // warp 0: TMA, warp 1: MMA + TMEM alloc, warps 2..9: epilogue

using namespace tcx;

__device__ __forceinline__ uint32_t make_idesc(int bn, int a_mn, int b_mn) { return make_idesc_f16(BM, bn, a_mn, b_mn); }

// Epilogue inputs read from global memory: 1 = fp32 residual (aux), 2 = old fp32 C (dW accumulate),
// 3 = bf16 stored pre-activation (aux of ACT_BWD), 0 = none.
__device__ __forceinline__ int epi_in_kind(const EpiParams& e, int epi) {
  if (epi == HK_EPI_RESID_F32) return 1;
  if (epi == HK_EPI_ACC_F32 && e.accumulate) return 2;
  if (epi == HK_EPI_ACT_BWD) return 3;
  return 0;
}
__device__ __forceinline__ int epi_in_kind(const EpiParams& e) { return epi_in_kind(e, e.epi); }

// L2 prefetch of this thread's row segment [n_beg, n_end) of the epilogue input, issued before the
// accumulator wait so the (cold, HBM) residual / dW / pre-activation read overlaps the mainloop.
__device__ __forceinline__ void epi_prefetch(const EpiParams& e, int m, int n_beg, int n_end, int64_t zoff) {
  const int kind = epi_in_kind(e);
  if (!kind || m >= e.M || n_beg >= n_end) return;
  const int esz = kind == 3 ? 2 : 4;
  const char* base = static_cast<const char*>(kind == 2 ? e.C : e.aux);
  const char* p = base + (zoff + (int64_t)m * e.ldc + n_beg) * esz;
  const int bytes = (n_end - n_beg) * esz;
  for (int o = 0; o < bytes; o += 128) asm volatile("prefetch.global.L2 [%0];" ::"l"(p + o));
  asm volatile("prefetch.global.L2 [%0];" ::"l"(p + bytes - 1));
}

__device__ __forceinline__ bool al16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }

// one epilogue warp's 32-column chunk: TMEM (thread = row) -> registers -> fused epilogue -> global in
// 32-byte row pieces (full sectors).  The chunk's global inputs are loaded before the TMEM load so
// their latency overlaps it.  A variant that transposed chunks through shared memory for 128-byte
// row segments measured 6% slower in the step (profiles/r01_epilogue_ab.txt) and was dropped.
__device__ __forceinline__ void drain_chunk(const EpiParams& e, uint32_t taddr, bool have_acc, int lane, int mrow0,
                                            int n, int64_t zoff) {
  const int m = mrow0 + lane;
  const int64_t off = zoff + (int64_t)m * e.ldc + n;
  const int kind = epi_in_kind(e);
  const void* src = kind == 2 ? e.C : e.aux;
  const bool fast = kind != 0 && m < e.M && n + 32 <= e.N && al16(static_cast<float*>(e.C) + (kind == 3 ? 0 : off)) &&
                    (kind == 3 ? al16(static_cast<const __nv_bfloat16*>(src) + off) &&
                                     al16(static_cast<__nv_bfloat16*>(e.C) + off)
                               : al16(static_cast<const float*>(src) + off));
  float4 in[8];
  if (fast) {
    if (kind == 3) {
      const uint4* s4 = reinterpret_cast<const uint4*>(static_cast<const __nv_bfloat16*>(src) + off);
#pragma unroll
      for (int q = 0; q < 4; ++q) { uint4 u = s4[q]; in[q] = *reinterpret_cast<float4*>(&u); }
    } else {
      const float4* s4 = reinterpret_cast<const float4*>(static_cast<const float*>(src) + off);
#pragma unroll
      for (int q = 0; q < 8; ++q) in[q] = s4[q];
    }
  }
  float v[32];
  if (have_acc) {
    tmem_ld32(taddr, v);
  } else {
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = 0.f;
  }
  if (m >= e.M) return;
  if (fast) {
    if (kind == 3) {  // dH = dG * act'(H), bf16 out
      const __nv_bfloat16* h = reinterpret_cast<const __nv_bfloat16*>(in);
      uint4 o[4];
      __nv_bfloat162* op = reinterpret_cast<__nv_bfloat162*>(o);
#pragma unroll
      for (int j = 0; j < 16; ++j)
        op[j] = __floats2bfloat162_rn(v[2 * j] * act_grad_f<true>(e.act, __bfloat162float(h[2 * j])),
                                      v[2 * j + 1] * act_grad_f<true>(e.act, __bfloat162float(h[2 * j + 1])));
      uint4* cp = reinterpret_cast<uint4*>(static_cast<__nv_bfloat16*>(e.C) + off);
#pragma unroll
      for (int q = 0; q < 4; ++q) cp[q] = o[q];
    } else {
      float4* c4 = reinterpret_cast<float4*>(static_cast<float*>(e.C) + off);
      if (kind == 1) {  // C = aux + (acc + b)
        float bb[32];
        load_bias32(e, n, bb);
#pragma unroll
        for (int q = 0; q < 8; ++q)
          c4[q] = make_float4(in[q].x + (v[4 * q] + bb[4 * q]), in[q].y + (v[4 * q + 1] + bb[4 * q + 1]),
                              in[q].z + (v[4 * q + 2] + bb[4 * q + 2]), in[q].w + (v[4 * q + 3] + bb[4 * q + 3]));
      } else {  // C = C + alpha * acc
#pragma unroll
        for (int q = 0; q < 8; ++q)
          c4[q] = make_float4(in[q].x + e.alpha * v[4 * q], in[q].y + e.alpha * v[4 * q + 1],
                              in[q].z + e.alpha * v[4 * q + 2], in[q].w + e.alpha * v[4 * q + 3]);
      }
    }
    return;
  }
  epi_row16<__nv_bfloat16>(e, zoff + (int64_t)m * e.ldc, n, v);
  if (n + 16 < e.N) epi_row16<__nv_bfloat16>(e, zoff + (int64_t)m * e.ldc, n + 16, v + 16);
}

struct TcParams {
  int M, N, K, nz0, nz, a_mn, b_mn;
  int tma_epi;  // 1: epilogue through shared-memory staging + TMA stores (maps tmC / tmIn / tmO2)
  int group_m;  // tile raster: GROUP_M consecutive m-tiles per n sweep (order only; results unchanged)
  int diag;     // experiments only (HARMONY_GEMM_DIAG): bit 0 = epilogue warps drain nothing (timing of the
                // mainloop alone; the output is not written); bit 1 = no TMEM loads (zeros stored);
                // bit 2 = no TMA stores of the (first) output
  EpiParams e;
};

// ------------------------------------------------------------------ TMA-store epilogue
// Each epilogue warp owns two 4 KB staging boxes of 32 rows x 128 bytes (32 fp32 or 64 bf16
// columns) in the 128-byte swizzle of the tensor map, so a thread writing its own row in 16-byte
// pieces is bank-conflict free, plus its columns' bias as fp32.  Per box: TMEM -> registers ->
// fused epilogue -> staging -> one TMA store (full-line writes, asynchronous: the warp moves on).
// Epilogues that read global data (residual, old dW, stored pre-activation) TMA-load the box into
// the staging buffer ahead of use: the first box before the accumulator wait (overlapping the
// mainloop), each next one while the current one is processed.  BIAS_ACT writes its two bf16
// outputs through both boxes.  (BIAS_ACT_F32, an fp32 second output, keeps the register path.)
constexpr int EPI_BUF = 4096;
// fp32 bias of a warp's (at most 128) columns, staged once per (accumulator buffer, column half): the
// four row-quadrant warps of a half write the same values, and a warp is never more than one tile
// ahead of another (the accumulator hand-off), so the tile-parity double buffer is race-free
constexpr int EPI_BIAS_SET = 128 * 4;  // fp32
constexpr int EPI_BIAS = 4 * EPI_BIAS_SET;  // [2 accumulators][2 halves]
constexpr int EPI_SMEM = EPI_WARPS * 2 * EPI_BUF + EPI_BIAS + EPI_WARPS * 2 * 8;

struct EpiWarp {
  uint32_t buf;   // shared address of the two staging boxes
  uint32_t bias;  // shared address of the fp32 bias
  uint64_t* bar;  // input-load barriers of the two boxes
  uint32_t ph;    // parity bit per box
  uint32_t j;     // boxes processed
};

__device__ __forceinline__ uint32_t swz128(int r, int k) { return (uint32_t)(r * 128 + ((k ^ (r & 7)) << 4)); }
__device__ __forceinline__ void sts128(uint32_t a, uint32_t x, uint32_t y, uint32_t z, uint32_t w) {
  asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(x), "r"(y), "r"(z), "r"(w) : "memory");
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.b32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ float4 lds128f(uint32_t a) {
  uint4 v = lds128(a);
  return make_float4(__uint_as_float(v.x), __uint_as_float(v.y), __uint_as_float(v.z), __uint_as_float(v.w));
}
// four bf16 at a shared address (8-byte aligned) as fp32
__device__ __forceinline__ float4 lds_bf16x4(uint32_t a) {
  uint32_t x, y;
  asm volatile("ld.shared.v2.b32 {%0, %1}, [%2];" : "=r"(x), "=r"(y) : "r"(a) : "memory");
  const float2 lo = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&x));
  const float2 hi = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&y));
  return make_float4(lo.x, lo.y, hi.x, hi.y);
}
__device__ __forceinline__ uint32_t pack_bf16(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}
__device__ __forceinline__ void tma_load_box(uint32_t dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                             int c3, uint32_t bytes) {
  mbar_expect_tx(bar, bytes);
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(
          dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void tma_store_box(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2, int c3) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group [%0, {%2, %3, %4, %5}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
               : "memory");
}
// the same with an L2 eviction-priority policy (createpolicy) for the written lines
__device__ __forceinline__ void tma_store_box_hint(const CUtensorMap* map, uint32_t src, int c0, int c1, int c2, int c3,
                                                   uint64_t pol) {
  asm volatile("cp.async.bulk.tensor.4d.global.shared::cta.bulk_group.L2::cache_hint [%0, {%2, %3, %4, %5}], [%1], %6;" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(src), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "l"(pol)
               : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}

// One warp writes a staged 32-row x 128-byte box (128B-swizzled) to global memory with coalesced
// 16-byte stores (8 lanes per 128-byte row) — the LSU path instead of a TMA store, which leaves the
// TMA unit to the mainloop's loads.  Rows / columns past M / N are not written.
template <int ESZ>
__device__ __forceinline__ void warp_store_box(void* base, int64_t ld, uint32_t sb, int row0, int n, int M, int N,
                                               int lane) {
  constexpr int EPC = 16 / ESZ;  // elements per 16-byte chunk
#pragma unroll
  for (int it = 0; it < 8; ++it) {
    const int idx = it * 32 + lane, r = idx >> 3, k = idx & 7;
    const int grow = row0 + r, gcol = n + k * EPC;
    if (grow >= M || gcol >= N) continue;
    const uint4 v = lds128(sb + swz128(r, k));
    char* dst = static_cast<char*>(base) + ((int64_t)grow * ld + gcol) * ESZ;
    if (gcol + EPC <= N) {
      *reinterpret_cast<uint4*>(dst) = v;
    } else {
      const char* src = reinterpret_cast<const char*>(&v);
      for (int q = 0; q < (N - gcol) * ESZ; ++q) dst[q] = src[q];
    }
  }
}

// Is the TMA epilogue usable for this epilogue kind / tile width (host and device agree)?
__host__ __device__ __forceinline__ bool tma_epi_kind_ok(int epi) { return epi != HK_EPI_BIAS_ACT_F32; }

// One warp's share of one tile: 32 rows (row0..) x columns [n_beg, n_end) (n_end - n_beg <= 128),
// TMEM columns from tacc.  ESZ = output element size (4: fp32 outputs, 2: bf16 outputs).  EK >= 0:
// the epilogue kind fixed at compile time (only its code is emitted, no diagnostics); -1: read
// from the parameters (every kind and the HARMONY_GEMM_DIAG experiments in one body).
template <int ESZ, int EK = -1>
__device__ __forceinline__ void tma_epi_tile(const TcParams& p, const CUtensorMap* mC, const CUtensorMap* mIn,
                                             const CUtensorMap* mO2, EpiWarp& w, uint32_t tacc, bool have_acc,
                                             int lane, int row0, int n_beg, int n_end, int z0, int z1,
                                             uint64_t* full_bar, uint32_t full_par) {
  constexpr int CPB = 128 / ESZ;  // columns per box
  const EpiParams& e = p.e;
  const int epi = EK >= 0 ? EK : e.epi;
  const int diag = EK >= 0 ? 0 : p.diag;
  const int kind = epi_in_kind(e, epi);
  const bool two = epi == HK_EPI_BIAS_ACT;
  const int nbox = n_end > n_beg ? (n_end - n_beg + CPB - 1) / CPB : 0;
  const bool has_bias = e.bias != nullptr && (epi == HK_EPI_STORE_T || epi == HK_EPI_BIAS_ACT ||
                                              epi == HK_EPI_ACT_T || epi == HK_EPI_STORE_F32 ||
                                              epi == HK_EPI_RESID_F32);
  if (kind && nbox > 0 && lane == 0) {
    const int b = w.j & 1;
    bulk_wait_read<1>();  // the store two boxes back has left this box
    tma_load_box(w.buf + b * EPI_BUF, mIn, &w.bar[b], n_beg, row0, z0, z1, EPI_BUF);
  }
  if (has_bias) {  // this warp's bias columns as fp32 (while the mainloop runs)
    const __nv_bfloat16* bp = static_cast<const __nv_bfloat16*>(e.bias);
    for (int c = lane; c < nbox * CPB; c += 32) {
      const int n = n_beg + c;
      const float bv = n < e.N ? __bfloat162float(bp[n]) : 0.f;
      asm volatile("st.shared.f32 [%0], %1;" ::"r"(w.bias + 4 * c), "f"(bv) : "memory");
    }
    __syncwarp();
  }
  mbar_wait(full_bar, full_par);
  tc_fence_after();
  const int r = lane;
#pragma unroll 1
  for (int bi = 0; bi < nbox; ++bi) {
    const int b = w.j & 1;
    const int n = n_beg + CPB * bi;
    const uint32_t sb = two ? w.buf : w.buf + b * EPI_BUF;
    if (kind) {
      if (bi + 1 < nbox && lane == 0) {
        bulk_wait_read<0>();  // the previous box's store has left the other buffer
        tma_load_box(w.buf + (b ^ 1) * EPI_BUF, mIn, &w.bar[b ^ 1], n + CPB, row0, z0, z1, EPI_BUF);
      }
    } else if (lane == 0) {
      // <= 1 store group pending: one buffer back (plain), or for BIAS_ACT the previous box's G
      // store may still be reading buffer B while this box's H goes into buffer A
      bulk_wait_read<1>();
    }
    float v[CPB];
    uint32_t hkeep[ESZ == 2 ? 32 : 1];  // BIAS_ACT: this box's packed H, the input of G
    if (have_acc && !(diag & 2)) {
#pragma unroll
      for (int h = 0; h < CPB / 32; ++h) tmem_ld32(tacc + CPB * bi + 32 * h, v + 32 * h);
    } else {
#pragma unroll
      for (int i = 0; i < CPB; ++i) v[i] = 0.f;
    }
    if (kind) {
      mbar_wait(&w.bar[b], (w.ph >> b) & 1);
      w.ph ^= 1u << b;
    } else {
      __syncwarp();
    }
    const uint32_t bias_row = w.bias + 4 * CPB * bi;
    if (ESZ == 4) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t ad = sb + swz128(r, k);
        float o0 = e.alpha * v[4 * k], o1 = e.alpha * v[4 * k + 1], o2 = e.alpha * v[4 * k + 2],
              o3 = e.alpha * v[4 * k + 3];
        if (epi == HK_EPI_RESID_F32) {  // C = aux + (acc + b)
          float4 bb = has_bias ? lds128f(bias_row + 16 * k) : make_float4(0.f, 0.f, 0.f, 0.f);
          const float4 in = lds128f(ad);
          o0 = in.x + (v[4 * k] + bb.x); o1 = in.y + (v[4 * k + 1] + bb.y);
          o2 = in.z + (v[4 * k + 2] + bb.z); o3 = in.w + (v[4 * k + 3] + bb.w);
        } else if (epi == HK_EPI_ACC_F32) {  // C (+)= alpha * acc
          if (kind) {
            const float4 in = lds128f(ad);
            o0 = in.x + o0; o1 = in.y + o1; o2 = in.z + o2; o3 = in.w + o3;
          }
        } else if (has_bias) {  // STORE_F32
          float4 bb = lds128f(bias_row + 16 * k);
          o0 += bb.x; o1 += bb.y; o2 += bb.z; o3 += bb.w;
        }
        sts128(ad, __float_as_uint(o0), __float_as_uint(o1), __float_as_uint(o2), __float_as_uint(o3));
      }
    } else {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const uint32_t ad = sb + swz128(r, k);
        const float* x = v + 8 * k;
        uint32_t o[4];
        if (epi == HK_EPI_ACT_BWD) {  // dH = dG * act'(H)
          const uint4 in = lds128(ad);
          const uint32_t hw[4] = {in.x, in.y, in.z, in.w};
#pragma unroll
          for (int t = 0; t < 4; ++t) {
            const float2 h = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&hw[t]));
            o[t] = pack_bf16(x[2 * t] * act_grad_f<true>(e.act, h.x), x[2 * t + 1] * act_grad_f<true>(e.act, h.y));
          }
        } else {
          float bb[8];
          if (has_bias) {
            const float4 b0 = lds128f(bias_row + 32 * k), b1 = lds128f(bias_row + 32 * k + 16);
            bb[0] = b0.x; bb[1] = b0.y; bb[2] = b0.z; bb[3] = b0.w; bb[4] = b1.x; bb[5] = b1.y; bb[6] = b1.z; bb[7] = b1.w;
          } else {
#pragma unroll
            for (int t = 0; t < 8; ++t) bb[t] = 0.f;
          }
          if (epi == HK_EPI_STORE_T) {
#pragma unroll
            for (int t = 0; t < 4; ++t)
              o[t] = pack_bf16(e.alpha * x[2 * t] + bb[2 * t], e.alpha * x[2 * t + 1] + bb[2 * t + 1]);
          } else if (epi == HK_EPI_ACT_T) {  // G = act(H as it would be stored), H not written
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              const uint32_t hz = pack_bf16(x[2 * t] + bb[2 * t], x[2 * t + 1] + bb[2 * t + 1]);
              const float2 zr = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&hz));
              o[t] = pack_bf16(act_f<true>(e.act, zr.x), act_f<true>(e.act, zr.y));
            }
          } else {  // BIAS_ACT: H = acc + b (bf16) now; G = act(H as stored) after H's store is issued
#pragma unroll
            for (int t = 0; t < 4; ++t) {
              o[t] = pack_bf16(x[2 * t] + bb[2 * t], x[2 * t + 1] + bb[2 * t + 1]);
              hkeep[ESZ == 2 ? 4 * k + t : 0] = o[t];
            }
          }
        }
        sts128(ad, o[0], o[1], o[2], o[3]);
      }
      if (EK == HK_EPI_ACT_BWD && e.colsum != nullptr && row0 < e.M) {
        // gemm_colsum: this box's column sums over its 32 rows, from the staged (stored) bf16 values;
        // lane = a column pair, rows in increasing order
        __syncwarp();
        const int c = n + 2 * lane;
        float s0 = 0.f, s1 = 0.f;
        const uint32_t col_off = (uint32_t)((lane & 3) * 4);
#pragma unroll 8
        for (int rr = 0; rr < 32; ++rr) {
          if (row0 + rr < e.M) {
            uint32_t wv;
            asm volatile("ld.shared.b32 %0, [%1];" : "=r"(wv) : "r"(sb + swz128(rr, lane >> 2) + col_off) : "memory");
            const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&wv));
            s0 += f.x;
            s1 += f.y;
          }
        }
        float* dst = e.colsum + (int64_t)(row0 / 32) * e.N + c;
        if (c + 1 < e.N) *reinterpret_cast<float2*>(dst) = make_float2(s0, s1);
        else if (c < e.N) dst[0] = s0;
      }
    }
    const bool lsu = diag & 16;  // experiment: LSU stores instead of TMA stores
    const int64_t zoff_c = (int64_t)z0 * e.c_sz0 + (int64_t)z1 * e.c_sz1;
    if (lsu) {
      __syncwarp();
      warp_store_box<ESZ>(static_cast<char*>(e.C) + zoff_c * ESZ, e.ldc, sb, row0, n, e.M, e.N, lane);
      fence_proxy_async_smem();  // these generic reads before a later TMA load into the buffer
      __syncwarp();
    } else {
      fence_proxy_async_smem();
      __syncwarp();
    }
    if (!lsu && lane == 0 && !(diag & 4)) {
      if (diag & 8) tma_store_box_hint(mC, sb, n, row0, z0, z1, policy_evict_first());
      else tma_store_box(mC, sb, n, row0, z0, z1);
      bulk_commit();
    }
    if (ESZ == 2 && two) {
      // G = act(H as stored), from the packed H kept in registers; G goes into buffer B once the
      // previous box's G store has left it
      if (lane == 0) bulk_wait_read<1>();
      __syncwarp();
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        uint32_t g[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const float2 zr = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&hkeep[ESZ == 2 ? 4 * k + t : 0]));
          g[t] = pack_bf16(act_f<true>(e.act, zr.x), act_f<true>(e.act, zr.y));
        }
        sts128(w.buf + EPI_BUF + swz128(r, k), g[0], g[1], g[2], g[3]);
      }
      if (lsu) {
        __syncwarp();
        warp_store_box<ESZ>(static_cast<char*>(e.aux_out) + zoff_c * ESZ, e.ldc, w.buf + EPI_BUF, row0, n, e.M, e.N,
                            lane);
        fence_proxy_async_smem();
        __syncwarp();
        ++w.j;
        continue;
      }
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) {
        if (diag & 8) tma_store_box_hint(mO2, w.buf + EPI_BUF, n, row0, z0, z1, policy_evict_first());
        else tma_store_box(mO2, w.buf + EPI_BUF, n, row0, z0, z1);
        bulk_commit();
      }
    }
    ++w.j;
  }
}

template <int BN, int STAGES>
struct TcCfg {
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + EPI_SMEM + 1024 /*align*/ + 256 /*barriers*/;
  static_assert(SMEM <= 232448, "shared memory per CTA");
  static constexpr int ACC_COLS = BN;               // one fp32 accumulator = BN TMEM columns
  static constexpr int TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;  // double-buffered accumulator
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Persistent tile walk shared by the three roles: tile t -> (z, m_blk, n_blk), grouped along M
// (GROUP_M row-blocks share their B column panels in L2).
// HARMONY_GEMM_GROUP_M (default 8): raster width of the persistent tile order, an A/B knob
static int gemm_diag() {
  static const int v = [] {
    const char* e = getenv("HARMONY_GEMM_DIAG");
    return e ? atoi(e) : 0;
  }();
  return v;
}
static int gemm_group_m() {
  static const int g = [] {
    const char* v = getenv("HARMONY_GEMM_GROUP_M");
    const int x = v ? atoi(v) : 8;
    return x >= 1 ? x : 8;
  }();
  return g;
}

struct TileMap {
  int tiles_m, tiles_n, per_z, total, GROUP_M;
  __device__ __forceinline__ void get(int t, int& z, int& mb, int& nb) const {
    z = t / per_z;
    int r = t - z * per_z;
    int group = r / (GROUP_M * tiles_n);
    int first_m = group * GROUP_M;
    int gsize = min(tiles_m - first_m, GROUP_M);
    int local = r - group * GROUP_M * tiles_n;
    mb = first_m + local % gsize;
    nb = local / gsize;
  }
};

template <int BN, int STAGES>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                   const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmIn,
                   const __grid_constant__ CUtensorMap tmO2, TcParams p) {
  using Cfg = TcCfg<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint8_t* sE = smem + STAGES * Cfg::STAGE_BYTES;  // epilogue staging boxes
  uint64_t* ebar = reinterpret_cast<uint64_t*>(sE + EPI_WARPS * 2 * EPI_BUF + EPI_BIAS);
  uint64_t* full = ebar + EPI_WARPS * 2;
  uint64_t* empty = full + STAGES;
  uint64_t* tmem_full = empty + STAGES;   // [2]
  uint64_t* tmem_empty = tmem_full + 2;   // [2]
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(tmem_empty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nkb = (p.K + BK - 1) / BK;
  TileMap tm;
  tm.tiles_m = (p.M + BM - 1) / BM;
  tm.tiles_n = (p.N + BN - 1) / BN;
  tm.per_z = tm.tiles_m * tm.tiles_n;
  tm.total = tm.per_z * p.nz;
  tm.GROUP_M = p.group_m;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tmem_full[a], 1); mbar_init(&tmem_empty[a], 32 * EPI_WARPS); }
    for (int i = 0; i < EPI_WARPS * 2; ++i) mbar_init(&ebar[i], 1);
    if (p.tma_epi) { prefetch_tmap(&tmC); prefetch_tmap(&tmIn); prefetch_tmap(&tmO2); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(Cfg::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer: runs ahead across tiles, bounded by the smem ring =====
      int s = 0;
      uint32_t ph = 0;
      for (int t = blockIdx.x; t < tm.total; t += gridDim.x) {
        int z, mb, nb;
        tm.get(t, z, mb, nb);
        const int z0 = z % p.nz0, z1 = z / p.nz0, m0 = mb * BM, n0 = nb * BN;
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&empty[s], ph ^ 1);
          mbar_expect_tx(&full[s], Cfg::STAGE_BYTES);
          uint8_t* a = sA + s * Cfg::A_BYTES;
          uint8_t* b = sB + s * Cfg::B_BYTES;
          const int k0 = kb * BK;
          if (!p.a_mn) {
            tma_load_4d(a, &tmA, &full[s], k0, m0, z0, z1);
          } else {
#pragma unroll
            for (int j = 0; j < BM / 64; ++j) tma_load_4d(a + j * (BK * 128), &tmA, &full[s], m0 + 64 * j, k0, z0, z1);
          }
          if (!p.b_mn) {
            tma_load_4d(b, &tmB, &full[s], k0, n0, z0, z1);
          } else {
#pragma unroll
            for (int j = 0; j < BN / 64; ++j) tma_load_4d(b + j * (BK * 128), &tmB, &full[s], n0 + 64 * j, k0, z0, z1);
          }
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ===== MMA issuer (single thread), accumulator double-buffered in TMEM =====
      const uint32_t idesc = make_idesc(BN, p.a_mn, p.b_mn);
      int s = 0;
      uint32_t ph = 0;
      int it = 0;
      const uint64_t a_d0 = make_sdesc(smem_u32(sA), p.a_mn ? BK * 128 : 16, 1024);
      const uint64_t b_d0 = make_sdesc(smem_u32(sB), p.b_mn ? BK * 128 : 16, 1024);
      const uint32_t a_kst = p.a_mn ? 2048 >> 4 : 32 >> 4, b_kst = p.b_mn ? 2048 >> 4 : 32 >> 4;
      static_assert(BK / 16 == 4, "four UMMAs per k-block");
      for (int t = blockIdx.x; t < tm.total; t += gridDim.x, ++it) {
        const int acc = it & 1;
        const uint32_t aph = (it >> 1) & 1;
        mbar_wait(&tmem_empty[acc], aph ^ 1);  // epilogue drained this accumulator
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * Cfg::ACC_COLS;
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[s], ph);
          tc_fence_after();
          // K-major: 16 k = 32 bytes along the swizzled row; SBO = 8 rows * 128 B.
          // MN-major: 16 k = 16 rows of 128 B; LBO = next 64-wide MN chunk (BK*128 B), SBO = 8 k-rows.
          const uint64_t ad = a_d0 + (uint64_t)(s * (Cfg::A_BYTES >> 4));
          const uint64_t bd = b_d0 + (uint64_t)(s * (Cfg::B_BYTES >> 4));
          mma4_bf16(tmem_d, ad, bd, a_kst, b_kst, idesc, kb ? 1u : 0u);
          mma_commit(&empty[s]);  // frees the smem stage once these MMAs complete
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
        mma_commit(&tmem_full[acc]);  // accumulator ready for the epilogue
      }
    }
    __syncwarp();
  } else {
    // ===== epilogue warps 2..5: TMEM -> registers -> fused epilogue -> global (overlaps next tile's MMA) =====
    const int q = warp & 3;  // TMEM lane quadrant this warp may access
    const int half = (warp - 2) >> 2;  // which half of the tile's columns this warp drains
    const EpiParams& e = p.e;
    const uint32_t bias_base = smem_u32(sE) + EPI_WARPS * 2 * EPI_BUF;
    EpiWarp ew{smem_u32(sE) + (warp - 2) * 2 * EPI_BUF, bias_base, ebar + (warp - 2) * 2, 0u, 0u};
    const bool out_f32 = e.epi == HK_EPI_STORE_F32 || e.epi == HK_EPI_RESID_F32 || e.epi == HK_EPI_ACC_F32;
    int it = 0;
    for (int t = blockIdx.x; t < tm.total; t += gridDim.x, ++it) {
      int z, mb, nb;
      tm.get(t, z, mb, nb);
      const int z0 = z % p.nz0, z1 = z / p.nz0, m0 = mb * BM, n0 = nb * BN;
      const int acc = it & 1;
      const int64_t zoff = z0 * e.c_sz0 + z1 * e.c_sz1;
      const int ncols = min(BN, p.N - n0);
      const int c_beg = half * (BN / 2), c_end = min(ncols, c_beg + BN / 2);
      const uint32_t tacc = tmem_base + acc * Cfg::ACC_COLS + ((uint32_t)(q * 32) << 16);
      ew.bias = bias_base + (uint32_t)((acc << 1) | half) * EPI_BIAS_SET;
      if (p.tma_epi) {
        if (out_f32)
          tma_epi_tile<4>(p, &tmC, &tmIn, &tmO2, ew, tacc + c_beg, nkb > 0, lane, m0 + q * 32, n0 + c_beg, n0 + c_end,
                          z0, z1, &tmem_full[acc], (it >> 1) & 1);
        else
          tma_epi_tile<2>(p, &tmC, &tmIn, &tmO2, ew, tacc + c_beg, nkb > 0, lane, m0 + q * 32, n0 + c_beg, n0 + c_end,
                          z0, z1, &tmem_full[acc], (it >> 1) & 1);
      } else {
        epi_prefetch(e, m0 + q * 32 + lane, n0 + c_beg, n0 + c_end, zoff);
        mbar_wait(&tmem_full[acc], (it >> 1) & 1);
        tc_fence_after();
#pragma unroll 1
        for (int c = c_beg; c < c_end; c += 32) drain_chunk(e, tacc + c, nkb > 0, lane, m0 + q * 32, n0 + c, zoff);
      }
      tc_fence_before();
      mbar_arrive(&tmem_empty[acc]);
    }
    if (p.tma_epi && lane == 0) bulk_wait_all();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(Cfg::TMEM_COLS)
                 : "memory");
  }
}

// Operand (rows r, K) as a 4-D bf16 map (inner, outer, z0, z1).  K-major: inner = K, box (64, box_r);
// MN-major: inner = r, box (64, BK).
// Epilogue maps (C, input, second output); p.tma_epi = 0 when any is not TMA-addressable or
// HARMONY_GEMM_TMA_EPI=0 (register epilogue).
static void make_epi_maps(const hk_gemm_args& a, const EpiParams& e, int bn, CUtensorMap* mc, CUtensorMap* mi,
                          CUtensorMap* mo, TcParams& p) {
  static const int enabled = [] {
    const char* v = getenv("HARMONY_GEMM_TMA_EPI");
    return v ? atoi(v) : 1;
  }();
  memset(mc, 0, sizeof(CUtensorMap)); memset(mi, 0, sizeof(CUtensorMap)); memset(mo, 0, sizeof(CUtensorMap));
  p.tma_epi = 0;
  const int epi = e.epi;
  const int esz = (epi == HK_EPI_STORE_F32 || epi == HK_EPI_RESID_F32 || epi == HK_EPI_ACC_F32) ? 4 : 2;
  // a warp drains bn/2 columns: at least one 128-byte box of the output type
  if (!enabled || !tma_epi_kind_ok(epi) || (bn / 2) * esz < 128) return;
  auto mk = [&](CUtensorMap* m, const void* ptr, int sz) {
    return make_epi_map(m, ptr, sz, a.N, a.M, e.ldc, a.nz0, e.c_sz0, a.nz1, e.c_sz1);
  };
  bool ok = mk(mc, e.C, esz);
  if (epi == HK_EPI_RESID_F32) ok = ok && mk(mi, e.aux, 4);
  else if (epi == HK_EPI_ACC_F32 && e.accumulate) ok = ok && mk(mi, e.C, 4);
  else if (epi == HK_EPI_ACT_BWD) ok = ok && mk(mi, e.aux, 2);
  if (epi == HK_EPI_BIAS_ACT) ok = ok && mk(mo, e.aux_out, 2);
  p.tma_epi = ok ? 1 : 0;
}

static void make_operand_map(CUtensorMap* map, const void* ptr, int mn_major, int64_t rows, int64_t K, int64_t ld,
                             int64_t nz0, int64_t sz0, int64_t nz1, int64_t sz1, int box_r) {
  const int64_t inner = mn_major ? rows : K, outer = mn_major ? K : rows;
  make_map_4d(map, ptr, inner, outer, nz0, nz1, ld, sz0, sz1, 64, mn_major ? BK : box_r);
}

template <int BN, int STAGES>
static void launch_tc(const hk_gemm_args& a, const EpiParams& e, cudaStream_t st) {
  using Cfg = TcCfg<BN, STAGES>;
  CUtensorMap ma, mb;
  make_operand_map(&ma, a.A, a.a_mn_major, a.M, a.K, a.lda, a.nz0, a.a_sz0, a.nz1, a.a_sz1, BM);
  make_operand_map(&mb, a.B, a.b_mn_major, a.N, a.K, a.ldb, a.nz0, a.b_sz0, a.nz1, a.b_sz1, BN);
  TcParams p;
  p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0; p.nz = a.nz0 * a.nz1; p.a_mn = a.a_mn_major; p.b_mn = a.b_mn_major;
  p.group_m = gemm_group_m();
  p.diag = gemm_diag();
  p.e = e;
  CUtensorMap mc, mi, mo;
  make_epi_maps(a, e, BN, &mc, &mi, &mo, p);
  static bool attr_set = false;  // per instantiation
  if (!attr_set) {
    HM_CUDA(cudaFuncSetAttribute(gemm_tc_kernel<BN, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_set = true;
  }
  static int num_sms = 0;
  if (!num_sms) {
    int dev = 0;
    HM_CUDA(cudaGetDevice(&dev));
    HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int64_t tiles = ceil_div(a.M, BM) * ceil_div(a.N, BN) * (int64_t)a.nz0 * a.nz1;
  dim3 grid((unsigned)std::min<int64_t>(tiles, num_sms));  // persistent: at most one CTA per SM
  // profiling events bracket only the device work (tensor maps are encoded before)
  const int e0 = g_prof.begin(st);
  launch_k(gemm_tc_kernel<BN, STAGES>, dim3(grid), dim3(NUM_THREADS), Cfg::SMEM, st, ma, mb, mc, mi, mo, p);
  check_launch("gemm_tc_kernel");
  g_prof.end(PROF_GEMM, e0, st, 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1);
}


// ============================================================================================ 2-CTA
// cta_group::2: a CTA pair (cluster of 2 on one TPC) computes a 256 x BN tile with M=256 UMMAs.
// Each CTA stages its own 128 rows of A and BN/2 rows of B per k-block (so each SM moves half
// the B bytes of the 1-CTA kernel through L2/smem); the leader CTA issues the MMAs, which read A
// and B from both CTAs' shared memory and write rows 0-127 of the accumulator to the leader's
// TMEM and rows 128-255 to the peer's.  Both CTAs' producers signal the leader's full barrier;
// the leader's commits are multicast to both CTAs' empty / tmem_full barriers; both epilogues
// drain their own TMEM and arrive on the leader's tmem_empty barrier.
__device__ __forceinline__ uint32_t cluster_ctarank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t cluster_id_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
  return r;
}
__device__ __forceinline__ uint32_t nclusters_x() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__device__ __forceinline__ uint32_t to_leader(uint32_t smem_addr) { return smem_addr & 0xFEFFFFFFu; }
__device__ __forceinline__ void tma_load_4d_2sm(void* dst, const CUtensorMap* map, uint32_t leader_bar, int c0, int c1,
                                                int c2, int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, "
      "%6}], [%2];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(leader_bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void mbar_arrive_cluster(uint32_t cluster_addr) {
  // default (.release, .cta scope) semantics: no cluster-scope fence per arrive (the TMA bytes are
  // tracked by complete_tx; TMEM reads are ordered by tcgen05.fence::before_thread_sync)
  asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ uint32_t mapa_leader(const void* local) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, 0;" : "=r"(r) : "r"(smem_u32(local)));
  return r;
}
__device__ __forceinline__ void mma_bf16_2sm(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                             uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}
// the four K=16 UMMAs of one 64-deep k-block in one asm block (one operand hand-off to the
// uniform datapath instead of four); the first accumulates only if acc != 0, the rest always
__device__ __forceinline__ void mma4_bf16_2sm(uint32_t tmem_d, uint64_t ad, uint64_t bd, uint32_t a_kst, uint32_t b_kst,
                                              uint32_t idesc, uint32_t acc) {
  const uint64_t a1 = ad + a_kst, a2 = ad + 2 * a_kst, a3 = ad + 3 * a_kst;
  const uint64_t b1 = bd + b_kst, b2 = bd + 2 * b_kst, b3 = bd + 3 * b_kst;
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t"
      "setp.ne.b32 p, %10, 0;\n\t"
      "setp.eq.b32 q, %0, %0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %9, p;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %3, %4, %9, q;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %5, %6, %9, q;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %7, %8, %9, q;\n\t}" ::"r"(tmem_d),
      "l"(ad), "l"(bd), "l"(a1), "l"(b1), "l"(a2), "l"(b2), "l"(a3), "l"(b3), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit_2sm_mc(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}

template <int BN, int STAGES>
struct Tc2Cfg {
  static constexpr int HB = BN / 2;            // B rows staged per CTA
  static constexpr int A_BYTES = 128 * BK * 2; // 16 KB
  static constexpr int B_BYTES = HB * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  // no alignment slack: dynamic shared memory starts right after the 1 KB the system reserves, i.e.
  // 1024-aligned (checked in the kernel, which traps otherwise)
  static constexpr int SMEM = STAGES * STAGE_BYTES + EPI_SMEM + 256;
  static_assert(SMEM <= 232448, "shared memory per CTA");
  static constexpr int TMEM_COLS = 2 * BN;     // double-buffered accumulator (BN fp32 columns each)
};

// EK: the epilogue kind compiled in (>= 0: that kind through the TMA-store epilogue only, a kernel a
// fraction of the generic one's size — the generic body, every kind plus the register epilogue and
// the diagnostics, overflowed the instruction cache: its epilogue warps stalled on instruction
// fetch); -1: the generic kernel
template <int BN, int STAGES, int EK = -1>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                    const __grid_constant__ CUtensorMap tmC, const __grid_constant__ CUtensorMap tmIn,
                    const __grid_constant__ CUtensorMap tmO2, TcParams p) {
  using Cfg = Tc2Cfg<BN, STAGES>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  if (smem_u32(smem_raw) & 1023) __trap();  // the layout below assumes a 1024-aligned base (128B-swizzle atoms)
  uint8_t* smem = smem_raw;
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint8_t* sE = smem + STAGES * Cfg::STAGE_BYTES;  // epilogue staging boxes
  uint64_t* ebar = reinterpret_cast<uint64_t*>(sE + EPI_WARPS * 2 * EPI_BUF + EPI_BIAS);
  uint64_t* full = ebar + EPI_WARPS * 2;
  uint64_t* empty = full + STAGES;
  uint64_t* tmem_full = empty + STAGES;  // [2]
  uint64_t* tmem_empty = tmem_full + 2;  // [2] (used in the leader)
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(tmem_empty + 2);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;
  const int nkb = (p.K + BK - 1) / BK;
  TileMap tm;
  tm.tiles_m = (p.M + 255) / 256;
  tm.tiles_n = (p.N + BN - 1) / BN;
  tm.per_z = tm.tiles_m * tm.tiles_n;
  tm.total = tm.per_z * p.nz;
  tm.GROUP_M = p.group_m;
  const int pair = (int)cluster_id_x(), npairs = (int)nclusters_x();

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 2); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tmem_full[a], 1); mbar_init(&tmem_empty[a], 2 * 32 * EPI_WARPS); }
    for (int i = 0; i < EPI_WARPS * 2; ++i) mbar_init(&ebar[i], 1);
    if (EK >= 0 || p.tma_epi) { prefetch_tmap(&tmC); prefetch_tmap(&tmIn); prefetch_tmap(&tmO2); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(Cfg::TMEM_COLS)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  cluster_sync_all();  // barriers of both CTAs initialised, TMEM allocated in both
  tc_fence_after();
  const uint32_t tmem_base = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer (both CTAs): own half of A and B, completion on the leader's barrier =====
      int s = 0;
      uint32_t ph = 0;
      for (int t = pair; t < tm.total; t += npairs) {
        int z, mb, nb;
        tm.get(t, z, mb, nb);
        const int z0 = z % p.nz0, z1 = z / p.nz0;
        const int m0 = mb * 256 + (int)rank * 128, n0 = nb * BN + (int)rank * Cfg::HB;
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&empty[s], ph ^ 1);
          const uint32_t fb = to_leader(smem_u32(&full[s]));
          if (leader) mbar_expect_tx(&full[s], 2 * Cfg::STAGE_BYTES);
          else mbar_arrive_cluster(fb);
          uint8_t* a = sA + s * Cfg::A_BYTES;
          uint8_t* b = sB + s * Cfg::B_BYTES;
          const int k0 = kb * BK;
          if (!p.a_mn) {
            tma_load_4d_2sm(a, &tmA, fb, k0, m0, z0, z1);
          } else {
#pragma unroll
            for (int j = 0; j < 2; ++j) tma_load_4d_2sm(a + j * (BK * 128), &tmA, fb, m0 + 64 * j, k0, z0, z1);
          }
          if (!p.b_mn) {
            tma_load_4d_2sm(b, &tmB, fb, k0, n0, z0, z1);
          } else {
#pragma unroll
            for (int j = 0; j < Cfg::HB / 64; ++j) tma_load_4d_2sm(b + j * (BK * 128), &tmB, fb, n0 + 64 * j, k0, z0, z1);
          }
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (leader && lane == 0) {
      // ===== MMA issuer (leader CTA, single thread): M=256 x N=BN UMMAs over the pair =====
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)p.a_mn << 15) |
                             ((uint32_t)p.b_mn << 16) | ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(256 >> 4) << 24);
      // descriptors built once: stage s, sub-step kk is base + s * stage stride + kk * k-step in the
      // 14-bit start-address field (shared addresses < 2^18, so the adds never carry out of it)
      const uint64_t a_d0 = make_sdesc(smem_u32(sA), p.a_mn ? BK * 128 : 16, 1024);
      const uint64_t b_d0 = make_sdesc(smem_u32(sB), p.b_mn ? BK * 128 : 16, 1024);
      const uint32_t a_kst = p.a_mn ? 2048 >> 4 : 32 >> 4, b_kst = p.b_mn ? 2048 >> 4 : 32 >> 4;
      static_assert(BK / 16 == 4, "four UMMAs per k-block");
      int s = 0;
      uint32_t ph = 0;
      int it = 0;
      for (int t = pair; t < tm.total; t += npairs, ++it) {
        const int acc = it & 1;
        mbar_wait(&tmem_empty[acc], ((it >> 1) & 1) ^ 1);
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * BN;
        for (int kb = 0; kb < nkb; ++kb) {
          mbar_wait(&full[s], ph);
          tc_fence_after();
          const uint64_t ad = a_d0 + (uint64_t)(s * (Cfg::A_BYTES >> 4));
          const uint64_t bd = b_d0 + (uint64_t)(s * (Cfg::B_BYTES >> 4));
          mma4_bf16_2sm(tmem_d, ad, bd, a_kst, b_kst, idesc, kb ? 1u : 0u);
          mma_commit_2sm_mc(&empty[s]);  // frees this stage in both CTAs
          if (++s == STAGES) { s = 0; ph ^= 1; }
        }
        mma_commit_2sm_mc(&tmem_full[acc]);  // both CTAs' accumulator halves ready
      }
    }
    __syncwarp();
  } else {
    // ===== epilogue warps 2..5 of each CTA: its 128 accumulator rows =====
    const int q = warp & 3;
    const int half = (warp - 2) >> 2;
    const EpiParams& e = p.e;
    const uint32_t te = mapa_leader(&tmem_empty[0]);
    const uint32_t bias_base = smem_u32(sE) + EPI_WARPS * 2 * EPI_BUF;
    EpiWarp ew{smem_u32(sE) + (warp - 2) * 2 * EPI_BUF, bias_base, ebar + (warp - 2) * 2, 0u, 0u};
    const int epi = EK >= 0 ? EK : e.epi;
    const bool tma_epi = EK >= 0 || p.tma_epi;
    const bool out_f32 = epi == HK_EPI_STORE_F32 || epi == HK_EPI_RESID_F32 || epi == HK_EPI_ACC_F32;
    int it = 0;
    for (int t = pair; t < tm.total; t += npairs, ++it) {
      int z, mb, nb;
      tm.get(t, z, mb, nb);
      const int z0 = z % p.nz0, z1 = z / p.nz0, n0 = nb * BN;
      const int acc = it & 1;
      const int64_t zoff = z0 * e.c_sz0 + z1 * e.c_sz1;
      const int ncols = min(BN, p.N - n0);
      const int c_beg = half * (BN / 2), c_end = min(ncols, c_beg + BN / 2);
      const int row0 = mb * 256 + (int)rank * 128 + q * 32;
      const uint32_t tacc = tmem_base + acc * BN + ((uint32_t)(q * 32) << 16);
      ew.bias = bias_base + (uint32_t)((acc << 1) | half) * EPI_BIAS_SET;
      if (EK < 0 && (p.diag & 1)) {
        mbar_wait(&tmem_full[acc], (it >> 1) & 1);
        tc_fence_after();
      } else if (tma_epi) {
        if (out_f32)
          tma_epi_tile<4, EK>(p, &tmC, &tmIn, &tmO2, ew, tacc + c_beg, nkb > 0, lane, row0, n0 + c_beg, n0 + c_end, z0,
                              z1, &tmem_full[acc], (it >> 1) & 1);
        else
          tma_epi_tile<2, EK>(p, &tmC, &tmIn, &tmO2, ew, tacc + c_beg, nkb > 0, lane, row0, n0 + c_beg, n0 + c_end, z0,
                              z1, &tmem_full[acc], (it >> 1) & 1);
      } else if (EK < 0) {
        epi_prefetch(e, row0 + lane, n0 + c_beg, n0 + c_end, zoff);
        mbar_wait(&tmem_full[acc], (it >> 1) & 1);
        tc_fence_after();
#pragma unroll 1
        for (int c = c_beg; c < c_end; c += 32) drain_chunk(e, tacc + c, nkb > 0, lane, row0, n0 + c, zoff);
      }
      tc_fence_before();
      mbar_arrive_cluster(te + acc * 8);
    }
    if (tma_epi && lane == 0) bulk_wait_all();
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(Cfg::TMEM_COLS)
                 : "memory");
  }
}

template <int BN, int STAGES, int EK>
static void launch_tc2_k(const CUtensorMap& ma, const CUtensorMap& mb, const CUtensorMap& mc, const CUtensorMap& mi,
                         const CUtensorMap& mo, const TcParams& p, dim3 grid, cudaStream_t st) {
  using Cfg = Tc2Cfg<BN, STAGES>;
  static bool attr_set = false;
  if (!attr_set) {
    HM_CUDA(cudaFuncSetAttribute(gemm_tc2_kernel<BN, STAGES, EK>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 Cfg::SMEM));
    attr_set = true;
  }
  launch_k(gemm_tc2_kernel<BN, STAGES, EK>, dim3(grid), dim3(NUM_THREADS), Cfg::SMEM, st, ma, mb, mc, mi, mo, p);
}

// HARMONY_GEMM_SPECIALIZE=0: always the generic kernel (A/B of the per-kind specialisation)
static bool gemm_specialize() {
  static const bool v = [] {
    const char* e = getenv("HARMONY_GEMM_SPECIALIZE");
    return !(e && *e == '0');
  }();
  return v;
}

template <int BN, int STAGES>
static bool launch_tc2(const hk_gemm_args& a, const EpiParams& e, cudaStream_t st) {
  using Cfg = Tc2Cfg<BN, STAGES>;
  CUtensorMap ma, mb;
  make_operand_map(&ma, a.A, a.a_mn_major, a.M, a.K, a.lda, a.nz0, a.a_sz0, a.nz1, a.a_sz1, 128);
  make_operand_map(&mb, a.B, a.b_mn_major, a.N, a.K, a.ldb, a.nz0, a.b_sz0, a.nz1, a.b_sz1, Cfg::HB);
  TcParams p;
  p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0; p.nz = a.nz0 * a.nz1; p.a_mn = a.a_mn_major; p.b_mn = a.b_mn_major;
  p.group_m = gemm_group_m();
  p.diag = gemm_diag();
  p.e = e;
  CUtensorMap mc, mi, mo;
  make_epi_maps(a, e, BN, &mc, &mi, &mo, p);
  static int num_sms = 0;
  if (!num_sms) {
    int dev = 0;
    HM_CUDA(cudaGetDevice(&dev));
    HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int64_t tiles = ceil_div(a.M, 256) * ceil_div(a.N, BN) * (int64_t)a.nz0 * a.nz1;
  dim3 grid((unsigned)(2 * std::min<int64_t>(tiles, num_sms / 2)));  // persistent pairs
  const int e0 = g_prof.begin(st);
  // the per-kind kernels for the TMA-store epilogue (same code path as the generic one for that kind,
  // so the results are bit-identical); the generic kernel for the register epilogue and diagnostics
  const bool spec = BN == 256 && p.tma_epi && p.diag == 0 && gemm_specialize();
  // the ACT_BWD kernel sums its output boxes for gemm_colsum (plain products, 8-column-aligned rows)
  const bool fused_colsum = spec && e.epi == HK_EPI_ACT_BWD && e.colsum != nullptr && p.nz == 1 && a.N % 2 == 0 &&
                            (reinterpret_cast<uintptr_t>(e.colsum) & 7) == 0;
  if (!fused_colsum) p.e.colsum = nullptr;
  if constexpr (BN != 256) {
    launch_tc2_k<BN, STAGES, -1>(ma, mb, mc, mi, mo, p, grid, st);
  } else switch (spec ? e.epi : -1) {
    case HK_EPI_STORE_T: launch_tc2_k<BN, STAGES, HK_EPI_STORE_T>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_STORE_F32: launch_tc2_k<BN, STAGES, HK_EPI_STORE_F32>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_RESID_F32: launch_tc2_k<BN, STAGES, HK_EPI_RESID_F32>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_ACC_F32: launch_tc2_k<BN, STAGES, HK_EPI_ACC_F32>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_BIAS_ACT: launch_tc2_k<BN, STAGES, HK_EPI_BIAS_ACT>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_ACT_BWD: launch_tc2_k<BN, STAGES, HK_EPI_ACT_BWD>(ma, mb, mc, mi, mo, p, grid, st); break;
    case HK_EPI_ACT_T: launch_tc2_k<BN, STAGES, HK_EPI_ACT_T>(ma, mb, mc, mi, mo, p, grid, st); break;
    default: launch_tc2_k<BN, STAGES, -1>(ma, mb, mc, mi, mo, p, grid, st); break;
  }
  check_launch("gemm_tc2_kernel");
  g_prof.end(PROF_GEMM, e0, st, 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1);
  return fused_colsum;
}

}  // namespace tc

// returns true when the GEMM itself produced the gemm_colsum partials
static bool gemm_impl(const hk_gemm_args& a, float* colsum, cudaStream_t st) {
  HM_CHECK(a.M >= 0 && a.N >= 0 && a.K >= 0 && a.nz0 >= 1 && a.nz1 >= 1, HARMONY_E_INVALID_ARG, "gemm: bad shape");
  if (a.M == 0 || a.N == 0) return false;
  EpiParams e;
  e.C = a.C; e.ldc = a.ldc; e.c_sz0 = a.c_sz0; e.c_sz1 = a.c_sz1;
  e.epi = a.epilogue; e.act = a.act; e.accumulate = a.accumulate; e.alpha = a.alpha;
  e.bias = a.bias; e.aux = a.aux; e.aux_out = a.aux_out; e.M = a.M; e.N = a.N;
  e.colsum = colsum;
  HM_CHECK(a.accumulate != 2 || (a.dtype == 0 && a.epilogue == HK_EPI_ACC_F32 && a.alpha == 1.f),
           HARMONY_E_UNSUPPORTED, "gemm: accumulate = 2 (continue C's reduction) is the fp32 ACC_F32 path only");
  if (a.dtype == 0) {
    const int e0 = g_prof.begin(st);
    const double flops = 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1;
    SimtParams p;
    p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0;
    p.A = static_cast<const float*>(a.A); p.a_mn = a.a_mn_major; p.lda = a.lda; p.a_sz0 = a.a_sz0; p.a_sz1 = a.a_sz1;
    p.B = static_cast<const float*>(a.B); p.b_mn = a.b_mn_major; p.ldb = a.ldb; p.b_sz0 = a.b_sz0; p.b_sz1 = a.b_sz1;
    p.e = e;
    dim3 grid((unsigned)ceil_div(a.N, SBN), (unsigned)ceil_div(a.M, SBM), (unsigned)(a.nz0 * a.nz1));
    launch_k(gemm_simt_kernel, dim3(grid), dim3(256), 0, st, p);
    check_launch("gemm_simt_kernel");
    g_prof.end(PROF_GEMM, e0, st, flops);
    return false;
  }
  // Tile shape from the problem shape only (never from the memory cap): bit-exact capped == uncapped.
  static const int mode = [] {
    const char* v = getenv("HARMONY_GEMM_2SM");
    return v ? atoi(v) : 1;
  }();
  const int64_t nz = (int64_t)a.nz0 * a.nz1;
  // CTA-pair tiles unless they would leave most pairs idle (e.g. the d x d weight gradient: 16 pair
  // tiles on 74 pairs) — then 128 x 128 single-CTA tiles spread the work over 4x more SMs
  const int64_t pair_tiles = ceil_div(a.M, 256) * ceil_div(a.N, 256) * nz;
  if (mode && a.M >= 256 && a.N >= 256 && pair_tiles >= 37) {
    // CTA-pair 256 x 256 tiles (measured best for every cfg2 shape, tools/gemm_bench.py);
    // HARMONY_GEMM_2SM=3 selects 256 x 128 pair tiles, 0 the single-CTA kernel
    // five 32 KB stages for plain products, four for batched ones (split-K weight gradients:
    // measured 2-6% faster / 4% slower, profiles/r02_gemm_stages_cfg2.txt); HARMONY_GEMM_STAGES
    // forces one (the stage count only paces the loads: results are bitwise the same)
    static const int force = [] {
      const char* v = getenv("HARMONY_GEMM_STAGES");
      return v ? atoi(v) : 0;
    }();
    const int stages = force ? force : (nz == 1 ? 5 : 4);
    if (mode == 3) return tc::launch_tc2<128, 6>(a, e, st);
    if (stages == 5) return tc::launch_tc2<256, 5>(a, e, st);
    return tc::launch_tc2<256, 4>(a, e, st);
  }
  e.colsum = nullptr;
  if (a.N <= 64)
    tc::launch_tc<64, 6>(a, e, st);
  else if (a.N <= 128 || (int64_t)ceil_div(a.M, 128) * ceil_div(a.N, 256) * nz < 148)
    tc::launch_tc<128, 4>(a, e, st);
  else
    tc::launch_tc<256, 3>(a, e, st);
  return false;
}

void gemm(const hk_gemm_args& a, cudaStream_t st) { gemm_impl(a, nullptr, st); }

void gemm_colsum(const hk_gemm_args& a, float* partial, cudaStream_t st) {
  HM_CHECK(a.dtype == 1 && a.nz0 == 1 && a.nz1 == 1 && partial != nullptr, HARMONY_E_INVALID_ARG,
           "gemm_colsum: a plain bf16 product and a partial buffer");
  if (!gemm_impl(a, partial, st)) colsum32_partial(a.M, a.N, a.C, a.ldc, partial, st);
}

}  // namespace hm
