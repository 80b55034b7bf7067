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
  __shared__ float As[SBK][SBM + 4];
  __shared__ float Bs[SBK][SBN + 4];
  const int tid = threadIdx.x;
  const int z = blockIdx.z, z0 = z % p.nz0, z1 = z / p.nz0;
  const int m0 = blockIdx.y * SBM, n0 = blockIdx.x * SBN;
  const float* A = p.A + z0 * p.a_sz0 + z1 * p.a_sz1;
  const float* B = p.B + z0 * p.b_sz0 + z1 * p.b_sz1;
  const int tx = tid % 16, ty = tid / 16;
  float acc[4][4] = {};
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
      epi_scalar<float>(e, off, n, acc[i][j]);
    }
  }
}

// ----------------------------------------------------------------------------------------- tcgen05
namespace tc {

constexpr int BM = 128;
constexpr int BK = 64;                 // 64 bf16 = 128 bytes = one 128B swizzle row
constexpr int NUM_THREADS = 192;       // warp 0: TMA, warp 1: MMA + TMEM alloc, warps 2-5: epilogue

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t addr, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(addr), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t a = smem_u32(bar);
  while (!mbar_try_wait(a, parity)) {
  }
}
__device__ __forceinline__ void tma_load_4d(void* dst, const CUtensorMap* map, uint64_t* bar, int c0, int c1, int c2,
                                            int c3) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5, %6}], [%2];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(smem_u32(bar)), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
      : "memory");
}
__device__ __forceinline__ void prefetch_tmap(const CUtensorMap* map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
// UMMA shared-memory descriptor (sm_100): start>>4 [0,14), LBO>>4 [16,30), SBO>>4 [32,46),
// version 1 [46,48), base offset 0, layout type SWIZZLE_128B = 2 at [61,64).
__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) |
         ((uint64_t)((sbo >> 4) & 0x3FFFu) << 32) | (1ull << 46) | (2ull << 61);
}
// Instruction descriptor, kind::f16: D=F32 [4,6)=1, A=BF16 [7,10)=1, B=BF16 [10,13)=1,
// a_major bit 15, b_major bit 16 (1 = MN-major), N>>3 at [17,23), M>>4 at [24,29).
__device__ __forceinline__ uint32_t make_idesc(int bn, int a_mn, int b_mn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)a_mn << 15) | ((uint32_t)b_mn << 16) |
         ((uint32_t)(bn >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}
__device__ __forceinline__ void mma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float* v) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

struct TcParams {
  int M, N, K, nz0, a_mn, b_mn;
  EpiParams e;
};

template <int BN, int STAGES>
struct TcCfg {
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
  static constexpr int TMEM_COLS = BN < 32 ? 32 : BN;
};

template <int BN, int STAGES>
__global__ void __launch_bounds__(NUM_THREADS, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, TcParams p) {
  using Cfg = TcCfg<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES);
  uint64_t* empty = full + STAGES;
  uint64_t* tmem_full = empty + STAGES;
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(tmem_full + 1);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int n0 = blockIdx.x * BN, m0 = blockIdx.y * BM;
  const int z0 = blockIdx.z % p.nz0, z1 = blockIdx.z / p.nz0;
  const int nkb = (p.K + BK - 1) / BK;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    mbar_init(tmem_full, 1);
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
  const uint32_t tmem_acc = *tmem_base_s;

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer =====
      int s = 0;
      uint32_t ph = 0;
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
  } else if (warp == 1) {
    if (lane == 0) {
      // ===== MMA issuer (single thread) =====
      const uint32_t idesc = make_idesc(BN, p.a_mn, p.b_mn);
      int s = 0;
      uint32_t ph = 0;
      for (int kb = 0; kb < nkb; ++kb) {
        mbar_wait(&full[s], ph);
        tc_fence_after();
        const uint32_t a = smem_u32(sA + s * Cfg::A_BYTES);
        const uint32_t b = smem_u32(sB + s * Cfg::B_BYTES);
#pragma unroll
        for (int kk = 0; kk < BK / 16; ++kk) {
          // K-major: 16 k = 32 bytes along the swizzled row; SBO = 8 rows * 128 B.
          // MN-major: 16 k = 16 rows of 128 B; LBO = next 64-wide MN chunk (BK*128 B), SBO = 8 k-rows.
          uint64_t ad = p.a_mn ? make_sdesc(a + kk * 2048, BK * 128, 1024) : make_sdesc(a + kk * 32, 16, 1024);
          uint64_t bd = p.b_mn ? make_sdesc(b + kk * 2048, BK * 128, 1024) : make_sdesc(b + kk * 32, 16, 1024);
          mma_bf16(tmem_acc, ad, bd, idesc, (kb | kk) ? 1u : 0u);
        }
        mma_commit(&empty[s]);  // frees the smem stage once these MMAs complete
        if (++s == STAGES) { s = 0; ph ^= 1; }
      }
      mma_commit(tmem_full);  // accumulator ready
    }
    __syncwarp();
  } else {
    // ===== epilogue warps 2..5: TMEM -> registers -> fused epilogue -> global =====
    const int q = warp & 3;  // TMEM lane quadrant this warp may access
    if (nkb > 0) {
      mbar_wait(tmem_full, 0);
      tc_fence_after();
    }
    const int m = m0 + q * 32 + lane;
    const EpiParams& e = p.e;
    const int64_t row_off = z0 * e.c_sz0 + z1 * e.c_sz1 + (int64_t)m * e.ldc;
#pragma unroll 1
    for (int c = 0; c < BN; c += 16) {
      float v[16];
      if (nkb > 0) {
        tmem_ld16(tmem_acc + ((uint32_t)(q * 32) << 16) + c, v);
      } else {
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] = 0.f;
      }
      if (m < p.M && n0 + c < p.N) epi_row16<__nv_bfloat16>(e, row_off, n0 + c, v);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem_acc), "r"(Cfg::TMEM_COLS)
                 : "memory");
  }
}

// ----- host: tensor maps through the driver entry point (no link-time libcuda dependency)
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

// Operand (rows r, K) as a 4-D bf16 map (inner, outer, z0, z1).  K-major: inner = K, box (64, box_r);
// MN-major: inner = r, box (64, BK).
static void make_operand_map(CUtensorMap* map, const void* ptr, int mn_major, int64_t rows, int64_t K, int64_t ld,
                             int64_t nz0, int64_t sz0, int64_t nz1, int64_t sz1, int box_r) {
  auto enc = get_encode();
  HM_CHECK(enc != nullptr, HARMONY_E_CUDA, "cuTensorMapEncodeTiled unavailable (driver too old?)");
  HM_CHECK((reinterpret_cast<uintptr_t>(ptr) & 15) == 0, HARMONY_E_UNSUPPORTED, "bf16 GEMM operand not 16-byte aligned");
  HM_CHECK(ld % 8 == 0, HARMONY_E_UNSUPPORTED, "bf16 GEMM leading dimension must be a multiple of 8");
  cuuint64_t dims[4];
  cuuint64_t strides[3];
  cuuint32_t box[4];
  cuuint32_t estr[4] = {1, 1, 1, 1};
  int64_t inner = mn_major ? rows : K, outer = mn_major ? K : rows;
  dims[0] = (cuuint64_t)inner;
  dims[1] = (cuuint64_t)outer;
  dims[2] = (cuuint64_t)nz0;
  dims[3] = (cuuint64_t)nz1;
  strides[0] = (cuuint64_t)ld * 2;
  int64_t s1 = nz0 > 1 ? sz0 * 2 : (int64_t)align_up((uint64_t)(ld * outer * 2), 16);
  int64_t s2 = nz1 > 1 ? sz1 * 2 : (int64_t)align_up((uint64_t)(s1 * nz0), 16);
  HM_CHECK(s1 % 16 == 0 && s2 % 16 == 0, HARMONY_E_UNSUPPORTED, "bf16 GEMM batch strides must be multiples of 8");
  strides[1] = (cuuint64_t)s1;
  strides[2] = (cuuint64_t)s2;
  box[0] = 64;
  box[1] = mn_major ? BK : box_r;
  box[2] = 1;
  box[3] = 1;
  CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(ptr), dims, strides, box, estr,
                   CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                   CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  HM_CHECK(r == CUDA_SUCCESS, HARMONY_E_CUDA, "cuTensorMapEncodeTiled failed: " + std::to_string((int)r));
}

template <int BN, int STAGES>
static void launch_tc(const hk_gemm_args& a, const EpiParams& e, cudaStream_t st) {
  using Cfg = TcCfg<BN, STAGES>;
  CUtensorMap ma, mb;
  make_operand_map(&ma, a.A, a.a_mn_major, a.M, a.K, a.lda, a.nz0, a.a_sz0, a.nz1, a.a_sz1, BM);
  make_operand_map(&mb, a.B, a.b_mn_major, a.N, a.K, a.ldb, a.nz0, a.b_sz0, a.nz1, a.b_sz1, BN);
  TcParams p;
  p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0; p.a_mn = a.a_mn_major; p.b_mn = a.b_mn_major; p.e = e;
  static bool attr_set = false;  // per instantiation
  if (!attr_set) {
    HM_CUDA(cudaFuncSetAttribute(gemm_tc_kernel<BN, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_set = true;
  }
  dim3 grid((unsigned)ceil_div(a.N, BN), (unsigned)ceil_div(a.M, BM), (unsigned)(a.nz0 * a.nz1));
  gemm_tc_kernel<BN, STAGES><<<grid, NUM_THREADS, Cfg::SMEM, st>>>(ma, mb, p);
  check_launch("gemm_tc_kernel");
}

}  // namespace tc

void gemm(const hk_gemm_args& a, cudaStream_t st) {
  HM_CHECK(a.M >= 0 && a.N >= 0 && a.K >= 0 && a.nz0 >= 1 && a.nz1 >= 1, HARMONY_E_INVALID_ARG, "gemm: bad shape");
  if (a.M == 0 || a.N == 0) return;
  EpiParams e;
  e.C = a.C; e.ldc = a.ldc; e.c_sz0 = a.c_sz0; e.c_sz1 = a.c_sz1;
  e.epi = a.epilogue; e.act = a.act; e.accumulate = a.accumulate; e.alpha = a.alpha;
  e.bias = a.bias; e.aux = a.aux; e.aux_out = a.aux_out; e.M = a.M; e.N = a.N;
  const int e0 = g_prof.begin(st);
  const double flops = 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1;
  if (a.dtype == 0) {
    SimtParams p;
    p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0;
    p.A = static_cast<const float*>(a.A); p.a_mn = a.a_mn_major; p.lda = a.lda; p.a_sz0 = a.a_sz0; p.a_sz1 = a.a_sz1;
    p.B = static_cast<const float*>(a.B); p.b_mn = a.b_mn_major; p.ldb = a.ldb; p.b_sz0 = a.b_sz0; p.b_sz1 = a.b_sz1;
    p.e = e;
    dim3 grid((unsigned)ceil_div(a.N, SBN), (unsigned)ceil_div(a.M, SBM), (unsigned)(a.nz0 * a.nz1));
    gemm_simt_kernel<<<grid, 256, 0, st>>>(p);
    check_launch("gemm_simt_kernel");
    g_prof.end(PROF_GEMM, e0, st, flops);
    return;
  }
  // Tile width from the shape only (never from the memory cap): bit-exact capped == uncapped.
  if (a.N <= 64)
    tc::launch_tc<64, 8>(a, e, st);
  else if (a.N <= 128 || (int64_t)ceil_div(a.M, 128) * ceil_div(a.N, 256) * a.nz0 * a.nz1 < 148)
    tc::launch_tc<128, 6>(a, e, st);
  else
    tc::launch_tc<256, 4>(a, e, st);
  g_prof.end(PROF_GEMM, e0, st, flops);
}

}  // namespace hm
