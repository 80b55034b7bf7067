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
constexpr int EPI_WARPS = 8;           // two epilogue warps per TMEM lane quadrant (column halves)
constexpr int NUM_THREADS = 64 + 32 * EPI_WARPS;  // warp 0: TMA, warp 1: MMA + TMEM alloc, warps 2..9: epilogue

using namespace tcx;

__device__ __forceinline__ uint32_t make_idesc(int bn, int a_mn, int b_mn) { return make_idesc_f16(BM, bn, a_mn, b_mn); }

// one epilogue warp's 32-column chunk: TMEM (thread = row) -> registers -> fused epilogue -> global in
// 32-byte row pieces (full sectors).  A variant that transposed chunks through shared memory for
// 128-byte row segments measured 6% slower in the step (profiles/r01_epilogue_ab.txt) and was dropped.
__device__ __forceinline__ void drain_chunk(const EpiParams& e, uint32_t taddr, bool have_acc, int lane, int mrow0,
                                            int n, int64_t zoff) {
  float v[32];
  if (have_acc) {
    tmem_ld16(taddr, v);
    tmem_ld16(taddr + 16, v + 16);
  } else {
#pragma unroll
    for (int i = 0; i < 32; ++i) v[i] = 0.f;
  }
  const int m = mrow0 + lane;
  if (m < e.M) {
    epi_row16<__nv_bfloat16>(e, zoff + (int64_t)m * e.ldc, n, v);
    if (n + 16 < e.N) epi_row16<__nv_bfloat16>(e, zoff + (int64_t)m * e.ldc, n + 16, v + 16);
  }
}

struct TcParams {
  int M, N, K, nz0, nz, a_mn, b_mn;
  EpiParams e;
};

template <int BN, int STAGES>
struct TcCfg {
  static constexpr int A_BYTES = BM * BK * 2;  // 16 KB
  static constexpr int B_BYTES = BN * BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 /*align*/ + 256 /*barriers*/;
  static constexpr int ACC_COLS = BN;               // one fp32 accumulator = BN TMEM columns
  static constexpr int TMEM_COLS = 2 * BN < 32 ? 32 : 2 * BN;  // double-buffered accumulator
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// Persistent tile walk shared by the three roles: tile t -> (z, m_blk, n_blk), grouped along M
// (GROUP_M row-blocks share their B column panels in L2).
struct TileMap {
  int tiles_m, tiles_n, per_z, total;
  __device__ __forceinline__ void get(int t, int& z, int& mb, int& nb) const {
    constexpr int GROUP_M = 8;
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
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, TcParams p) {
  using Cfg = TcCfg<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES);
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

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tmem_full[a], 1); mbar_init(&tmem_empty[a], 32 * EPI_WARPS); }
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
      for (int t = blockIdx.x; t < tm.total; t += gridDim.x, ++it) {
        const int acc = it & 1;
        const uint32_t aph = (it >> 1) & 1;
        mbar_wait(&tmem_empty[acc], aph ^ 1);  // epilogue drained this accumulator
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * Cfg::ACC_COLS;
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
            mma_bf16(tmem_d, ad, bd, idesc, (kb | kk) ? 1u : 0u);
          }
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
    int it = 0;
    for (int t = blockIdx.x; t < tm.total; t += gridDim.x, ++it) {
      int z, mb, nb;
      tm.get(t, z, mb, nb);
      const int z0 = z % p.nz0, z1 = z / p.nz0, m0 = mb * BM, n0 = nb * BN;
      const int acc = it & 1;
      mbar_wait(&tmem_full[acc], (it >> 1) & 1);
      tc_fence_after();
      const int64_t zoff = z0 * e.c_sz0 + z1 * e.c_sz1;
      const uint32_t tacc = tmem_base + acc * Cfg::ACC_COLS + ((uint32_t)(q * 32) << 16);
      const int ncols = min(BN, p.N - n0);
      const int c_beg = half * (BN / 2), c_end = min(ncols, c_beg + BN / 2);
#pragma unroll 1
      for (int c = c_beg; c < c_end; c += 32) drain_chunk(e, tacc + c, nkb > 0, lane, m0 + q * 32, n0 + c, zoff);
      tc_fence_before();
      mbar_arrive(&tmem_empty[acc]);
    }
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
  p.e = e;
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
  gemm_tc_kernel<BN, STAGES><<<grid, NUM_THREADS, Cfg::SMEM, st>>>(ma, mb, p);
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
  static constexpr int SMEM = STAGES * STAGE_BYTES + 1024 + 256;
  static constexpr int TMEM_COLS = 2 * BN;     // double-buffered accumulator (BN fp32 columns each)
};

template <int BN, int STAGES>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(NUM_THREADS, 1)
    gemm_tc2_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB, TcParams p) {
  using Cfg = Tc2Cfg<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + STAGES * Cfg::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + STAGES * Cfg::STAGE_BYTES);
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
  const int pair = (int)cluster_id_x(), npairs = (int)nclusters_x();

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmA);
    prefetch_tmap(&tmB);
    for (int s = 0; s < STAGES; ++s) { mbar_init(&full[s], 2); mbar_init(&empty[s], 1); }
    for (int a = 0; a < 2; ++a) { mbar_init(&tmem_full[a], 1); mbar_init(&tmem_empty[a], 2 * 32 * EPI_WARPS); }
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
          const uint32_t a = smem_u32(sA + s * Cfg::A_BYTES);
          const uint32_t b = smem_u32(sB + s * Cfg::B_BYTES);
#pragma unroll
          for (int kk = 0; kk < BK / 16; ++kk) {
            uint64_t ad = p.a_mn ? make_sdesc(a + kk * 2048, BK * 128, 1024) : make_sdesc(a + kk * 32, 16, 1024);
            uint64_t bd = p.b_mn ? make_sdesc(b + kk * 2048, BK * 128, 1024) : make_sdesc(b + kk * 32, 16, 1024);
            mma_bf16_2sm(tmem_d, ad, bd, idesc, (kb | kk) ? 1u : 0u);
          }
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
    int it = 0;
    for (int t = pair; t < tm.total; t += npairs, ++it) {
      int z, mb, nb;
      tm.get(t, z, mb, nb);
      const int z0 = z % p.nz0, z1 = z / p.nz0, n0 = nb * BN;
      const int acc = it & 1;
      mbar_wait(&tmem_full[acc], (it >> 1) & 1);
      tc_fence_after();
      const int64_t zoff = z0 * e.c_sz0 + z1 * e.c_sz1;
      const uint32_t tacc = tmem_base + acc * BN + ((uint32_t)(q * 32) << 16);
      const int ncols = min(BN, p.N - n0);
      const int c_beg = half * (BN / 2), c_end = min(ncols, c_beg + BN / 2);
#pragma unroll 1
      for (int c = c_beg; c < c_end; c += 32)
        drain_chunk(e, tacc + c, nkb > 0, lane, mb * 256 + (int)rank * 128 + q * 32, n0 + c, zoff);
      tc_fence_before();
      mbar_arrive_cluster(te + acc * 8);
    }
  }
  tc_fence_before();
  cluster_sync_all();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem_base), "r"(Cfg::TMEM_COLS)
                 : "memory");
  }
}

template <int BN, int STAGES>
static void launch_tc2(const hk_gemm_args& a, const EpiParams& e, cudaStream_t st) {
  using Cfg = Tc2Cfg<BN, STAGES>;
  CUtensorMap ma, mb;
  make_operand_map(&ma, a.A, a.a_mn_major, a.M, a.K, a.lda, a.nz0, a.a_sz0, a.nz1, a.a_sz1, 128);
  make_operand_map(&mb, a.B, a.b_mn_major, a.N, a.K, a.ldb, a.nz0, a.b_sz0, a.nz1, a.b_sz1, Cfg::HB);
  TcParams p;
  p.M = a.M; p.N = a.N; p.K = a.K; p.nz0 = a.nz0; p.nz = a.nz0 * a.nz1; p.a_mn = a.a_mn_major; p.b_mn = a.b_mn_major;
  p.e = e;
  static bool attr_set = false;
  if (!attr_set) {
    HM_CUDA(cudaFuncSetAttribute(gemm_tc2_kernel<BN, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, Cfg::SMEM));
    attr_set = true;
  }
  static int num_sms = 0;
  if (!num_sms) {
    int dev = 0;
    HM_CUDA(cudaGetDevice(&dev));
    HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int64_t tiles = ceil_div(a.M, 256) * ceil_div(a.N, BN) * (int64_t)a.nz0 * a.nz1;
  dim3 grid((unsigned)(2 * std::min<int64_t>(tiles, num_sms / 2)));  // persistent pairs
  const int e0 = g_prof.begin(st);
  gemm_tc2_kernel<BN, STAGES><<<grid, NUM_THREADS, Cfg::SMEM, st>>>(ma, mb, p);
  check_launch("gemm_tc2_kernel");
  g_prof.end(PROF_GEMM, e0, st, 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1);
}

}  // namespace tc

void gemm(const hk_gemm_args& a, cudaStream_t st) {
  HM_CHECK(a.M >= 0 && a.N >= 0 && a.K >= 0 && a.nz0 >= 1 && a.nz1 >= 1, HARMONY_E_INVALID_ARG, "gemm: bad shape");
  if (a.M == 0 || a.N == 0) return;
  EpiParams e;
  e.C = a.C; e.ldc = a.ldc; e.c_sz0 = a.c_sz0; e.c_sz1 = a.c_sz1;
  e.epi = a.epilogue; e.act = a.act; e.accumulate = a.accumulate; e.alpha = a.alpha;
  e.bias = a.bias; e.aux = a.aux; e.aux_out = a.aux_out; e.M = a.M; e.N = a.N;
  if (a.dtype == 0) {
    const int e0 = g_prof.begin(st);
    const double flops = 2.0 * a.M * a.N * (double)a.K * a.nz0 * a.nz1;
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
  // Tile shape from the problem shape only (never from the memory cap): bit-exact capped == uncapped.
  static const int mode = [] {
    const char* v = getenv("HARMONY_GEMM_2SM");
    return v ? atoi(v) : 1;
  }();
  const int64_t nz = (int64_t)a.nz0 * a.nz1;
  if (mode && a.M >= 256 && a.N >= 256) {
    // CTA-pair 256 x 256 tiles (measured best for every cfg2 shape, tools/gemm_bench.py);
    // HARMONY_GEMM_2SM=3 selects 256 x 128 pair tiles, 0 the single-CTA kernel
    if (mode == 3) tc::launch_tc2<128, 6>(a, e, st);
    else tc::launch_tc2<256, 6>(a, e, st);
    return;
  }
  if (a.N <= 64)
    tc::launch_tc<64, 8>(a, e, st);
  else if (a.N <= 128 || (int64_t)ceil_div(a.M, 128) * ceil_div(a.N, 256) * nz < 148)
    tc::launch_tc<128, 6>(a, e, st);
  else
    tc::launch_tc<256, 4>(a, e, st);
}

}  // namespace hm
