// attention_fwd2.cu — fused multi-head attention forward for dh = 64 with two query tiles per CTA
// (the same contract as attn_fwd_kernel in attention.cu).
//
// An A/B alternative to attn_fwd_kernel (selected with HARMONY_ATTN_FWD=2; the default stays the
// one-tile kernel).  Measured on B200 at the cfg2 shape (b=32, h=16, S=512): both take 79-84 us
// (ncu: 20% tensor-pipe activity, 29% issue utilisation; the softmax warps' samples sit on the
// scores-ready barrier, i.e. the MMA -> softmax -> MMA round trip, not the exponentials (removing
// them: -2%) nor the TMEM reads (halving them: 0%) nor the item order or K/V stage count).  Causal
// it is slower (76 vs 62 us): the pair's two tiles have unequal key ranges.  DESIGN.md §6.
// Design: each CTA owns TWO query tiles (A, B) of one (sequence, head) and streams the key / value
// tiles once for both:
//   warp 0: TMA (Q_A, Q_B once per item; K_j, V_j per key tile),
//   warp 1: MMA (S_A = Q_A K_j^T, S_B = Q_B K_j^T into TMEM; O_X += P_X V_j with P_X in TMEM),
//   warps 4-7: softmax of tile A, warps 8-11: softmax of tile B — one thread per query row holding all
//   128 scores of the key tile, so the row maximum needs no exchange, and while one tile's warps
//   wait for their scores the other tile's warps keep the SFU busy.
// TMEM (512 columns): S_A [0,128), S_B [128,256), O_A [256,320), O_B [320,384), P_A [384,448),
// P_B [448,512) (P as bf16 pairs).  Numerics as attn_fwd_kernel (reading c11): one pass with a lazily
// raised running max (raised only when a tile's max exceeds it by more than 8 in log2 units; O then
// rescaled in TMEM), exact zeros above the causal diagonal, O / l and the row LSE at the end.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <type_traits>

#include "../common.hpp"
#include "kernels.hpp"
#include "tc_common.cuh"

namespace hm {
namespace attn2 {

// HM_ATTN_TRACE builds (diagnostics only): CTA 0 records clock64 stamps — row 0: softmax warp 4
// lane 0 (tile A), row 1: the MMA issuer, row 2: softmax warp 8 lane 0 (tile B)
#ifdef HM_ATTN_TRACE
__device__ unsigned long long g_attn2_trace[3][2048];
__device__ int g_attn2_trace_n[3];
#define TR(row, code)                                                                                   \
  do {                                                                                                  \
    if (blockIdx.x == 0 && (row == 1 || (threadIdx.x == 128 || threadIdx.x == 256))) {                 \
      const int i_ = g_attn2_trace_n[row]++;                                                            \
      if (i_ < 2048) g_attn2_trace[row][i_] = ((unsigned long long)(code) << 56) | (clock64() & 0xffffffffffffffull); \
    }                                                                                                   \
  } while (0)
#else
#define TR(row, code) do { } while (0)
#endif

using namespace tcx;

__device__ __forceinline__ float fast_exp2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}



// 128 consecutive columns of this thread's lane, both loads and the wait in ONE asm statement: the
// destination registers are written asynchronously until tcgen05.wait::ld, so the compiler must not
// be able to move, spill or read them in between
__device__ __forceinline__ void tmem_ld128_sync(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%128];\n\t"
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%64,%65,%66,%67,%68,%69,%70,%71,%72,%73,%74,%75,%76,%77,%78,%79,%80,%81,%82,%83,%84,%85,%86,%87,%88,%89,%90,%91,%92,%93,%94,%95,%96,%97,%98,%99,%100,%101,%102,%103,%104,%105,%106,%107,%108,%109,%110,%111,%112,%113,%114,%115,%116,%117,%118,%119,%120,%121,%122,%123,%124,%125,%126,%127}, [%129];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]), "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]), "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]), "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]), "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]), "=r"(r[61]), "=r"(r[62]), "=r"(r[63]), "=r"(r[64]), "=r"(r[65]), "=r"(r[66]), "=r"(r[67]), "=r"(r[68]), "=r"(r[69]), "=r"(r[70]), "=r"(r[71]), "=r"(r[72]), "=r"(r[73]), "=r"(r[74]), "=r"(r[75]), "=r"(r[76]), "=r"(r[77]), "=r"(r[78]), "=r"(r[79]), "=r"(r[80]), "=r"(r[81]), "=r"(r[82]), "=r"(r[83]), "=r"(r[84]), "=r"(r[85]), "=r"(r[86]), "=r"(r[87]), "=r"(r[88]), "=r"(r[89]), "=r"(r[90]), "=r"(r[91]), "=r"(r[92]), "=r"(r[93]), "=r"(r[94]), "=r"(r[95]), "=r"(r[96]), "=r"(r[97]), "=r"(r[98]), "=r"(r[99]), "=r"(r[100]), "=r"(r[101]), "=r"(r[102]), "=r"(r[103]), "=r"(r[104]), "=r"(r[105]), "=r"(r[106]), "=r"(r[107]), "=r"(r[108]), "=r"(r[109]), "=r"(r[110]), "=r"(r[111]), "=r"(r[112]), "=r"(r[113]), "=r"(r[114]), "=r"(r[115]), "=r"(r[116]), "=r"(r[117]), "=r"(r[118]), "=r"(r[119]), "=r"(r[120]), "=r"(r[121]), "=r"(r[122]), "=r"(r[123]), "=r"(r[124]), "=r"(r[125]), "=r"(r[126]), "=r"(r[127])
      : "r"(taddr), "r"(taddr + 64));
}

// 64 columns, load and wait in one asm statement (see tmem_ld128_sync)
__device__ __forceinline__ void tmem_ld64_sync(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x64.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32,%33,%34,%35,%36,%37,%38,%39,%40,%41,%42,%43,%44,%45,%46,%47,%48,%49,%50,%51,%52,%53,%54,%55,%56,%57,%58,%59,%60,%61,%62,%63}, [%64];\n\t"
      "tcgen05.wait::ld.sync.aligned;"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31]), "=r"(r[32]), "=r"(r[33]), "=r"(r[34]), "=r"(r[35]), "=r"(r[36]), "=r"(r[37]), "=r"(r[38]), "=r"(r[39]), "=r"(r[40]), "=r"(r[41]), "=r"(r[42]), "=r"(r[43]), "=r"(r[44]), "=r"(r[45]), "=r"(r[46]), "=r"(r[47]), "=r"(r[48]), "=r"(r[49]), "=r"(r[50]), "=r"(r[51]), "=r"(r[52]), "=r"(r[53]), "=r"(r[54]), "=r"(r[55]), "=r"(r[56]), "=r"(r[57]), "=r"(r[58]), "=r"(r[59]), "=r"(r[60]), "=r"(r[61]), "=r"(r[62]), "=r"(r[63])
      : "r"(taddr));
}

constexpr int DH = 64;
constexpr int BQ = 128;   // query rows per tile (two tiles per CTA item)
constexpr int BKV = 128;  // keys per tile
constexpr int THREADS = 384;  // warpgroup 0: TMA (warp 0), MMA (warp 1); warpgroups 1, 2: softmax of tiles A, B
constexpr int KST = 4, VST = 4;                 // K / V stages
constexpr int Q_BYTES = BQ * DH * 2;            // 16 KB per tile
constexpr int KV_BYTES = BKV * DH * 2;          // 16 KB
constexpr int O_BYTES = BQ * DH * 2;            // output staging per tile
constexpr int SMEM = 2 * 2 * Q_BYTES + KST * KV_BYTES + VST * KV_BYTES + 2 * O_BYTES + 1024 + 512;
static_assert(SMEM <= 232448, "shared memory per CTA");
constexpr int S_COL = 0, O_COL = 256, P_COL = 384;

struct Params {
  int S, H, B, causal;
  float scale_log2, scale;
  float* lse;  // [b, H, S]
  int order;   // item order (HARMONY_ATTN2_ORDER): 0 pair-major, 1 (sequence, head)-major
};

__device__ __forceinline__ int snake(int r) {
  return r * (int)gridDim.x + ((r & 1) ? (int)(gridDim.x - 1 - blockIdx.x) : (int)blockIdx.x);
}
__global__ void __launch_bounds__(THREADS, 1)
    attn_fwd2_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                     const __grid_constant__ CUtensorMap tmV, const __grid_constant__ CUtensorMap tmC, Params p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                          // [2 stages][A, B] 16 KB each
  uint8_t* sK = sQ + 4 * Q_BYTES;
  uint8_t* sV = sK + KST * KV_BYTES;
  uint8_t* sO = sV + VST * KV_BYTES;           // [A, B] output staging
  uint64_t* bars = reinterpret_cast<uint64_t*>(sO + 2 * O_BYTES);
  uint64_t* q_full = bars;            // [2]
  uint64_t* q_empty = q_full + 2;     // [2]
  uint64_t* k_full = q_empty + 2;     // [KST]
  uint64_t* k_empty = k_full + KST;   // [KST]
  uint64_t* v_full = k_empty + KST;   // [VST]
  uint64_t* v_empty = v_full + VST;   // [VST]
  uint64_t* s_full = v_empty + VST;   // [2] per tile
  uint64_t* s_empty = s_full + 2;     // [2]
  uint64_t* p_full = s_empty + 2;     // [2]
  uint64_t* p_empty = p_full + 2;     // [2]
  uint64_t* o_full = p_empty + 2;     // [2]
  uint64_t* o_empty = o_full + 2;     // [2]
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(o_empty + 2);
  static_assert((16 + 2 * KST + 2 * VST) * 8 + 4 <= 512, "barrier area");

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nq = p.S / BQ, npair = nq / 2;
  const int items = npair * p.H * p.B;
  // Items are (sequence, head)-major: the npair query-tile pairs of one (b, h) are dealt to adjacent
  // CTAs of the same round, so they stream the same K / V tiles at about the same time and all but
  // the first read hit L2 (the kernel is bound by these loads, not by its math).  Within a (b, h) the
  // causal pairs go longest first.
  auto decode = [&](int item, int& b, int& h, int& t) {
    if (p.order) {  // (sequence, head)-major: the pairs of one (b, h) on adjacent CTAs (shared K / V in L2)
      t = npair - 1 - item % npair;
      const int bh = item / npair;
      h = bh % p.H;
      b = bh / p.H;
    } else {  // pair-major, longest causal pairs first
      const int hb = p.H * p.B;
      t = npair - 1 - item / hb;
      const int rem = item % hb;
      h = rem % p.H;
      b = rem / p.H;
    }
  };

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); prefetch_tmap(&tmC);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1);
      mbar_init(&s_full[i], 1); mbar_init(&s_empty[i], 128);
      mbar_init(&p_full[i], 128); mbar_init(&p_empty[i], 1);
      mbar_init(&o_full[i], 1); mbar_init(&o_empty[i], 128);
    }
    for (int i = 0; i < KST; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < VST; ++i) { mbar_init(&v_full[i], 1); mbar_init(&v_empty[i], 1); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(512) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  // registers move to the softmax warpgroups (the per-SM-subpartition file holds one warp of each
  // CTA: 4 x 80 + 8 x 208 <= 12 x 168 registers per lane, the launch allocation)
  if (warp < 4) {
  asm volatile("setmaxnreg.dec.sync.aligned.u32 80;" ::: "memory");
  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer =====
      int ks = 0; uint32_t kph = 0;
      int vs = 0; uint32_t vph = 0;
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, t;
        decode(item, b, h, t);
        const int nB = p.causal ? 2 * t + 2 : nq;  // key tiles of the pair's later tile B
        const int qs = n & 1;
        mbar_wait(&q_empty[qs], ((n >> 1) & 1) ^ 1);
        mbar_expect_tx(&q_full[qs], 2 * Q_BYTES);
        tma_load_4d(sQ + (2 * qs) * Q_BYTES, &tmQ, &q_full[qs], 0, (2 * t) * BQ, h, b);
        tma_load_4d(sQ + (2 * qs + 1) * Q_BYTES, &tmQ, &q_full[qs], 0, (2 * t + 1) * BQ, h, b);
        for (int j = 0; j < nB; ++j) {
          mbar_wait(&k_empty[ks], kph ^ 1);
          mbar_expect_tx(&k_full[ks], KV_BYTES);
          tma_load_4d(sK + ks * KV_BYTES, &tmK, &k_full[ks], 0, j * BKV, h, b);
          if (++ks == KST) { ks = 0; kph ^= 1; }
          mbar_wait(&v_empty[vs], vph ^ 1);
          mbar_expect_tx(&v_full[vs], KV_BYTES);
#pragma unroll
          for (int ka = 0; ka < 2; ++ka)
            tma_load_4d(sV + vs * KV_BYTES + ka * 8192, &tmV, &v_full[vs], 0, j * BKV + ka * 64, h, b);
          if (++vs == VST) { vs = 0; vph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ===== MMA issuer =====
      const uint32_t idesc_s = make_idesc_f16(128, BKV, 0, 0);  // S = Q K^T: K-major operands
      const uint32_t idesc_o = make_idesc_f16(128, DH, 0, 1);   // O += P V: P from TMEM, V MN-major
      int ks = 0; uint32_t kph = 0;
      int vs = 0; uint32_t vph = 0;
      int su[2] = {0, 0}, pu[2] = {0, 0};  // S fills / P uses per tile
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, t;
        decode(item, b, h, t);
        const int nt[2] = {p.causal ? 2 * t + 1 : nq, p.causal ? 2 * t + 2 : nq};
        const int nB = nt[1];
        const int qs = n & 1;
        mbar_wait(&q_full[qs], (n >> 1) & 1);
        const uint32_t qa[2] = {smem_u32(sQ + (2 * qs) * Q_BYTES), smem_u32(sQ + (2 * qs + 1) * Q_BYTES)};
        auto issue_s = [&](int j) {  // S_A(j), S_B(j) from K_j
          mbar_wait(&k_full[ks], kph);
          const uint32_t ka = smem_u32(sK + ks * KV_BYTES);
#pragma unroll
          for (int x = 0; x < 2; ++x) {
            if (j >= nt[x]) continue;
            mbar_wait(&s_empty[x], (su[x] & 1) ^ 1);
            // the item's first tile: B's scores only once A has read its own, so the two softmax groups
            // start half a phase apart (one reads scores from TMEM while the other exponentiates)
            if (x == 1 && j == 0 && nt[0] > 0) mbar_wait(&s_empty[0], (su[0] & 1) ^ 1);
            TR(1, x ? 12 : 10);
            tc_fence_after();
            mma4_bf16(tmem + S_COL + x * BKV, make_sdesc(qa[x], 16, 1024), make_sdesc(ka, 16, 1024), 2, 2, idesc_s, 0u);
            mma_commit(&s_full[x]);
            ++su[x];
          }
          mma_commit(&k_empty[ks]);
          if (++ks == KST) { ks = 0; kph ^= 1; }
          if (j == nB - 1) mma_commit(&q_empty[qs]);
        };
        auto issue_pv = [&](int j) {  // O_A += P_A V_j, O_B += P_B V_j
          mbar_wait(&v_full[vs], vph);
          const uint32_t va = smem_u32(sV + vs * KV_BYTES);
#pragma unroll
          for (int x = 0; x < 2; ++x) {
            if (j >= nt[x]) continue;
            mbar_wait(&p_full[x], pu[x] & 1);
            if (j == 0) mbar_wait(&o_empty[x], (n & 1) ^ 1);  // the previous item's O_X has been drained
            TR(1, x ? 13 : 11);
            tc_fence_after();
            const uint32_t pa = tmem + P_COL + x * (BKV / 2);
#pragma unroll
            for (int kk = 0; kk < BKV / 16; ++kk) {
              const int atom = kk / 4, sub = kk % 4;
              const uint64_t bd = make_sdesc(va + atom * 8192 + sub * 2048, 8192, 1024);
              mma_bf16_ts(tmem + O_COL + x * DH, pa + kk * 8, bd, idesc_o, (j | kk) ? 1u : 0u);
            }
            mma_commit(&p_empty[x]);
            ++pu[x];
            if (j == nt[x] - 1) mma_commit(&o_full[x]);
          }
          mma_commit(&v_empty[vs]);
          if (++vs == VST) { vs = 0; vph ^= 1; }
        };
        // scores of key tile j+1 are queued before the PV of tile j, so the softmax of j+1 overlaps it
        issue_s(0);
        for (int j = 0; j < nB; ++j) {
          if (j + 1 < nB) issue_s(j + 1);
          issue_pv(j);
        }
      }
    }
    __syncwarp();
  }
  } else {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 208;" ::: "memory");
    // ===== softmax: tile x = 0 (warps 4-7) or 1 (warps 8-11); thread = query row =====
    const int x = (warp - 4) >> 2;
    const int qd = warp & 3;            // TMEM lane quadrant of this warp
    const int r = qd * 32 + lane;       // row within the tile
    const uint32_t trow = (uint32_t)(qd * 32) << 16;
    const uint32_t tS = tmem + trow + S_COL + x * BKV, tO = tmem + trow + O_COL + x * DH,
                   tP = tmem + trow + P_COL + x * (BKV / 2);
    const bool issuer = qd == 0 && lane == 0;  // of this tile's TMA store
    uint8_t* stage = sO + x * O_BYTES;
    int su = 0, pu = 0, n = 0;
    const float sl = p.scale_log2;
    for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
      int b, h, t;
      decode(item, b, h, t);
      const int qt = 2 * t + x;
      const int ntiles = p.causal ? qt + 1 : nq;
      const int qrow = qt * BQ + r;
      float m = -INFINITY;
      float2 la = make_float2(0.f, 0.f), lb = make_float2(0.f, 0.f);
      auto tile = [&](int j, auto diag_tag) {
        constexpr bool DIAG = decltype(diag_tag)::value;
        mbar_wait(&s_full[x], su & 1);
        TR(x ? 2 : 0, 20);
        tc_fence_after();
        uint32_t raw[128];
        tmem_ld128_sync(tS, raw);
        tc_fence_before();
        mbar_arrive_local(&s_empty[x]);  // S is in registers: the next tile's scores may land
        TR(x ? 2 : 0, 21);
        ++su;
        float* v = reinterpret_cast<float*>(raw);
        if constexpr (DIAG) {
          const int lim = qrow - j * BKV;  // keys i <= lim are visible
#pragma unroll
          for (int i = 0; i < BKV; ++i)
            if (i > lim) v[i] = -INFINITY;
        }
        float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
        for (int i = 0; i < BKV; ++i) m4[i & 3] = fmaxf(m4[i & 3], v[i]);
        const float tm = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
        const bool raise = (tm - m) * sl > 8.f;  // true on the first tile (m = -inf)
        float f = 1.f;
        if (raise) {
          f = j == 0 ? 0.f : fast_exp2((m - tm) * sl);
          m = tm;
          la = make_float2(la.x * f, la.y * f);
          lb = make_float2(lb.x * f, lb.y * f);
        }
        const float ms = m * sl;
        const float2 sl2 = make_float2(sl, sl), nms2 = make_float2(-ms, -ms), one2 = make_float2(1.f, 1.f);
        uint32_t pk[64];  // the tile's probabilities as bf16 pairs (the scores die as they are converted)
#pragma unroll
        for (int i = 0; i < 64; ++i) {
          const float2 z = ffma2(make_float2(v[2 * i], v[2 * i + 1]), sl2, nms2);
          const float2 e2 = make_float2(fast_exp2(z.x), fast_exp2(z.y));
          if (i & 1) lb = ffma2(e2, one2, lb);
          else la = ffma2(e2, one2, la);
          __nv_bfloat162 h2 = __floats2bfloat162_rn(e2.x, e2.y);
          pk[i] = *reinterpret_cast<uint32_t*>(&h2);
        }
        // P_X is single-buffered: the PV of the previous key tile must have consumed it (and, for a
        // rescale, must have landed in O_X) — waited for only now, so the exponentials overlap it
        TR(x ? 2 : 0, 23);
        mbar_wait(&p_empty[x], (pu & 1) ^ 1);
        TR(x ? 2 : 0, 24);
        tc_fence_after();
        tmem_st32(tP, pk);
        tmem_st32(tP + 32, pk + 32);
        // a raised max rescales this row of O_X (after the scores are consumed: fewer live registers;
        // the PV of this tile is issued only once p_full is signalled below)
        if (__any_sync(0xffffffffu, raise && j > 0)) {
#pragma unroll
          for (int c = 0; c < DH; c += 16) {
            uint32_t o[16];
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                : "=r"(o[0]), "=r"(o[1]), "=r"(o[2]), "=r"(o[3]), "=r"(o[4]), "=r"(o[5]), "=r"(o[6]), "=r"(o[7]),
                  "=r"(o[8]), "=r"(o[9]), "=r"(o[10]), "=r"(o[11]), "=r"(o[12]), "=r"(o[13]), "=r"(o[14]), "=r"(o[15])
                : "r"(tO + c));
            tmem_wait_ld();
#pragma unroll
            for (int i = 0; i < 16; ++i) o[i] = __float_as_uint(__uint_as_float(o[i]) * f);
            asm volatile(
                "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
                    tO + c),
                "r"(o[0]), "r"(o[1]), "r"(o[2]), "r"(o[3]), "r"(o[4]), "r"(o[5]), "r"(o[6]), "r"(o[7]), "r"(o[8]),
                "r"(o[9]), "r"(o[10]), "r"(o[11]), "r"(o[12]), "r"(o[13]), "r"(o[14]), "r"(o[15])
                : "memory");
          }
        }
        tmem_wait_st();
        tc_fence_before();
        mbar_arrive_local(&p_full[x]);
        TR(x ? 2 : 0, 25);
        ++pu;
      };
      const int nfull = p.causal ? ntiles - 1 : ntiles;
      for (int j = 0; j < nfull; ++j) tile(j, std::false_type{});
      if (p.causal) tile(ntiles - 1, std::true_type{});
      const float l = (la.x + la.y) + (lb.x + lb.y);
      const float inv_l = 1.f / l;
      // ---- epilogue: O_X (normalised, bf16) -> swizzled staging -> TMA store to C; then the LSE
      mbar_wait(&o_full[x], n & 1);
      TR(x ? 2 : 0, 26);
      tc_fence_after();
      uint32_t o[DH];
      tmem_ld64_sync(tO, o);
      tc_fence_before();
      mbar_arrive_local(&o_empty[x]);  // O_X is in registers: the next item's PV may start
      TR(x ? 2 : 0, 27);
      if (issuer) bulk_wait_read<0>();  // the previous item's store has left the staging box
      asm volatile("bar.sync %0, 128;" ::"r"(2 + x) : "memory");
      uint8_t* row = stage + r * 128;
#pragma unroll
      for (int u = 0; u < DH / 8; ++u) {
        uint32_t pk[4];
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          __nv_bfloat162 h2 = __floats2bfloat162_rn(__uint_as_float(o[8 * u + 2 * q]) * inv_l,
                                                    __uint_as_float(o[8 * u + 2 * q + 1]) * inv_l);
          pk[q] = *reinterpret_cast<uint32_t*>(&h2);
        }
        *reinterpret_cast<uint4*>(row + ((u ^ (r & 7)) << 4)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("bar.sync %0, 128;" ::"r"(2 + x) : "memory");
      if (issuer) {
        tma_store_4d(&tmC, stage, 0, qt * BQ, h, b);
        bulk_commit();
      }
      p.lse[((int64_t)b * p.H + h) * p.S + qrow] = m * p.scale + logf(l);
    }
    if (issuer) bulk_wait_all();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
  }
}

}  // namespace attn2

// dh = 64, S a multiple of 256: the two-tile forward; false otherwise (the caller falls back)
bool attention_fwd2_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, void* C, float* lse,
                          cudaStream_t st) {
  using namespace attn2;
  if (dh != DH || S % (2 * BQ) != 0) return false;
  const int d = H * dh;
  CUtensorMap mq, mk, mv, mc;
  tcx::make_map_4d(&mq, QKV, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BQ);
  tcx::make_map_4d(&mk, static_cast<const __nv_bfloat16*>(QKV) + d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BKV);
  tcx::make_map_4d(&mv, static_cast<const __nv_bfloat16*>(QKV) + 2 * d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64,
                   64);
  tcx::make_map_4d(&mc, C, dh, S, H, b, d, dh, (int64_t)S * d, 64, BQ);
  Params p;
  p.S = S; p.H = H; p.B = (int)b; p.causal = causal;
  p.scale = 1.0f / std::sqrt((float)dh);
  p.scale_log2 = p.scale * 1.4426950408889634f;
  p.lse = lse;
  static const int order = [] {
    const char* v = getenv("HARMONY_ATTN2_ORDER");
    return v ? atoi(v) : 0;
  }();
  p.order = order;
  static int num_sms = 0;
  if (!num_sms) {
    int dev = 0;
    HM_CUDA(cudaGetDevice(&dev));
    HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int64_t items = (int64_t)(S / (2 * BQ)) * H * b;
  static const int grid_cap = [] {
    const char* v = getenv("HARMONY_ATTN_GRID");
    return v ? atoi(v) : 0;
  }();
  dim3 grid((unsigned)std::min<int64_t>(items, grid_cap > 0 ? grid_cap : num_sms));
  static bool set = false;
  if (!set) {
    HM_CUDA(cudaFuncSetAttribute(attn_fwd2_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM));
    set = true;
  }
  const int e0 = g_prof.begin(st);
  launch_k(attn_fwd2_kernel, dim3(grid), dim3(THREADS), SMEM, st, mq, mk, mv, mc, p);
  check_launch("attn_fwd2_kernel");
  g_prof.end(PROF_ATTN, e0, st, 4.0 * b * H * (double)S * S * dh);
  return true;
}

#ifdef HM_ATTN_TRACE
extern "C" int hm_attn2_trace_read(unsigned long long* out, int* counts) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, attn2::g_attn2_trace, sizeof(attn2::g_attn2_trace));
  cudaMemcpyFromSymbol(counts, attn2::g_attn2_trace_n, sizeof(attn2::g_attn2_trace_n));
  int z[3] = {0, 0, 0};
  cudaMemcpyToSymbol(attn2::g_attn2_trace_n, z, sizeof(z));
  return 0;
}
#endif

}  // namespace hm
