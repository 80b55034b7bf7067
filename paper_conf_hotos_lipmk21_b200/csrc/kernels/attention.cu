// attention.cu — fused multi-head attention forward on tcgen05 (SURVEY §8(a) rows a4/a5, K4 + K9).
//
// Persistent CTAs loop over (128-query tile, head, sequence) items.  The scores never touch HBM:
// S = Q K^T lands in TMEM, eight softmax warps (two per TMEM lane quadrant, 64 keys each) read it
// with tcgen05.ld, and the bf16 probabilities are stored back into TMEM where they are the A
// operand of O += P V (accumulated in TMEM).  One pass over the key tiles with a lazily raised
// running max: S is read from TMEM once per tile (the TMEM read bandwidth, not the tensor pipe, is
// what bounds a dh = 64 tile), O is rescaled in TMEM only when a tile raises the row max by more
// than 2^8, and O is divided by the row sum in the epilogue.  Outputs: C (bf16, heads
// interleaved in [T, d]) and the row log-sum-exp (fp32 [b, h, S]) the backward needs.
// Numerics match the unfused path's reading c11: P = softmax(scale * Q K^T) with causal rows
// masked to exactly 0 above the diagonal.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <type_traits>

#include "../common.hpp"
#include "kernels.hpp"
#include "tc_common.cuh"

namespace hm {
namespace attn {

using namespace tcx;

// 2^x on the SFU (ex2.approx.ftz: ~2 ulp, the same unit __expf uses)
__device__ __forceinline__ float fast_exp2(float x) {
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

// HM_ATTN_TRACE builds (diagnostics only): CTA 0 of the forward records clock64 stamps of its
// pipeline events — row 0: softmax warp 2 lane 0, row 1: the MMA issuer, row 2: the TMA producer —
// read back with hm_attn_trace_read()
#ifdef HM_ATTN_TRACE
__device__ unsigned long long g_attn_trace[3][2048];
__device__ int g_attn_trace_n[3];
// the event index lives in a register of the recording thread (tr_cnt, declared at kernel entry):
// a stamp is one fire-and-forget global store
#define TR(row, code)                                                                                   \
  do {                                                                                                  \
    if (blockIdx.x == 0 && threadIdx.x == (row == 0 ? 64 : row == 1 ? 32 : 0)) {                         \
      if (tr_cnt < 2048) g_attn_trace[row][tr_cnt] = ((unsigned long long)(code) << 56) | (clock64() & 0xffffffffffffffull); \
      ++tr_cnt;                                                                                         \
    }                                                                                                   \
  } while (0)
#define TR_END()                                                                                        \
  do {                                                                                                  \
    if (blockIdx.x == 0 && (threadIdx.x == 64 || threadIdx.x == 32 || threadIdx.x == 0))                 \
      g_attn_trace_n[threadIdx.x == 64 ? 0 : threadIdx.x == 32 ? 1 : 2] = tr_cnt;                       \
  } while (0)
#else
#define TR(row, code) do { } while (0)
#define TR_END() do { } while (0)
#endif

// 2^x for a pair on the FMA pipe: x = j + f with j = rint(x) (the 1.5 * 2^23 rounding trick, whose
// low mantissa bits are j), f in [-0.5, 0.5]; 2^f by a degree-5 polynomial fitted for relative error
// (max 2.3e-7 in fp32 Horner, the accuracy of ex2.approx), and 2^j added to the exponent field.
// x is clamped to [-125, 126]: below that 2^x is < 2^-125 (ex2.approx.ftz gives 0 there), which no
// caller can tell from 0 after the bf16 rounding and the row sum.
__device__ __forceinline__ float2 exp2_poly2(float2 x) {
  x.x = fminf(fmaxf(x.x, -125.f), 126.f);
  x.y = fminf(fmaxf(x.y, -125.f), 126.f);
  const float2 one = make_float2(1.f, 1.f), magic = make_float2(12582912.f, 12582912.f);
  const float2 t = tcx::ffma2(x, one, magic);                                    // 1.5 * 2^23 + rint(x)
  const float2 r = tcx::ffma2(t, one, make_float2(-12582912.f, -12582912.f));    // rint(x)
  const float2 f = tcx::ffma2(r, make_float2(-1.f, -1.f), x);                    // x - rint(x)
  float2 q = tcx::ffma2(make_float2(1.32764e-3f, 1.32764e-3f), f, make_float2(9.67552e-3f, 9.67552e-3f));
  q = tcx::ffma2(q, f, make_float2(5.550713e-2f, 5.550713e-2f));
  q = tcx::ffma2(q, f, make_float2(2.402212e-1f, 2.402212e-1f));
  q = tcx::ffma2(q, f, make_float2(6.9314697e-1f, 6.9314697e-1f));
  q = tcx::ffma2(q, f, make_float2(1.00000007f, 1.00000007f));
  // low 9 bits of the magic's bit pattern are 0: (bits(t) << 23) == rint(x) << 23 (mod 2^32)
  return make_float2(__int_as_float(__float_as_int(q.x) + (__float_as_int(t.x) << 23)),
                     __int_as_float(__float_as_int(q.y) + (__float_as_int(t.y) << 23)));
}

constexpr int BQ = 128;   // query rows per CTA
constexpr int BKV = 128;  // keys per tile
constexpr int THREADS = 320;  // warp 0: TMA, warp 1: MMA + TMEM, warps 2-9: softmax (2 per row quadrant)

template <int DH>
struct FwdCfg {
  static constexpr int Q_BYTES = BQ * DH * 2;           // DH/64 K-atoms of 16 KB
  static constexpr int K_BYTES = BKV * DH * 2;
  static constexpr int V_BYTES = BKV * DH * 2;          // 2 key-atoms x DH/64 MN-chunks of 8 KB
  static constexpr int O_BYTES = BQ * DH * 2;           // output staging (DH/64 boxes of 64 columns)
  static constexpr int QST = DH == 64 ? 3 : 1, KST = DH == 64 ? 4 : 2, VST = DH == 64 ? 4 : 2;
  static constexpr int BAR_BYTES = 512;                 // mbarriers + the TMEM base
  static constexpr int SMEM = QST * Q_BYTES + KST * K_BYTES + VST * V_BYTES + O_BYTES + 1024 + BAR_BYTES + 2 * BQ * 4 + 4 * BQ * 4;
  static constexpr int S_COLS = BKV;                    // fp32 accumulator columns per S buffer
  // SPLIT (an A/B variant, off): the two warps of a lane quadrant run independent online softmaxes
  // over the two 64-key halves of every tile, each with its own O accumulator (combined in the
  // epilogue), so they never meet at a per-tile barrier.  Measured at dh = 64, b = 32, S = 512:
  // 80.6 vs 77.3 us — the exponential phase shrinks (1270 -> 880 cycles per tile) but the softmax
  // then waits on the scores: the MMA issue (about 145 cycles per tcgen05.mma here) paces the tile.
  static constexpr bool SPLIT = false;
  static constexpr int O_COL = 2 * BKV;                 // O (SPLIT: O_0, O_1) after the two S buffers
  static constexpr int P_COL = 2 * BKV + (SPLIT ? 2 : 1) * DH;  // two P buffers (bf16 pairs: BKV/2 columns each)
  static constexpr int TMEM_COLS = 512;
  static_assert(P_COL + BKV <= TMEM_COLS, "TMEM columns");
  static_assert(SMEM <= 232448, "shared memory per CTA");
};

struct FwdParams {
  int S, H, B, causal;
  float scale_log2;  // scale * log2(e)
  float scale;
  float* lse;        // [b, H, S]
};

// Persistent item order.  Items are numbered by decreasing work (causal: query tile nq-1 first,
// whose rows see every key tile) and dealt to the CTAs in a snake (round r: CTA c takes
// r*G + c, or r*G + G-1-c on odd rounds), so every CTA gets a mix of long and short items.  (A
// plain stride-G walk hands CTA c only items with one tile index when G is a multiple of the
// tile count — 148 = 37 * 4 — which left the causal kernels as slow as the non-causal ones.)
__device__ __forceinline__ int snake(int r) {
  return r * (int)gridDim.x + ((r & 1) ? (int)(gridDim.x - 1 - blockIdx.x) : (int)blockIdx.x);
}
// sorted item -> (sequence, head, query tile)
__device__ __forceinline__ void fwd_item(int item, int nq, int H, int B, int& b, int& h, int& qt) {
  const int hb = H * B;
  qt = nq - 1 - item / hb;
  const int rem = item % hb;
  h = rem % H;
  b = rem / H;
}

// Persistent: one CTA per SM loops over the (query tile, head, sequence) items.  All pipeline
// counters (Q / K / V stages, S and P buffers) run on across items, so the producer loads the next
// item's Q and K while the current one is in its second pass, the MMA issues the next item's
// first-pass scores while the softmax warps drain O of the current one (O has its own full /
// empty barriers), and the output leaves through shared memory with TMA stores.  P never touches
// shared memory: the softmax warps store it (bf16 pairs) into TMEM and O += P V takes its A
// operand from there.
template <int DH, int NPOLY>
__global__ void __launch_bounds__(THREADS, 1)
    attn_fwd_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                    const __grid_constant__ CUtensorMap tmV, const __grid_constant__ CUtensorMap tmC, FwdParams p) {
  using Cfg = FwdCfg<DH>;
  int tr_cnt = 0;  // HM_ATTN_TRACE event index (unused otherwise)
  (void)tr_cnt;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = sQ + Cfg::QST * Cfg::Q_BYTES;
  uint8_t* sV = sK + Cfg::KST * Cfg::K_BYTES;
  uint8_t* sO = sV + Cfg::VST * Cfg::V_BYTES;  // output staging
  uint64_t* bars = reinterpret_cast<uint64_t*>(sO + Cfg::O_BYTES);
  uint64_t* q_full = bars;                      // [QST]
  uint64_t* q_empty = q_full + Cfg::QST;        // [QST]
  uint64_t* k_full = q_empty + Cfg::QST;        // [KST]
  uint64_t* k_empty = k_full + Cfg::KST;        // [KST]
  uint64_t* v_full = k_empty + Cfg::KST;        // [VST]
  uint64_t* v_empty = v_full + Cfg::VST;        // [VST]
  uint64_t* s_full = v_empty + Cfg::VST;        // [2]
  uint64_t* s_empty = s_full + 2;               // [2]
  uint64_t* p_full = s_empty + 2;               // [2 buffers][2 key halves] (non-SPLIT: [b][0] only)
  uint64_t* p_empty = p_full + 4;               // [2][2]
  uint64_t* o_full = p_empty + 4;
  uint64_t* o_empty = o_full + 1;
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(o_empty + 1);
  static_assert((14 + 2 * Cfg::QST + 2 * Cfg::KST + 2 * Cfg::VST) * 8 + 4 <= Cfg::BAR_BYTES, "barrier area");
  float(*sm_x)[BQ] = reinterpret_cast<float(*)[BQ]>(reinterpret_cast<uint8_t*>(bars) + Cfg::BAR_BYTES);  // [2][BQ] row stats
  float(*sm_t)[2][BQ] = reinterpret_cast<float(*)[2][BQ]>(reinterpret_cast<uint8_t*>(bars) + Cfg::BAR_BYTES + 2 * BQ * 4);  // [2][2][BQ]

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nq = p.S / BQ;
  const int items = nq * p.H * p.B;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); prefetch_tmap(&tmC);
    for (int i = 0; i < Cfg::QST; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mbar_init(&s_full[i], 1); mbar_init(&s_empty[i], 256); }
    for (int i = 0; i < 4; ++i) { mbar_init(&p_full[i], Cfg::SPLIT ? 128 : 256); mbar_init(&p_empty[i], 1); }
    for (int i = 0; i < Cfg::KST; ++i) { mbar_init(&k_full[i], 1); mbar_init(&k_empty[i], 1); }
    for (int i = 0; i < Cfg::VST; ++i) { mbar_init(&v_full[i], 1); mbar_init(&v_empty[i], 1); }
    mbar_init(o_full, 1); mbar_init(o_empty, 256);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(Cfg::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  if (warp == 0) {
    if (lane == 0) {
      // ===== TMA producer: per item Q once, then a K and a V tile per key tile =====
      int ks = 0; uint32_t kph = 0;
      int vs = 0; uint32_t vph = 0;
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, qt;
        fwd_item(item, nq, p.H, p.B, b, h, qt);
        const int ntiles = p.causal ? qt + 1 : nq;
        const int qs = n % Cfg::QST;
        mbar_wait(&q_empty[qs], ((n / Cfg::QST) & 1) ^ 1);
        TR(2, 1);
        mbar_expect_tx(&q_full[qs], Cfg::Q_BYTES);
#pragma unroll
        for (int a = 0; a < DH / 64; ++a)
          tma_load_4d(sQ + qs * Cfg::Q_BYTES + a * (BQ * 128), &tmQ, &q_full[qs], a * 64, qt * BQ, h, b);
        for (int j = 0; j < ntiles; ++j) {
          mbar_wait(&k_empty[ks], kph ^ 1);
          TR(2, 2);
          mbar_expect_tx(&k_full[ks], Cfg::K_BYTES);
#pragma unroll
          for (int a = 0; a < DH / 64; ++a)
            tma_load_4d(sK + ks * Cfg::K_BYTES + a * (BKV * 128), &tmK, &k_full[ks], a * 64, j * BKV, h, b);
          if (++ks == Cfg::KST) { ks = 0; kph ^= 1; }
          mbar_wait(&v_empty[vs], vph ^ 1);
          TR(2, 3);
          mbar_expect_tx(&v_full[vs], Cfg::V_BYTES);
#pragma unroll
          for (int ka = 0; ka < 2; ++ka)
#pragma unroll
            for (int c = 0; c < DH / 64; ++c)
              tma_load_4d(sV + vs * Cfg::V_BYTES + ka * (DH / 64) * 8192 + c * 8192, &tmV, &v_full[vs], c * 64,
                          j * BKV + ka * 64, h, b);
          if (++vs == Cfg::VST) { vs = 0; vph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ===== MMA issuer =====
      // S = Q K^T: M=128, N=128 (keys), K=DH; both operands K-major.
      const uint32_t idesc_s = make_idesc_f16(128, BKV, 0, 0);
      // O += P V: M=128, N=DH, K=128 keys; P K-major (smem), V MN-major.
      const uint32_t idesc_o = make_idesc_f16(128, DH, 0, 1);
      int ks = 0; uint32_t kph = 0;
      int vs = 0; uint32_t vph = 0;
      int it = 0;  // S-buffer uses
      int pc = 0;  // P-buffer uses
      // Q of item n_ (waits for its TMA load)
      auto q_addr = [&](int n_) {
        const int qs_ = n_ % Cfg::QST;
        mbar_wait(&q_full[qs_], (n_ / Cfg::QST) & 1);
        return smem_u32(sQ + qs_ * Cfg::Q_BYTES);
      };
      auto issue_s = [&](uint32_t qa) {
        const int sb = it & 1;
        mbar_wait(&k_full[ks], kph);
        mbar_wait(&s_empty[sb], ((it >> 1) & 1) ^ 1);
        TR(1, 10);
        tc_fence_after();
        const uint32_t ka = smem_u32(sK + ks * Cfg::K_BYTES);
        if constexpr (DH == 64) {  // one swizzle atom: the four K=16 steps from one asm block
          mma4_bf16(tmem + sb * Cfg::S_COLS, make_sdesc(qa, 16, 1024), make_sdesc(ka, 16, 1024), 2, 2, idesc_s, 0u);
        } else {
#pragma unroll
          for (int kk = 0; kk < DH / 16; ++kk) {
            const int atom = kk / 4, sub = kk % 4;
            uint64_t ad = make_sdesc(qa + atom * (BQ * 128) + sub * 32, 16, 1024);
            uint64_t bd = make_sdesc(ka + atom * (BKV * 128) + sub * 32, 16, 1024);
            mma_bf16(tmem + sb * Cfg::S_COLS, ad, bd, idesc_s, kk ? 1u : 0u);
          }
        }
        mma_commit(&k_empty[ks]);
        mma_commit(&s_full[sb]);
        TR(1, 15);
        if (++ks == Cfg::KST) { ks = 0; kph ^= 1; }
        ++it;
      };
      // score cursor: S is issued two key tiles ahead of O += P V, across item boundaries, as soon
      // as the softmax has read the S buffer it reuses — so when the softmax finishes a tile the
      // scores of the one after next are already in TMEM, and a PV never delays the next scores
      // (the cursor may enter item n + QST - 1 at most: its Q slot is free once item n - 1 is done)
      int s_n = 0, s_item = snake(0), s_j = 0, s_nt = 0, s_cnt = 0;
      uint32_t s_qa = 0;
      auto issue_s_upto = [&](int target, int n_pv) {
        while (s_cnt < target && s_item < items && s_n <= n_pv + Cfg::QST - 1) {
          if (s_j == 0) {
            int b_, h_, qt_;
            fwd_item(s_item, nq, p.H, p.B, b_, h_, qt_);
            s_nt = p.causal ? qt_ + 1 : nq;
            s_qa = q_addr(s_n);
          }
          issue_s(s_qa);
          ++s_cnt;
          if (++s_j == s_nt) { s_j = 0; ++s_n; s_item = snake(s_n); }
        }
      };
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, qt;
        fwd_item(item, nq, p.H, p.B, b, h, qt);
        const int ntiles = p.causal ? qt + 1 : nq;
        const int qs = n % Cfg::QST;
        for (int j = 0; j < ntiles; ++j) {
          issue_s_upto(pc + 3, n);  // scores up to two tiles past this PV's
          const int pb = pc & 1;
          mbar_wait(&v_full[vs], vph);
          if (j == 0) mbar_wait(o_empty, (n & 1) ^ 1);  // the previous item's O has been drained
          const uint32_t pa = tmem + Cfg::P_COL + pb * (BKV / 2);
          const uint32_t va = smem_u32(sV + vs * Cfg::V_BYTES);
          if constexpr (Cfg::SPLIT) {
            // O_h += P[:, 64h .. 64h+63] V[64h .. 64h+63, :], each half as soon as its P is stored
#pragma unroll
            for (int hh = 0; hh < 2; ++hh) {
              mbar_wait(&p_full[pb * 2 + hh], (pc >> 1) & 1);
              if (hh == 0) TR(1, 11);
              tc_fence_after();
#pragma unroll
              for (int sub = 0; sub < 4; ++sub) {
                uint64_t bd = make_sdesc(va + hh * 8192 + sub * 2048, 8192, 1024);
                mma_bf16_ts(tmem + Cfg::O_COL + hh * DH, pa + hh * 32 + sub * 8, bd, idesc_o, (j | sub) ? 1u : 0u);
              }
              mma_commit(&p_empty[pb * 2 + hh]);
            }
          } else {
            mbar_wait(&p_full[pb * 2], (pc >> 1) & 1);
            TR(1, 11);
            tc_fence_after();
#pragma unroll
            for (int kk = 0; kk < BKV / 16; ++kk) {
              const int atom = kk / 4, sub = kk % 4;
              uint64_t bd = make_sdesc(va + atom * (DH / 64) * 8192 + sub * 2048, 8192, 1024);
              mma_bf16_ts(tmem + Cfg::O_COL, pa + kk * 8, bd, idesc_o, (j | kk) ? 1u : 0u);
            }
            mma_commit(&p_empty[pb * 2]);
          }
          mma_commit(&v_empty[vs]);
          TR(1, 14);
          if (++vs == Cfg::VST) { vs = 0; vph ^= 1; }
          ++pc;
        }
        mma_commit(&q_empty[qs]);
        mma_commit(o_full);
      }
    }
    __syncwarp();
  } else {
    // ===== softmax warps: thread = query row; the two warps of a row quadrant split the 128 keys
    // of a tile into halves (= the two 64-key atoms of P) =====
    const int qd = warp & 3;
    const int half = (warp - 2) >> 2;
    const int cb = half * 64;
    const int r = qd * 32 + lane;        // row within the tile
    const uint32_t trow = (uint32_t)(qd * 32) << 16;
    const bool issuer = qd == 0 && lane == 0;  // of this half's TMA store of O
    int it = 0, pc = 0, n = 0, tp = 0;
    // deferred epilogue state: the item whose O is still in TMEM
    bool pend = false;
    int e_n = 0, e_b = 0, e_h = 0, e_qt = 0;
    float e_m = 0.f, e_l = 0.f;
    auto epilogue = [&]() {
      float l = e_l;
      if (issuer) bulk_wait_read<0>();  // the previous item's O store has left the staging boxes
      asm volatile("bar.sync 1, 256;" ::: "memory");  // every thread has read sm_x before it is reused
      sm_x[half][r] = l;
      if constexpr (Cfg::SPLIT) sm_t[0][half][r] = e_m;
      asm volatile("bar.sync 1, 256;" ::: "memory");
      float f0 = 1.f, f1 = 1.f, mrow = e_m;
      if constexpr (Cfg::SPLIT) {
        // combine the two key halves' softmaxes: shift both to the row max (a half with no visible
        // key has m = -inf and l = 0: factor 0)
        const float m0 = sm_t[0][0][r], m1 = sm_t[0][1][r];
        mrow = fmaxf(m0, m1);
        f0 = fast_exp2((m0 - mrow) * p.scale_log2);
        f1 = fast_exp2((m1 - mrow) * p.scale_log2);
        l = sm_x[0][r] * f0 + sm_x[1][r] * f1;
      } else {
        l = sm_x[0][r] + sm_x[1][r];
      }
      const float inv_l = 1.f / l;
      // ---- epilogue: O row (normalised, bf16) -> this half's DH/2 columns in a swizzled staging
      // box (P buffer `half`, free once O is complete) -> TMA store to C; then the LSE
      mbar_wait(o_full, e_n & 1);
      TR(0, 26);
      tc_fence_after();
      float v[DH / 2];
#pragma unroll
      for (int c = 0; c < DH / 2; c += 32) tmem_ld32(tmem + trow + Cfg::O_COL + half * (DH / 2) + c, v + c);
      if constexpr (Cfg::SPLIT) {
        float w[DH / 2];
#pragma unroll
        for (int c = 0; c < DH / 2; c += 32) tmem_ld32(tmem + trow + Cfg::O_COL + DH + half * (DH / 2) + c, w + c);
#pragma unroll
        for (int i = 0; i < DH / 2; ++i) v[i] = v[i] * f0 + w[i] * f1;
      }
      tc_fence_before();
      mbar_arrive_local(o_empty);  // O is in registers: the next item's PV may start
      TR(0, 27);
      // staging: boxes of 64 bf16 columns (128 B rows, 128B swizzle); DH=64: half h -> 32 columns
      // of box 0 (chunks 4h..4h+3); DH=128: half h -> box h
      uint8_t* box = sO + (DH == 64 ? 0 : half * (BQ * 128)) + r * 128;
      const int ch0 = DH == 64 ? half * 4 : 0;
#pragma unroll
      for (int u = 0; u < DH / 16; ++u) {
        uint32_t pk[4];
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          __nv_bfloat162 h2 = __floats2bfloat162_rn(v[8 * u + 2 * t] * inv_l, v[8 * u + 2 * t + 1] * inv_l);
          pk[t] = *reinterpret_cast<uint32_t*>(&h2);
        }
        *reinterpret_cast<uint4*>(box + (((ch0 + u) ^ (r & 7)) << 4)) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      if (DH == 64) {
        asm volatile("bar.sync 1, 256;" ::: "memory");  // both halves wrote the box
        if (half == 0 && issuer) {
          tma_store_4d(&tmC, sO, 0, e_qt * BQ, e_h, e_b);
          bulk_commit();
        }
      } else {
        asm volatile("bar.sync %0, 128;" ::"r"(2 + half) : "memory");
        if (issuer) {
          tma_store_4d(&tmC, sO + half * (BQ * 128), half * 64, e_qt * BQ, e_h, e_b);
          bulk_commit();
        }
      }
      // natural-log LSE of the scaled scores: lse = scale*m + ln(l)
      if (half == 0) p.lse[((int64_t)e_b * p.H + e_h) * p.S + e_qt * BQ + r] = mrow * p.scale + logf(l);
    };
    for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
      int b, h, qt;
      fwd_item(item, nq, p.H, p.B, b, h, qt);
      const int ntiles = p.causal ? qt + 1 : nq;
      const int qrow = qt * BQ + r;  // query index within the sequence
      // ---- one pass over the key tiles (online softmax with lazy rescaling): the row's running
      // max m is raised only when a tile's max exceeds it by more than 8 (log2 units of the
      // scaled scores), so P = 2^((s - m) scale log2e) stays in (0, 256] and O (in TMEM) is
      // rescaled only on those rare raises; O and the row sum l carry the same shift, so O / l and
      // the LSE are the softmax of reading c11 whatever m ends up being.
      float m = -INFINITY;
      float2 l2a = make_float2(0.f, 0.f), l2b = make_float2(0.f, 0.f);  // row-sum partials
      // one key tile; DIAG (the causal diagonal tile) is a compile-time copy of the body, so the
      // other tiles carry no masking instructions at all (masked scores are -inf, whose
      // exponential is exactly 0)
      auto tile = [&](int j, auto diag_tag) {
        constexpr bool DIAG = decltype(diag_tag)::value;
        const int sb = it & 1, pb = pc & 1;
        mbar_wait(&s_full[sb], (it >> 1) & 1);
        TR(0, 20);
        tc_fence_after();
        float v[64];
        tmem_ld64(tmem + trow + sb * Cfg::S_COLS + cb, v);
        tc_fence_before();
        mbar_arrive_local(&s_empty[sb]);  // S is in registers: the MMA may overwrite the buffer
        TR(0, 21);
        if constexpr (DIAG) {
          const int lim = qrow - (j * BKV + cb);  // keys cb + i with i <= lim are visible
#pragma unroll
          for (int i = 0; i < 64; ++i)
            if (i > lim) v[i] = -INFINITY;
        }
        float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
        for (int i = 0; i < 64; ++i) m4[i & 3] = fmaxf(m4[i & 3], v[i]);
        float tm = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3]));
        if constexpr (!Cfg::SPLIT) {
          // the other half of the row (the partner warp of this lane quadrant)
          sm_t[tp][half][r] = tm;
          asm volatile("bar.sync %0, 64;" ::"r"(4 + qd) : "memory");
          tm = fmaxf(tm, sm_t[tp][half ^ 1][r]);
          tp ^= 1;
        }
        TR(0, 22);
        const bool raise = (tm - m) * p.scale_log2 > 8.f;  // true on the first tile (m = -inf)
        float f = 1.f;
        if (raise) {
          f = j == 0 ? 0.f : fast_exp2((m - tm) * p.scale_log2);
          m = tm;
          l2a = make_float2(l2a.x * f, l2a.y * f);
          l2b = make_float2(l2b.x * f, l2b.y * f);
        }
        if (__any_sync(0xffffffffu, raise && j > 0)) {
          // rescale this warp's rows of O once PV_{j-1} has landed: its DH/2 columns of O, or
          // (SPLIT) all of O_half
          const int u = pc - 1;
          mbar_wait(&p_empty[(u & 1) * 2 + (Cfg::SPLIT ? half : 0)], (u >> 1) & 1);
          tc_fence_after();
          constexpr int OC = Cfg::SPLIT ? DH : DH / 2;
          const uint32_t o_base = tmem + trow + Cfg::O_COL + half * OC;
#pragma unroll
          for (int c = 0; c < OC; c += 32) {
            float o[32];
            tmem_ld32(o_base + c, o);
            uint32_t ou[32];
#pragma unroll
            for (int i = 0; i < 32; ++i) ou[i] = __float_as_uint(o[i] * f);
            tmem_st32(o_base + c, ou);
          }
          tmem_wait_st();
        }
        // (SPLIT: a key half with no visible key yet keeps m = -inf; its probabilities are 0)
        const float ms = (Cfg::SPLIT && m == -INFINITY) ? 0.f : m * p.scale_log2;
        uint32_t pk[32];
        const float2 sl2 = make_float2(p.scale_log2, p.scale_log2), nms2 = make_float2(-ms, -ms);
        const float2 one2 = make_float2(1.f, 1.f);
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const float2 x = ffma2(make_float2(v[2 * i], v[2 * i + 1]), sl2, nms2);
          // NPOLY of the 32 pairs take 2^x on the FMA pipe instead of the SFU (A/B variant);
          // the causal diagonal tile keeps ex2 for all, so masked scores give exactly 0
          const bool poly = !DIAG && (i * NPOLY) % 32 < NPOLY;
          const float2 e2 = poly ? exp2_poly2(x) : make_float2(fast_exp2(x.x), fast_exp2(x.y));
          if (i & 1) l2b = ffma2(e2, one2, l2b);
          else l2a = ffma2(e2, one2, l2a);
          __nv_bfloat162 h2 = __floats2bfloat162_rn(e2.x, e2.y);
          pk[i] = *reinterpret_cast<uint32_t*>(&h2);
        }
        TR(0, 23);
        mbar_wait(&p_empty[pb * 2 + (Cfg::SPLIT ? half : 0)], ((pc >> 1) & 1) ^ 1);
        TR(0, 24);
        tc_fence_after();
        // this thread's 64 keys -> 32 TMEM columns (bf16 pairs) of P buffer pb, row = its lane
        tmem_st32(tmem + trow + Cfg::P_COL + pb * (BKV / 2) + half * 32, pk);
        tmem_wait_st();
        tc_fence_before();
        mbar_arrive_local(&p_full[pb * 2 + (Cfg::SPLIT ? half : 0)]);
        TR(0, 25);
        ++it; ++pc;
      };
      // the previous item's epilogue runs after this item's first tile: by then its last PV has
      // landed in O (no wait), and the scores of this tile were computed while that PV ran
      const int nfull = p.causal ? ntiles - 1 : ntiles;
      for (int j = 0; j < nfull; ++j) {
        tile(j, std::false_type{});
        if (j == 0 && pend) { epilogue(); pend = false; }
      }
      if (p.causal) {
        tile(ntiles - 1, std::true_type{});
        if (ntiles == 1 && pend) { epilogue(); pend = false; }
      }
      pend = true;
      e_n = n; e_b = b; e_h = h; e_qt = qt; e_m = m;
      e_l = (l2a.x + l2a.y) + (l2b.x + l2b.y);
    }
    if (pend) epilogue();
    if (issuer) bulk_wait_all();
  }
  TR_END();
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS) : "memory");
  }
}


// ============================================================================================ backward
// One CTA per (128-key tile j, head, sequence), looping over the query tiles i that see it.  With
// M = keys, the CTA keeps dK_j and dV_j in TMEM for the whole loop.  Per query tile:
//   S^T = K_j Q_i^T,  dP^T = V_j dO_i^T                      (TMEM, fp32)
//   P^T = exp(scale S^T - lse_i),  dS^T = scale P^T (dP^T - D_i)   (softmax warps, thread = key)
//   dV_j += P^T dO_i,  dK_j += dS^T Q_i                       (P^T, dS^T from shared memory)
// D_i = rowsum(dO_i . O_i) comes from attn_bwd_prep.  dS^T is also written to global memory so that
// dQ = dS K is one deterministic batched GEMM afterwards (no atomics).  Q_i and dO_i are each
// staged once: their K-major smem tiles double as the MN-major B operands of dK and dV.
template <int DH>
struct BwdCfg {
  static constexpr int KV_BYTES = BKV * DH * 2;   // K_j or V_j
  static constexpr int QT_BYTES = BQ * DH * 2;    // Q_i or dO_i
  static constexpr int ST = DH == 64 ? 2 : 1;     // (Q, dO) stages
  static constexpr int PB = DH == 64 ? 2 : 1;     // (P^T, dS^T) buffers: 2 lets the softmax of tile n+1
                                                  // overlap the dV/dK MMAs of tile n
  static constexpr int PS_BYTES = BKV * BQ * 2;   // P^T or dS^T
  static constexpr int SMEM = 2 * KV_BYTES + ST * 2 * QT_BYTES + PB * 2 * PS_BYTES + 1024 + 512;
  static constexpr int ST_COL = 0, DP_COL = 128, DV_COL = 256, DK_COL = 256 + DH;
  static constexpr int TMEM_COLS = 512;
};

struct BwdParams {
  int S, H, causal;
  float scale;
  float scale_log2;    // scale * log2(e)
  const float* lse2;   // [b, H, S]: -lse * log2(e)
  const float* sD;     // [b, H, S]: -scale * D
  __nv_bfloat16* dqkv; // [b*S, 3d]: dK, dV columns written here
  __nv_bfloat16* dst;  // [b, H, S(keys), S(queries)]: scale * dS^T
  int d;
};

template <int DH>
__global__ void __launch_bounds__(THREADS, 1)
    attn_bwd_kernel(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                    const __grid_constant__ CUtensorMap tmV, const __grid_constant__ CUtensorMap tmdO,
                    const __grid_constant__ CUtensorMap tmdS, BwdParams p) {
  using Cfg = BwdCfg<DH>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sK = smem;
  uint8_t* sV = sK + Cfg::KV_BYTES;
  uint8_t* sQ = sV + Cfg::KV_BYTES;                  // [ST] (Q_i, dO_i)
  uint8_t* sPS = sQ + Cfg::ST * 2 * Cfg::QT_BYTES;   // [PB] (P^T, dS^T)
  uint64_t* bars = reinterpret_cast<uint64_t*>(sPS + Cfg::PB * 2 * Cfg::PS_BYTES);
  uint64_t* kv_full = bars;
  uint64_t* q_full = bars + 1;   // [2]
  uint64_t* q_empty = bars + 3;  // [2]
  uint64_t* s_full = bars + 5;
  uint64_t* p_full = bars + 6;   // [2]: softmax wrote P^T/dS^T buffer and finished reading S^T/dP^T
  uint64_t* p_empty = bars + 8;  // [2]
  uint64_t* kd_full = bars + 10;
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(bars + 11);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int kt = blockIdx.x, h = blockIdx.y, b = blockIdx.z;
  const int k0 = kt * BKV;
  const int nq = p.S / BQ;
  const int i0 = p.causal ? kt : 0;
  const int niter = nq - i0;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); prefetch_tmap(&tmdO); prefetch_tmap(&tmdS);
    mbar_init(kv_full, 1);
    for (int i = 0; i < 2; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    mbar_init(s_full, 1);
    for (int i = 0; i < 2; ++i) { mbar_init(&p_full[i], 256); mbar_init(&p_empty[i], 1); }
    mbar_init(kd_full, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(Cfg::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  if (warp == 0) {
    if (lane == 0) {
      mbar_expect_tx(kv_full, 2 * Cfg::KV_BYTES);
#pragma unroll
      for (int a = 0; a < DH / 64; ++a) {
        tma_load_4d(sK + a * (BKV * 128), &tmK, kv_full, a * 64, k0, h, b);
        tma_load_4d(sV + a * (BKV * 128), &tmV, kv_full, a * 64, k0, h, b);
      }
      int st = 0; uint32_t ph = 0;
      for (int n = 0; n < niter; ++n) {
        const int q0 = (i0 + n) * BQ;
        mbar_wait(&q_empty[st], ph ^ 1);
        mbar_expect_tx(&q_full[st], 2 * Cfg::QT_BYTES);
        uint8_t* q = sQ + st * 2 * Cfg::QT_BYTES;
        uint8_t* o = q + Cfg::QT_BYTES;
#pragma unroll
        for (int a = 0; a < DH / 64; ++a) {
          tma_load_4d(q + a * (BQ * 128), &tmQ, &q_full[st], a * 64, q0, h, b);
          tma_load_4d(o + a * (BQ * 128), &tmdO, &q_full[st], a * 64, q0, h, b);
        }
        if (++st == Cfg::ST) { st = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc_s = make_idesc_f16(128, BQ, 0, 0);   // S^T, dP^T: M=keys, N=queries, K=DH
      const uint32_t idesc_g = make_idesc_f16(128, DH, 0, 1);   // dV, dK: M=keys, N=DH, K=queries
      mbar_wait(kv_full, 0);
      const uint32_t ka = smem_u32(sK), va = smem_u32(sV);
      // order: S_0, dP_0 | for n: [wait P_n] S_{n+1}, dP_{n+1} | dV_n, dK_n — the tensor pipe computes the
      // next scores while the softmax warps are still writing nothing (they wait), then the gradients
      // of tile n run while the softmax warps turn S_{n+1} into P_{n+1} (PB = 2 buffers)
      auto issue_s = [&](int n) {
        const int st = n % Cfg::ST;
        mbar_wait(&q_full[st], (n / Cfg::ST) & 1);
        tc_fence_after();
        const uint32_t qa = smem_u32(sQ + st * 2 * Cfg::QT_BYTES), oa = qa + Cfg::QT_BYTES;
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const int atom = kk / 4, sub = kk % 4;
          const uint32_t off = atom * (128 * 128) + sub * 32;
          mma_bf16(tmem + Cfg::ST_COL, make_sdesc(ka + off, 16, 1024), make_sdesc(qa + off, 16, 1024), idesc_s, kk ? 1u : 0u);
          mma_bf16(tmem + Cfg::DP_COL, make_sdesc(va + off, 16, 1024), make_sdesc(oa + off, 16, 1024), idesc_s, kk ? 1u : 0u);
        }
        mma_commit(s_full);
      };
      issue_s(0);
      for (int n = 0; n < niter; ++n) {
        const int pb = n % Cfg::PB;
        mbar_wait(&p_full[pb], (n / Cfg::PB) & 1);  // P^T/dS^T of tile n written, S/dP TMEM read
        tc_fence_after();
        if (n + 1 < niter && Cfg::PB == 2) issue_s(n + 1);
        const int st = n % Cfg::ST;
        const uint32_t qa = smem_u32(sQ + st * 2 * Cfg::QT_BYTES), oa = qa + Cfg::QT_BYTES;
        const uint32_t pa = smem_u32(sPS + pb * 2 * Cfg::PS_BYTES), da = pa + Cfg::PS_BYTES;
#pragma unroll
        for (int kk = 0; kk < BQ / 16; ++kk) {
          const int atom = kk / 4, sub = kk % 4;
          const uint32_t aoff = atom * (128 * 128) + sub * 32;  // P^T / dS^T: K-major (K = queries)
          const uint32_t boff = kk * 2048;                      // dO / Q as MN-major B (k = query rows)
          const uint32_t acc = (n | kk) ? 1u : 0u;
          mma_bf16(tmem + Cfg::DV_COL, make_sdesc(pa + aoff, 16, 1024), make_sdesc(oa + boff, 128 * 128, 1024), idesc_g, acc);
          mma_bf16(tmem + Cfg::DK_COL, make_sdesc(da + aoff, 16, 1024), make_sdesc(qa + boff, 128 * 128, 1024), idesc_g, acc);
        }
        mma_commit(&p_empty[pb]);
        mma_commit(&q_empty[st]);
        if (n + 1 < niter && Cfg::PB == 1) issue_s(n + 1);
      }
      mma_commit(kd_full);
    }
    __syncwarp();
  } else {
    const int qd = warp & 3;
    const int half = (warp - 2) >> 2;  // which 64 queries of the tile (= which atom of P^T / dS^T)
    const int r = qd * 32 + lane;   // key row within the tile
    const int key = k0 + r;
    const uint32_t trow = (uint32_t)(qd * 32) << 16;
    const float* lse2 = p.lse2 + ((int64_t)b * p.H + h) * p.S;
    const float* sDv = p.sD + ((int64_t)b * p.H + h) * p.S;
    // this half's dS^T atom goes to global by one TMA store (the smem tile is already in the
    // 128B-swizzled layout of a (64 queries x 128 keys) box); its issuer is lane 0 of quadrant 0
    const bool issuer = qd == 0 && lane == 0;
    for (int n = 0; n < niter; ++n) {
      const int q0 = (i0 + n) * BQ;
      const int pb = n % Cfg::PB;
      mbar_wait(s_full, n & 1);
      mbar_wait(&p_empty[pb], ((n / Cfg::PB) & 1) ^ 1);
      tc_fence_after();
      const bool diag = p.causal && (i0 + n) == kt;
      if (Cfg::PB == 1) {  // single buffer: the previous tile's dS^T store must have left it
        if (issuer) bulk_wait_read<0>();
        asm volatile("bar.sync %0, 128;" ::"r"(2 + half) : "memory");
      }
      uint8_t* prow = sPS + pb * 2 * Cfg::PS_BYTES + half * (128 * 128) + r * 128;
      uint8_t* drow = prow + Cfg::PS_BYTES;
#pragma unroll 1
      for (int c = 0; c < 64; c += 32) {
        const int qc = q0 + half * 64 + c;  // first query of this 32-column batch
        // per-query statistics (same for every thread: L1 broadcast), loaded ahead of the TMEM reads
        float l2[32], sd[32];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          const float4 a4 = __ldg(reinterpret_cast<const float4*>(lse2 + qc) + i);
          const float4 d4 = __ldg(reinterpret_cast<const float4*>(sDv + qc) + i);
          l2[4 * i] = a4.x; l2[4 * i + 1] = a4.y; l2[4 * i + 2] = a4.z; l2[4 * i + 3] = a4.w;
          sd[4 * i] = d4.x; sd[4 * i + 1] = d4.y; sd[4 * i + 2] = d4.z; sd[4 * i + 3] = d4.w;
        }
        uint32_t rs[32], rd[32];
        tmem_ld32_nw(tmem + trow + Cfg::ST_COL + half * 64 + c, rs);
        tmem_ld32_nw(tmem + trow + Cfg::DP_COL + half * 64 + c, rd);
        tmem_wait_ld();
        uint32_t pk[16], dk[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          float pr[2], dr[2];
#pragma unroll
          for (int u = 0; u < 2; ++u) {
            const int e = 2 * i + u;
            float pv = fast_exp2(fmaf(__uint_as_float(rs[e]), p.scale_log2, l2[e]));
            if (diag && key > qc + e) pv = 0.f;
            pr[u] = pv;
            dr[u] = pv * fmaf(__uint_as_float(rd[e]), p.scale, sd[e]);
          }
          __nv_bfloat162 a2 = __floats2bfloat162_rn(pr[0], pr[1]);
          __nv_bfloat162 b2 = __floats2bfloat162_rn(dr[0], dr[1]);
          pk[i] = *reinterpret_cast<uint32_t*>(&a2);
          dk[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        const int ch0 = c / 8;  // 16-byte chunk of the 128-byte row
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const int sw = ((ch0 + u) ^ (r & 7)) << 4;
          *reinterpret_cast<uint4*>(prow + sw) = make_uint4(pk[4 * u], pk[4 * u + 1], pk[4 * u + 2], pk[4 * u + 3]);
          *reinterpret_cast<uint4*>(drow + sw) = make_uint4(dk[4 * u], dk[4 * u + 1], dk[4 * u + 2], dk[4 * u + 3]);
        }
      }
      tc_fence_before();
      if (issuer) bulk_wait_read<0>();  // the previous tile's dS^T store has left shared memory
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive_local(&p_full[pb]);
      asm volatile("bar.sync %0, 128;" ::"r"(2 + half) : "memory");  // the half's 128 rows are written
      if (issuer) {
        tma_store_4d(&tmdS, sPS + pb * 2 * Cfg::PS_BYTES + Cfg::PS_BYTES + half * (128 * 128), q0 + half * 64, k0, h, b);
        bulk_commit();
      }
    }
    if (issuer) bulk_wait_all();
    // epilogue: dV_j, dK_j rows -> dQKV (bf16)
    mbar_wait(kd_full, 0);
    tc_fence_after();
    __nv_bfloat16* base = p.dqkv + ((int64_t)b * p.S + key) * 3 * p.d + h * DH;
    {
      const int part = half;  // half 0 drains dV, half 1 dK
      __nv_bfloat16* out = base + (part == 0 ? 2 * p.d : p.d);  // dV, then dK
      const int col = part == 0 ? Cfg::DV_COL : Cfg::DK_COL;
#pragma unroll 1
      for (int c = 0; c < DH; c += 16) {
        float v[16];
        tmem_ld16(tmem + trow + col + c, v);
        uint32_t pk[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          __nv_bfloat162 h2 = __floats2bfloat162_rn(v[2 * i], v[2 * i + 1]);
          pk[i] = *reinterpret_cast<uint32_t*>(&h2);
        }
        uint4* dst = reinterpret_cast<uint4*>(out + c);
        dst[0] = make_uint4(pk[0], pk[1], pk[2], pk[3]);
        dst[1] = make_uint4(pk[4], pk[5], pk[6], pk[7]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS) : "memory");
  }
}

// ------------------------------------------------------------------ persistent backward (dh = 64)
// Same per-element mathematics as attn_bwd_kernel; one CTA per SM loops over the (key tile, head,
// sequence) items, and each item over 64-query sub-tiles, with every pipeline counter running on
// across items.  TMEM holds TWO S^T / dP^T buffer pairs (128 keys x 64 queries each), so the MMA
// computes the scores of sub-tile g+2 while the softmax warps turn sub-tile g+1 into P^T / dS^T:
//   MMA:     S(0) S(1) | per g: [wait P(g)] dV += P^T(g) dO, dK += dS^T(g) Q, S(g+2)
//   softmax: per g: [wait S(g)] P^T -> TMEM (A operand of dV), dS^T -> smem (A operand of dK and
//            the source of its TMA store for the deterministic dQ GEMM)
// K_j / V_j are double-buffered (the next item's load overlaps the current one), (Q_i, dO_i, the
// sub-tile's statistics) run in a 4-deep ring, and dK / dV drain with their own full / empty
// barriers so the next item's scores start while they are written out.
struct BwdPCfg {
  static constexpr int DH = 64;
  static constexpr int BQS = 64;                  // queries per sub-tile
  static constexpr int KV_BYTES = BKV * DH * 2;   // K_j or V_j
  static constexpr int QT_BYTES = BQS * DH * 2;   // Q_i or dO_i sub-tile
  static constexpr int KVST = 2, QST = 4, DSB = 2;
  static constexpr int DS_BYTES = BKV * BQS * 2;  // dS^T sub-tile (128 keys x 128 B)
  static constexpr int STAT_BYTES = 2 * BQS * 4;  // lse2 and sD of a sub-tile
  static constexpr int SMEM = KVST * 2 * KV_BYTES + QST * (2 * QT_BYTES + STAT_BYTES) + DSB * DS_BYTES + 1024 + 256;
  static constexpr int ST_COL = 0, DP_COL = 2 * BQS, DV_COL = 4 * BQS, DK_COL = 4 * BQS + DH, PT_COL = 4 * BQS + 2 * DH;
  static constexpr int TMEM_COLS = 512;
  static_assert(PT_COL + 2 * (BQS / 2) <= TMEM_COLS, "TMEM columns");
  static_assert(SMEM <= 232448, "shared memory per CTA");
};

// sorted item -> (sequence, head, key tile); causal: small key tiles see the most query tiles
__device__ __forceinline__ void bwd_item(int item, int nk, int H, int B, int& b, int& h, int& kt) {
  const int hb = H * B;
  kt = item / hb;
  const int rem = item % hb;
  h = rem % H;
  b = rem / H;
}

template <bool ALT>
__global__ void __launch_bounds__(THREADS, 1)
    attn_bwd_persistent(const __grid_constant__ CUtensorMap tmQ, const __grid_constant__ CUtensorMap tmK,
                        const __grid_constant__ CUtensorMap tmV, const __grid_constant__ CUtensorMap tmdO,
                        const __grid_constant__ CUtensorMap tmdS, BwdParams p, int B) {
  using Cfg = BwdPCfg;
  constexpr int DH = Cfg::DH, BQS = Cfg::BQS;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sKV = smem;                                   // [KVST] (K_j, V_j)
  uint8_t* sQ = sKV + Cfg::KVST * 2 * Cfg::KV_BYTES;     // [QST] (Q_i, dO_i)
  uint8_t* sDS = sQ + Cfg::QST * 2 * Cfg::QT_BYTES;      // [DSB] dS^T
  float* sStat = reinterpret_cast<float*>(sDS + Cfg::DSB * Cfg::DS_BYTES);  // [QST] (lse2[BQS], sD[BQS])
  uint64_t* bars = reinterpret_cast<uint64_t*>(reinterpret_cast<uint8_t*>(sStat) + Cfg::QST * Cfg::STAT_BYTES);
  uint64_t* kv_full = bars;          // [2]
  uint64_t* kv_empty = bars + 2;     // [2]
  uint64_t* q_full = bars + 4;       // [QST]
  uint64_t* q_empty = bars + 8;      // [QST]
  uint64_t* s_full = bars + 12;      // [2]: S^T / dP^T buffer pair written by the MMA
  uint64_t* p_full = bars + 14;      // [2]: P^T in TMEM, dS^T in smem, S^T / dP^T pair read
  uint64_t* p_empty = bars + 16;     // [2]: dV / dK MMAs of the buffer's sub-tile done
  uint64_t* kd_full = bars + 18;
  uint64_t* kd_empty = bars + 19;
  uint32_t* tmem_base_s = reinterpret_cast<uint32_t*>(bars + 20);

  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  const int nk = p.S / BKV, nqs = p.S / BQS;
  const int items = nk * p.H * B;

  if (warp == 0 && lane == 0) {
    prefetch_tmap(&tmQ); prefetch_tmap(&tmK); prefetch_tmap(&tmV); prefetch_tmap(&tmdO); prefetch_tmap(&tmdS);
    for (int i = 0; i < 2; ++i) {
      mbar_init(&kv_full[i], 1); mbar_init(&kv_empty[i], 1);
      mbar_init(&s_full[i], 1);
      mbar_init(&p_full[i], ALT ? 128 : 256); mbar_init(&p_empty[i], 1);
    }
    for (int i = 0; i < Cfg::QST; ++i) { mbar_init(&q_full[i], 1); mbar_init(&q_empty[i], 1); }
    mbar_init(kd_full, 1); mbar_init(kd_empty, 256);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_base_s)),
                 "r"(Cfg::TMEM_COLS) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_base_s;
  pdl_wait();  // (after the setup, which touches no global data: it overlaps the previous kernel's tail)

  if (warp == 0) {
    if (lane == 0) {
      int qs = 0; uint32_t qph = 0;
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, kt;
        bwd_item(item, nk, p.H, B, b, h, kt);
        const int i0 = p.causal ? kt * (BKV / BQS) : 0;
        const int kvs = n & 1;
        mbar_wait(&kv_empty[kvs], ((n >> 1) & 1) ^ 1);
        mbar_expect_tx(&kv_full[kvs], 2 * Cfg::KV_BYTES);
        uint8_t* kb = sKV + kvs * 2 * Cfg::KV_BYTES;
        tma_load_4d(kb, &tmK, &kv_full[kvs], 0, kt * BKV, h, b);
        tma_load_4d(kb + Cfg::KV_BYTES, &tmV, &kv_full[kvs], 0, kt * BKV, h, b);
        for (int i = i0; i < nqs; ++i) {
          mbar_wait(&q_empty[qs], qph ^ 1);
          mbar_expect_tx(&q_full[qs], 2 * Cfg::QT_BYTES + Cfg::STAT_BYTES);
          uint8_t* q = sQ + qs * 2 * Cfg::QT_BYTES;
          tma_load_4d(q, &tmQ, &q_full[qs], 0, i * BQS, h, b);
          tma_load_4d(q + Cfg::QT_BYTES, &tmdO, &q_full[qs], 0, i * BQS, h, b);
          // the sub-tile's per-query statistics (lse2, sD: 256 B each) ride on the same barrier
          const int64_t so = ((int64_t)b * p.H + h) * p.S + i * BQS;
          float* st = sStat + qs * (2 * BQS);
          bulk_load_1d(st, p.lse2 + so, BQS * 4, &q_full[qs]);
          bulk_load_1d(st + BQS, p.sD + so, BQS * 4, &q_full[qs]);
          if (++qs == Cfg::QST) { qs = 0; qph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc_s = make_idesc_f16(128, BQS, 0, 0);  // S^T, dP^T: M=keys, N=queries, K=DH
      const uint32_t idesc_g = make_idesc_f16(128, DH, 0, 1);   // dV, dK: M=keys, N=DH, K=queries
      // score-issue cursor (runs two sub-tiles ahead of the gradient cursor, across items)
      int s_item = snake(0), s_sub = 0, s_n = 0;
      int qs = 0; uint32_t qph = 0;  // (Q, dO) ring position of the next score issue
      int sc = 0;                    // score issues (buffer pair sc & 1)
      auto issue_s = [&]() {
        if (s_item >= items) return;
        int b, h, kt;
        bwd_item(s_item, nk, p.H, B, b, h, kt);
        const int nt = nqs - (p.causal ? kt * (BKV / BQS) : 0);
        const int kvs = s_n & 1;
        if (s_sub == 0) mbar_wait(&kv_full[kvs], (s_n >> 1) & 1);
        mbar_wait(&q_full[qs], qph);
        tc_fence_after();
        const uint32_t ka = smem_u32(sKV + kvs * 2 * Cfg::KV_BYTES), va = ka + Cfg::KV_BYTES;
        const uint32_t qa = smem_u32(sQ + qs * 2 * Cfg::QT_BYTES), oa = qa + Cfg::QT_BYTES;
        const int sb = sc & 1;
#pragma unroll
        for (int kk = 0; kk < DH / 16; ++kk) {
          const uint32_t off = kk * 32;
          mma_bf16(tmem + Cfg::ST_COL + sb * BQS, make_sdesc(ka + off, 16, 1024), make_sdesc(qa + off, 16, 1024),
                   idesc_s, kk ? 1u : 0u);
          mma_bf16(tmem + Cfg::DP_COL + sb * BQS, make_sdesc(va + off, 16, 1024), make_sdesc(oa + off, 16, 1024),
                   idesc_s, kk ? 1u : 0u);
        }
        mma_commit(&s_full[sb]);
        if (++qs == Cfg::QST) { qs = 0; qph ^= 1; }
        ++sc;
        if (++s_sub == nt) { s_sub = 0; s_item = snake(s_n + 1); ++s_n; }
      };
      issue_s();
      issue_s();
      int gq = 0;  // (Q, dO) ring position of the next dV/dK
      int pc = 0;  // sub-tiles whose gradients were issued (P/dS buffer pc & 1)
      int n = 0;
      for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
        int b, h, kt;
        bwd_item(item, nk, p.H, B, b, h, kt);
        const int nt = nqs - (p.causal ? kt * (BKV / BQS) : 0);
        const int kvs = n & 1;
        for (int t = 0; t < nt; ++t) {
          const int pb = pc & 1;
          mbar_wait(&p_full[pb], (pc >> 1) & 1);  // P^T / dS^T of this sub-tile ready, its S^T / dP^T read
          if (t == 0) mbar_wait(kd_empty, (n & 1) ^ 1);  // previous item's dK / dV drained
          tc_fence_after();
          const uint32_t qa = smem_u32(sQ + gq * 2 * Cfg::QT_BYTES), oa = qa + Cfg::QT_BYTES;
          const uint32_t pa = tmem + Cfg::PT_COL + pb * (BQS / 2);
          const uint32_t da = smem_u32(sDS + pb * Cfg::DS_BYTES);
#pragma unroll
          for (int kk = 0; kk < BQS / 16; ++kk) {
            const uint32_t boff = kk * 2048;  // dO / Q as MN-major B (k = query rows)
            const uint32_t acc = (t | kk) ? 1u : 0u;
            mma_bf16_ts(tmem + Cfg::DV_COL, pa + kk * 8, make_sdesc(oa + boff, 128 * 128, 1024), idesc_g, acc);
            mma_bf16(tmem + Cfg::DK_COL, make_sdesc(da + kk * 32, 16, 1024), make_sdesc(qa + boff, 128 * 128, 1024),
                     idesc_g, acc);
          }
          mma_commit(&p_empty[pb]);
          mma_commit(&q_empty[gq]);
          if (++gq == Cfg::QST) gq = 0;
          ++pc;
          if (t == nt - 1) {
            mma_commit(&kv_empty[kvs]);
            mma_commit(kd_full);
          }
          issue_s();  // the scores two sub-tiles ahead go into the pair this sub-tile just released
        }
      }
    }
    __syncwarp();
  } else {
    const int qd = warp & 3;
    const int half = (warp - 2) >> 2;  // which 32 queries of the sub-tile
    const int r = qd * 32 + lane;      // key row within the tile
    const uint32_t trow = (uint32_t)(qd * 32) << 16;
    const bool issuer = half == 0 && lane == 0;  // of this lane quadrant's dS^T store
    int g = 0, n = 0;
    int qsl = 0;        // (Q, dO, statistics) ring position of the current sub-tile
    uint32_t qslph = 0; // its phase
    for (int item = snake(0); item < items; item = snake(n + 1), ++n) {
      int b, h, kt;
      bwd_item(item, nk, p.H, B, b, h, kt);
      const int i0 = p.causal ? kt * (BKV / BQS) : 0;
      const int nt = nqs - i0;
      const int key = kt * BKV + r;
      for (int t = 0; t < nt; ++t, ++g) {
        const int cur = qsl;  // this sub-tile's (Q, dO, statistics) ring slot
        const uint32_t curph = qslph;
        if (++qsl == Cfg::QST) { qsl = 0; qslph ^= 1; }
        const int buf = g & 1;
        // ALT: the two warps of a lane quadrant take alternate sub-tiles (half h: buffer pair h), all 64
        // queries each, so on every SM sub-partition one warp reads scores from TMEM while the other
        // exponentiates; otherwise both take the same sub-tile, 32 queries each
        if (ALT && buf != half) continue;
        mbar_wait(&q_full[cur], curph);  // the TMA-written statistics are visible to this thread
        const int q0 = (i0 + t) * BQS;
        mbar_wait(&s_full[buf], (g >> 1) & 1);
        tc_fence_after();
        const bool diag = p.causal && q0 < kt * BKV + BKV;  // the sub-tile overlaps the key range
        if (ALT && lane == 0) bulk_wait_read<0>();  // this warp's store of sub-tile g-2 left the dS^T buffer
        bool waited_empty = false;
#pragma unroll 1
        for (int c = ALT ? 0 : half * 32; c < (ALT ? 64 : half * 32 + 32); c += 32) {
        const float* sl2 = sStat + cur * (2 * BQS) + c;
        const float* ssd = sl2 + BQS;
        const int qc = q0 + c;  // first query of this thread's 32 columns
        uint32_t rs[32], rd[32];
        tmem_ld32_nw(tmem + trow + Cfg::ST_COL + buf * BQS + c, rs);
        tmem_ld32_nw(tmem + trow + Cfg::DP_COL + buf * BQS + c, rd);
        float2 l2[16], sd[16];  // broadcast reads of the staged statistics (-lse2, -sD), in pairs
#pragma unroll
        for (int i = 0; i < 8; ++i) {
          float4 a4, d4;
          asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(a4.x), "=f"(a4.y), "=f"(a4.z), "=f"(a4.w)
                       : "r"(smem_u32(sl2) + 16 * i));
          asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(d4.x), "=f"(d4.y), "=f"(d4.z), "=f"(d4.w)
                       : "r"(smem_u32(ssd) + 16 * i));
          l2[2 * i] = make_float2(a4.x, a4.y); l2[2 * i + 1] = make_float2(a4.z, a4.w);
          sd[2 * i] = make_float2(d4.x, d4.y); sd[2 * i + 1] = make_float2(d4.z, d4.w);
        }
        tmem_wait_ld();
        if (diag) {  // keys after the query: score -inf, so P = 0 and dS = 0 exactly
#pragma unroll
          for (int e = 0; e < 32; ++e)
            if (key > qc + e) rs[e] = __float_as_uint(-INFINITY);
        }
        uint32_t pk[16], dk[16];
        const float2 sl2v = make_float2(p.scale_log2, p.scale_log2), sc2 = make_float2(p.scale, p.scale);
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          // P = 2^(s scale log2e - lse2); dS = P (dp scale - sD): three packed FP ops per pair
          const float2 x = ffma2(make_float2(__uint_as_float(rs[2 * i]), __uint_as_float(rs[2 * i + 1])), sl2v, l2[i]);
          const float2 pv = make_float2(fast_exp2(x.x), fast_exp2(x.y));
          const float2 t = ffma2(make_float2(__uint_as_float(rd[2 * i]), __uint_as_float(rd[2 * i + 1])), sc2, sd[i]);
          const float2 dr = fmul2(pv, t);
          __nv_bfloat162 a2 = __floats2bfloat162_rn(pv.x, pv.y);
          __nv_bfloat162 b2 = __floats2bfloat162_rn(dr.x, dr.y);
          pk[i] = *reinterpret_cast<uint32_t*>(&a2);
          dk[i] = *reinterpret_cast<uint32_t*>(&b2);
        }
        // the P^T / dS^T buffers are free once the dV / dK MMAs of sub-tile g-2 are done (waited only
        // now, so the score loads and the exponentials above overlap those MMAs)
        if (!waited_empty) {
          mbar_wait(&p_empty[buf], ((g >> 1) & 1) ^ 1);
          tc_fence_after();
          waited_empty = true;
        }
        // P^T: this thread's 32 queries -> 16 TMEM columns (bf16 pairs) of P buffer `buf`
        asm volatile(
            "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
                tmem + trow + Cfg::PT_COL + buf * (BQS / 2) + c / 2),
            "r"(pk[0]), "r"(pk[1]), "r"(pk[2]), "r"(pk[3]), "r"(pk[4]), "r"(pk[5]), "r"(pk[6]), "r"(pk[7]), "r"(pk[8]),
            "r"(pk[9]), "r"(pk[10]), "r"(pk[11]), "r"(pk[12]), "r"(pk[13]), "r"(pk[14]), "r"(pk[15])
            : "memory");
        // dS^T: the row's 16-byte chunks c/8 .. c/8+3 of the 128-byte (64-query) row, swizzled
        if (ALT && c == 0) __syncwarp();  // lane 0's wait for the buffer's previous store precedes every write
        const uint32_t drow = smem_u32(sDS + buf * Cfg::DS_BYTES + r * 128);
#pragma unroll
        for (int u = 0; u < 4; ++u)
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(drow + (((c / 8 + u) ^ (r & 7)) << 4)),
                       "r"(dk[4 * u]), "r"(dk[4 * u + 1]), "r"(dk[4 * u + 2]), "r"(dk[4 * u + 3])
                       : "memory");
        }
        tmem_wait_st();
        tc_fence_before();
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        mbar_arrive_local(&p_full[buf]);
        if (ALT) {
          // the warp wrote its quadrant's 32 keys x 64 queries: one TMA store from lane 0
          __syncwarp();
          if (lane == 0) {
            tma_store_4d(&tmdS, sDS + buf * Cfg::DS_BYTES + qd * 32 * 128, q0, kt * BKV + qd * 32, h, b);
            bulk_commit();
          }
        } else {
          // this lane quadrant's 32 keys x 64 queries are written (both halves): one TMA store per
          // quadrant, synchronised by the quadrant's two warps only.  The quadrant's store of the
          // sub-tile two back (same buffer) was waited for before the previous instance of this
          // barrier, so its rows were free when they were written above.
          if (issuer) bulk_wait_read<0>();
          asm volatile("bar.sync %0, 64;" ::"r"(4 + qd) : "memory");
          if (issuer) {
            tma_store_4d(&tmdS, sDS + buf * Cfg::DS_BYTES + qd * 32 * 128, q0, kt * BKV + qd * 32, h, b);
            bulk_commit();
          }
        }
      }
      // epilogue: dV_j (half 0) / dK_j (half 1) rows -> dQKV (bf16)
      mbar_wait(kd_full, n & 1);
      tc_fence_after();
      float v[DH];
      tmem_ld64(tmem + trow + (half == 0 ? Cfg::DV_COL : Cfg::DK_COL), v);
      tc_fence_before();
      mbar_arrive_local(kd_empty);  // accumulators in registers: the next item may overwrite them
      __nv_bfloat16* out = p.dqkv + ((int64_t)b * p.S + key) * 3 * p.d + h * DH + (half == 0 ? 2 * p.d : p.d);
#pragma unroll
      for (int c = 0; c < DH; c += 8) {
        uint32_t pk[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          __nv_bfloat162 h2 = __floats2bfloat162_rn(v[c + 2 * i], v[c + 2 * i + 1]);
          pk[i] = *reinterpret_cast<uint32_t*>(&h2);
        }
        *reinterpret_cast<uint4*>(out + c) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
    }
    if (ALT ? lane == 0 : issuer) bulk_wait_all();
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(Cfg::TMEM_COLS) : "memory");
  }
}

// sD[b, h, q] = -scale * sum_e dO[b*S+q][h*dh+e] * O[b*S+q][h*dh+e] and lse2 = -lse * log2(e): the
// per-query terms of dS = P (dP - D) in the forms the backward's FFMAs take.  One thread per 8
// consecutive elements of the [tokens, d] rows (one 16-byte load of dO and of O, fully coalesced,
// a few registers, so the grid is many small resident blocks); each head's dh/8 adjacent lanes
// reduce their 8-term partial sums with shuffles in a fixed order.
__global__ void __launch_bounds__(256) attn_bwd_prep(int64_t ntok, int S, int H, int dh, float scale,
                                                     const __nv_bfloat16* __restrict__ dO,
                                                     const __nv_bfloat16* __restrict__ O, const float* __restrict__ lse,
                                                     float* __restrict__ sD, float* __restrict__ lse2) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int d = H * dh, lph = dh / 8;  // lanes per head (8 or 16: a head never straddles a warp)
  const int64_t v = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;  // 8-element vector index
  const int64_t nvec = ntok * (d / 8);
  const bool in = v < nvec;
  const int64_t tok = in ? v / (d / 8) : 0;
  const int e = in ? (int)(v - tok * (d / 8)) * 8 : 0;
  float s = 0.f;
  if (in) {
    const uint4 xa = __ldg(reinterpret_cast<const uint4*>(dO) + v);
    const uint4 ya = __ldg(reinterpret_cast<const uint4*>(O) + v);
    const __nv_bfloat162* xp = reinterpret_cast<const __nv_bfloat162*>(&xa);
    const __nv_bfloat162* yp = reinterpret_cast<const __nv_bfloat162*>(&ya);
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      const float2 fx = __bfloat1622float2(xp[k]), fy = __bfloat1622float2(yp[k]);
      s += fx.x * fy.x + fx.y * fy.y;
    }
  }
  for (int w = lph / 2; w > 0; w >>= 1) s += __shfl_xor_sync(0xffffffffu, s, w);
  if (in && (threadIdx.x % lph) == 0) {
    const int h = e / dh;
    const int64_t bseq = tok / S, q = tok % S;
    const int64_t i = (bseq * H + h) * S + q;
    sD[i] = -(scale * s);                     // -scale * D
    lse2[i] = -(lse[i] * 1.4426950408889634f);  // -lse * log2(e)
  }
}
}  // namespace attn

// Returns false when the fused path does not apply (then the caller uses GEMM + softmax + GEMM).
bool attention_fwd_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, void* C, float* lse,
                         cudaStream_t st) {
  using namespace attn;
  if (S % BQ != 0 || (dh != 64 && dh != 128)) return false;
  {  // HARMONY_ATTN_FWD=2: the two-query-tile kernel for dh = 64 (an A/B alternative, attention_fwd2.cu)
    static const int which = [] {
      const char* v = getenv("HARMONY_ATTN_FWD");
      return v ? atoi(v) : 1;
    }();
    if (which == 2 && attention_fwd2_fused(b, S, H, dh, causal, QKV, C, lse, st)) return true;
  }
  const int d = H * dh;
  CUtensorMap mq, mk, mv, mc;
  // Q, K: K-major operands (inner = dh, rows = S, z0 = head, z1 = sequence); V: MN-major (inner = dh)
  tcx::make_map_4d(&mq, QKV, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BQ);
  tcx::make_map_4d(&mk, static_cast<const __nv_bfloat16*>(QKV) + d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BKV);
  tcx::make_map_4d(&mv, static_cast<const __nv_bfloat16*>(QKV) + 2 * d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64,
                   64);
  // C [b*S][d], head h in columns h*dh..: stored in (64 columns x 128 rows) boxes
  tcx::make_map_4d(&mc, C, dh, S, H, b, d, dh, (int64_t)S * d, 64, BQ);
  FwdParams p;
  p.S = S; p.H = H; p.B = (int)b; p.causal = causal;
  p.scale = 1.0f / std::sqrt((float)dh);
  p.scale_log2 = p.scale * 1.4426950408889634f;
  p.lse = lse;
  static int num_sms = 0;
  if (!num_sms) {
    int dev = 0;
    HM_CUDA(cudaGetDevice(&dev));
    HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
  }
  const int64_t items = (int64_t)(S / BQ) * H * b;
  dim3 grid((unsigned)std::min<int64_t>(items, num_sms));  // persistent
  const int e0 = g_prof.begin(st);
  // pairs of exponentials (of 32 per thread and tile) computed on the FMA pipe instead of the SFU;
  // HARMONY_ATTN_POLY = 8 / 12 / 16 for A/B runs (measured 78.7 / 79.1 / 82.3 us against 77.9 with
  // none: the exponentials are not what paces the tile)
  static const int npoly = [] {
    const char* v = getenv("HARMONY_ATTN_POLY");
    const int k = v ? atoi(v) : 0;
    return (k == 8 || k == 12 || k == 16) ? k : 0;
  }();
  static bool attr_set[5] = {false, false, false, false, false};  // per kernel variant
  auto launch = [&](int variant, auto kern, int smem) {
    if (!attr_set[variant]) {
      HM_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
      attr_set[variant] = true;
    }
    launch_k(kern, dim3(grid), dim3(THREADS), smem, st, mq, mk, mv, mc, p);
  };
  if (dh == 64) {
    if (npoly == 8) launch(1, attn_fwd_kernel<64, 8>, FwdCfg<64>::SMEM);
    else if (npoly == 12) launch(3, attn_fwd_kernel<64, 12>, FwdCfg<64>::SMEM);
    else if (npoly == 16) launch(2, attn_fwd_kernel<64, 16>, FwdCfg<64>::SMEM);
    else launch(0, attn_fwd_kernel<64, 0>, FwdCfg<64>::SMEM);
  } else {
    launch(4, attn_fwd_kernel<128, 0>, FwdCfg<128>::SMEM);
  }
  check_launch("attn_fwd_kernel");
  // algorithmic FLOPs of the attention contractions (QK^T and PV, causal or not)
  g_prof.end(PROF_ATTN, e0, st, 4.0 * b * H * (double)S * S * dh);
  return true;
}


size_t attention_bwd_scratch_bytes(int64_t b, int S, int H) {
  return align_up((uint64_t)b * H * S * S * 2, 256) + 2 * align_up((uint64_t)b * H * S * 4, 256);
}

// Fused attention backward: dQKV (bf16 [b*S, 3d]) from QKV, O (= C), dO (= dC), lse.
bool attention_bwd_fused(int64_t b, int S, int H, int dh, int causal, const void* QKV, const void* O, const void* dO,
                         const float* lse, void* dQKV, void* scratch, cudaStream_t st) {
  using namespace attn;
  if (S % BQ != 0 || (dh != 64 && dh != 128)) return false;
  const int d = H * dh;
  uint8_t* sc = static_cast<uint8_t*>(scratch);
  __nv_bfloat16* dst = reinterpret_cast<__nv_bfloat16*>(sc);
  float* sD = reinterpret_cast<float*>(sc + align_up((uint64_t)b * H * S * S * 2, 256));
  float* lse2 = sD + align_up((uint64_t)b * H * S * 4, 256) / 4;
  const float scale = 1.0f / std::sqrt((float)dh);
  const int e0 = g_prof.begin(st);
  launch_k(attn_bwd_prep, dim3((unsigned)ceil_div(b * S * (d / 8), 256)), dim3(256), 0, st, b * S, S, H, dh, scale, static_cast<const __nv_bfloat16*>(dO),
                                                             static_cast<const __nv_bfloat16*>(O), lse, sD, lse2);
  check_launch("attn_bwd_prep");
  if (causal) HM_CUDA(cudaMemsetAsync(dst, 0, (size_t)b * H * S * S * 2, st));  // key tiles never visited by a query tile
  CUtensorMap mq, mk, mv, mo, mds;
  const __nv_bfloat16* q = static_cast<const __nv_bfloat16*>(QKV);
  // dS^T [b][H][S keys][S queries]: stored from the kernel's swizzled (64 queries x 128 keys) atoms
  tcx::make_map_4d(&mds, dst, S, S, H, b, S, (int64_t)S * S, (int64_t)H * S * S, 64, BKV);
  tcx::make_map_4d(&mq, q, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BQ);
  tcx::make_map_4d(&mk, q + d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BKV);
  tcx::make_map_4d(&mv, q + 2 * d, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BKV);
  tcx::make_map_4d(&mo, dO, dh, S, H, b, d, dh, (int64_t)S * d, 64, BQ);
  BwdParams p;
  p.S = S; p.H = H; p.causal = causal;
  p.scale = scale;
  p.scale_log2 = scale * 1.4426950408889634f;
  p.lse2 = lse2; p.sD = sD;
  p.dqkv = static_cast<__nv_bfloat16*>(dQKV);
  p.dst = dst;
  p.d = d;
  dim3 grid((unsigned)(S / BKV), (unsigned)H, (unsigned)b);
  if (dh == 64) {
    // HARMONY_ATTN_BWD_ALT=1 alternates sub-tiles between the two warps of a lane quadrant (each
    // takes all 64 queries of its sub-tiles) instead of splitting every sub-tile between them: an
    // A/B variant, measured 169.6 vs 164.8 us at b = 32, S = 512 (the softmax is not the bound)
    static const bool alt = [] {
      const char* v = getenv("HARMONY_ATTN_BWD_ALT");
      return v && v[0] == '1';
    }();
    static bool set = false;
    if (!set) {
      HM_CUDA(cudaFuncSetAttribute(attn_bwd_persistent<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, BwdPCfg::SMEM));
      HM_CUDA(cudaFuncSetAttribute(attn_bwd_persistent<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, BwdPCfg::SMEM));
      set = true;
    }
    static int num_sms = 0;
    if (!num_sms) {
      int dev = 0;
      HM_CUDA(cudaGetDevice(&dev));
      HM_CUDA(cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev));
    }
    const int64_t items = (int64_t)(S / BKV) * H * b;
    // Q / dO in 64-query sub-tiles
    CUtensorMap mq64, mo64, mds32;
    tcx::make_map_4d(&mds32, dst, S, S, H, b, S, (int64_t)S * S, (int64_t)H * S * S, 64, 32);  // per-quadrant boxes
    tcx::make_map_4d(&mq64, q, dh, S, H, b, 3LL * d, dh, (int64_t)S * 3 * d, 64, BwdPCfg::BQS);
    tcx::make_map_4d(&mo64, dO, dh, S, H, b, d, dh, (int64_t)S * d, 64, BwdPCfg::BQS);
    auto kern = alt ? attn_bwd_persistent<true> : attn_bwd_persistent<false>;
    launch_k(kern, dim3((unsigned)std::min<int64_t>(items, num_sms)), dim3(THREADS), BwdPCfg::SMEM, st, mq64, mk, mv, mo64, mds32, p, (int)b);
  } else {
    static bool set = false;
    if (!set) { HM_CUDA(cudaFuncSetAttribute(attn_bwd_kernel<128>, cudaFuncAttributeMaxDynamicSharedMemorySize, BwdCfg<128>::SMEM)); set = true; }
    launch_k(attn_bwd_kernel<128>, dim3(grid), dim3(THREADS), BwdCfg<128>::SMEM, st, mq, mk, mv, mo, mds, p);
  }
  check_launch("attn_bwd_kernel");
  g_prof.end(PROF_ATTN, e0, st, 8.0 * b * H * (double)S * S * dh);  // S^T, dP^T, dV, dK contractions
  // dQ = dS K: A(m=q, k=key) = dS^T[key][q] (MN-major), B(n=e, k=key) = K[key][e] (MN-major)
  hk_gemm_args a = gemm_args(1, S, dh, S);
  a.nz0 = H; a.nz1 = (int)b;
  a.A = dst; a.a_mn_major = 1; a.lda = S; a.a_sz0 = (int64_t)S * S; a.a_sz1 = (int64_t)H * S * S;
  a.B = q + d; a.b_mn_major = 1; a.ldb = 3 * d; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * d;
  a.C = dQKV; a.ldc = 3 * d; a.c_sz0 = dh; a.c_sz1 = (int64_t)S * 3 * d;
  a.epilogue = HK_EPI_STORE_T;
  gemm(a, st);
  return true;
}

#ifdef HM_ATTN_TRACE
extern "C" int hm_attn_trace_read(unsigned long long* out, int* counts) {
  cudaDeviceSynchronize();
  cudaMemcpyFromSymbol(out, attn::g_attn_trace, sizeof(attn::g_attn_trace));
  cudaMemcpyFromSymbol(counts, attn::g_attn_trace_n, sizeof(attn::g_attn_trace_n));
  int z[3] = {0, 0, 0};
  cudaMemcpyToSymbol(attn::g_attn_trace_n, z, sizeof(z));
  return 0;
}
#endif

}  // namespace hm
