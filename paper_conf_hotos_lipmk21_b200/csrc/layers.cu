// layers.cu — forward / backward task bodies of the registered layer kinds.
// Math: oracle-independent restatement of the pre-LN block (reading c1) and the
// MLP layer; every contraction runs on hk gemm (tcgen05 for bf16, SIMT for fp32).
#include <cmath>

#include "common.hpp"
#include "kernels/kernels.hpp"
#include "layers.hpp"

namespace hm {

void act_fwd_T(int dtype, int act, int64_t n, const void* Z, void* out, cudaStream_t st);

int64_t layer_n_params(const harmony_layer_desc& d) {
  if (d.kind == HARMONY_LAYER_MLP) return (int64_t)d.d_in * d.d_out + d.d_out;
  int64_t D = d.d_in;
  return 12 * D * D + 13 * D;
}

// scratch of the backward: LN column partials, bias-grad partials, or 2 rows of recomputed LN stats
static uint64_t bwd_scratch_bytes(int64_t R, int D) {
  return std::max<uint64_t>(std::max<uint64_t>(layernorm_bwd_scratch_bytes(R, D), colsum_scratch_bytes(R, 4 * D)),
                            (uint64_t)R * 8);
}

static uint64_t bump(uint64_t& cur, uint64_t bytes) {
  uint64_t o = cur;
  cur = align_up(cur + bytes, 256);
  return o;
}

// Split-K factor of a weight gradient dW[k][n] += X^T dY over `rows` tokens: when its 256 x 256
// CTA-pair tiles would leave most of the 74 pairs idle (the d x d output projection: 16 tiles),
// the token (K) range is cut into S slices computed as S batched GEMMs into a workspace and added
// in slice order by splitk_sum (deterministic; shape-only, so capped == uncapped).
static int wgrad_splits(const LayerGeom& g, int64_t rows, int n, int k) {
  if (g.dtype != 1) return 1;
  const int64_t tiles = ceil_div(k, 256) * ceil_div(n, 256);
  if (k < 256 || n < 256 || tiles >= 37) return 1;
  int S = 1;
  while (S < 4 && tiles * S * 2 <= 74 && rows % (S * 2 * 64) == 0) S *= 2;
  return S;
}
static uint64_t wgrad_split_ws_bytes(const LayerGeom& g, int64_t rows, int n, int k) {
  const int S = wgrad_splits(g, rows, n, k);
  return S > 1 ? (uint64_t)S * k * n * 4 : 0;
}
LayerGeom make_panel_geom(const harmony_layer_desc& full, int b, int dtype, int stash_policy, int panel, int npanel) {
  HM_CHECK(full.kind == HARMONY_LAYER_MLP && npanel >= 1 && full.d_out % (16 * npanel) == 0, HARMONY_E_INVALID_ARG,
           "column panels: MLP layers with d_out a multiple of 16 * panels");
  harmony_layer_desc d = full;
  d.d_out = full.d_out / npanel;
  LayerGeom g = make_geom(d, b, dtype, stash_policy);
  g.npanel = npanel;
  g.panel = panel;
  g.col0 = panel * d.d_out;
  g.ld_out = full.d_out;
  if (npanel > 1) {  // contiguous copies of the panel's output / output-gradient columns
    const uint64_t tmp = align_up((uint64_t)g.rows * d.d_out * 4, 256);
    g.ws_fwd += tmp;
    g.ws_bwd += tmp;
  }
  return g;
}

LayerGeom make_geom(const harmony_layer_desc& desc, int b, int dtype, int stash_policy) {
  if ((stash_policy == 2 || stash_policy == 3) && desc.kind == HARMONY_LAYER_TRANSFORMER) {
    // Block recompute ([7] P:881): the stash is the block input X; the forward and the
    // backward both run the policy-0 block on a workspace-resident copy of the full stash.
    // Policy 3 also stashes the fused attention's output C (bf16) and row log-sum-exp, so the
    // recompute skips the attention forward (8.25 MB more per cfg2 task, usually host-swapped).
    LayerGeom core = make_geom(desc, b, dtype, 0);
    LayerGeom g = core;
    g.stash_policy = stash_policy == 3 && core.fused_attn ? 3 : 2;
    g.core_st = core.st;
    g.core_ws_fwd = core.ws_fwd;
    g.core_ws_bwd = core.ws_bwd;
    g.st = StashLayout{};
    uint64_t c = 0;
    g.st.X = bump(c, (uint64_t)core.rows * core.d * 4);
    if (g.stash_policy == 3) {
      g.st.C = bump(c, (uint64_t)core.rows * core.d * core.ts);
      g.st.P = bump(c, (uint64_t)core.b * core.h * core.S * 4);  // row log-sum-exp
    }
    g.st.total = c;
    const uint64_t full = align_up(core.st.total, 256);
    g.core_off = 0;
    g.ws_fwd = full + core.ws_fwd;
    g.ws_bwd = full + std::max(core.ws_fwd, core.ws_bwd) + align_up((uint64_t)core.rows * core.d * 4, 256);
    return g;
  }
  if (stash_policy >= 2) stash_policy = 0;  // MLP: the op-input stash is already minimal
  LayerGeom g;
  g.desc = desc;
  g.dtype = dtype;
  g.ts = dtype == 1 ? 2 : 4;
  g.stash_policy = stash_policy;
  g.b = b;
  g.n_params = layer_n_params(desc);
  g.ld_out = desc.d_out;
  if (desc.kind == HARMONY_LAYER_MLP) {
    g.S = 1;
    g.rows = b;
    g.d = desc.d_in;
    g.off[P_MLP_W] = 0;
    g.off[P_MLP_B] = (int64_t)desc.d_in * desc.d_out;
    uint64_t c = 0;
    g.st.X = bump(c, (uint64_t)g.rows * desc.d_in * g.ts);  // Xc: the GEMM operand (T)
    g.st.Z = bump(c, (uint64_t)g.rows * desc.d_out * g.ts); // pre-activation
    g.st.total = c;
    uint64_t w = 0;
    bump(w, (uint64_t)g.rows * desc.d_out * g.ts);  // dZ
    bump(w, std::max(colsum_scratch_bytes(g.rows, desc.d_out), (size_t)256));
    g.ws_bwd = w;
    g.ws_fwd = 256;
    g.flops_fwd = 2.0 * g.rows * desc.d_in * desc.d_out;
    return g;
  }
  const int64_t D = desc.d_in;
  g.d = desc.d_in;
  g.h = desc.n_heads;
  g.dh = desc.d_in / desc.n_heads;
  g.S = desc.seq_len;
  g.rows = (int64_t)b * g.S;
  int64_t o = 0;
  const int64_t seg[12] = {D, D, 3 * D * D, 3 * D, D * D, D, D, D, 4 * D * D, 4 * D, 4 * D * D, D};
  for (int i = 0; i < 12; ++i) { g.off[i] = o; o += seg[i]; }
  const uint64_t R = (uint64_t)g.rows, ts = (uint64_t)g.ts;
  const uint64_t SS = (uint64_t)b * g.h * g.S * g.S;
  // fused tcgen05 attention (scores in TMEM, no S x S tensor in HBM) when the shape qualifies
  g.fused_attn = dtype == 1 && g.S % 128 == 0 && (g.dh == 64 || g.dh == 128);
  const uint64_t BHS = (uint64_t)b * g.h * g.S;
  uint64_t c = 0;
  g.st.X = bump(c, R * D * 4);
  g.st.mean1 = bump(c, R * 4);
  g.st.rstd1 = bump(c, R * 4);
  if (stash_policy == 0) g.st.U = bump(c, R * D * ts);
  g.st.QKV = bump(c, R * 3 * D * ts);
  g.st.P = bump(c, g.fused_attn ? BHS * 4 : SS * ts);  // fused: row log-sum-exp instead of P
  g.st.C = bump(c, R * D * ts);
  g.st.X2 = bump(c, R * D * 4);
  g.st.mean2 = bump(c, R * 4);
  g.st.rstd2 = bump(c, R * 4);
  if (stash_policy == 0) g.st.U2 = bump(c, R * D * ts);
  g.st.H = bump(c, R * 4 * D * ts);
  if (stash_policy == 0) g.st.G = bump(c, R * 4 * D * ts);
  g.st.total = c;
  // forward workspace: scores Z (fp32) [+ recomputable U, U2, G under policy 1]
  uint64_t wf = 0;
  bump(wf, g.fused_attn ? 256 : SS * 4);
  if (stash_policy == 1) { bump(wf, R * D * ts); bump(wf, R * D * ts); bump(wf, R * 4 * D * ts); }
  g.ws_fwd = wf;
  // backward workspace (see layer_bwd for the aliasing)
  uint64_t wb = 0;
  bump(wb, R * D * ts);          // dYc / dX2c
  bump(wb, R * 4 * D * ts);      // dH / dQKV
  bump(wb, R * D * 4);           // dU2 / dU (fp32)
  bump(wb, R * D * 4);           // dX2 (fp32)
  bump(wb, R * D * ts);          // dC
  if (g.fused_attn) {
    bump(wb, attention_bwd_scratch_bytes(b, g.S, g.h));  // dS^T (bf16) + D
    bump(wb, 256);
  } else {
    bump(wb, SS * 4);              // dP (fp32)
    bump(wb, SS * ts);             // dZ
  }
  bump(wb, bwd_scratch_bytes(g.rows, (int)D));
  if (stash_policy == 1) bump(wb, R * 4 * D * ts);  // recomputed G / U2 / U
  // separate buffers read by the weight-gradient side stream (see bwd_core)
  bump(wb, R * D * ts);      // dX2c
  bump(wb, R * 3 * D * ts);  // dQKV
  bump(wb, colsum_scratch_bytes(g.rows, (int)(4 * D)));  // side-stream column-sum scratch
  bump(wb, std::max<uint64_t>(wgrad_split_ws_bytes(g, g.rows, (int)D, (int)D), 256));  // split-K dW_o partials
  if (dtype == 1) bump(wb, colsum32_partial_bytes(g.rows, (int)(4 * D)));  // db_fc1 partials (FC2 dgrad epilogue)
  g.ws_bwd = wb;
  g.flops_fwd = 24.0 * (double)R * D * D + 4.0 * (double)b * g.S * g.S * D;
  return g;
}

// ------------------------------------------------------------------------------------------------ side stream
// The executor lends the backward a second stream: the weight-gradient GEMMs and bias column sums
// of a block (which feed only dW) run there, concurrently with the data-gradient chain
// (dgrad -> LN backward -> attention -> dgrad) on the task's stream; the task joins it before it
// ends, so to the planner a BWD task is still one op on the compute stream.
static thread_local cudaStream_t t_side = nullptr;
static thread_local cudaEvent_t t_side_ev[4] = {nullptr, nullptr, nullptr, nullptr};
void set_side_stream(void* st, void* const* events) {
  t_side = static_cast<cudaStream_t>(st);
  for (int i = 0; i < 4; ++i) t_side_ev[i] = events ? static_cast<cudaEvent_t>(events[i]) : nullptr;
}

// ------------------------------------------------------------------------------------------------ helpers
static inline const uint8_t* wseg(const LayerGeom& g, const void* W, int seg) {
  return static_cast<const uint8_t*>(W) + g.off[seg] * g.ts;
}
static inline float* gseg(const LayerGeom& g, float* dW, int seg) { return dW + g.off[seg]; }

// Linear Y[rows][n] = X[rows][k] . W[k][n]  (W stored [k][n]: MN-major B)
static hk_gemm_args lin_fwd(const LayerGeom& g, int64_t rows, int n, int k, const void* X, const void* W) {
  hk_gemm_args a = gemm_args(g.dtype, (int)rows, n, k);
  a.A = X; a.a_mn_major = 0; a.lda = k;
  a.B = W; a.b_mn_major = 1; a.ldb = n;
  a.ldc = n;
  return a;
}
// dX[rows][k] = dY[rows][n] . W^T  (W[k][n] read as (n=k-index, k=n-index): K-major B)
static hk_gemm_args lin_dgrad(const LayerGeom& g, int64_t rows, int n, int k, const void* dY, const void* W) {
  hk_gemm_args a = gemm_args(g.dtype, (int)rows, k, n);
  a.A = dY; a.a_mn_major = 0; a.lda = n;
  a.B = W; a.b_mn_major = 0; a.ldb = n;
  a.ldc = k;
  return a;
}
// dW[k][n] (+)= X^T . dY  (both MN-major), fp32 accumulate (one writer per element: deterministic)
static hk_gemm_args lin_wgrad(const LayerGeom& g, int64_t rows, int n, int k, const void* X, const void* dY, float* dW,
                              int first) {
  hk_gemm_args a = gemm_args(g.dtype, k, n, (int)rows);
  a.A = X; a.a_mn_major = 1; a.lda = k;
  a.B = dY; a.b_mn_major = 1; a.ldb = n;
  a.C = dW; a.ldc = n;
  a.epilogue = HK_EPI_ACC_F32;
  a.accumulate = first ? 0 : 1;
  return a;
}

static void wgrad(const LayerGeom& g, int64_t rows, int n, int k, const void* X, const void* dY, float* dW, int first,
                  float* ws, cudaStream_t st) {
  const int S = wgrad_splits(g, rows, n, k);
  if (S == 1) return gemm(lin_wgrad(g, rows, n, k, X, dY, dW, first), st);
  const int64_t ks = rows / S;
  hk_gemm_args a = lin_wgrad(g, ks, n, k, X, dY, ws, 1);
  a.nz0 = S;
  a.a_sz0 = ks * k;  // X^T slice z: token rows [z ks, (z+1) ks) of X[rows][k]
  a.b_sz0 = ks * n;
  a.c_sz0 = (int64_t)k * n;
  a.epilogue = HK_EPI_STORE_F32;
  a.accumulate = 0;
  gemm(a, st);
  splitk_sum(S, (int64_t)k * n, ws, dW, first ? 0 : 1, st);
}

// ------------------------------------------------------------------------------------------------ forward
// Attention output C and row LSE kept outside the core stash (stash policy 3): where they live and
// whether they already hold this block's values (the backward's recompute skips the attention)
struct AttnStash {
  uint8_t* C;
  float* lse;
  bool have;
};

static void fwd_core(const LayerGeom& g, const void* W, const float* X, float* Y, uint8_t* stash, uint8_t* ws,
                     void* stv, bool stash_x = true, const AttnStash* as = nullptr, float* x_copy = nullptr,
                     float* x_copy2 = nullptr) {
  cudaStream_t st = static_cast<cudaStream_t>(stv);
  const harmony_layer_desc& d = g.desc;
  if (d.kind == HARMONY_LAYER_MLP) {
    void* Xc = stash + g.st.X;
    void* Z = stash + g.st.Z;
    if (g.dtype == 1) cast(1, g.rows * d.d_in, X, Xc, st);
    else copy_f32(g.rows * d.d_in, X, static_cast<float*>(Xc), st);
    hk_gemm_args a = lin_fwd(g, g.rows, d.d_out, d.d_in, Xc, wseg(g, W, P_MLP_W));
    a.C = Z; a.epilogue = HK_EPI_BIAS_ACT_F32; a.act = d.act; a.bias = wseg(g, W, P_MLP_B); a.aux_out = Y;
    gemm(a, st);
    return;
  }
  const int64_t R = g.rows;
  const int D = g.d, S = g.S, H = g.h, dh = g.dh, b = g.b;
  const size_t ts = g.ts;
  float* Xs = reinterpret_cast<float*>(stash + g.st.X);
  float* mean1 = reinterpret_cast<float*>(stash + g.st.mean1);
  float* rstd1 = reinterpret_cast<float*>(stash + g.st.rstd1);
  uint8_t* QKV = stash + g.st.QKV;
  uint8_t* P = as ? reinterpret_cast<uint8_t*>(as->lse) : stash + g.st.P;
  uint8_t* C = as ? as->C : stash + g.st.C;
  float* X2 = reinterpret_cast<float*>(stash + g.st.X2);
  float* mean2 = reinterpret_cast<float*>(stash + g.st.mean2);
  float* rstd2 = reinterpret_cast<float*>(stash + g.st.rstd2);
  uint8_t* Hh = stash + g.st.H;
  uint64_t wc = 0;
  float* Z = reinterpret_cast<float*>(ws + bump(wc, g.fused_attn ? 256 : (uint64_t)b * H * S * S * 4));
  uint8_t *U, *U2, *G;
  if (g.stash_policy == 0) {
    U = stash + g.st.U; U2 = stash + g.st.U2; G = stash + g.st.G;
  } else {
    U = ws + bump(wc, R * D * ts); U2 = ws + bump(wc, R * D * ts); G = ws + bump(wc, R * 4 * D * ts);
  }
  // stash the layer input (Fig. 5(a) "Stashed X"); under block recompute the caller keeps X itself
  if (stash_x) copy_f32(R * D, X, Xs, st);
  // U = LN1(X)
  // (block recompute: the LN reads X once and also writes the stashed copy of the block input)
  if (x_copy2) {
    // a forward pack of two microbatches: each half of the rows stashes its block input in its own
    // microbatch's stash (LayerNorm is per row: the same bits as one launch)
    const int64_t h = R / 2;
    layernorm_fwd(g.dtype, h, D, X, wseg(g, W, P_LN1_G), wseg(g, W, P_LN1_B), U, mean1, rstd1, st, x_copy);
    layernorm_fwd(g.dtype, h, D, X + h * D, wseg(g, W, P_LN1_G), wseg(g, W, P_LN1_B), U + (size_t)h * D * ts,
                  mean1 + h, rstd1 + h, st, x_copy2);
  } else {
    layernorm_fwd(g.dtype, R, D, X, wseg(g, W, P_LN1_G), wseg(g, W, P_LN1_B), U, mean1, rstd1, st, x_copy);
  }
  // QKV = U W_qkv + b_qkv
  {
    hk_gemm_args a = lin_fwd(g, R, 3 * D, D, U, wseg(g, W, P_WQKV));
    a.C = QKV; a.epilogue = HK_EPI_STORE_T; a.bias = wseg(g, W, P_BQKV);
    gemm(a, st);
  }
  if (as && as->have) {
    // C and the LSE of this block are in the stash (policy 3): the recompute needs only Q, K, V
  } else if (g.fused_attn) {
    // C = softmax(Q K^T / sqrt(dh)) V per head, scores kept in TMEM; stash the row LSE
    HM_CHECK(attention_fwd_fused(b, S, H, dh, d.causal, QKV, C, reinterpret_cast<float*>(P), st), HARMONY_E_INVALID_ARG,
             "fused attention rejected a qualifying shape");
  } else {
  // Z[b,h] = Q_h K_h^T (fp32), batched over heads (z0) and sequences (z1)
  {
    hk_gemm_args a = gemm_args(g.dtype, S, S, dh);
    a.nz0 = H; a.nz1 = b;
    a.A = QKV; a.a_mn_major = 0; a.lda = 3 * D; a.a_sz0 = dh; a.a_sz1 = (int64_t)S * 3 * D;
    a.B = QKV + (size_t)D * ts; a.b_mn_major = 0; a.ldb = 3 * D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * D;
    a.C = Z; a.ldc = S; a.c_sz0 = (int64_t)S * S; a.c_sz1 = (int64_t)H * S * S;
    a.epilogue = HK_EPI_STORE_F32;
    gemm(a, st);
  }
  // P = softmax(Z / sqrt(dh)) (+ causal mask)
  softmax_fwd(g.dtype, (int64_t)b * H * S, S, d.causal, 1.0f / std::sqrt((float)dh), Z, P, st);
  // C_h = P V_h, written head-interleaved into C [R][D]
  {
    hk_gemm_args a = gemm_args(g.dtype, S, dh, S);
    a.nz0 = H; a.nz1 = b;
    a.A = P; a.a_mn_major = 0; a.lda = S; a.a_sz0 = (int64_t)S * S; a.a_sz1 = (int64_t)H * S * S;
    a.B = QKV + (size_t)2 * D * ts; a.b_mn_major = 1; a.ldb = 3 * D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * D;
    a.C = C; a.ldc = D; a.c_sz0 = dh; a.c_sz1 = (int64_t)S * D;
    a.epilogue = HK_EPI_STORE_T;
    gemm(a, st);
  }
  }
  // X2 = X + C W_o + b_o   (fp32 residual stream)
  {
    hk_gemm_args a = lin_fwd(g, R, D, D, C, wseg(g, W, P_WO));
    a.C = X2; a.epilogue = HK_EPI_RESID_F32; a.aux = X; a.bias = wseg(g, W, P_BO);
    gemm(a, st);
  }
  // U2 = LN2(X2)
  layernorm_fwd(g.dtype, R, D, X2, wseg(g, W, P_LN2_G), wseg(g, W, P_LN2_B), U2, mean2, rstd2, st);
  // H = U2 W_fc1 + b_fc1 ; G = GeLU(H).  The block-recompute forward (stash_x false, output wanted)
  // needs only G: H is recomputed in the backward, so it is not written (identical G bits)
  {
    hk_gemm_args a = lin_fwd(g, R, 4 * D, D, U2, wseg(g, W, P_WFC1));
    a.act = HARMONY_ACT_GELU_TANH; a.bias = wseg(g, W, P_BFC1);
    if (!stash_x && Y && g.dtype == 1) {
      a.C = G; a.epilogue = HK_EPI_ACT_T;
    } else {
      a.C = Hh; a.epilogue = HK_EPI_BIAS_ACT; a.aux_out = G;
    }
    gemm(a, st);
  }
  // Y = X2 + G W_fc2 + b_fc2   (skipped when Y == nullptr: the backward's recompute needs only
  // the block's internals, not its output)
  if (Y) {
    hk_gemm_args a = lin_fwd(g, R, D, 4 * D, G, wseg(g, W, P_WFC2));
    a.C = Y; a.epilogue = HK_EPI_RESID_F32; a.aux = X2; a.bias = wseg(g, W, P_BFC2);
    gemm(a, st);
  }
}

// ------------------------------------------------------------------------------------------------ backward
static void bwd_core(const LayerGeom& g, const void* W, const uint8_t* stash, const float* dY, float* dX, float* dW,
                     int first, uint8_t* ws, void* stv, const float* Xs_in = nullptr,
                     const AttnStash* as = nullptr) {
  cudaStream_t st = static_cast<cudaStream_t>(stv);
  const harmony_layer_desc& d = g.desc;
  const int acc = first ? 0 : 1;
  if (d.kind == HARMONY_LAYER_MLP) {
    uint64_t wc = 0;
    uint8_t* dZ = ws + bump(wc, (uint64_t)g.rows * d.d_out * g.ts);
    float* scratch = reinterpret_cast<float*>(ws + bump(wc, colsum_scratch_bytes(g.rows, d.d_out)));
    const uint8_t* Xc = stash + g.st.X;
    const uint8_t* Z = stash + g.st.Z;
    act_bwd(g.dtype, d.act, g.rows * d.d_out, dY, Z, dZ, st);
    gemm(lin_wgrad(g, g.rows, d.d_out, d.d_in, Xc, dZ, gseg(g, dW, P_MLP_W), first), st);
    colsum(g.dtype, g.rows, d.d_out, dZ, d.d_out, gseg(g, dW, P_MLP_B), acc, scratch, st);
    if (dX) {
      hk_gemm_args a = lin_dgrad(g, g.rows, d.d_out, d.d_in, dZ, wseg(g, W, P_MLP_W));
      a.C = dX; a.epilogue = HK_EPI_STORE_F32;
      // a later column panel continues the K reduction of dX where the previous panel left it: the
      // panels, run in order, reproduce the unsplit dgrad bit for bit (fp32 path)
      if (g.panel > 0) { a.epilogue = HK_EPI_ACC_F32; a.accumulate = 2; }
      gemm(a, st);
    }
    return;
  }
  const int64_t R = g.rows;
  const int D = g.d, S = g.S, H = g.h, dh = g.dh, b = g.b;
  const size_t ts = g.ts;
  const int dt = g.dtype;
  const float* Xs = Xs_in ? Xs_in : reinterpret_cast<const float*>(stash + g.st.X);
  const float* mean1 = reinterpret_cast<const float*>(stash + g.st.mean1);
  const float* rstd1 = reinterpret_cast<const float*>(stash + g.st.rstd1);
  const uint8_t* QKV = stash + g.st.QKV;
  const uint8_t* P = as ? reinterpret_cast<const uint8_t*>(as->lse) : stash + g.st.P;
  const uint8_t* C = as ? as->C : stash + g.st.C;
  const float* X2 = reinterpret_cast<const float*>(stash + g.st.X2);
  const float* mean2 = reinterpret_cast<const float*>(stash + g.st.mean2);
  const float* rstd2 = reinterpret_cast<const float*>(stash + g.st.rstd2);
  const uint8_t* Hh = stash + g.st.H;
  const uint64_t SS = (uint64_t)b * H * S * S;
  uint64_t wc = 0;
  uint8_t* dYc = ws + bump(wc, R * D * ts);            // later dX2c
  uint8_t* dHb = ws + bump(wc, R * 4 * D * ts);        // later dQKV
  float* dUf = reinterpret_cast<float*>(ws + bump(wc, R * D * 4));
  float* dX2 = reinterpret_cast<float*>(ws + bump(wc, R * D * 4));
  uint8_t* dC = ws + bump(wc, R * D * ts);
  float* dP = nullptr;
  uint8_t* dZ = nullptr;
  uint8_t* attn_scratch = nullptr;
  if (g.fused_attn) {
    attn_scratch = ws + bump(wc, attention_bwd_scratch_bytes(b, S, H));
    bump(wc, 256);
  } else {
    dP = reinterpret_cast<float*>(ws + bump(wc, SS * 4));
    dZ = ws + bump(wc, SS * ts);
  }
  float* scratch = reinterpret_cast<float*>(ws + bump(wc, bwd_scratch_bytes(R, D)));
  uint8_t* rec = g.stash_policy == 1 ? ws + bump(wc, R * 4 * D * ts) : nullptr;
  uint8_t* dX2c_buf = ws + bump(wc, R * D * ts);
  uint8_t* dQKV_buf = ws + bump(wc, R * 3 * D * ts);
  float* side_scratch = reinterpret_cast<float*>(ws + bump(wc, colsum_scratch_bytes(R, 4 * D)));
  float* split_ws = reinterpret_cast<float*>(ws + bump(wc, std::max<uint64_t>(wgrad_split_ws_bytes(g, R, D, D), 256)));
  float* bfc1_part = dt == 1 ? reinterpret_cast<float*>(ws + bump(wc, colsum32_partial_bytes(R, (int)(4 * D)))) : nullptr;
  // weight gradients on the side stream (not with policy 1: its recompute buffer is reused in place)
  const bool overlap = t_side != nullptr && g.stash_policy != 1;
  cudaStream_t sw = overlap ? t_side : st;     // stream of the weight-gradient work
  float* wscratch = overlap ? side_scratch : scratch;
  auto fork = [&](int k) {
    if (!overlap) return;
    HM_CUDA(cudaEventRecord(t_side_ev[k], st));
    HM_CUDA(cudaStreamWaitEvent(t_side, t_side_ev[k], 0));
  };

  // dY as a GEMM operand; bf16: its copy and the FC2 bias gradient (column sums) in one pass
  const void* dYop = dY;
  if (dt == 1) {
    cast_colsum(1, R, D, dY, dYc, gseg(g, dW, P_BFC2), acc, scratch, st);
    dYop = dYc;
  }
  // ---- FC2: dG = dY W_fc2^T, fused with GeLU': dH = dG * gelu'(H); bf16: the same epilogue also
  // column-sums dH per 32-row block (the FC1 bias gradient's partials)
  {
    hk_gemm_args a = lin_dgrad(g, R, D, 4 * D, dYop, wseg(g, W, P_WFC2));
    a.C = dHb; a.epilogue = HK_EPI_ACT_BWD; a.act = HARMONY_ACT_GELU_TANH; a.aux = Hh;
    if (dt == 1) gemm_colsum(a, bfc1_part, st);
    else gemm(a, st);
  }
  const uint8_t* G = g.stash_policy == 0 ? stash + g.st.G : rec;
  if (g.stash_policy == 1) act_fwd_T(dt, HARMONY_ACT_GELU_TANH, R * 4 * D, Hh, rec, st);
  fork(0);
  gemm(lin_wgrad(g, R, D, 4 * D, G, dYop, gseg(g, dW, P_WFC2), first), sw);
  if (dt == 0) colsum(0, R, D, dY, D, gseg(g, dW, P_BFC2), acc, wscratch, sw);
  // ---- FC1: dU2 = dH W_fc1^T (fp32 for the LN backward); dW_fc1 += U2^T dH
  {
    hk_gemm_args a = lin_dgrad(g, R, 4 * D, D, dHb, wseg(g, W, P_WFC1));
    a.C = dUf; a.epilogue = HK_EPI_STORE_F32;
    gemm(a, st);
  }
  const uint8_t* U2 = stash + g.st.U2;
  if (g.stash_policy == 1) {
    // recompute U2 = LN2(X2) from the stashed X2 (identical kernel => identical bits)
    float* tmp_mean = reinterpret_cast<float*>(scratch);
    float* tmp_rstd = tmp_mean + R;
    layernorm_fwd(dt, R, D, X2, wseg(g, W, P_LN2_G), wseg(g, W, P_LN2_B), rec, tmp_mean, tmp_rstd, st);
    U2 = rec;
  }
  if (g.stash_policy == 1) fork(0);
  gemm(lin_wgrad(g, R, 4 * D, D, U2, dHb, gseg(g, dW, P_WFC1), first), sw);
  if (dt == 1) colsum32_reduce(R, (int)(4 * D), bfc1_part, gseg(g, dW, P_BFC1), acc, sw);
  else colsum(dt, R, 4 * D, dHb, 4 * D, gseg(g, dW, P_BFC1), acc, wscratch, sw);
  // ---- LN2 backward: dX2 = dY + LN2'(dU2), fused with the bf16 copy of dX2 (the O-projection
  // GEMM operand) and db_o (+)= sum_rows dX2
  const void* dX2op = dt == 1 ? (const void*)dX2c_buf : (const void*)dX2;
  layernorm_bwd_ex(dt, R, D, dUf, X2, mean2, rstd2, wseg(g, W, P_LN2_G), dY, dX2, gseg(g, dW, P_LN2_G),
                   gseg(g, dW, P_LN2_B), acc, dt == 1 ? dX2c_buf : nullptr, gseg(g, dW, P_BO), acc, scratch, st);
  fork(1);
  // ---- O projection: dC = dX2 W_o^T; dW_o += C^T dX2
  {
    hk_gemm_args a = lin_dgrad(g, R, D, D, dX2op, wseg(g, W, P_WO));
    a.C = dC; a.epilogue = HK_EPI_STORE_T;
    gemm(a, st);
  }
  wgrad(g, R, D, D, C, dX2op, gseg(g, dW, P_WO), first, split_ws, sw);
  // ---- attention backward (batched over heads z0 and sequences z1)
  uint8_t* dQKV = dQKV_buf;
  const float scale = 1.0f / std::sqrt((float)dh);
  if (g.fused_attn) {
    HM_CHECK(attention_bwd_fused(b, S, H, dh, d.causal, QKV, C, dC, reinterpret_cast<const float*>(P), dQKV,
                                 attn_scratch, st),
             HARMONY_E_INVALID_ARG, "fused attention rejected a qualifying shape");
  } else {
  {  // dP = dC_h V_h^T
    hk_gemm_args a = gemm_args(dt, S, S, dh);
    a.nz0 = H; a.nz1 = b;
    a.A = dC; a.a_mn_major = 0; a.lda = D; a.a_sz0 = dh; a.a_sz1 = (int64_t)S * D;
    a.B = QKV + (size_t)2 * D * ts; a.b_mn_major = 0; a.ldb = 3 * D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * D;
    a.C = dP; a.ldc = S; a.c_sz0 = (int64_t)S * S; a.c_sz1 = (int64_t)H * S * S;
    a.epilogue = HK_EPI_STORE_F32;
    gemm(a, st);
  }
  {  // dV_h = P^T dC_h
    hk_gemm_args a = gemm_args(dt, S, dh, S);
    a.nz0 = H; a.nz1 = b;
    a.A = P; a.a_mn_major = 1; a.lda = S; a.a_sz0 = (int64_t)S * S; a.a_sz1 = (int64_t)H * S * S;
    a.B = dC; a.b_mn_major = 1; a.ldb = D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * D;
    a.C = dQKV + (size_t)2 * D * ts; a.ldc = 3 * D; a.c_sz0 = dh; a.c_sz1 = (int64_t)S * 3 * D;
    a.epilogue = HK_EPI_STORE_T;
    gemm(a, st);
  }
  // dZ = scale * P.(dP - rowsum(dP.P))
  softmax_bwd(dt, (int64_t)b * H * S, S, scale, dP, P, dZ, st);
  {  // dQ_h = dZ K_h
    hk_gemm_args a = gemm_args(dt, S, dh, S);
    a.nz0 = H; a.nz1 = b;
    a.A = dZ; a.a_mn_major = 0; a.lda = S; a.a_sz0 = (int64_t)S * S; a.a_sz1 = (int64_t)H * S * S;
    a.B = QKV + (size_t)D * ts; a.b_mn_major = 1; a.ldb = 3 * D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * D;
    a.C = dQKV; a.ldc = 3 * D; a.c_sz0 = dh; a.c_sz1 = (int64_t)S * 3 * D;
    a.epilogue = HK_EPI_STORE_T;
    gemm(a, st);
  }
  {  // dK_h = dZ^T Q_h
    hk_gemm_args a = gemm_args(dt, S, dh, S);
    a.nz0 = H; a.nz1 = b;
    a.A = dZ; a.a_mn_major = 1; a.lda = S; a.a_sz0 = (int64_t)S * S; a.a_sz1 = (int64_t)H * S * S;
    a.B = QKV; a.b_mn_major = 1; a.ldb = 3 * D; a.b_sz0 = dh; a.b_sz1 = (int64_t)S * 3 * D;
    a.C = dQKV + (size_t)D * ts; a.ldc = 3 * D; a.c_sz0 = dh; a.c_sz1 = (int64_t)S * 3 * D;
    a.epilogue = HK_EPI_STORE_T;
    gemm(a, st);
  }
  }
  // ---- QKV projection: dU = dQKV W_qkv^T; dW_qkv += U^T dQKV; db_qkv += sum dQKV.  The weight
  // gradient (and db) go to the side stream FIRST: both products only read dQKV, and with the data
  // gradient and the LN1 backward after the fork this stream has ~150 us of work beside the weight
  // gradient's ~150 instead of ~70 — the task's closing join no longer idles this stream (measured:
  // ~125 us per task, profiles/r02_kernel_timeline_join.txt)
  const uint8_t* U = stash + g.st.U;
  if (g.stash_policy == 1) {
    float* tmp_mean = reinterpret_cast<float*>(scratch);
    float* tmp_rstd = tmp_mean + R;
    layernorm_fwd(dt, R, D, Xs, wseg(g, W, P_LN1_G), wseg(g, W, P_LN1_B), rec, tmp_mean, tmp_rstd, st);
    U = rec;
  }
  static const bool wgrad_first = [] {  // HARMONY_QKV_WGRAD_FIRST=0: the dgrad first (A/B)
    const char* e = getenv("HARMONY_QKV_WGRAD_FIRST");
    return !(e && *e == '0');
  }();
  auto qkv_dgrad = [&]() {
    hk_gemm_args a = lin_dgrad(g, R, 3 * D, D, dQKV, wseg(g, W, P_WQKV));
    a.C = dUf; a.epilogue = HK_EPI_STORE_F32;
    gemm(a, st);
  };
  if (!wgrad_first) qkv_dgrad();
  fork(2);
  gemm(lin_wgrad(g, R, 3 * D, D, U, dQKV, gseg(g, dW, P_WQKV), first), sw);
  colsum(dt, R, 3 * D, dQKV, 3 * D, gseg(g, dW, P_BQKV), acc, wscratch, sw);
  if (wgrad_first) qkv_dgrad();
  // ---- LN1 backward: dX = dX2 + LN1'(dU)
  layernorm_bwd(dt, R, D, dUf, Xs, mean1, rstd1, wseg(g, W, P_LN1_G), dX2, dX, gseg(g, dW, P_LN1_G),
                gseg(g, dW, P_LN1_B), acc, scratch, st);
  if (overlap) {  // join: the task ends when its weight gradients are in dW
    HM_CUDA(cudaEventRecord(t_side_ev[3], t_side));
    HM_CUDA(cudaStreamWaitEvent(st, t_side_ev[3], 0));
  }
}

// ------------------------------------------------------------------------------------------------ dispatch
static LayerGeom core_geom(const LayerGeom& g) {
  LayerGeom c = g;
  c.stash_policy = 0;
  c.st = g.core_st;
  c.ws_fwd = g.core_ws_fwd;
  c.ws_bwd = g.core_ws_bwd;
  return c;
}

void layer_fwd(const LayerGeom& g, const void* W, const float* X, float* Y, uint8_t* stash, uint8_t* ws, void* st) {
  if (g.npanel > 1) {  // column panel: its output columns into Y[:, col0 ..] (row stride ld_out)
    float* Yt = reinterpret_cast<float*>(ws);
    const uint64_t tmp = align_up((uint64_t)g.rows * g.desc.d_out * 4, 256);
    fwd_core(g, W, X, Yt, stash, ws + tmp, st);
    HM_CUDA(cudaMemcpy2DAsync(Y + g.col0, (size_t)g.ld_out * 4, Yt, (size_t)g.desc.d_out * 4, (size_t)g.desc.d_out * 4,
                              (size_t)g.rows, cudaMemcpyDeviceToDevice, static_cast<cudaStream_t>(st)));
    return;
  }
  if (g.stash_policy < 2) return fwd_core(g, W, X, Y, stash, ws, st);
  const LayerGeom c = core_geom(g);
  uint8_t* full = ws + g.core_off;
  uint8_t* rest = ws + align_up(c.st.total, 256);
  // policy 3: the attention writes C and its LSE straight into the stash
  const AttnStash as{stash + g.st.C, reinterpret_cast<float*>(stash + g.st.P), false};
  fwd_core(c, W, X, Y, full, rest, st, /*stash_x=*/false, g.stash_policy == 3 ? &as : nullptr,
           reinterpret_cast<float*>(stash + g.st.X));
}

// A forward pack (fwd_pack = 2): gp is the layer's geometry at two microbatches (block recompute);
// X / Y span both microbatches' rows, and each writes its block input into its own stash.
void layer_fwd_pack2(const LayerGeom& gp, const void* W, const float* X, float* Y, uint8_t* stash0, uint8_t* stash1,
                     uint8_t* ws, void* st) {
  HM_CHECK(gp.stash_policy == 2 && gp.desc.kind == HARMONY_LAYER_TRANSFORMER, HARMONY_E_UNSUPPORTED,
           "forward packs: block-recompute transformer layers");
  const LayerGeom c = core_geom(gp);
  uint8_t* full = ws + gp.core_off;
  uint8_t* rest = ws + align_up(c.st.total, 256);
  fwd_core(c, W, X, Y, full, rest, st, /*stash_x=*/false, nullptr, reinterpret_cast<float*>(stash0 + gp.st.X),
           reinterpret_cast<float*>(stash1 + gp.st.X));
}

void layer_bwd(const LayerGeom& g, const void* W, const uint8_t* stash, const float* dY, float* dX, float* dW,
               int first, uint8_t* ws, void* st) {
  if (g.npanel > 1) {  // column panel: its columns of dY; dX written (panel 0) or continued (later panels)
    float* dYt = reinterpret_cast<float*>(ws);
    const uint64_t tmp = align_up((uint64_t)g.rows * g.desc.d_out * 4, 256);
    HM_CUDA(cudaMemcpy2DAsync(dYt, (size_t)g.desc.d_out * 4, dY + g.col0, (size_t)g.ld_out * 4, (size_t)g.desc.d_out * 4,
                              (size_t)g.rows, cudaMemcpyDeviceToDevice, static_cast<cudaStream_t>(st)));
    return bwd_core(g, W, stash, dYt, dX, dW, first, ws + tmp, st);
  }
  if (g.stash_policy < 2) return bwd_core(g, W, stash, dY, dX, dW, first, ws, st);
  const LayerGeom c = core_geom(g);
  uint8_t* full = ws + g.core_off;
  uint8_t* rest = ws + align_up(c.st.total, 256);
  // recompute the block's forward from its stashed input: the same kernels, hence the same bits;
  // the LN1 backward reads the stashed input in place (policy 3: and the stashed C / LSE)
  const float* Xst = reinterpret_cast<const float*>(stash + g.st.X);
  const AttnStash as{const_cast<uint8_t*>(stash) + g.st.C, reinterpret_cast<float*>(const_cast<uint8_t*>(stash) + g.st.P),
                     true};
  const AttnStash* asp = g.stash_policy == 3 ? &as : nullptr;
  fwd_core(c, W, Xst, nullptr, full, rest, st, /*stash_x=*/false, asp);
  bwd_core(c, W, full, dY, dX, dW, first, rest, st, Xst, asp);
}

}  // namespace hm
