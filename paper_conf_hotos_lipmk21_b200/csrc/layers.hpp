// layers.hpp — geometry of one layer task instance (layer x microbatch) and the task bodies.
//
// A task instance is "tied to a specific micro-batch of input data".  The
// forward task of layer l on microbatch i reads the layer input X (fp32 residual stream,
// reading c23) and the compute copy of W, writes the layer output and the op inputs the
// backward needs ("Stashed X", Fig. 5(a); reading c13).  The backward task
// reads dY, W and the stash, writes dX and accumulates dW in fp32 across microbatches
// ("Accumulated dW"; grouping P:546-548).
#pragma once
#include <stdint.h>
#include <stddef.h>

#include "harmony.h"

namespace hm {

// Byte offsets of the stash of one (layer, microbatch) inside its stash block.
struct StashLayout {
  uint64_t X = 0, mean1 = 0, rstd1 = 0, U = 0, QKV = 0, P = 0, C = 0, X2 = 0, mean2 = 0, rstd2 = 0, U2 = 0, H = 0,
           G = 0, Z = 0;
  uint64_t total = 0;
};

struct LayerGeom {
  harmony_layer_desc desc{};
  int dtype = 0;            // 0 = fp32 activations / SIMT GEMM, 1 = bf16 / tcgen05
  int ts = 4;               // bytes per activation element
  int stash_policy = 0;     // 0 = all op inputs, 1 = recompute LN outputs and GeLU in the backward,
                            // 2 = stash only the block input; the backward recomputes the block,
                            // 3 = 2 + the attention output and LSE (the recompute skips attention)
  int64_t core_off = 0;     // policy 2/3: offset of the full (policy-0) stash inside the workspace
  int b = 0;                // samples per microbatch
  int64_t rows = 0;         // tokens per microbatch (b*S; MLP: b)
  int d = 0, dh = 0, h = 0, S = 1;
  bool fused_attn = false;  // tcgen05 fused attention (bf16, S % 128 == 0, dh in {64, 128})
  int64_t n_params = 0;     // canonical packing length
  int64_t off[12] = {};     // parameter segment offsets (elements): transformer order of harmony.h
  StashLayout st;
  uint64_t ws_fwd = 0, ws_bwd = 0;  // workspace bytes
  double flops_fwd = 0;             // algorithmic GEMM FLOPs of one forward task
  StashLayout core_st;              // policy 2: the policy-0 layout the recompute materialises
  uint64_t core_ws_fwd = 0, core_ws_bwd = 0;
  // operator split (row a15): this task is column panel `panel` of `npanel` of an fp32 MLP layer whose
  // full output width is ld_out; it writes / reads output columns [col0, col0 + desc.d_out)
  int npanel = 1, panel = 0, col0 = 0, ld_out = 0;
};
// A layer's geometry as column panel `panel` of `npanel` (MLP, d_out % (16 npanel) == 0).
LayerGeom make_panel_geom(const harmony_layer_desc& full, int b, int dtype, int stash_policy, int panel, int npanel);

enum { P_LN1_G = 0, P_LN1_B, P_WQKV, P_BQKV, P_WO, P_BO, P_LN2_G, P_LN2_B, P_WFC1, P_BFC1, P_WFC2, P_BFC2 };
enum { P_MLP_W = 0, P_MLP_B = 1 };

LayerGeom make_geom(const harmony_layer_desc& desc, int b, int dtype, int stash_policy);
int64_t layer_n_params(const harmony_layer_desc& desc);

// Task bodies (launch kernels on st).  W: compute copy of the layer (T elements, canonical packing).
void layer_fwd(const LayerGeom& g, const void* W, const float* X, float* Y, uint8_t* stash, uint8_t* ws, void* st);
void layer_fwd_pack2(const LayerGeom& gp, const void* W, const float* X, float* Y, uint8_t* stash0, uint8_t* stash1,
                     uint8_t* ws, void* st);
// Lend the backward tasks a second stream (and 4 events) for weight-gradient work; nullptr = none.
void set_side_stream(void* st, void* const* events);
void layer_bwd(const LayerGeom& g, const void* W, const uint8_t* stash, const float* dY, float* dX, float* dW,
               int first, uint8_t* ws, void* st);

}  // namespace hm
