// plan.hpp — task decomposition and late binding of the Harmony-DP step (host only, no CUDA calls).
//
// decompose: the step becomes tasks FWD(l,i), LOSS(i), BWD(l,i), UPD(l)
//   for layers l and microbatches i of this rank, plus copy / collective ops.
// plan: under the per-GPU cap, choose which tensors stay
//   resident in HBM (compute weights first, then fp32 master/m/v, then the activation stash in
//   LIFO order), lay out double-buffered slots for the rest, attach each task's swap-in /
//   swap-out set (Fig. 5(a)), and emit one static per-stream program (compute,
//   h2d, d2h, comm) whose cross-stream edges are derived from buffer read/write sets
//   (the tensor-lifetime state machine of P:532-533).  The program is replayed every step.
#pragma once
#include <stdint.h>

#include <string>
#include <vector>

#include "harmony.h"
#include "layers.hpp"

namespace hm {

enum StreamId { S_COMPUTE = 0, S_H2D = 1, S_D2H = 2, S_COMM = 3, S_NUM = 4 };
enum OpKind {
  OP_INPUT = 0,      // user X / T -> arena (host or device source)
  OP_H2D = 1,        // pinned host store -> arena
  OP_D2H = 2,        // arena -> pinned host store
  OP_FWD = 3,
  OP_LOSS = 4,
  OP_BWD = 5,
  OP_UPD = 6,
  OP_ALLGATHER = 7,      // in-place all-gather of a layer's shards (weights)
  OP_REDUCESCATTER = 8,  // dW -> this rank's summed shard
  OP_LOSS_GATHER = 9,    // all-gather of every rank's per-microbatch loss partials
  OP_LOSS_OUT = 10,      // loss partials -> host
  OP_P2P = 11            // Harmony-PP: a peer rank's arena -> this rank's arena (activation / gradient hand-off)
};
enum Cat { CAT_WEIGHT = 0, CAT_STATE = 1, CAT_STASH = 2, CAT_INPUT = 3, CAT_OUTPUT = 4, CAT_GRAD = 5, CAT_NONE = 6 };
enum HostBuf { HB_NONE = -1, HB_WC = 0, HB_STATE = 1, HB_STASH = 2, HB_USER_X = 3, HB_USER_T = 4, HB_GRAD = 5 };

struct Op {
  int kind = 0, stream = 0, cat = CAT_NONE;
  int layer = -1, mb = -1;
  int first = 0;  // BWD: first microbatch of the group (dW written, not accumulated)
  int pack = 1;   // FWD: microbatches mb .. mb+pack-1 in one task (rows contiguous in the activation buffers)
  // copies: host side (buffer kind, index = layer or layer*m+mb, byte offset), device side arena offset
  int hbuf = HB_NONE;
  int64_t hidx = -1;
  uint64_t hoff = 0, dev = 0, bytes = 0;
  // compute operands: arena byte offsets
  uint64_t w = 0, in = 0, out = 0, stash = 0, ws = 0, dw = 0, state = 0, grad = 0, tgt = 0, loss = 0;
  uint64_t stash2 = 0;  // FWD with pack = 2: the second microbatch's stash
  uint64_t count = 0;  // collectives: elements per rank
  int peer = -1;       // OP_P2P: source rank; peer_off: byte offset in its arena
  uint64_t peer_off = 0;
  std::vector<int> waits;  // ops on other streams this op waits for
  int event = -1;          // event slot recorded after this op
};

struct LayerPlan {
  LayerGeom g;
  LayerGeom gp;                        // fwd_pack = 2: the same layer on two microbatches (2*b rows)
  int64_t P = 0, Ppad = 0, shard = 0;  // params, padded to N*1024, per-rank shard (elements)
  uint64_t wc_bytes = 0;               // full compute copy on device
  uint64_t state_bytes = 0;            // master|m|v shard (fp32)
  int64_t wc_res = -1, state_res = -1; // resident offsets (-1 = streamed)
  std::vector<int64_t> stash_res;      // per microbatch: resident offset or -1 (spilled)
  int user = 0;                        // the registered layer this task layer belongs to (column panels)
};

struct Plan {
  int N = 1, rank = 0, m = 1, b = 1, dtype = 0, stash_policy = 0, schedule = 0, retain_grads = 0;
  int fwd_pack = 1;
  uint64_t cap = 0;
  int upd_lag = 0;
  std::vector<LayerPlan> layers;   // task layers: a registered layer, or its column panels (operator split)
  int n_user = 0;                  // registered layers
  std::vector<int> user_first, user_count;  // registered layer -> its task layers
  // arena layout
  uint64_t arena_bytes = 0, min_ws_bytes = 0;
  // fp32 activation / gradient buffers of m microbatch rows each: [0], [1] the ping-pong of the DP step;
  // Harmony-PP uses four (layer input, layer output, incoming gradient, outgoing gradient)
  uint64_t bnd[4] = {0, 0, 0, 0}, bnd_bytes = 0, bnd_row_stride = 0;
  int n_bnd = 2;
  uint64_t tgt = 0, tgt_row_stride = 0;
  uint64_t ws = 0, ws_bytes = 0;
  std::vector<uint64_t> dw;  // fp32 dW accumulators (two alternating when N > 1; one per layer with groups)
  uint64_t gsh[2] = {0, 0};
  uint64_t loss = 0, loss_scratch = 0, tstep = 0;  // tstep: device int holding Adam's t
  std::vector<uint64_t> wslot, sslot, stage;  // slot offsets
  uint64_t wslot_bytes = 0, sslot_bytes = 0, stage_bytes = 0;
  // program
  std::vector<Op> ops;
  int n_events = 0;
  harmony_plan_summary summary{};
  int64_t n_params = 0;
  int d_in0 = 0, d_out_last = 0;
  int64_t in_elems_per_mb = 0, out_elems_per_mb = 0;
  std::string hazard_msg;
};

// Throws hm::Error (HARMONY_E_INVALID_ARG / UNSUPPORTED / CAP_TOO_SMALL).
// layout_only: residency, slots and arena layout for a sub-stack (Harmony-PP: one rank's layers,
// which need not chain), with n_bnd activation buffers, and no program.
Plan make_plan(const harmony_config& cfg, int n_layers, const harmony_layer_desc* descs, bool layout_only = false,
               int n_bnd = 2);

// ---- Harmony-PP (Fig. 4; reading c27): layer l runs on rank l % N;
// every layer-level task runs its group of m microbatches back to back; activations (forward) and
// gradients (backward) are handed to the next rank peer to peer; each layer's weights are swapped in
// once for its forward group and once for its backward group and out once after its JIT update.
// One program for the whole group: ops tagged with their rank, waits are global op indices.
struct GOp {
  int rank = 0;
  Op op;  // op.waits: indices into GroupPlan::ops; op.event: event slot of op.rank's context
};
struct GroupPlan {
  int N = 1;
  std::vector<Plan> ranks;                  // per-rank layout (local layers; their own ops unused)
  std::vector<int> layer_rank, layer_local;  // global layer -> (rank, local index)
  std::vector<GOp> ops;
  int n_events = 0;
  harmony_plan_summary summary{};           // box totals (bytes summed over ranks, arena = max)
  std::string hazard_msg;
};
GroupPlan make_plan_pp(const harmony_config& cfg, int num_ranks, int n_layers, const harmony_layer_desc* descs);
std::string dump_group_plan(const GroupPlan& g);
std::string dump_plan(const Plan& p);
void validate_config(const harmony_config& cfg);
int validate_program(const Plan& p, std::string* first);

}  // namespace hm
