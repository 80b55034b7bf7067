// plan.cpp — decompose + plan (see plan.hpp).  Host-only: runs without a GPU (harmony_plan_dry).
#include "plan.hpp"

#include <algorithm>
#include <array>
#include <cstdlib>
#include <deque>
#include <map>
#include <sstream>
#include <unordered_map>

#include "common.hpp"
#include "kernels/kernels.hpp"

namespace hm {

static const uint64_t ALIGN = 1024;  // every arena buffer 1 KiB aligned: identical code paths capped/uncapped

void validate_config(const harmony_config& c) {
  HM_CHECK(c.struct_size == sizeof(harmony_config), HARMONY_E_INVALID_ARG, "harmony_config.struct_size mismatch");
  HM_CHECK(c.world_size >= 1 && c.world_size <= 64, HARMONY_E_INVALID_ARG, "world_size must be in 1..64");
  HM_CHECK(c.rank >= 0 && c.rank < c.world_size, HARMONY_E_INVALID_ARG, "rank out of range");
  HM_CHECK(c.microbatches >= 1, HARMONY_E_INVALID_ARG, "microbatches must be >= 1");
  HM_CHECK(c.microbatch_size >= 1, HARMONY_E_INVALID_ARG, "microbatch_size must be >= 1");
  HM_CHECK(c.precision == HARMONY_FP32 || c.precision == HARMONY_BF16_FP32MASTER, HARMONY_E_INVALID_ARG,
           "unknown precision");
  HM_CHECK(c.schedule == HARMONY_SCHED_HARMONY_DP || c.schedule == HARMONY_SCHED_PER_GPU_VIRT ||
               c.schedule == HARMONY_SCHED_HARMONY_PP,
           HARMONY_E_INVALID_ARG, "unknown schedule");
  HM_CHECK(c.stash_policy >= 0 && c.stash_policy <= 3, HARMONY_E_INVALID_ARG, "stash_policy must be 0..3");
  HM_CHECK(c.groups >= 0 && c.groups <= 64, HARMONY_E_INVALID_ARG, "groups must be in 0..64");
  HM_CHECK(c.fwd_pack >= 0 && c.fwd_pack <= 2, HARMONY_E_INVALID_ARG, "fwd_pack must be 0, 1 or 2");
  HM_CHECK(c.weight_decay == 0.0, HARMONY_E_UNSUPPORTED, "weight_decay must be 0 (reading c3)");
  HM_CHECK(c.lr > 0 && c.beta1 >= 0 && c.beta1 < 1 && c.beta2 >= 0 && c.beta2 < 1 && c.eps > 0,
           HARMONY_E_INVALID_ARG, "bad Adam hyper-parameters");
}

static void validate_layers(const harmony_config& c, int n, const harmony_layer_desc* d, bool chain = true) {
  HM_CHECK(n >= 1 && d != nullptr, HARMONY_E_INVALID_ARG, "need >= 1 layer");
  for (int l = 0; l < n; ++l) {
    const harmony_layer_desc& x = d[l];
    HM_CHECK(x.d_in >= 1 && x.d_out >= 1, HARMONY_E_INVALID_ARG, "layer widths must be >= 1");
    if (x.kind == HARMONY_LAYER_MLP) {
      HM_CHECK(x.act >= 0 && x.act <= 2, HARMONY_E_INVALID_ARG, "unknown activation");
      if (c.precision == HARMONY_BF16_FP32MASTER)
        HM_CHECK(x.d_in % 8 == 0 && x.d_out % 8 == 0, HARMONY_E_UNSUPPORTED, "bf16 path needs widths % 8 == 0 (c24)");
    } else if (x.kind == HARMONY_LAYER_TRANSFORMER) {
      HM_CHECK(x.d_out == x.d_in, HARMONY_E_INVALID_ARG, "transformer layer needs d_out == d_in");
      HM_CHECK(x.n_heads >= 1 && x.d_in % x.n_heads == 0, HARMONY_E_INVALID_ARG, "d % h must be 0 (c24)");
      HM_CHECK(x.seq_len >= 1, HARMONY_E_INVALID_ARG, "seq_len must be >= 1");
      if (c.precision == HARMONY_BF16_FP32MASTER)
        HM_CHECK(x.d_in % 8 == 0 && (x.d_in / x.n_heads) % 8 == 0 && x.seq_len % 8 == 0, HARMONY_E_UNSUPPORTED,
                 "bf16 path needs d, d/h and S multiples of 8 (16-byte TMA strides, c24)");
    } else {
      HM_CHECK(false, HARMONY_E_INVALID_ARG, "unknown layer kind");
    }
    if (l > 0) {
      HM_CHECK(!chain || d[l - 1].d_out == x.d_in, HARMONY_E_INVALID_ARG, "layer widths do not chain");
      HM_CHECK(d[l - 1].kind == x.kind, HARMONY_E_UNSUPPORTED, "mixed layer kinds in one stack");
      if (x.kind == HARMONY_LAYER_TRANSFORMER)
        HM_CHECK(d[l - 1].seq_len == x.seq_len, HARMONY_E_INVALID_ARG, "seq_len must match across layers");
    }
  }
}

// ------------------------------------------------------------------------------------ resource tracking
namespace {
enum ResKind : uint64_t {
  R_BND = 1, R_TGT, R_LOSS, R_WSLOT, R_WRES, R_SSLOT, R_SRES, R_STAGE, R_STASHRES, R_DW, R_GSH,
  H_WC, H_STATE, H_STASH, H_GRAD, R_LOSSALL
};
inline uint64_t key(ResKind k, uint64_t a, uint64_t b = 0) { return ((uint64_t)k << 56) | (a << 28) | b; }

struct Tracker {
  struct Res {
    int writer = -1;
    std::vector<int> readers;
  };
  std::unordered_map<uint64_t, Res> res;
  std::vector<Op>* ops;

  int add(Op op, const std::vector<uint64_t>& reads, const std::vector<uint64_t>& writes) {
    const int idx = (int)ops->size();
    std::vector<int> deps;
    for (uint64_t r : reads) {
      auto it = res.find(r);
      if (it != res.end() && it->second.writer >= 0) deps.push_back(it->second.writer);
    }
    for (uint64_t w : writes) {
      auto it = res.find(w);
      if (it == res.end()) continue;
      if (it->second.writer >= 0) deps.push_back(it->second.writer);
      for (int rd : it->second.readers) deps.push_back(rd);
    }
    // keep only the latest dependency per other stream (streams execute in order)
    int latest[S_NUM] = {-1, -1, -1, -1};
    for (int dpi : deps) {
      int s = (*ops)[dpi].stream;
      if (s != op.stream) latest[s] = std::max(latest[s], dpi);
    }
    op.waits.clear();
    for (int s = 0; s < S_NUM; ++s)
      if (latest[s] >= 0) op.waits.push_back(latest[s]);
    for (uint64_t r : reads) res[r].readers.push_back(idx);
    for (uint64_t w : writes) {
      Res& x = res[w];
      x.writer = idx;
      x.readers.clear();
    }
    ops->push_back(op);
    return idx;
  }
};

struct Arena {
  uint64_t cur = 0;
  uint64_t take(uint64_t bytes) {
    uint64_t o = cur;
    cur = align_up(cur + std::max<uint64_t>(bytes, 1), ALIGN);
    return o;
  }
};
}  // namespace


// ------------------------------------------------------------------------------------ program validator
// Independent of the resource keys used to derive the edges: every op's arena (and host-store)
// byte ranges are recomputed from its operands, happens-before is derived from stream order
// plus the wait edges (vector clocks), and any two unordered ops touching overlapping bytes,
// at least one writing, count as a hazard.  (race detection.)
namespace {
struct Acc {
  int space;  // 0 = arena, 1 + host buffer kind
  int64_t idx;
  uint64_t lo, hi;
  bool write;
};
}  // namespace

static std::vector<Acc> accesses(const Plan& p, const Op& o) {
  std::vector<Acc> v;
  auto ar = [&](uint64_t off, uint64_t bytes, bool w) {
    if (bytes) v.push_back({0, 0, off, off + bytes, w});
  };
  auto hb = [&](int hbuf, int64_t idx, uint64_t off, uint64_t bytes, bool w) {
    if (bytes) v.push_back({1 + hbuf, idx, off, off + bytes, w});
  };
  const uint64_t ts = p.dtype ? 2 : 4;
  switch (o.kind) {
    case OP_INPUT: ar(o.dev, o.bytes, true); break;
    case OP_H2D: ar(o.dev, o.bytes, true); hb(o.hbuf, o.hidx, o.hoff, o.bytes, false); break;
    case OP_D2H: ar(o.dev, o.bytes, false); hb(o.hbuf, o.hidx, o.hoff, o.bytes, true); break;
    case OP_FWD: {
      const LayerPlan& lp = p.layers[o.layer];
      const uint64_t pk = (uint64_t)o.pack;  // a pack spans its microbatches' contiguous rows
      ar(o.w, (uint64_t)lp.P * ts, false);
      ar(o.in, pk * lp.g.rows * lp.g.desc.d_in * 4, false);
      ar(o.out, pk * lp.g.rows * lp.g.ld_out * 4, true);  // (a column panel: within these rows)
      ar(o.stash, lp.g.st.total, true);
      if (o.pack == 2) ar(o.stash2, lp.g.st.total, true);
      ar(o.ws, o.pack == 2 ? lp.gp.ws_fwd : lp.g.ws_fwd, true);
      break;
    }
    case OP_BWD: {
      const LayerPlan& lp = p.layers[o.layer];
      ar(o.w, (uint64_t)lp.P * ts, false);
      ar(o.stash, lp.g.st.total, false);
      ar(o.in, (uint64_t)lp.g.rows * lp.g.ld_out * 4, false);
      ar(o.out, (uint64_t)lp.g.rows * lp.g.desc.d_in * 4, true);
      ar(o.dw, (uint64_t)lp.P * 4, true);
      ar(o.ws, lp.g.ws_bwd, true);
      break;
    }
    case OP_LOSS:
      ar(o.in, (uint64_t)p.out_elems_per_mb * 4, false);
      ar(o.tgt, (uint64_t)p.out_elems_per_mb * 4, false);
      ar(o.out, (uint64_t)p.out_elems_per_mb * 4, true);
      ar(o.loss, 8, true);
      ar(p.loss_scratch, mse_scratch_bytes(), true);
      break;
    case OP_UPD: {
      const LayerPlan& lp = p.layers[o.layer];
      ar(o.grad, (uint64_t)lp.shard * 4, false);
      ar(o.state, lp.state_bytes, true);
      ar(o.w + (uint64_t)p.rank * lp.shard * ts, (uint64_t)lp.shard * ts, true);
      break;
    }
    case OP_ALLGATHER: ar(o.dev, (uint64_t)p.N * o.count * ts, true); break;
    case OP_REDUCESCATTER: ar(o.dev, (uint64_t)p.N * o.count * 4, false); ar(o.grad, o.count * 4, true); break;
    case OP_LOSS_GATHER: ar(o.dev, (uint64_t)p.N * o.count * 8, true); break;
    case OP_LOSS_OUT: ar(o.dev, o.bytes, false); break;
    default: break;
  }
  return v;
}

int validate_program(const Plan& p, std::string* first) {
  const size_t n = p.ops.size();
  std::vector<std::array<int, S_NUM>> vc(n);
  std::vector<int> pos(n);
  std::array<int, S_NUM> cnt{};
  std::array<int, S_NUM> last{};
  last.fill(-1);
  for (size_t i = 0; i < n; ++i) {
    const Op& o = p.ops[i];
    std::array<int, S_NUM> c;
    c.fill(-1);
    if (last[o.stream] >= 0) c = vc[last[o.stream]];
    for (int w : o.waits)
      for (int s = 0; s < S_NUM; ++s) c[s] = std::max(c[s], vc[w][s]);
    pos[i] = cnt[o.stream]++;
    c[o.stream] = pos[i];
    vc[i] = c;
    last[o.stream] = (int)i;
  }
  auto hb = [&](size_t a, size_t b) { return vc[b][p.ops[a].stream] >= pos[a]; };
  std::vector<std::vector<Acc>> acc(n);
  for (size_t i = 0; i < n; ++i) acc[i] = accesses(p, p.ops[i]);
  int hazards = 0;
  // dataflow rule: a spilled stash is produced and consumed within the step, so every read of a
  // host stash buffer must be ordered after a write of it (else it would read the previous step's)
  for (size_t j = 0; j < n; ++j)
    for (const Acc& b : acc[j]) {
      if (b.write || b.space != 1 + HB_STASH) continue;
      bool produced = false;
      for (size_t i = 0; i < n && !produced; ++i)
        for (const Acc& a : acc[i])
          if (a.write && a.space == b.space && a.idx == b.idx && a.lo <= b.lo && a.hi >= b.hi && i != j && hb(i, j)) {
            produced = true;
            break;
          }
      if (!produced) {
        if (hazards == 0 && first)
          *first = "op " + std::to_string(j) + " reads host stash " + std::to_string(b.idx) + " before it is written";
        ++hazards;
      }
    }
  for (size_t j = 0; j < n; ++j)
    for (size_t i = 0; i < j; ++i) {
      if (p.ops[i].stream == p.ops[j].stream || hb(i, j)) continue;
      for (const Acc& a : acc[i])
        for (const Acc& b : acc[j])
          if ((a.write || b.write) && a.space == b.space && a.idx == b.idx && a.lo < b.hi && b.lo < a.hi) {
            if (hazards == 0 && first)
              *first = "ops " + std::to_string(i) + " and " + std::to_string(j) + " race on space " +
                       std::to_string(a.space) + "[" + std::to_string(a.idx) + "]";
            ++hazards;
            goto next_pair;
          }
    next_pair:;
    }
  return hazards;
}

// ------------------------------------------------------------------------------------ make_plan
static Plan make_plan_impl(const harmony_config& cfg, int n_layers, const harmony_layer_desc* descs, bool layout_only,
                           int n_bnd, const std::vector<int>& npanel);

// Operator split inside the step (row a15): when the cap cannot hold a registered layer's
// working set, fp32 MLP layers are decomposed into column panels — sub-tasks that each need only their
// W[:, panel] columns (compute copy, master / m / v, dW) — the widest layer halved first, until the
// plan fits.  Panels in order reproduce the unsplit layer bit for bit (the forward and the weight
// gradient split along N; dX continues one K reduction across the panels), so capped == uncapped
// stays exact (reading c21).
Plan make_plan(const harmony_config& cfg, int n_layers, const harmony_layer_desc* descs, bool layout_only,
               int n_bnd) {
  std::vector<int> np(n_layers > 0 ? n_layers : 0, 1);
  try {
    return make_plan_impl(cfg, n_layers, descs, layout_only, n_bnd, np);
  } catch (const Error& e) {
    if (e.code != HARMONY_E_CAP_TOO_SMALL || cfg.precision != HARMONY_FP32 || layout_only) throw;
    for (int round = 0; round < 16; ++round) {
      int best = -1;
      int64_t best_p = 0;
      for (int l = 0; l < n_layers; ++l) {
        const harmony_layer_desc& d = descs[l];
        if (d.kind != HARMONY_LAYER_MLP || d.d_out % (16 * 2 * np[l]) != 0) continue;
        const int64_t per = ((int64_t)d.d_in + 1) * d.d_out / np[l];
        if (per > best_p) { best_p = per; best = l; }
      }
      if (best < 0) throw;
      np[best] *= 2;
      try {
        return make_plan_impl(cfg, n_layers, descs, layout_only, n_bnd, np);
      } catch (const Error& e2) {
        if (e2.code != HARMONY_E_CAP_TOO_SMALL) throw;
      }
    }
    throw;
  }
}

static Plan make_plan_impl(const harmony_config& cfg, int n_layers, const harmony_layer_desc* descs, bool layout_only,
                           int n_bnd, const std::vector<int>& npanel) {
  validate_config(cfg);
  validate_layers(cfg, n_layers, descs, !layout_only);
  HM_CHECK(cfg.schedule != HARMONY_SCHED_HARMONY_PP, HARMONY_E_UNSUPPORTED,
           "Harmony-PP is planned for a group of ranks (harmony_init_group / harmony_plan_dry_group)");
  Plan p;
  p.n_bnd = n_bnd;
  p.N = cfg.world_size;
  p.rank = cfg.rank;
  p.m = cfg.microbatches;
  p.b = cfg.microbatch_size;
  p.dtype = cfg.precision == HARMONY_BF16_FP32MASTER ? 1 : 0;
  p.stash_policy = cfg.stash_policy;
  p.schedule = cfg.schedule;
  p.retain_grads = cfg.retain_grads;
  p.cap = cfg.hbm_cap_bytes;
  p.upd_lag = (p.N > 1 && p.schedule == HARMONY_SCHED_HARMONY_DP) ? 1 : 0;
  const int m = p.m, N = p.N, r = p.rank;
  const uint64_t ts = p.dtype ? 2 : 4;
  // task layers: each registered layer, or its column panels
  p.n_user = n_layers;
  std::vector<std::pair<int, int>> tl;  // (registered layer, panel)
  for (int u = 0; u < n_layers; ++u) {
    p.user_first.push_back((int)tl.size());
    p.user_count.push_back(npanel[u]);
    for (int k = 0; k < npanel[u]; ++k) tl.push_back({u, k});
  }
  const int L = (int)tl.size();
  const int LU = n_layers;

  p.layers.resize(L);
  int dmax = 0;
  for (int u = 0; u < LU; ++u) dmax = std::max({dmax, descs[u].d_in, descs[u].d_out});
  uint64_t ws_need = 256, maxP = 0, max_shard = 0;
  for (int l = 0; l < L; ++l) {
    LayerPlan& lp = p.layers[l];
    const int u = tl[l].first;
    lp.user = u;
    lp.g = npanel[u] > 1 ? make_panel_geom(descs[u], p.b, p.dtype, p.stash_policy, tl[l].second, npanel[u])
                         : make_geom(descs[u], p.b, p.dtype, p.stash_policy);
    lp.P = lp.g.n_params;
    lp.Ppad = (int64_t)align_up((uint64_t)lp.P, (uint64_t)N * 1024);
    lp.shard = lp.Ppad / N;
    lp.wc_bytes = (uint64_t)lp.Ppad * ts;
    lp.state_bytes = 3 * (uint64_t)lp.shard * 4;
    lp.stash_res.assign(m, -1);
    ws_need = std::max({ws_need, lp.g.ws_fwd, lp.g.ws_bwd});
    if (cfg.fwd_pack == 2) {  // the forward pass on two microbatches at once (NEXT-4 pack size)
      lp.gp = make_geom(descs[u], 2 * p.b, p.dtype, p.stash_policy);
      ws_need = std::max(ws_need, lp.gp.ws_fwd);
    }
    maxP = std::max<uint64_t>(maxP, (uint64_t)lp.Ppad);
    max_shard = std::max<uint64_t>(max_shard, (uint64_t)lp.shard);
    p.n_params += lp.P;
  }
  const int64_t rows = p.layers[0].g.rows;
  p.d_in0 = descs[0].d_in;
  p.d_out_last = descs[LU - 1].d_out;
  p.in_elems_per_mb = rows * descs[0].d_in;
  p.out_elems_per_mb = rows * descs[LU - 1].d_out;

  // ---------------------------------------------------------------- fixed working set
  const uint64_t bnd_stride = align_up((uint64_t)rows * dmax * 4, ALIGN);
  const uint64_t tgt_stride = align_up((uint64_t)p.out_elems_per_mb * 4, ALIGN);
  // microbatch groups (direction balance): G > 1 keeps every layer's fp32 dW accumulator from its
  // first group's backward to its last
  const int G = cfg.groups > 1 ? cfg.groups : 1;
  HM_CHECK(m % G == 0, HARMONY_E_INVALID_ARG, "microbatches must be a multiple of groups");
  HM_CHECK(G == 1 || p.schedule == HARMONY_SCHED_HARMONY_DP, HARMONY_E_UNSUPPORTED,
           "microbatch groups are a Harmony-DP schedule");
  const int mg = m / G;
  p.fwd_pack = cfg.fwd_pack == 2 ? 2 : 1;
  if (p.fwd_pack == 2) {
    bool ok = p.schedule == HARMONY_SCHED_HARMONY_DP && p.stash_policy == 2 && mg % 2 == 0 && L == LU;
    for (int l = 0; l < L && ok; ++l)
      ok = descs[l].kind == HARMONY_LAYER_TRANSFORMER && descs[l].d_in == dmax &&
           bnd_stride == (uint64_t)rows * dmax * 4;  // consecutive microbatches' rows are contiguous
    HM_CHECK(ok, HARMONY_E_UNSUPPORTED,
             "fwd_pack = 2 needs Harmony-DP, stash_policy 2, uniform transformer layers and "
             "microbatches per group a multiple of 2");
  }
  const int nDW = G > 1 ? L : (N > 1 ? 2 : 1);
  auto dwi = [&](int l) { return G > 1 ? l : l % nDW; };
  auto fixed_bytes = [&]() {
    uint64_t f = 0;
    f += (uint64_t)p.n_bnd * bnd_stride * m;          // activation / gradient buffers
    f += tgt_stride * m;                              // targets
    f += align_up(ws_need, ALIGN);                    // one task's transients
    f += nDW * align_up(maxP * 4, ALIGN);             // fp32 dW accumulators
    if (N > 1) f += 2 * align_up(max_shard * 4, ALIGN);  // reduced-gradient shards
    f += align_up((uint64_t)N * m * 8, ALIGN) + align_up(mse_scratch_bytes(), ALIGN) + ALIGN;
    return f;
  };
  const uint64_t fixed = fixed_bytes();

  // ---------------------------------------------------------------- residency (late binding of memory)
  const bool uncapped = p.cap == 0;
  const bool baseline = p.schedule == HARMONY_SCHED_PER_GPU_VIRT;
  uint64_t all_res = fixed;
  for (auto& lp : p.layers) all_res += align_up(lp.wc_bytes, ALIGN) + align_up(lp.state_bytes, ALIGN) +
                                       (uint64_t)m * align_up(lp.g.st.total, ALIGN);
  int nW = 0, nS = 0, nG = 0;
  {
    uint64_t mw = 0, ms = 0, mst = 0;
    for (auto& lp : p.layers) {
      mw = std::max(mw, align_up(lp.wc_bytes, ALIGN));
      ms = std::max(ms, align_up(lp.state_bytes, ALIGN));
      mst = std::max(mst, align_up(lp.g.st.total, ALIGN));
    }
    p.min_ws_bytes = std::min(all_res, fixed + mw + ms + mst);
  }
  if (uncapped || (!baseline && all_res <= p.cap)) {
    for (auto& lp : p.layers) {
      lp.wc_res = 0; lp.state_res = 0;
      for (int i = 0; i < m; ++i) lp.stash_res[i] = 0;
    }
  } else {
    uint64_t maxw = 0, maxs = 0, maxst = 0;
    for (auto& lp : p.layers) {
      maxw = std::max(maxw, align_up(lp.wc_bytes, ALIGN));
      maxs = std::max(maxs, align_up(lp.state_bytes, ALIGN));
      maxst = std::max(maxst, align_up(lp.g.st.total, ALIGN));
    }
    HM_CHECK(p.min_ws_bytes <= p.cap, HARMONY_E_CAP_TOO_SMALL,
             "hbm_cap_bytes " + std::to_string(p.cap) + " < minimum working set " + std::to_string(p.min_ws_bytes));
    // slot counts in order of preference (double buffering needs memory)
    // Small stash entries get four staging slots: a stash swap-in waits for its slot to be released
    // by the backward two entries back, and on the one H2D stream that wait would hold up the
    // state swap-ins queued behind it (head-of-line blocking; cfg3: 26 MB entries, 16 GiB cap)
    int gq = maxst > 0 && maxst * 4 <= p.cap / 64 ? 4 : 2;
    if (const char* e = getenv("HARMONY_STAGE_SLOTS")) gq = std::max(1, std::min(8, atoi(e)));  // experiments
    const int pref[][3] = {{2, 2, gq}, {2, 2, std::min(gq, 2)}, {2, 1, 2}, {2, 1, 1}, {1, 1, 2}, {1, 1, 1}};
    for (auto& c : pref) {
      if (fixed + c[0] * maxw + c[1] * maxs + c[2] * maxst <= p.cap) { nW = c[0]; nS = c[1]; nG = c[2]; break; }
    }
    // Fill residency with the room the slots leave, then shrink the slots to what is still streamed
    // and repeat (the freed room lets more become resident).  Greedy filling is not monotone in
    // the room, so every pass is checked: a pass whose streamed items fit its own slot sizes next
    // to its residency is a consistent layout; the last consistent one is kept (pass 0 always is,
    // its sizes are the global maxima).  Slot counts are upgraded (double buffering) only
    // afterwards and only where they fit — the layout can never exceed the cap.
    struct Res { std::vector<int> w, s, st; uint64_t mw, ms, mst, bytes; };
    Res best{};
    bool have_best = false;
    for (int pass = 0; pass < 16; ++pass) {
      for (auto& lp : p.layers) {
        lp.wc_res = -1; lp.state_res = -1;
        std::fill(lp.stash_res.begin(), lp.stash_res.end(), -1);
      }
      const uint64_t used = fixed + nW * maxw + nS * maxs + nG * maxst;
      uint64_t room = p.cap > used ? p.cap - used : 0;
      const uint64_t room0 = room;
      if (!baseline) {
        // compute weights: 3 B of transfer saved per resident byte; backward order
        for (int l = L - 1; l >= 0; --l) {
          uint64_t sz = align_up(p.layers[l].wc_bytes, ALIGN);
          if (sz <= room) { p.layers[l].wc_res = 0; room -= sz; }
        }
        // master/m/v: 2 B saved per byte, both in the backward (swap-in before the JIT update,
        // swap-out after it).  With equal per-layer state sizes the streamed layers are spread
        // evenly over the backward order instead of being the last ones updated: each streamed
        // layer's swap-in then overlaps the backward of the resident layers before it, rather
        // than a run of consecutive updates waiting on the host link.
        bool uniform = true;
        for (int l = 1; l < L; ++l) uniform = uniform && p.layers[l].state_bytes == p.layers[0].state_bytes;
        const uint64_t ssz = align_up(p.layers[0].state_bytes, ALIGN);
        if (uniform && ssz > 0 && (uint64_t)L * ssz > room) {
          const int keep = (int)std::min<uint64_t>(room / ssz, (uint64_t)L);
          const int nstream = L - keep;
          // backward position j (0 = layer L-1) is streamed iff floor((j+1) n / L) > floor(j n / L)
          for (int j = 0; j < L; ++j) {
            const bool streamed = (int64_t)(j + 1) * nstream / L > (int64_t)j * nstream / L;
            if (!streamed) { p.layers[L - 1 - j].state_res = 0; room -= ssz; }
          }
        } else {
          for (int l = L - 1; l >= 0; --l) {
            uint64_t sz = align_up(p.layers[l].state_bytes, ALIGN);
            if (sz <= room) { p.layers[l].state_res = 0; room -= sz; }
          }
        }
      }
      // stash: 2 B saved per byte.  Equal-size entries: the spilled (layer, microbatch) entries are
      // spread evenly over the backward order (as the streamed state above), so each one's swap-in
      // overlaps the backward of resident entries instead of a run of spilled entries at the end
      // of the backward waiting on the host link; otherwise LIFO (consumed first in the backward).
      bool st_uniform = true;
      for (int l = 1; l < L; ++l) st_uniform = st_uniform && p.layers[l].g.st.total == p.layers[0].g.st.total;
      const uint64_t gsz = align_up(p.layers[0].g.st.total, ALIGN);
      const int nent = L * m;
      if (st_uniform && gsz > 0 && (uint64_t)nent * gsz > room && !baseline) {
        const int keep = (int)std::min<uint64_t>(room / gsz, (uint64_t)nent);
        const int nspill = nent - keep;
        for (int j = 0; j < nent; ++j) {  // backward position j: layer L-1-j/m, microbatch j%m
          const bool spilled = (int64_t)(j + 1) * nspill / nent > (int64_t)j * nspill / nent;
          if (!spilled) { p.layers[L - 1 - j / m].stash_res[j % m] = 0; room -= gsz; }
        }
      } else {
        for (int l = L - 1; l >= 0; --l)
          for (int i = 0; i < m; ++i) {
            uint64_t sz = align_up(p.layers[l].g.st.total, ALIGN);
            if (sz <= room) { p.layers[l].stash_res[i] = 0; room -= sz; }
          }
      }
      Res r{};
      r.bytes = room0 - room;
      r.mw = r.ms = r.mst = 0;
      for (auto& lp : p.layers) {
        r.w.push_back(lp.wc_res); r.s.push_back(lp.state_res);
        r.st.insert(r.st.end(), lp.stash_res.begin(), lp.stash_res.end());
        if (lp.wc_res < 0) r.mw = std::max(r.mw, align_up(lp.wc_bytes, ALIGN));
        if (lp.state_res < 0) r.ms = std::max(r.ms, align_up(lp.state_bytes, ALIGN));
        for (int i = 0; i < m; ++i)
          if (lp.stash_res[i] < 0) r.mst = std::max(r.mst, align_up(lp.g.st.total, ALIGN));
      }
      const bool fits = r.mw <= maxw && r.ms <= maxs && r.mst <= maxst;  // streamed items fit the slots
      const bool fixed_point = r.mw == maxw && r.ms == maxs && r.mst == maxst;
      if (fits) { best = r; have_best = true; }
      if (fixed_point || !fits) break;
      maxw = r.mw; maxs = r.ms; maxst = r.mst;
    }
    HM_CHECK(have_best, HARMONY_E_CAP_TOO_SMALL, "internal: no consistent residency");
    {
      size_t k = 0, ks = 0;
      for (auto& lp : p.layers) {
        lp.wc_res = best.w[k]; lp.state_res = best.s[k]; ++k;
        for (int i = 0; i < m; ++i) lp.stash_res[i] = best.st[ks++];
      }
    }
    maxw = best.mw; maxs = best.ms; maxst = best.mst;
    const uint64_t resident_bytes = best.bytes;
    nW = maxw ? std::max(nW, 1) : 0;
    nS = maxs ? std::max(nS, 1) : 0;
    nG = maxst ? std::max(nG, 1) : 0;
    HM_CHECK(fixed + nW * maxw + nS * maxs + nG * maxst + resident_bytes <= p.cap, HARMONY_E_CAP_TOO_SMALL,
             "internal: residency exceeds the cap");
    // upgrade slot counts (double buffering) where the residency above still leaves room
    for (auto& c : pref) {
      const int w = maxw ? std::max(nW, c[0]) : 0, s2 = maxs ? std::max(nS, c[1]) : 0,
                g2 = maxst ? std::max(nG, c[2]) : 0;
      if (fixed + w * maxw + s2 * maxs + g2 * maxst + resident_bytes <= p.cap) { nW = w; nS = s2; nG = g2; break; }
    }
    p.wslot_bytes = maxw; p.sslot_bytes = maxs; p.stage_bytes = maxst;
  }
  // A lagged update (N > 1) writes the compute copy back into the slot its backward used;
  // with a single weight slot that slot already holds the next layer, so update immediately.
  if (nW == 1) p.upd_lag = 0;

  // ---------------------------------------------------------------- arena layout
  Arena a;
  p.bnd_row_stride = bnd_stride;
  p.tgt_row_stride = tgt_stride;
  p.bnd_bytes = bnd_stride * m;
  for (int j = 0; j < p.n_bnd; ++j) p.bnd[j] = a.take(p.bnd_bytes);
  p.tgt = a.take(tgt_stride * m);
  p.ws_bytes = ws_need;
  p.ws = a.take(ws_need);
  p.dw.assign(nDW, 0);
  for (int j = 0; j < nDW; ++j) p.dw[j] = a.take(maxP * 4);
  if (N > 1) for (int j = 0; j < 2; ++j) p.gsh[j] = a.take(max_shard * 4);
  p.loss = a.take((uint64_t)N * m * 8);
  p.loss_scratch = a.take(mse_scratch_bytes());
  p.tstep = a.take(256);
  for (int j = 0; j < nW; ++j) p.wslot.push_back(a.take(p.wslot_bytes));
  for (int j = 0; j < nS; ++j) p.sslot.push_back(a.take(p.sslot_bytes));
  for (int j = 0; j < nG; ++j) p.stage.push_back(a.take(p.stage_bytes));
  for (auto& lp : p.layers) {
    if (lp.wc_res >= 0) lp.wc_res = (int64_t)a.take(lp.wc_bytes);
    if (lp.state_res >= 0) lp.state_res = (int64_t)a.take(lp.state_bytes);
  }
  for (int l = L - 1; l >= 0; --l)
    for (int i = 0; i < m; ++i)
      if (p.layers[l].stash_res[i] >= 0) p.layers[l].stash_res[i] = (int64_t)a.take(p.layers[l].g.st.total);
  p.arena_bytes = a.cur;
  HM_CHECK(uncapped || p.arena_bytes <= p.cap, HARMONY_E_CAP_TOO_SMALL, "internal: arena layout exceeds the cap");
  if (layout_only) {
    harmony_plan_summary& s = p.summary;
    s.arena_bytes = p.arena_bytes;
    s.min_working_set_bytes = p.min_ws_bytes;
    s.n_params = p.n_params;
    s.weight_slots = nW; s.state_slots = nS; s.stash_slots = nG;
    return p;
  }

  // ---------------------------------------------------------------- program
  Tracker tr;
  tr.ops = &p.ops;
  auto bnd_row = [&](int buf, int i) { return p.bnd[buf] + (uint64_t)i * bnd_stride; };

  // Input items (prefetchable swap-ins) and their slot occupancies.
  struct Item {
    int need = 0;                 // task index that needs it
    int release = -1;             // task after which the slot is free
    std::vector<std::pair<Op, std::pair<std::vector<uint64_t>, std::vector<uint64_t>>>> ops;
  };
  struct Task {
    Op op;
    std::vector<uint64_t> rd, wr;
    std::vector<std::pair<Op, std::pair<std::vector<uint64_t>, std::vector<uint64_t>>>> post;
  };
  std::vector<Task> tasks;
  std::vector<Item> items;

  // slot bookkeeping: last task index using each slot
  std::vector<int> wslot_last(nW, -1), sslot_last(nS, -1), stage_last(nG, -1);
  int wnext = 0, snext = 0, gnext = 0;

  // weight location for each layer use (fwd / bwd)
  auto weight_use = [&](int l, int need_task, int& slot) -> uint64_t {
    LayerPlan& lp = p.layers[l];
    if (lp.wc_res >= 0) { slot = -1; return (uint64_t)lp.wc_res; }
    slot = wnext;
    wnext = (wnext + 1) % nW;
    Item it;
    it.need = need_task;
    it.release = wslot_last[slot];
    const uint64_t dst = p.wslot[slot];
    const uint64_t sh_bytes = (uint64_t)lp.shard * ts;
    Op h;
    h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_WEIGHT; h.layer = l;
    h.hbuf = HB_WC; h.hidx = l; h.hoff = 0; h.dev = dst + (uint64_t)r * sh_bytes; h.bytes = sh_bytes;
    it.ops.push_back({h, {{key(H_WC, l)}, {key(R_WSLOT, slot)}}});
    if (N > 1) {
      Op g;
      g.kind = OP_ALLGATHER; g.stream = S_COMM; g.cat = CAT_WEIGHT; g.layer = l;
      g.dev = dst; g.count = (uint64_t)lp.shard; g.bytes = sh_bytes * (N - 1);
      it.ops.push_back({g, {{key(R_WSLOT, slot)}, {key(R_WSLOT, slot)}}});
    }
    items.push_back(it);
    return dst;
  };
  auto wkey = [&](int l, int slot) { return slot >= 0 ? key(R_WSLOT, slot) : key(R_WRES, l); };

  // ---- forward
  std::vector<int> fwd_wslot(L, -1);
  // FWD task that spills each (l, i): a backward swap-in of that stash may not be issued before it
  std::vector<int> spill_task((size_t)L * m, -1);
  {
    Task t;  // inputs are issued as the first ops (not prefetch items)
    (void)t;
  }
  auto fwd_task = [&](int l, int i, bool gfirst, int pack) {
    LayerPlan& lp = p.layers[l];
    const int in_buf = lp.user % 2, out_buf = (lp.user + 1) % 2;  // a registered layer's panels share its buffers
    int slot = -1;
    uint64_t wdev;
    if (baseline || gfirst) wdev = weight_use(l, (int)tasks.size(), slot);  // grouping: one swap-in per layer and group
    else { slot = fwd_wslot[l]; wdev = slot >= 0 ? p.wslot[slot] : (uint64_t)lp.wc_res; }
    fwd_wslot[l] = slot;
    Task t;
    t.op.kind = OP_FWD; t.op.stream = S_COMPUTE; t.op.layer = l; t.op.mb = i; t.op.pack = pack;
    t.op.w = wdev; t.op.in = bnd_row(in_buf, i); t.op.out = bnd_row(out_buf, i); t.op.ws = p.ws;
    t.rd = {wkey(l, slot)};
    // a pack reads / writes the consecutive (contiguous) rows of its microbatches and writes each one's stash
    for (int k = 0; k < pack; ++k) {
      const int ik = i + k;
      t.rd.push_back(key(R_BND, in_buf, ik));
      t.wr.push_back(key(R_BND, out_buf, ik));
      uint64_t& dst = k == 0 ? t.op.stash : t.op.stash2;
      if (lp.stash_res[ik] >= 0) {
        dst = (uint64_t)lp.stash_res[ik];
        t.wr.push_back(key(R_STASHRES, l, ik));
      } else {
        int g = gnext;
        gnext = (gnext + 1) % nG;
        dst = p.stage[g];
        t.wr.push_back(key(R_STAGE, g));
        Op d;
        d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_STASH; d.layer = l; d.mb = ik;
        d.hbuf = HB_STASH; d.hidx = (int64_t)l * m + ik; d.dev = p.stage[g]; d.bytes = lp.g.st.total;
        t.post.push_back({d, {{key(R_STAGE, g)}, {key(H_STASH, l, ik)}}});
        stage_last[g] = (int)tasks.size();
        spill_task[(size_t)l * m + ik] = (int)tasks.size();
      }
    }
    HM_CHECK(pack == 1 || t.op.stash != t.op.stash2, HARMONY_E_CAP_TOO_SMALL,
             "fwd_pack = 2 needs two staging slots for two spilled stashes");
    if (slot >= 0) wslot_last[slot] = (int)tasks.size();
    if (baseline && slot >= 0) {  // per-GPU virtualization: weights out again after each forward
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_WEIGHT; d.layer = l; d.mb = i;
      d.hbuf = HB_WC; d.hidx = l; d.dev = wdev + (uint64_t)r * lp.shard * ts; d.bytes = (uint64_t)lp.shard * ts;
      t.post.push_back({d, {{key(R_WSLOT, slot)}, {key(H_WC, l)}}});
    }
    tasks.push_back(t);
  };
  // ---- loss
  const int Lb = LU % 2, dYb = (LU + 1) % 2;
  auto loss_task = [&](int i) {
    Task t;
    t.op.kind = OP_LOSS; t.op.stream = S_COMPUTE; t.op.mb = i;
    t.op.in = bnd_row(Lb, i); t.op.tgt = p.tgt + (uint64_t)i * tgt_stride; t.op.out = bnd_row(dYb, i);
    t.op.loss = p.loss + (uint64_t)(r * m + i) * 8;
    t.rd = {key(R_BND, Lb, i), key(R_TGT, i)};
    t.wr = {key(R_BND, dYb, i), key(R_LOSS, i)};
    if (i == m - 1) {
      Op o;
      if (N > 1) {
        o.kind = OP_LOSS_GATHER; o.stream = S_COMM; o.dev = p.loss; o.count = (uint64_t)m; o.bytes = (uint64_t)m * 8 * (N - 1);
        std::vector<uint64_t> rds;
        for (int j = 0; j < m; ++j) rds.push_back(key(R_LOSS, j));
        t.post.push_back({o, {rds, {key(R_LOSSALL, 0)}}});
        Op d;
        d.kind = OP_LOSS_OUT; d.stream = S_D2H; d.cat = CAT_OUTPUT; d.dev = p.loss; d.bytes = (uint64_t)N * m * 8;
        t.post.push_back({d, {{key(R_LOSSALL, 0)}, {}}});
      } else {
        o.kind = OP_LOSS_OUT; o.stream = S_D2H; o.cat = CAT_OUTPUT; o.dev = p.loss; o.bytes = (uint64_t)m * 8;
        std::vector<uint64_t> rds;
        for (int j = 0; j < m; ++j) rds.push_back(key(R_LOSS, j));
        t.post.push_back({o, {rds, {}}});
      }
    }
    tasks.push_back(t);
  };
  // ---- backward + JIT update
  std::vector<int> bwd_wslot(L, -1);
  std::vector<int> pending_upd;
  auto emit_upd = [&](int l) {
    LayerPlan& lp = p.layers[l];
    Task t;
    t.op.kind = OP_UPD; t.op.stream = S_COMPUTE; t.op.layer = l;
    const int j = dwi(l);
    uint64_t gkey = key(R_DW, j);
    if (N > 1) { t.op.grad = p.gsh[l % 2]; gkey = key(R_GSH, l % 2); }
    else t.op.grad = p.dw[j];
    t.rd = {gkey};
    if (baseline) {
      // the baseline updates after the whole backward: this layer's gradient was
      // swapped out after its backward and comes back now
      Item it;
      it.need = (int)tasks.size();
      it.release = (int)tasks.size() - 1;
      Op h;
      h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_GRAD; h.layer = l;
      h.hbuf = HB_GRAD; h.hidx = l; h.dev = t.op.grad; h.bytes = (uint64_t)lp.shard * 4;
      it.ops.push_back({h, {{key(H_GRAD, l)}, {gkey}}});
      items.push_back(it);
    }
    int sslot = -1;
    if (lp.state_res >= 0) {
      t.op.state = (uint64_t)lp.state_res;
      t.rd.push_back(key(R_SRES, l));
      t.wr.push_back(key(R_SRES, l));
    } else {
      sslot = snext;
      snext = (snext + 1) % nS;
      Item it;
      it.need = (int)tasks.size();
      it.release = sslot_last[sslot];
      Op h;
      h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_STATE; h.layer = l;
      h.hbuf = HB_STATE; h.hidx = l; h.dev = p.sslot[sslot]; h.bytes = lp.state_bytes;
      it.ops.push_back({h, {{key(H_STATE, l)}, {key(R_SSLOT, sslot)}}});
      items.push_back(it);
      t.op.state = p.sslot[sslot];
      t.rd.push_back(key(R_SSLOT, sslot));
      t.wr.push_back(key(R_SSLOT, sslot));
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_STATE; d.layer = l;
      d.hbuf = HB_STATE; d.hidx = l; d.dev = p.sslot[sslot]; d.bytes = lp.state_bytes;
      t.post.push_back({d, {{key(R_SSLOT, sslot)}, {key(H_STATE, l)}}});
      sslot_last[sslot] = (int)tasks.size();
    }
    // the compute copy this rank's shard is written into (the baseline's backward slot of this layer
    // was reused long ago: it takes the next slot in turn)
    int wsl = bwd_wslot[l];
    if (baseline && lp.wc_res < 0) { wsl = wnext; wnext = (wnext + 1) % nW; }
    const uint64_t sh_bytes = (uint64_t)lp.shard * ts;
    if (lp.wc_res >= 0) {
      t.op.w = (uint64_t)lp.wc_res;
      t.wr.push_back(key(R_WRES, l));
      if (N > 1) {
        Op g;
        g.kind = OP_ALLGATHER; g.stream = S_COMM; g.cat = CAT_WEIGHT; g.layer = l;
        g.dev = (uint64_t)lp.wc_res; g.count = (uint64_t)lp.shard; g.bytes = sh_bytes * (N - 1);
        t.post.push_back({g, {{key(R_WRES, l)}, {key(R_WRES, l)}}});
      }
    } else {
      t.op.w = p.wslot[wsl];
      t.wr.push_back(key(R_WSLOT, wsl));
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_WEIGHT; d.layer = l;
      d.hbuf = HB_WC; d.hidx = l; d.dev = p.wslot[wsl] + (uint64_t)r * sh_bytes; d.bytes = sh_bytes;
      t.post.push_back({d, {{key(R_WSLOT, wsl)}, {key(H_WC, l)}}});
      wslot_last[wsl] = (int)tasks.size();
    }
    if (p.retain_grads) {
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_GRAD; d.layer = l;
      d.hbuf = HB_GRAD; d.hidx = l; d.dev = t.op.grad; d.bytes = (uint64_t)lp.shard * 4;
      t.post.push_back({d, {{gkey}, {key(H_GRAD, l)}}});
    }
    tasks.push_back(t);
  };

  // registered layers in reverse; a layer's column panels in order (the dX reduction runs through them)
  std::vector<int> bwd_order;
  for (int u = LU - 1; u >= 0; --u)
    for (int k = 0; k < p.user_count[u]; ++k) bwd_order.push_back(p.user_first[u] + k);
  auto bwd_task = [&](int l, int i, bool gfirst) {
    LayerPlan& lp = p.layers[l];
    const int in_buf = lp.user % 2, out_buf = (lp.user + 1) % 2;
    const int j = dwi(l);
    int slot = -1;
    uint64_t wdev;
    if (baseline || gfirst) wdev = weight_use(l, (int)tasks.size(), slot);
    else { slot = bwd_wslot[l]; wdev = slot >= 0 ? p.wslot[slot] : (uint64_t)lp.wc_res; }
    bwd_wslot[l] = slot;
    Task t;
    t.op.kind = OP_BWD; t.op.stream = S_COMPUTE; t.op.layer = l; t.op.mb = i; t.op.first = i == 0;
    t.op.w = wdev; t.op.in = bnd_row(in_buf, i); t.op.out = bnd_row(out_buf, i); t.op.ws = p.ws; t.op.dw = p.dw[j];
    t.rd = {wkey(l, slot), key(R_BND, in_buf, i)};
    t.wr = {key(R_BND, out_buf, i), key(R_DW, j)};
    if (i > 0) t.rd.push_back(key(R_DW, j));
    if (lp.stash_res[i] >= 0) {
      t.op.stash = (uint64_t)lp.stash_res[i];
      t.rd.push_back(key(R_STASHRES, l, i));
    } else {
      int g = gnext;
      gnext = (gnext + 1) % nG;
      Item it;
      it.need = (int)tasks.size();
      // free staging slot AND the spill of this very stash already issued (read after write)
      it.release = std::max(stage_last[g], spill_task[(size_t)l * m + i]);
      Op h;
      h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_STASH; h.layer = l; h.mb = i;
      h.hbuf = HB_STASH; h.hidx = (int64_t)l * m + i; h.dev = p.stage[g]; h.bytes = lp.g.st.total;
      it.ops.push_back({h, {{key(H_STASH, l, i)}, {key(R_STAGE, g)}}});
      items.push_back(it);
      t.op.stash = p.stage[g];
      t.rd.push_back(key(R_STAGE, g));
      stage_last[g] = (int)tasks.size();
    }
    if (slot >= 0) wslot_last[slot] = (int)tasks.size();
    if (i == m - 1 && N > 1) {
      Op rs;
      rs.kind = OP_REDUCESCATTER; rs.stream = S_COMM; rs.cat = CAT_GRAD; rs.layer = l;
      rs.dev = p.dw[j]; rs.grad = p.gsh[l % 2]; rs.count = (uint64_t)lp.shard;
      rs.bytes = (uint64_t)lp.shard * 4 * (N - 1);
      t.post.push_back({rs, {{key(R_DW, j)}, {key(R_GSH, l % 2)}}});
    }
    if (baseline) {
      // per-GPU virtualization swaps the layer's weights out again after every microbatch's
      // backward (Fig. 5(b); clean, so the bytes are those already on the host), and
      // parks the finished gradient on the host until the update at the end of the backward
      if (slot >= 0) {
        Op d;
        d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_WEIGHT; d.layer = l; d.mb = i;
        d.hbuf = HB_WC; d.hidx = l; d.dev = wdev + (uint64_t)r * lp.shard * ts; d.bytes = (uint64_t)lp.shard * ts;
        t.post.push_back({d, {{key(R_WSLOT, slot)}, {key(H_WC, l)}}});
      }
      if (i == m - 1) {
        const uint64_t gk = N > 1 ? key(R_GSH, l % 2) : key(R_DW, j);
        Op d;
        d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_GRAD; d.layer = l;
        d.hbuf = HB_GRAD; d.hidx = l; d.dev = N > 1 ? p.gsh[l % 2] : p.dw[j]; d.bytes = (uint64_t)lp.shard * 4;
        t.post.push_back({d, {{gk}, {key(H_GRAD, l)}}});
      }
    }
    tasks.push_back(t);
  };
  auto bwd_layer_done = [&](int l) {  // after the layer's last microbatch: its update, just in time
  if (!baseline) {
    pending_upd.push_back(l);
    while ((int)pending_upd.size() > p.upd_lag) {
      emit_upd(pending_upd.front());
      pending_upd.erase(pending_upd.begin());
    }
  } else {
    pending_upd.push_back(l);  // baseline: every update after the whole backward
  }
  };
  // Microbatch groups (direction balance): group 0's forward, then each group's
  // backward interleaved layer by layer with the next group's forward, so stash swap-ins (backward)
  // and spills (forward) use both directions of the host link at once.  The microbatches stay in
  // canonical order in every dW accumulation: the result is bit-identical for every G (reading c21).
  auto fwd_group = [&](int g, int l) {
    for (int i = g * mg; i < (g + 1) * mg; i += p.fwd_pack) fwd_task(l, i, i == g * mg, p.fwd_pack);
  };
  auto loss_group = [&](int g) {
    for (int i = g * mg; i < (g + 1) * mg; ++i) loss_task(i);
  };
  for (int l = 0; l < L; ++l) fwd_group(0, l);
  loss_group(0);
  for (int g = 0; g < G; ++g) {
    for (int k = 0; k < (int)bwd_order.size(); ++k) {
      const int l = bwd_order[k];
      for (int i = g * mg; i < (g + 1) * mg; ++i) bwd_task(l, i, i == g * mg);
      if (g == G - 1) bwd_layer_done(l);
      if (g + 1 < G) fwd_group(g + 1, k);
    }
    if (g + 1 < G) loss_group(g + 1);
  }
  for (int l : pending_upd) emit_upd(l);

  // ---- merge tasks and prefetch items into one program
  {
    // inputs first (user X into the layer-0 activation rows, targets)
    Op x;
    x.kind = OP_INPUT; x.stream = S_H2D; x.cat = CAT_INPUT; x.hbuf = HB_USER_X; x.dev = p.bnd[0];
    x.bytes = (uint64_t)p.in_elems_per_mb * 4;
    for (int i = 0; i < m; ++i) {
      Op xi = x;
      xi.mb = i; xi.dev = bnd_row(0, i); xi.hoff = (uint64_t)i * p.in_elems_per_mb * 4;
      tr.add(xi, {}, {key(R_BND, 0, i)});
    }
    for (int i = 0; i < m; ++i) {
      Op ti = x;
      ti.hbuf = HB_USER_T; ti.mb = i; ti.dev = p.tgt + (uint64_t)i * tgt_stride;
      ti.hoff = (uint64_t)i * p.out_elems_per_mb * 4; ti.bytes = (uint64_t)p.out_elems_per_mb * 4;
      tr.add(ti, {}, {key(R_TGT, i)});
    }
    // items are created in need order per class; merge them by need
    std::stable_sort(items.begin(), items.end(), [](const Item& a2, const Item& b2) { return a2.need < b2.need; });
    size_t next = 0;
    auto emit_item = [&](Item& it) {
      for (auto& o : it.ops) tr.add(o.first, o.second.first, o.second.second);
    };
    for (int k = 0; k < (int)tasks.size(); ++k) {
      while (next < items.size() && items[next].need <= k) emit_item(items[next++]);
      Task& t = tasks[k];
      tr.add(t.op, t.rd, t.wr);
      for (auto& o : t.post) tr.add(o.first, o.second.first, o.second.second);
      while (next < items.size() && items[next].release <= k) emit_item(items[next++]);
    }
    while (next < items.size()) emit_item(items[next++]);
  }
  // events: one per op that another stream waits on
  {
    std::vector<int> ev(p.ops.size(), -1);
    int ne = 0;
    for (auto& o : p.ops)
      for (int w : o.waits)
        if (ev[w] < 0) ev[w] = ne++;
    for (size_t i = 0; i < p.ops.size(); ++i) p.ops[i].event = ev[i];
    p.n_events = ne;
  }

  // ---------------------------------------------------------------- summary
  harmony_plan_summary& s = p.summary;
  s.arena_bytes = p.arena_bytes;
  s.min_working_set_bytes = p.min_ws_bytes;
  s.n_params = p.n_params;
  s.weight_slots = nW; s.state_slots = nS; s.stash_slots = nG;
  double fl = 0;
  for (auto& lp : p.layers) {
    s.total_weight_bytes += lp.wc_bytes;
    s.total_state_bytes += lp.state_bytes;
    s.total_stash_bytes += (uint64_t)m * lp.g.st.total;
    if (lp.wc_res >= 0) s.resident_weight_bytes += lp.wc_bytes;
    if (lp.state_res >= 0) s.resident_state_bytes += lp.state_bytes;
    for (int i = 0; i < m; ++i)
      if (lp.stash_res[i] >= 0) s.resident_stash_bytes += lp.g.st.total;
    fl += 3.0 * lp.g.flops_fwd * m;
  }
  s.flops_per_step = (uint64_t)fl;
  for (auto& o : p.ops) {
    const bool copy_in = o.kind == OP_H2D || o.kind == OP_INPUT;
    const bool copy_out = o.kind == OP_D2H || o.kind == OP_LOSS_OUT;
    if (copy_in) s.pred_h2d_bytes += o.bytes;
    if (copy_out) s.pred_d2h_bytes += o.bytes;
    if (copy_in && o.cat == CAT_WEIGHT) s.pred_h2d_weight_bytes += o.bytes;
    if (copy_out && o.cat == CAT_WEIGHT) s.pred_d2h_weight_bytes += o.bytes;
    if (o.stream == S_COMPUTE) s.n_compute_ops++;
    else if (o.stream == S_COMM) s.n_comm_ops++;
    else s.n_copy_ops++;
  }
  s.n_ops = (int32_t)p.ops.size();
  std::string why;
  s.hazards = validate_program(p, &why);
  p.hazard_msg = why;
  return p;
}

std::string dump_plan(const Plan& p) {
  static const char* kn[] = {"INPUT", "H2D", "D2H", "FWD", "LOSS", "BWD", "UPD", "ALLGATHER", "REDUCESCATTER",
                             "LOSS_GATHER", "LOSS_OUT"};
  static const char* sn[] = {"compute", "h2d", "d2h", "comm"};
  static const char* cn[] = {"weight", "state", "stash", "input", "output", "grad", "-"};
  std::ostringstream os;
  os << "# plan N=" << p.N << " rank=" << p.rank << " m=" << p.m << " b=" << p.b << " dtype=" << p.dtype
     << " cap=" << p.cap << " arena=" << p.arena_bytes << " wslots=" << p.wslot.size() << " sslots=" << p.sslot.size()
     << " stage=" << p.stage.size() << " ops=" << p.ops.size() << " events=" << p.n_events << "\n";
  for (size_t i = 0; i < p.ops.size(); ++i) {
    const Op& o = p.ops[i];
    os << i << " " << kn[o.kind] << " " << sn[o.stream] << " cat=" << cn[o.cat] << " l=" << o.layer << " i=" << o.mb
       << " bytes=" << o.bytes;
    if (o.kind == OP_BWD) os << " first=" << o.first;
    os << " waits=";
    for (size_t k = 0; k < o.waits.size(); ++k) os << (k ? "," : "") << o.waits[k];
    os << "\n";
  }
  return os.str();
}


// ------------------------------------------------------------------------------------ Harmony-PP
namespace {
// resource keys of one rank (bits 48..55 = rank; key() keeps a < 2^20, b < 2^28)
inline uint64_t rkey(int rank, ResKind k, uint64_t a, uint64_t b = 0) { return key(k, a, b) | ((uint64_t)rank << 48); }

struct GTracker {
  int N;
  std::unordered_map<uint64_t, Tracker::Res> res;
  std::vector<GOp>* ops;
  int add(int rank, Op op, const std::vector<uint64_t>& reads, const std::vector<uint64_t>& writes) {
    const int idx = (int)ops->size();
    std::vector<int> deps;
    for (uint64_t r : reads) {
      auto it = res.find(r);
      if (it != res.end() && it->second.writer >= 0) deps.push_back(it->second.writer);
    }
    for (uint64_t w : writes) {
      auto it = res.find(w);
      if (it == res.end()) continue;
      if (it->second.writer >= 0) deps.push_back(it->second.writer);
      for (int rd : it->second.readers) deps.push_back(rd);
    }
    // the latest dependency per other (rank, stream): each stream executes in order
    std::map<int, int> latest;
    const int self = rank * S_NUM + op.stream;
    for (int d : deps) {
      const int s = (*ops)[d].rank * S_NUM + (*ops)[d].op.stream;
      if (s != self) latest[s] = std::max(latest.count(s) ? latest[s] : -1, d);
    }
    op.waits.clear();
    for (auto& kv : latest) op.waits.push_back(kv.second);
    for (uint64_t r : reads) res[r].readers.push_back(idx);
    for (uint64_t w : writes) {
      Tracker::Res& x = res[w];
      x.writer = idx;
      x.readers.clear();
    }
    ops->push_back(GOp{rank, op});
    return idx;
  }
};

// The independent race check of validate_program over the whole group: per-rank arenas and host
// stores are separate address spaces; happens-before over every (rank, stream).
int validate_group(const GroupPlan& g, std::string* first) {
  const size_t n = g.ops.size();
  const int NS = g.N * S_NUM;
  std::vector<std::vector<int>> vc(n, std::vector<int>(NS, -1));
  std::vector<int> pos(n), cnt(NS, 0), last(NS, -1);
  auto sid = [&](size_t i) { return g.ops[i].rank * S_NUM + g.ops[i].op.stream; };
  for (size_t i = 0; i < n; ++i) {
    const int s = sid(i);
    std::vector<int> c(NS, -1);
    if (last[s] >= 0) c = vc[last[s]];
    for (int w : g.ops[i].op.waits)
      for (int k = 0; k < NS; ++k) c[k] = std::max(c[k], vc[w][k]);
    pos[i] = cnt[s]++;
    c[s] = pos[i];
    vc[i] = c;
    last[s] = (int)i;
  }
  auto hb = [&](size_t a, size_t b) { return vc[b][sid(a)] >= pos[a]; };
  std::vector<std::vector<Acc>> acc(n);
  for (size_t i = 0; i < n; ++i) {
    const GOp& o = g.ops[i];
    if (o.op.kind == OP_P2P) {
      acc[i].push_back({16 * o.rank, 0, o.op.dev, o.op.dev + o.op.bytes, true});
      acc[i].push_back({16 * o.op.peer, 0, o.op.peer_off, o.op.peer_off + o.op.bytes, false});
      continue;
    }
    for (Acc a : accesses(g.ranks[o.rank], o.op)) {
      a.space += 16 * o.rank;
      acc[i].push_back(a);
    }
  }
  int hazards = 0;
  for (size_t j = 0; j < n; ++j)
    for (size_t i = 0; i < j; ++i) {
      if (sid(i) == sid(j) || hb(i, j)) continue;
      for (const Acc& a : acc[i])
        for (const Acc& b : acc[j])
          if ((a.write || b.write) && a.space == b.space && a.idx == b.idx && a.lo < b.hi && b.lo < a.hi) {
            if (hazards == 0 && first)
              *first = "ops " + std::to_string(i) + " and " + std::to_string(j) + " race on space " +
                       std::to_string(a.space) + "[" + std::to_string(a.idx) + "]";
            ++hazards;
            goto next_pair;
          }
    next_pair:;
    }
  return hazards;
}
}  // namespace

GroupPlan make_plan_pp(const harmony_config& cfg, int N, int L, const harmony_layer_desc* descs) {
  validate_config(cfg);
  validate_layers(cfg, L, descs);
  HM_CHECK(N >= 2 && N <= 16, HARMONY_E_INVALID_ARG, "Harmony-PP needs a group of 2..16 ranks");
  HM_CHECK(L >= N, HARMONY_E_INVALID_ARG, "Harmony-PP needs at least as many layers as ranks");
  GroupPlan G;
  G.N = N;
  G.layer_rank.resize(L);
  G.layer_local.resize(L);
  for (int l = 0; l < L; ++l) { G.layer_rank[l] = l % N; G.layer_local[l] = l / N; }
  // per-rank layout: the rank's layers as one stack of one rank (the update is not sharded: each layer
  // lives on one GPU), four activation buffers (A_in, A_out, G_in, G_out)
  HM_CHECK(cfg.groups <= 1, HARMONY_E_UNSUPPORTED, "microbatch groups are a Harmony-DP schedule");
  HM_CHECK(cfg.fwd_pack <= 1, HARMONY_E_UNSUPPORTED, "forward packs are a Harmony-DP schedule");
  harmony_config rc = cfg;
  rc.world_size = 1; rc.rank = 0; rc.schedule = HARMONY_SCHED_HARMONY_DP; rc.groups = 1;
  for (int r = 0; r < N; ++r) {
    std::vector<harmony_layer_desc> sub;
    for (int l = r; l < L; l += N) sub.push_back(descs[l]);
    G.ranks.push_back(make_plan(rc, (int)sub.size(), sub.data(), /*layout_only=*/true, /*n_bnd=*/4));
  }
  const int m = cfg.microbatches;
  const uint64_t ts = cfg.precision == HARMONY_BF16_FP32MASTER ? 2 : 4;
  GTracker tr{N, {}, &G.ops};
  auto row = [&](int r, int buf, int i) { return G.ranks[r].bnd[buf] + (uint64_t)i * G.ranks[r].bnd_row_stride; };
  enum { A_IN = 0, A_OUT = 1, G_IN = 2, G_OUT = 3 };

  struct Rec { int rank; Op op; std::vector<uint64_t> rd, wr; };
  struct Item { int need = 0, release = -1; std::vector<Rec> ops; };
  struct Task { Rec t; std::vector<Rec> post; };
  std::vector<Task> tasks;
  std::vector<Item> items;
  struct Slots { std::vector<int> wlast, slast, glast; int wn = 0, sn = 0, gn = 0; };
  std::vector<Slots> sl(N);
  for (int r = 0; r < N; ++r) {
    sl[r].wlast.assign(G.ranks[r].wslot.size(), -1);
    sl[r].slast.assign(G.ranks[r].sslot.size(), -1);
    sl[r].glast.assign(G.ranks[r].stage.size(), -1);
  }
  auto weight_use = [&](int r, int k, int need, int& slot) -> uint64_t {
    Plan& P = G.ranks[r];
    LayerPlan& lp = P.layers[k];
    if (lp.wc_res >= 0) { slot = -1; return (uint64_t)lp.wc_res; }
    Slots& S = sl[r];
    slot = S.wn;
    S.wn = (S.wn + 1) % (int)P.wslot.size();
    Item it;
    it.need = need;
    it.release = S.wlast[slot];
    Op h;
    h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_WEIGHT; h.layer = k;
    h.hbuf = HB_WC; h.hidx = k; h.dev = P.wslot[slot]; h.bytes = (uint64_t)lp.shard * ts;
    it.ops.push_back({r, h, {rkey(r, H_WC, k)}, {rkey(r, R_WSLOT, slot)}});
    items.push_back(it);
    return P.wslot[slot];
  };
  auto wkey = [&](int r, int k, int slot) { return slot >= 0 ? rkey(r, R_WSLOT, slot) : rkey(r, R_WRES, k); };

  // ---- forward: layer by layer, each layer's m microbatches back to back on its rank (grouping)
  std::vector<int> fwd_slot(L, -1), spill_task((size_t)L * m, -1);
  for (int l = 0; l < L; ++l) {
    const int r = G.layer_rank[l], k = G.layer_local[l];
    Plan& P = G.ranks[r];
    LayerPlan& lp = P.layers[k];
    for (int i = 0; i < m; ++i) {
      int slot = fwd_slot[l];
      uint64_t w;
      if (i == 0) { w = weight_use(r, k, (int)tasks.size(), slot); fwd_slot[l] = slot; }
      else w = slot >= 0 ? P.wslot[slot] : (uint64_t)lp.wc_res;
      Task t;
      t.t.rank = r;
      Op& o = t.t.op;
      o.kind = OP_FWD; o.stream = S_COMPUTE; o.layer = k; o.mb = i;
      o.w = w; o.in = row(r, A_IN, i); o.out = row(r, A_OUT, i); o.ws = P.ws;
      t.t.rd = {wkey(r, k, slot), rkey(r, R_BND, A_IN, i)};
      t.t.wr = {rkey(r, R_BND, A_OUT, i)};
      if (lp.stash_res[i] >= 0) {
        o.stash = (uint64_t)lp.stash_res[i];
        t.t.wr.push_back(rkey(r, R_STASHRES, k, i));
      } else {
        Slots& S = sl[r];
        const int gq = S.gn;
        S.gn = (S.gn + 1) % (int)P.stage.size();
        o.stash = P.stage[gq];
        t.t.wr.push_back(rkey(r, R_STAGE, gq));
        Op d;
        d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_STASH; d.layer = k; d.mb = i;
        d.hbuf = HB_STASH; d.hidx = (int64_t)k * m + i; d.dev = P.stage[gq]; d.bytes = lp.g.st.total;
        t.post.push_back({r, d, {rkey(r, R_STAGE, gq)}, {rkey(r, H_STASH, k, i)}});
        S.glast[gq] = (int)tasks.size();
        spill_task[(size_t)l * m + i] = (int)tasks.size();
      }
      if (slot >= 0) sl[r].wlast[slot] = (int)tasks.size();
      if (l + 1 < L) {  // hand the activation rows to the next layer's rank, peer to peer
        const int r2 = G.layer_rank[l + 1];
        Op x;
        x.kind = OP_P2P; x.stream = S_COMM; x.cat = CAT_NONE; x.layer = G.layer_local[l + 1]; x.mb = i;
        x.dev = row(r2, A_IN, i); x.peer = r; x.peer_off = row(r, A_OUT, i);
        x.bytes = (uint64_t)lp.g.rows * lp.g.desc.d_out * 4;
        t.post.push_back({r2, x, {rkey(r, R_BND, A_OUT, i)}, {rkey(r2, R_BND, A_IN, i)}});
      }
      tasks.push_back(t);
    }
  }
  // ---- loss on the last layer's rank: dY of the last layer into its incoming-gradient rows
  const int rl = G.layer_rank[L - 1];
  {
    Plan& P = G.ranks[rl];
    for (int i = 0; i < m; ++i) {
      Task t;
      t.t.rank = rl;
      Op& o = t.t.op;
      o.kind = OP_LOSS; o.stream = S_COMPUTE; o.mb = i;
      o.in = row(rl, A_OUT, i); o.tgt = P.tgt + (uint64_t)i * P.tgt_row_stride; o.out = row(rl, G_IN, i);
      o.loss = P.loss + (uint64_t)i * 8;
      t.t.rd = {rkey(rl, R_BND, A_OUT, i), rkey(rl, R_TGT, i)};
      t.t.wr = {rkey(rl, R_BND, G_IN, i), rkey(rl, R_LOSS, i)};
      if (i == m - 1) {
        Op d;
        d.kind = OP_LOSS_OUT; d.stream = S_D2H; d.cat = CAT_OUTPUT; d.dev = P.loss; d.bytes = (uint64_t)m * 8;
        std::vector<uint64_t> rds;
        for (int j = 0; j < m; ++j) rds.push_back(rkey(rl, R_LOSS, j));
        t.post.push_back({rl, d, rds, {}});
      }
      tasks.push_back(t);
    }
  }
  // ---- backward (reverse layers, grouped) + JIT update of each layer right after its group
  std::vector<int> bwd_slot(L, -1);
  for (int l = L - 1; l >= 0; --l) {
    const int r = G.layer_rank[l], k = G.layer_local[l];
    Plan& P = G.ranks[r];
    LayerPlan& lp = P.layers[k];
    for (int i = 0; i < m; ++i) {
      int slot = bwd_slot[l];
      uint64_t w;
      if (i == 0) { w = weight_use(r, k, (int)tasks.size(), slot); bwd_slot[l] = slot; }
      else w = slot >= 0 ? P.wslot[slot] : (uint64_t)lp.wc_res;
      Task t;
      t.t.rank = r;
      Op& o = t.t.op;
      o.kind = OP_BWD; o.stream = S_COMPUTE; o.layer = k; o.mb = i; o.first = i == 0;
      o.w = w; o.in = row(r, G_IN, i); o.out = row(r, G_OUT, i); o.ws = P.ws; o.dw = P.dw[0];
      t.t.rd = {wkey(r, k, slot), rkey(r, R_BND, G_IN, i)};
      t.t.wr = {rkey(r, R_BND, G_OUT, i), rkey(r, R_DW, 0)};
      if (i > 0) t.t.rd.push_back(rkey(r, R_DW, 0));
      if (lp.stash_res[i] >= 0) {
        o.stash = (uint64_t)lp.stash_res[i];
        t.t.rd.push_back(rkey(r, R_STASHRES, k, i));
      } else {
        Slots& S = sl[r];
        const int gq = S.gn;
        S.gn = (S.gn + 1) % (int)P.stage.size();
        Item it;
        it.need = (int)tasks.size();
        it.release = std::max(S.glast[gq], spill_task[(size_t)l * m + i]);
        Op h;
        h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_STASH; h.layer = k; h.mb = i;
        h.hbuf = HB_STASH; h.hidx = (int64_t)k * m + i; h.dev = P.stage[gq]; h.bytes = lp.g.st.total;
        it.ops.push_back({r, h, {rkey(r, H_STASH, k, i)}, {rkey(r, R_STAGE, gq)}});
        items.push_back(it);
        o.stash = P.stage[gq];
        t.t.rd.push_back(rkey(r, R_STAGE, gq));
        S.glast[gq] = (int)tasks.size();
      }
      if (slot >= 0) sl[r].wlast[slot] = (int)tasks.size();
      if (l > 0) {  // the input gradient to the previous layer's rank
        const int r2 = G.layer_rank[l - 1];
        Op x;
        x.kind = OP_P2P; x.stream = S_COMM; x.cat = CAT_NONE; x.layer = G.layer_local[l - 1]; x.mb = i;
        x.dev = row(r2, G_IN, i); x.peer = r; x.peer_off = row(r, G_OUT, i);
        x.bytes = (uint64_t)lp.g.rows * lp.g.desc.d_in * 4;
        t.post.push_back({r2, x, {rkey(r, R_BND, G_OUT, i)}, {rkey(r2, R_BND, G_IN, i)}});
      }
      tasks.push_back(t);
    }
    // UPD(l) just in time: dW is this rank's whole (unsharded) accumulator
    Task t;
    t.t.rank = r;
    Op& o = t.t.op;
    o.kind = OP_UPD; o.stream = S_COMPUTE; o.layer = k; o.grad = P.dw[0];
    t.t.rd = {rkey(r, R_DW, 0)};
    if (lp.state_res >= 0) {
      o.state = (uint64_t)lp.state_res;
      t.t.rd.push_back(rkey(r, R_SRES, k));
      t.t.wr.push_back(rkey(r, R_SRES, k));
    } else {
      Slots& S = sl[r];
      const int ss = S.sn;
      S.sn = (S.sn + 1) % (int)P.sslot.size();
      Item it;
      it.need = (int)tasks.size();
      it.release = S.slast[ss];
      Op h;
      h.kind = OP_H2D; h.stream = S_H2D; h.cat = CAT_STATE; h.layer = k;
      h.hbuf = HB_STATE; h.hidx = k; h.dev = P.sslot[ss]; h.bytes = lp.state_bytes;
      it.ops.push_back({r, h, {rkey(r, H_STATE, k)}, {rkey(r, R_SSLOT, ss)}});
      items.push_back(it);
      o.state = P.sslot[ss];
      t.t.rd.push_back(rkey(r, R_SSLOT, ss));
      t.t.wr.push_back(rkey(r, R_SSLOT, ss));
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_STATE; d.layer = k;
      d.hbuf = HB_STATE; d.hidx = k; d.dev = P.sslot[ss]; d.bytes = lp.state_bytes;
      t.post.push_back({r, d, {rkey(r, R_SSLOT, ss)}, {rkey(r, H_STATE, k)}});
      S.slast[ss] = (int)tasks.size();
    }
    const int ws = bwd_slot[l];
    if (lp.wc_res >= 0) {
      o.w = (uint64_t)lp.wc_res;
      t.t.wr.push_back(rkey(r, R_WRES, k));
    } else {
      o.w = P.wslot[ws];
      t.t.wr.push_back(rkey(r, R_WSLOT, ws));
      Op d;  // the updated compute copy out once (the third |W| of P:773-775)
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_WEIGHT; d.layer = k;
      d.hbuf = HB_WC; d.hidx = k; d.dev = P.wslot[ws]; d.bytes = (uint64_t)lp.shard * ts;
      t.post.push_back({r, d, {rkey(r, R_WSLOT, ws)}, {rkey(r, H_WC, k)}});
      sl[r].wlast[ws] = (int)tasks.size();
    }
    if (P.retain_grads) {
      Op d;
      d.kind = OP_D2H; d.stream = S_D2H; d.cat = CAT_GRAD; d.layer = k;
      d.hbuf = HB_GRAD; d.hidx = k; d.dev = P.dw[0]; d.bytes = (uint64_t)lp.shard * 4;
      t.post.push_back({r, d, {rkey(r, R_DW, 0)}, {rkey(r, H_GRAD, k)}});
    }
    tasks.push_back(t);
  }

  // ---- one program: inputs, then tasks with their prefetch items merged by need
  {
    Plan& P0 = G.ranks[0];
    for (int i = 0; i < m; ++i) {
      Op x;
      x.kind = OP_INPUT; x.stream = S_H2D; x.cat = CAT_INPUT; x.hbuf = HB_USER_X; x.mb = i;
      x.dev = row(0, A_IN, i); x.hoff = (uint64_t)i * P0.in_elems_per_mb * 4; x.bytes = (uint64_t)P0.in_elems_per_mb * 4;
      tr.add(0, x, {}, {rkey(0, R_BND, A_IN, i)});
    }
    Plan& PL = G.ranks[rl];
    for (int i = 0; i < m; ++i) {
      Op x;
      x.kind = OP_INPUT; x.stream = S_H2D; x.cat = CAT_INPUT; x.hbuf = HB_USER_T; x.mb = i;
      x.dev = PL.tgt + (uint64_t)i * PL.tgt_row_stride; x.hoff = (uint64_t)i * PL.out_elems_per_mb * 4;
      x.bytes = (uint64_t)PL.out_elems_per_mb * 4;
      tr.add(rl, x, {}, {rkey(rl, R_TGT, i)});
    }
    std::stable_sort(items.begin(), items.end(), [](const Item& a, const Item& b) { return a.need < b.need; });
    size_t next = 0;
    auto emit = [&](Item& it) {
      for (auto& x : it.ops) tr.add(x.rank, x.op, x.rd, x.wr);
    };
    for (int k = 0; k < (int)tasks.size(); ++k) {
      while (next < items.size() && items[next].need <= k) emit(items[next++]);
      Task& t = tasks[k];
      tr.add(t.t.rank, t.t.op, t.t.rd, t.t.wr);
      for (auto& x : t.post) tr.add(x.rank, x.op, x.rd, x.wr);
      while (next < items.size() && items[next].release <= k) emit(items[next++]);
    }
    while (next < items.size()) emit(items[next++]);
  }
  {  // events: one per op another stream waits on (owned by the op's rank)
    std::vector<int> ev(G.ops.size(), -1);
    int ne = 0;
    for (auto& o : G.ops)
      for (int w : o.op.waits)
        if (ev[w] < 0) ev[w] = ne++;
    for (size_t i = 0; i < G.ops.size(); ++i) G.ops[i].op.event = ev[i];
    G.n_events = ne;
  }
  // ---- box summary
  harmony_plan_summary& s = G.summary;
  double fl = 0;
  for (auto& P : G.ranks) {
    s.arena_bytes = std::max(s.arena_bytes, P.arena_bytes);
    s.min_working_set_bytes = std::max(s.min_working_set_bytes, P.min_ws_bytes);
    s.weight_slots = std::max(s.weight_slots, (int32_t)P.wslot.size());
    s.state_slots = std::max(s.state_slots, (int32_t)P.sslot.size());
    s.stash_slots = std::max(s.stash_slots, (int32_t)P.stage.size());
    s.n_params += P.n_params;
    for (auto& lp : P.layers) {
      s.total_weight_bytes += lp.wc_bytes;
      s.total_state_bytes += lp.state_bytes;
      s.total_stash_bytes += (uint64_t)m * lp.g.st.total;
      if (lp.wc_res >= 0) s.resident_weight_bytes += lp.wc_bytes;
      if (lp.state_res >= 0) s.resident_state_bytes += lp.state_bytes;
      for (int i = 0; i < m; ++i)
        if (lp.stash_res[i] >= 0) s.resident_stash_bytes += lp.g.st.total;
      fl += 3.0 * lp.g.flops_fwd * m;
    }
  }
  s.flops_per_step = (uint64_t)fl;
  for (auto& g : G.ops) {
    const Op& o = g.op;
    const bool in = o.kind == OP_H2D || o.kind == OP_INPUT, out = o.kind == OP_D2H || o.kind == OP_LOSS_OUT;
    if (in) s.pred_h2d_bytes += o.bytes;
    if (out) s.pred_d2h_bytes += o.bytes;
    if (in && o.cat == CAT_WEIGHT) s.pred_h2d_weight_bytes += o.bytes;
    if (out && o.cat == CAT_WEIGHT) s.pred_d2h_weight_bytes += o.bytes;
    if (o.stream == S_COMPUTE) s.n_compute_ops++;
    else if (o.stream == S_COMM) s.n_comm_ops++;
    else s.n_copy_ops++;
  }
  s.n_ops = (int32_t)G.ops.size();
  std::string why;
  s.hazards = validate_group(G, &why);
  G.hazard_msg = why;
  return G;
}

std::string dump_group_plan(const GroupPlan& g) {
  static const char* kn[] = {"INPUT", "H2D", "D2H", "FWD", "LOSS", "BWD", "UPD", "ALLGATHER", "REDUCESCATTER",
                             "LOSS_GATHER", "LOSS_OUT", "P2P"};
  static const char* sn[] = {"compute", "h2d", "d2h", "comm"};
  static const char* cn[] = {"weight", "state", "stash", "input", "output", "grad", "-"};
  std::ostringstream os;
  os << "# group plan N=" << g.N << " ops=" << g.ops.size() << " events=" << g.n_events << "\n";
  std::vector<std::vector<int>> glob(g.N);  // local layer -> global layer
  for (size_t l = 0; l < g.layer_rank.size(); ++l) glob[g.layer_rank[l]].push_back((int)l);
  for (size_t i = 0; i < g.ops.size(); ++i) {
    const GOp& x = g.ops[i];
    const Op& o = x.op;
    const int gl = o.layer >= 0 && o.kind != OP_P2P ? glob[x.rank][o.layer]
                   : o.kind == OP_P2P ? glob[x.rank][o.layer] : -1;
    os << i << " " << kn[o.kind] << " " << sn[o.stream] << " rank=" << x.rank << " cat=" << cn[o.cat]
       << " l=" << gl << " i=" << o.mb << " bytes=" << o.bytes;
    if (o.kind == OP_P2P) os << " peer=" << o.peer;
    os << " waits=";
    for (size_t k = 0; k < o.waits.size(); ++k) os << (k ? "," : "") << o.waits[k];
    os << "\n";
  }
  return os.str();
}

}  // namespace hm
