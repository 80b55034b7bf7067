// harmony.cpp — runtime and C ABI of libharmony (include/harmony.h).
//
// Runtime pieces: the capped device arena (one block, laid out by the planner),
// the pinned host store (this rank's shards of the fp32 master W, Adam m and v, the compute copy
// of W, and the spilled activation stash), four CUDA streams {compute, h2d, d2h, comm} with the
// plan's events, the collectives, and the copy ledger (bytes per tensor class, per step).
// The executor replays the static program of plan.cpp every step: for each op it waits on the
// events of its cross-stream dependencies, issues the op on its stream, and records its event.
//
// Two process models share the executor:
//  - one process per GPU (harmony_init; rank r of world_size, NCCL loaded with dlopen);
//  - one process driving N ranks as "one virtual device" (harmony_init_group; SURVEY §8(b)
//    primary mode): the context the caller holds owns N rank contexts, issues their
//    programs op by op in lock step from one thread, and runs the collectives itself as pulls
//    from the peers' arenas (kernels/collective.cu) — over NVLink between GPUs, or inside one
//    GPU when ranks share it (the loopback that exercises N > 1 on a single B200).
#include <cuda_runtime.h>
#include <string.h>

#include <algorithm>
#include <cmath>
#include <memory>
#include <stdexcept>
#include <string>
#include <thread>
#include <vector>

#include "comm.hpp"
#include "harmony_kernels.h"
#include "common.hpp"
#include "kernels/kernels.hpp"
#include "layers.hpp"
#include "plan.hpp"

namespace hm {
thread_local uint64_t g_kernel_launches = 0;
thread_local KProf g_prof;
static thread_local std::string g_err;
void set_global_error(const std::string& msg) { g_err = msg; }
const char* global_error() { return g_err.c_str(); }

static inline uint16_t f32_to_bf16_rne(float f) {
  uint32_t u;
  memcpy(&u, &f, 4);
  if ((u & 0x7F800000u) == 0x7F800000u) return (uint16_t)((u >> 16) | ((u & 0xFFFF) ? 0x40 : 0));  // inf / nan
  return (uint16_t)((u + 0x7FFFu + ((u >> 16) & 1u)) >> 16);
}
}  // namespace hm

using namespace hm;

// One captured instance of the step program (all ranks of a group in one graph).
struct StepGraph {
  cudaGraph_t graph = nullptr;
  cudaGraphExec_t exec = nullptr;
  int sig = -1;                           // (x on device) | (target on device) << 1 at capture
  struct In { int rank; const Op* op; cudaGraphNode_t node; };
  std::vector<In> in_nodes;               // input copies, re-pointed every step
  std::vector<harmony_step_stats> stats;  // per rank
  uint64_t launches = 0;
  std::vector<KProf::Rec> recs;           // profiled graph: timing-event pairs of its kernels
  std::vector<KProf::OpRec> oprecs;       // profiled graph: timing-event pairs of its ops
};

struct harmony_ctx {
  harmony_config cfg{};
  std::string err;
  bool broken = false;
  cudaStream_t st[S_NUM] = {};
  std::vector<cudaEvent_t> events;
  cudaEvent_t ev_begin = nullptr, ev_end[S_NUM] = {};
  cudaEvent_t ev_caller = nullptr;  // caller's default-stream work the step's input copies wait for
  uint8_t* arena = nullptr;
  bool own_arena = false;
  ncclComm_t comm = nullptr;
  bool registered = false;
  Plan plan;
  std::vector<uint8_t*> h_wc;     // per layer: compute-copy shard (T)
  std::vector<float*> h_state;    // per layer: [master | m | v] shard
  std::vector<uint8_t*> h_stash;  // per (layer, microbatch): spilled stash, nullptr if resident
  std::vector<float*> h_grad;     // retain_grads: reduced gradient shard
  double* h_loss = nullptr;
  float* h_gather = nullptr;      // read_state at world_size > 1: pinned staging of the gathered tensor
  int t = 0;
  harmony_step_stats last{};
  bool profiling = false;
  harmony_kernel_profile prof{};
  std::vector<harmony_timeline_rec> timeline;  // last profiled step, one record per op
  std::vector<harmony_kernel_rec> ktimeline;   // last profiled step, one record per kernel launch
  int* h_step = nullptr;  // pinned: Adam's t, copied to the device at the start of every step
  bool use_graph = true;
  StepGraph g_plain, g_prof;  // the step as CUDA graphs: plain, and with per-kernel timing events
  cudaEvent_t ev_fork = nullptr, ev_join[S_NUM] = {};
  cudaStream_t side = nullptr;          // weight-gradient stream lent to the backward tasks
  cudaEvent_t side_ev[4] = {};
  // group mode: the caller's context owns the rank contexts (members); a member knows its group
  std::vector<harmony_ctx*> members;
  harmony_ctx* group = nullptr;
  bool one_device = true;               // group: every rank on the same GPU (loopback)
  cudaEvent_t lb_ready = nullptr, lb_done = nullptr;  // member: rendezvous of a group collective
  std::unique_ptr<GroupPlan> gplan;     // group under Harmony-PP: the one program of all ranks
  // pageable inputs are copied here first (pinned), so the step still replays its CUDA graph
  uint8_t* h_stage[2] = {nullptr, nullptr};
  size_t h_stage_bytes[2] = {0, 0};
};

namespace {

void free_host(void* p) {
  if (p) cudaFreeHost(p);
}

void* alloc_host(size_t bytes) {
  void* p = nullptr;
  cudaError_t e = cudaHostAlloc(&p, std::max<size_t>(bytes, 64), cudaHostAllocPortable);
  if (e != cudaSuccess) throw Error{HARMONY_E_HOST_OOM, std::string("cudaHostAlloc(") + std::to_string(bytes) +
                                                            ") failed: " + cudaGetErrorString(e)};
  return p;
}

void check_nccl(ncclResult_t r, const char* what) {
  if (r != ncclSuccess)
    throw Error{HARMONY_E_NCCL, std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "?")};
}

harmony_status fail(harmony_ctx* ctx, const Error& e) {
  if (ctx) {
    ctx->err = e.msg;
    if (e.code == HARMONY_E_CUDA || e.code == HARMONY_E_NCCL) ctx->broken = true;
  }
  set_global_error(e.msg);
  return e.code;
}

#define HM_API_BEGIN try {
#define HM_API_END(ctx)                                               \
  }                                                                   \
  catch (const Error& e) {                                            \
    return fail(ctx, e);                                              \
  }                                                                   \
  catch (const std::exception& e) {                                   \
    return fail(ctx, Error{HARMONY_E_INVALID_ARG, e.what()});         \
  }                                                                   \
  return HARMONY_OK;

void drop_graph(StepGraph& g);

// The rank contexts a context drives: itself, or a group's members.
std::vector<harmony_ctx*> ranks_of(harmony_ctx* c) {
  if (c->members.empty()) return {c};
  return c->members;
}

void sync_all(harmony_ctx* c) {
  for (harmony_ctx* r : ranks_of(c)) {
    if (r->st[0] == nullptr) continue;
    cudaSetDevice(r->cfg.device);
    for (int s = 0; s < S_NUM; ++s)
      if (r->st[s]) cudaStreamSynchronize(r->st[s]);
    if (r->side) cudaStreamSynchronize(r->side);
  }
}

void destroy(harmony_ctx* c) {
  if (!c) return;
  sync_all(c);
  drop_graph(c->g_plain);  // a group's graphs span its ranks' streams: dropped before the ranks
  drop_graph(c->g_prof);
  for (harmony_ctx* m : c->members) destroy(m);
  c->members.clear();
  cudaSetDevice(c->cfg.device);
  if (c->side) cudaStreamSynchronize(c->side);
  for (auto e : c->side_ev)
    if (e) cudaEventDestroy(e);
  if (c->side) cudaStreamDestroy(c->side);
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_caller) cudaEventDestroy(c->ev_caller);
  if (c->lb_ready) cudaEventDestroy(c->lb_ready);
  if (c->lb_done) cudaEventDestroy(c->lb_done);
  for (int s = 0; s < S_NUM; ++s)
    if (c->ev_join[s]) cudaEventDestroy(c->ev_join[s]);
  free_host(c->h_step);
  for (auto e : c->events) cudaEventDestroy(e);
  if (c->ev_begin) cudaEventDestroy(c->ev_begin);
  for (int s = 0; s < S_NUM; ++s) {
    if (c->ev_end[s]) cudaEventDestroy(c->ev_end[s]);
    if (c->st[s]) cudaStreamDestroy(c->st[s]);
  }
  if (c->comm && nccl().CommDestroy) nccl().CommDestroy(c->comm);
  if (c->own_arena && c->arena) cudaFree(c->arena);
  for (auto p : c->h_wc) free_host(p);
  for (auto p : c->h_state) free_host(p);
  for (auto p : c->h_stash) free_host(p);
  for (auto p : c->h_grad) free_host(p);
  free_host(c->h_loss);
  free_host(c->h_gather);
  free_host(c->h_stage[0]);
  free_host(c->h_stage[1]);
  delete c;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

// Streams, events and (world_size > 1, one process per GPU) the NCCL communicator of one rank.
void init_rank(harmony_ctx* c, const harmony_config& cfg, bool want_nccl) {
  c->cfg = cfg;
  int ndev = 0;
  HM_CUDA(cudaGetDeviceCount(&ndev));
  HM_CHECK(cfg.device >= 0 && cfg.device < ndev, HARMONY_E_INVALID_ARG, "device ordinal out of range");
  HM_CUDA(cudaSetDevice(cfg.device));
  cudaDeviceProp prop;
  HM_CUDA(cudaGetDeviceProperties(&prop, cfg.device));
  HM_CHECK(prop.major == 10, HARMONY_E_UNSUPPORTED,
           std::string("libharmony is built for sm_100a (B200); device is ") + prop.name);
  // Stream priorities: the compute stream carries the step's critical path (the dgrad chain), the
  // side stream the weight-gradient work that only feeds dW — when SMs free up, the block scheduler
  // places the compute stream's CTAs first (HARMONY_PRIO=0: all default priority)
  int prio_lo = 0, prio_hi = 0;
  HM_CUDA(cudaDeviceGetStreamPriorityRange(&prio_lo, &prio_hi));
  {
    const char* e = getenv("HARMONY_PRIO");
    if (e && *e == '0') prio_lo = prio_hi = 0;
  }
  for (int s = 0; s < S_NUM; ++s) {
    HM_CUDA(cudaStreamCreateWithPriority(&c->st[s], cudaStreamNonBlocking, s == S_COMPUTE ? prio_hi : 0));
    HM_CUDA(cudaEventCreate(&c->ev_end[s]));
  }
  HM_CUDA(cudaEventCreate(&c->ev_begin));
  HM_CUDA(cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
  HM_CUDA(cudaEventCreateWithFlags(&c->ev_caller, cudaEventDisableTiming));
  HM_CUDA(cudaEventCreateWithFlags(&c->lb_ready, cudaEventDisableTiming));
  HM_CUDA(cudaEventCreateWithFlags(&c->lb_done, cudaEventDisableTiming));
  for (int s = 0; s < S_NUM; ++s) HM_CUDA(cudaEventCreateWithFlags(&c->ev_join[s], cudaEventDisableTiming));
  c->h_step = static_cast<int*>(alloc_host(sizeof(int)));
  HM_CUDA(cudaStreamCreateWithPriority(&c->side, cudaStreamNonBlocking, prio_lo));
  for (auto& e : c->side_ev) HM_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  {
    const char* e = getenv("HARMONY_NO_GRAPH");
    c->use_graph = !(e && *e && *e != '0');
  }
  if (want_nccl && cfg.world_size > 1) {
    HM_CHECK(nccl().load(), HARMONY_E_NCCL, nccl().err);
    ncclUniqueId id;
    memcpy(&id, cfg.nccl_id, 128);
    check_nccl(nccl().CommInitRank(&c->comm, cfg.world_size, id, cfg.rank), "ncclCommInitRank");
  }
}

// ---------------------------------------------------------------------------------------- executor
enum PtrKind { PTR_PAGEABLE = 0, PTR_PINNED = 1, PTR_DEVICE = 2 };
PtrKind ptr_kind(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return PTR_PAGEABLE;
  }
  if (a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged) return PTR_DEVICE;
  if (a.type == cudaMemoryTypeHost) return PTR_PINNED;
  return PTR_PAGEABLE;
}

// Host copy on the host's cores (pageable -> pinned staging of the step's inputs): every buffer of
// the step cut into 16 MB pieces, the pieces dealt round-robin to min(cores, 16) threads.
void parallel_memcpy_multi(void* const* dst, const void* const* src, const size_t* n, int count) {
  const size_t chunk = 16u << 20;
  struct Piece { char* d; const char* s; size_t n; };
  std::vector<Piece> pieces;
  for (int b = 0; b < count; ++b)
    for (size_t lo = 0; lo < n[b]; lo += chunk)
      pieces.push_back({static_cast<char*>(dst[b]) + lo, static_cast<const char*>(src[b]) + lo, std::min(chunk, n[b] - lo)});
  const unsigned hw = std::max(1u, std::thread::hardware_concurrency());
  const int nt = (int)std::min<size_t>(std::min(16u, hw), pieces.size());
  if (nt <= 1) {
    for (const Piece& q : pieces) memcpy(q.d, q.s, q.n);
    return;
  }
  std::vector<std::thread> th;
  for (int i = 0; i < nt; ++i)
    th.emplace_back([&, i] {
      for (size_t k = (size_t)i; k < pieces.size(); k += (size_t)nt) memcpy(pieces[k].d, pieces[k].s, pieces[k].n);
    });
  for (auto& t : th) t.join();
}

// This rank's view of the step's user inputs.
struct RankIn {
  const float* x = nullptr;
  const float* tg = nullptr;
  bool x_dev = false, t_dev = false;
};

bool is_group_collective(int kind) {
  return kind == OP_ALLGATHER || kind == OP_REDUCESCATTER || kind == OP_LOSS_GATHER;
}

void issue_prologue(harmony_ctx* c) {
  // Adam's step t lives in device memory (read by the update kernels at execution time)
  HM_CUDA(cudaMemcpyAsync(c->arena + c->plan.tstep, c->h_step, sizeof(int), cudaMemcpyHostToDevice, c->st[S_COMPUTE]));
}

// cross-stream waits of op oi; returns the profiling event opened after them (-1: not profiling)
int op_pre(harmony_ctx* c, size_t oi) {
  const Plan& p = c->plan;
  const Op& o = p.ops[oi];
  cudaStream_t st = c->st[o.stream];
  for (int w : o.waits) HM_CUDA(cudaStreamWaitEvent(st, c->events[p.ops[w].event], 0));
  return g_prof.begin(st);  // profiling: the op's span on its stream (after its waits)
}

void op_post(harmony_ctx* c, size_t oi, int op_e0) {
  const Op& o = c->plan.ops[oi];
  cudaStream_t st = c->st[o.stream];
  if (op_e0 >= 0) {
    const int op_e1 = g_prof.begin(st);
    if (op_e1 >= 0) g_prof.oprecs.push_back({(int)oi, op_e0, op_e1});
  }
  if (o.event >= 0) HM_CUDA(cudaEventRecord(c->events[o.event], st));
}

// The zero padding of a dW buffer beyond the layer's P parameters is part of every rank's reduce-
// scatter input: keep it zero (another layer of a larger P may have left values there).
void zero_dw_padding(harmony_ctx* c, const Op& o) {
  const LayerPlan& lp = c->plan.layers[o.layer];
  const uint64_t tot = (uint64_t)c->plan.N * o.count;
  if (tot > (uint64_t)lp.P)
    HM_CUDA(cudaMemsetAsync(c->arena + o.dev + (uint64_t)lp.P * 4, 0, (tot - (uint64_t)lp.P) * 4, c->st[o.stream]));
}

void op_body(harmony_ctx* c, const Op& o, const RankIn& in, harmony_step_stats& s) {
  Plan& p = c->plan;
  uint8_t* A = c->arena;
  const int dt = p.dtype;
  cudaStream_t st = c->st[o.stream];
  switch (o.kind) {
    case OP_INPUT: {
      const uint8_t* src = reinterpret_cast<const uint8_t*>(o.hbuf == HB_USER_X ? (const void*)in.x : (const void*)in.tg);
      const bool dev = o.hbuf == HB_USER_X ? in.x_dev : in.t_dev;
      HM_CUDA(cudaMemcpyAsync(A + o.dev, src + o.hoff, o.bytes, cudaMemcpyDefault, st));
      if (!dev) { s.h2d_bytes += o.bytes; s.h2d_input_bytes += o.bytes; }
      break;
    }
    case OP_H2D:
    case OP_D2H: {
      uint8_t* h = nullptr;
      switch (o.hbuf) {
        case HB_WC: h = c->h_wc[o.hidx]; break;
        case HB_STATE: h = reinterpret_cast<uint8_t*>(c->h_state[o.hidx]); break;
        case HB_STASH: h = c->h_stash[o.hidx]; break;
        case HB_GRAD: h = reinterpret_cast<uint8_t*>(c->h_grad[o.hidx]); break;
        default: throw Error{HARMONY_E_INVALID_ARG, "bad host buffer in plan"};
      }
      h += o.hoff;
      if (o.kind == OP_H2D) {
        HM_CUDA(cudaMemcpyAsync(A + o.dev, h, o.bytes, cudaMemcpyHostToDevice, st));
        s.h2d_bytes += o.bytes;
        if (o.cat == CAT_WEIGHT) s.h2d_weight_bytes += o.bytes;
        else if (o.cat == CAT_STATE) s.h2d_state_bytes += o.bytes;
        else if (o.cat == CAT_STASH) s.h2d_stash_bytes += o.bytes;
        else if (o.cat == CAT_GRAD) s.h2d_grad_bytes += o.bytes;
      } else {
        HM_CUDA(cudaMemcpyAsync(h, A + o.dev, o.bytes, cudaMemcpyDeviceToHost, st));
        s.d2h_bytes += o.bytes;
        if (o.cat == CAT_WEIGHT) s.d2h_weight_bytes += o.bytes;
        else if (o.cat == CAT_STATE) s.d2h_state_bytes += o.bytes;
        else if (o.cat == CAT_STASH) s.d2h_stash_bytes += o.bytes;
        else if (o.cat == CAT_GRAD) s.d2h_grad_bytes += o.bytes;
      }
      break;
    }
    case OP_FWD: {
      const LayerPlan& lp = p.layers[o.layer];
      if (o.pack == 2)
        layer_fwd_pack2(lp.gp, A + o.w, reinterpret_cast<const float*>(A + o.in), reinterpret_cast<float*>(A + o.out),
                        A + o.stash, A + o.stash2, A + o.ws, st);
      else
        layer_fwd(lp.g, A + o.w, reinterpret_cast<const float*>(A + o.in), reinterpret_cast<float*>(A + o.out),
                  A + o.stash, A + o.ws, st);
      break;
    }
    case OP_LOSS: {
      const float inv_batch = 1.0f / (float)((int64_t)p.N * p.m * p.b);
      mse(p.out_elems_per_mb, reinterpret_cast<const float*>(A + o.in), reinterpret_cast<const float*>(A + o.tgt),
          inv_batch, reinterpret_cast<float*>(A + o.out), reinterpret_cast<double*>(A + o.loss),
          reinterpret_cast<double*>(A + p.loss_scratch), st);
      break;
    }
    case OP_BWD: {
      const LayerPlan& lp = p.layers[o.layer];
      const char* e = getenv("HARMONY_NO_SIDE");
      if (!(e && *e && *e != '0')) {
        void* ev[4] = {c->side_ev[0], c->side_ev[1], c->side_ev[2], c->side_ev[3]};
        set_side_stream(c->side, ev);
      } else {
        set_side_stream(nullptr, nullptr);
      }
      layer_bwd(lp.g, A + o.w, A + o.stash, reinterpret_cast<const float*>(A + o.in),
                reinterpret_cast<float*>(A + o.out), reinterpret_cast<float*>(A + o.dw), o.first, A + o.ws, st);
      set_side_stream(nullptr, nullptr);
      break;
    }
    case OP_UPD: {
      const LayerPlan& lp = p.layers[o.layer];
      float* state = reinterpret_cast<float*>(A + o.state);
      const uint64_t sh = (uint64_t)lp.shard;
      uint8_t* wc = A + o.w + (uint64_t)p.rank * sh * (dt ? 2 : 4);
      adam(dt, (int64_t)sh, state, state + sh, state + 2 * sh, reinterpret_cast<const float*>(A + o.grad), wc,
           c->cfg.lr, c->cfg.beta1, c->cfg.beta2, c->cfg.eps, c->t, reinterpret_cast<const int*>(A + p.tstep), st);
      break;
    }
    case OP_ALLGATHER: {
      const size_t esz = dt ? 2 : 4;
      uint8_t* buf = A + o.dev;
      check_nccl(nccl().AllGather(buf + (uint64_t)p.rank * o.count * esz, buf, o.count, dt ? ncclBfloat16 : ncclFloat32,
                                  c->comm, st),
                 "ncclAllGather");
      s.nvlink_bytes += o.bytes;
      break;
    }
    case OP_REDUCESCATTER: {
      zero_dw_padding(c, o);
      check_nccl(nccl().ReduceScatter(A + o.dev, A + o.grad, o.count, ncclFloat32, ncclSum, c->comm, st),
                 "ncclReduceScatter");
      s.nvlink_bytes += o.bytes;
      break;
    }
    case OP_LOSS_GATHER: {
      uint8_t* buf = A + o.dev;
      check_nccl(nccl().AllGather(buf + (uint64_t)p.rank * o.count * 8, buf, o.count, ncclFloat64, c->comm, st),
                 "ncclAllGather(loss)");
      s.nvlink_bytes += o.bytes;
      break;
    }
    case OP_LOSS_OUT: {
      const uint64_t off = p.N > 1 ? 0 : (uint64_t)p.rank * p.m * 8;
      HM_CUDA(cudaMemcpyAsync(reinterpret_cast<uint8_t*>(c->h_loss) + off, A + o.dev + off, o.bytes,
                              cudaMemcpyDeviceToHost, st));
      s.d2h_bytes += o.bytes;
      s.d2h_output_bytes += o.bytes;
      break;
    }
    default:
      throw Error{HARMONY_E_INVALID_ARG, "unknown op kind in plan"};
  }
}

// A collective of a group, as three lock-step phases over the ranks: (1) every rank reaches the op
// (its plan waits) and marks its inputs ready; (2) every rank waits for all inputs and pulls what it
// receives from its peers' arenas; (3) every rank waits until all peers have finished pulling before
// its program may overwrite the buffers (the same ordering NCCL gives the one-process-per-GPU path).
void issue_group_collective(const std::vector<harmony_ctx*>& R, bool one_device, size_t oi,
                            std::vector<harmony_step_stats>& s) {
  const int N = (int)R.size();
  std::vector<int> e0(N);
  for (int r = 0; r < N; ++r) {
    harmony_ctx* c = R[r];
    if (!one_device) HM_CUDA(cudaSetDevice(c->cfg.device));
    e0[r] = op_pre(c, oi);
    const Op& o = c->plan.ops[oi];
    if (o.kind == OP_REDUCESCATTER) zero_dw_padding(c, o);
    HM_CUDA(cudaEventRecord(c->lb_ready, c->st[o.stream]));
  }
  for (int r = 0; r < N; ++r) {
    harmony_ctx* c = R[r];
    if (!one_device) HM_CUDA(cudaSetDevice(c->cfg.device));
    const Op& o = c->plan.ops[oi];
    cudaStream_t st = c->st[o.stream];
    for (int q = 0; q < N; ++q)
      if (q != r) HM_CUDA(cudaStreamWaitEvent(st, R[q]->lb_ready, 0));
    if (o.kind == OP_REDUCESCATTER) {
      const float* src[HM_MAX_GROUP];
      for (int q = 0; q < N; ++q)
        src[q] = reinterpret_cast<const float*>(R[q]->arena + R[q]->plan.ops[oi].dev) + (uint64_t)r * o.count;
      rank_sum(N, src, (int64_t)o.count, reinterpret_cast<float*>(c->arena + o.grad), st);
    } else {
      const size_t esz = o.kind == OP_LOSS_GATHER ? 8 : (c->plan.dtype ? 2 : 4);
      const uint64_t sh = o.count * esz;
      for (int q = 0; q < N; ++q) {
        if (q == r) continue;
        HM_CUDA(cudaMemcpyAsync(c->arena + o.dev + (uint64_t)q * sh, R[q]->arena + R[q]->plan.ops[oi].dev + (uint64_t)q * sh,
                                sh, cudaMemcpyDefault, st));
      }
    }
    s[r].nvlink_bytes += o.bytes;
    HM_CUDA(cudaEventRecord(c->lb_done, st));
  }
  for (int r = 0; r < N; ++r) {
    harmony_ctx* c = R[r];
    if (!one_device) HM_CUDA(cudaSetDevice(c->cfg.device));
    const Op& o = c->plan.ops[oi];
    for (int q = 0; q < N; ++q)
      if (q != r) HM_CUDA(cudaStreamWaitEvent(c->st[o.stream], R[q]->lb_done, 0));
    op_post(c, oi, e0[r]);
  }
}

// Harmony-PP: the group's one program in order; an op's waits may name other ranks' ops (the
// activation / gradient hand-offs), whose events live in those ranks' contexts.
void issue_program_pp(harmony_ctx* c, const std::vector<RankIn>& in, std::vector<harmony_step_stats>& s) {
  const std::vector<harmony_ctx*>& R = c->members;
  const GroupPlan& gp = *c->gplan;
  for (harmony_ctx* r : R) {
    if (!c->one_device) HM_CUDA(cudaSetDevice(r->cfg.device));
    issue_prologue(r);
  }
  for (const GOp& g : gp.ops) {
    harmony_ctx* rc = R[g.rank];
    const Op& o = g.op;
    if (!c->one_device) HM_CUDA(cudaSetDevice(rc->cfg.device));
    cudaStream_t st = rc->st[o.stream];
    for (int w : o.waits) HM_CUDA(cudaStreamWaitEvent(st, R[gp.ops[w].rank]->events[gp.ops[w].op.event], 0));
    if (o.kind == OP_P2P) {  // peer to peer over NVLink (or inside the GPU when the ranks share it)
      HM_CUDA(cudaMemcpyAsync(rc->arena + o.dev, R[o.peer]->arena + o.peer_off, o.bytes, cudaMemcpyDefault, st));
      s[g.rank].nvlink_bytes += o.bytes;
    } else {
      op_body(rc, o, in[g.rank], s[g.rank]);
    }
    if (o.event >= 0) HM_CUDA(cudaEventRecord(rc->events[o.event], st));
  }
  if (!c->one_device) HM_CUDA(cudaSetDevice(R[0]->cfg.device));
}

// The user-input copies of the step: (rank, op).
std::vector<std::pair<int, const Op*>> input_ops(harmony_ctx* c) {
  std::vector<std::pair<int, const Op*>> v;
  if (c->gplan) {
    for (const GOp& g : c->gplan->ops)
      if (g.op.kind == OP_INPUT) v.push_back({g.rank, &g.op});
    return v;
  }
  const std::vector<harmony_ctx*> R = ranks_of(c);
  for (size_t r = 0; r < R.size(); ++r)
    for (const Op& o : R[r]->plan.ops)
      if (o.kind == OP_INPUT) v.push_back({(int)r, &o});
  return v;
}

// Issue the static program once on every rank's streams (eagerly, or inside a stream capture).
void issue_program(harmony_ctx* c, const std::vector<RankIn>& in, std::vector<harmony_step_stats>& s) {
  if (c->gplan) return issue_program_pp(c, in, s);
  const std::vector<harmony_ctx*> R = ranks_of(c);
  const bool group = !c->members.empty();
  const bool one_device = c->one_device;
  for (size_t r = 0; r < R.size(); ++r) {
    if (!one_device) HM_CUDA(cudaSetDevice(R[r]->cfg.device));
    issue_prologue(R[r]);
  }
  const size_t n = R[0]->plan.ops.size();
  for (size_t oi = 0; oi < n; ++oi) {
    if (group && is_group_collective(R[0]->plan.ops[oi].kind)) {
      issue_group_collective(R, one_device, oi, s);
      continue;
    }
    for (size_t r = 0; r < R.size(); ++r) {
      if (!one_device) HM_CUDA(cudaSetDevice(R[r]->cfg.device));
      const int e0 = op_pre(R[r], oi);
      op_body(R[r], R[r]->plan.ops[oi], in[r], s[r]);
      op_post(R[r], oi, e0);
    }
  }
  if (!one_device) HM_CUDA(cudaSetDevice(R[0]->cfg.device));
}

void drop_graph(StepGraph& g) {
  if (g.exec) cudaGraphExecDestroy(g.exec);
  if (g.graph) cudaGraphDestroy(g.graph);
  g.exec = nullptr;
  g.graph = nullptr;
  g.in_nodes.clear();
  g.recs.clear();
  g.oprecs.clear();
  g.sig = -1;
}

// Capture the whole step (every rank's four streams, collectives included) as one CUDA graph;
// later steps only patch the source pointers of the input copies and replay it (one launch per
// step).  With `profiled`, every kernel of the step is bracketed by external event-record nodes, so
// the per-kernel durations come from the real step without host-issue gaps.
void capture_graph(harmony_ctx* c, StepGraph& G, const std::vector<RankIn>& in, bool profiled) {
  drop_graph(G);
  const std::vector<harmony_ctx*> R = ranks_of(c);
  harmony_ctx* c0 = R[0];
  cudaStream_t cs = c0->st[S_COMPUTE];
  std::vector<harmony_step_stats> s(R.size());
  g_kernel_launches = 0;
  g_prof.on = profiled;
  g_prof.external = profiled;
  g_prof.used = 0;
  g_prof.recs.clear();
  g_prof.oprecs.clear();
  HM_CUDA(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
  try {
    HM_CUDA(cudaEventRecord(c0->ev_fork, cs));
    for (harmony_ctx* r : R)
      for (int k = 0; k < S_NUM; ++k)
        if (r->st[k] != cs) HM_CUDA(cudaStreamWaitEvent(r->st[k], c0->ev_fork, 0));
    issue_program(c, in, s);
    for (harmony_ctx* r : R)
      for (int k = 0; k < S_NUM; ++k) {
        if (r->st[k] == cs) continue;
        HM_CUDA(cudaEventRecord(r->ev_join[k], r->st[k]));
        HM_CUDA(cudaStreamWaitEvent(cs, r->ev_join[k], 0));
      }
  } catch (...) {
    cudaGraph_t g = nullptr;
    cudaStreamEndCapture(cs, &g);
    if (g) cudaGraphDestroy(g);
    cudaGetLastError();
    g_prof.on = g_prof.external = false;
    throw;
  }
  g_prof.on = g_prof.external = false;
  HM_CUDA(cudaStreamEndCapture(cs, &G.graph));
  HM_CUDA(cudaGraphInstantiate(&G.exec, G.graph, cudaGraphInstantiateFlagUseNodePriority));
  G.stats = s;
  G.launches = g_kernel_launches;
  G.recs = g_prof.recs;
  G.oprecs = g_prof.oprecs;
  // find the input memcpy nodes by their destinations (every rank's arena is its own allocation)
  size_t n = 0;
  HM_CUDA(cudaGraphGetNodes(G.graph, nullptr, &n));
  std::vector<cudaGraphNode_t> nodes(n);
  HM_CUDA(cudaGraphGetNodes(G.graph, nodes.data(), &n));
  G.in_nodes.clear();
  for (auto& io : input_ops(c)) G.in_nodes.push_back({io.first, io.second, nullptr});
  for (auto nd : nodes) {
    cudaGraphNodeType ty;
    HM_CUDA(cudaGraphNodeGetType(nd, &ty));
    if (ty != cudaGraphNodeTypeMemcpy) continue;
    cudaMemcpy3DParms mp;
    HM_CUDA(cudaGraphMemcpyNodeGetParams(nd, &mp));
    const uint8_t* dst = static_cast<const uint8_t*>(mp.dstPtr.ptr);
    const uint8_t* srcp = static_cast<const uint8_t*>(mp.srcPtr.ptr);
    for (auto& e : G.in_nodes) {  // destination AND source: other copies may land in the same rows
      const uint8_t* want = reinterpret_cast<const uint8_t*>(e.op->hbuf == HB_USER_X ? (const void*)in[e.rank].x
                                                                                    : (const void*)in[e.rank].tg) +
                            e.op->hoff;
      if (dst == R[e.rank]->arena + e.op->dev && srcp == want) e.node = nd;
    }
  }
  for (auto& e : G.in_nodes) HM_CHECK(e.node != nullptr, HARMONY_E_CUDA, "graph capture: input copy node not found");
  G.sig = (in[0].x_dev ? 1 : 0) | (in[0].t_dev ? 2 : 0);
}

// One step of a rank context or a group.  x / tg: this context's rows (a group: the global batch).
void run_step(harmony_ctx* c, const float* x, const float* tg, double* loss_out, harmony_step_stats* out) {
  const std::vector<harmony_ctx*> R = ranks_of(c);
  const int NR = (int)R.size();
  harmony_ctx* c0 = R[0];
  const Plan& p0 = c0->plan;
  const int t_next = c->t + 1;
  for (harmony_ctx* r : R) {
    r->t = t_next;  // the value the update kernels of this step read (reverted below on failure)
    *r->h_step = t_next;
  }
  PtrKind xk = ptr_kind(x), tk = ptr_kind(tg);
  const bool pp = c->gplan != nullptr;  // Harmony-PP: the whole batch enters at rank 0, targets at the last rank
  {  // pageable host inputs: staged into pinned buffers (parallel host copy), then the graph replays
    static const bool stage = [] {
      const char* e = getenv("HARMONY_PAGEABLE_STAGE");
      return !(e && *e == '0');
    }();
    const size_t rows = (size_t)(pp ? 1 : NR) * p0.m;
    const size_t nb[2] = {rows * p0.in_elems_per_mb * 4, rows * p0.out_elems_per_mb * 4};
    const float* src[2] = {x, tg};
    PtrKind* kinds[2] = {&xk, &tk};
    bool staged[2] = {false, false};
    void* cd[2];
    const void* cs[2];
    size_t cn[2];
    int nc = 0;
    for (int q = 0; q < 2 && stage; ++q) {
      if (*kinds[q] != PTR_PAGEABLE) continue;
      staged[q] = true;
      if (c->h_stage_bytes[q] < nb[q]) {
        free_host(c->h_stage[q]);
        c->h_stage[q] = nullptr;
        c->h_stage[q] = static_cast<uint8_t*>(alloc_host(nb[q]));
        c->h_stage_bytes[q] = nb[q];
      }
      cd[nc] = c->h_stage[q]; cs[nc] = src[q]; cn[nc] = nb[q]; ++nc;
      *kinds[q] = PTR_PINNED;
    }
    if (nc) parallel_memcpy_multi(cd, cs, cn, nc);  // X and T together
    if (staged[0]) x = reinterpret_cast<const float*>(c->h_stage[0]);
    if (staged[1]) tg = reinterpret_cast<const float*>(c->h_stage[1]);
  }
  std::vector<RankIn> in(NR);
  for (int r = 0; r < NR; ++r) {
    in[r].x = pp ? x : x + (size_t)r * p0.m * p0.in_elems_per_mb;
    in[r].tg = pp ? tg : tg + (size_t)r * p0.m * p0.out_elems_per_mb;
    in[r].x_dev = xk == PTR_DEVICE;
    in[r].t_dev = tk == PTR_DEVICE;
  }
  // graphs need pinned or device inputs (a pageable copy cannot be captured); one graph spans the
  // ranks of a group only when they share a GPU
  const bool use_graph = c0->use_graph && xk != PTR_PAGEABLE && tk != PTR_PAGEABLE && c->one_device;
  std::vector<harmony_step_stats> s(NR);
  g_kernel_launches = 0;
  g_prof.on = c->profiling;
  g_prof.external = false;
  g_prof.used = 0;
  g_prof.recs.clear();
  g_prof.oprecs.clear();
  cudaStream_t cs = c0->st[S_COMPUTE];
  std::vector<KProf::Rec>* recs = &g_prof.recs;
  std::vector<KProf::OpRec>* oprecs = &g_prof.oprecs;
  uint64_t launches = 0;
  bool issued = false;
  try {
    // the caller's work on the legacy default stream (e.g. torch ops writing x / target) first
    HM_CUDA(cudaEventRecord(c0->ev_caller, cudaStreamLegacy));
    HM_CUDA(cudaStreamWaitEvent(cs, c0->ev_caller, 0));
    if (use_graph) {
      StepGraph& G = c->profiling ? c->g_prof : c->g_plain;
      const int sig = (in[0].x_dev ? 1 : 0) | (in[0].t_dev ? 2 : 0);
      issued = true;
      if (!G.exec || G.sig != sig) capture_graph(c, G, in, c->profiling);
      for (auto& e : G.in_nodes) {
        const Op& o = *e.op;
        const uint8_t* src = reinterpret_cast<const uint8_t*>(o.hbuf == HB_USER_X ? (const void*)in[e.rank].x
                                                                                  : (const void*)in[e.rank].tg);
        HM_CUDA(cudaGraphExecMemcpyNodeSetParams1D(G.exec, e.node, R[e.rank]->arena + o.dev, src + o.hoff, o.bytes,
                                                   cudaMemcpyDefault));
      }
      HM_CUDA(cudaEventRecord(c0->ev_begin, cs));
      HM_CUDA(cudaGraphLaunch(G.exec, cs));
      HM_CUDA(cudaEventRecord(c0->ev_end[0], cs));
      HM_CUDA(cudaEventSynchronize(c0->ev_end[0]));
      float ms = 0.f;
      HM_CUDA(cudaEventElapsedTime(&ms, c0->ev_begin, c0->ev_end[0]));
      s = G.stats;
      for (auto& x2 : s) x2.step_seconds = ms * 1e-3;
      launches = G.launches;
      recs = &G.recs;
      oprecs = &G.oprecs;
    } else {
      HM_CUDA(cudaEventRecord(c0->ev_begin, cs));
      for (harmony_ctx* r : R) {
        if (!c->one_device) HM_CUDA(cudaSetDevice(r->cfg.device));
        for (int k = 0; k < S_NUM; ++k)
          if (r->st[k] != cs) HM_CUDA(cudaStreamWaitEvent(r->st[k], c0->ev_begin, 0));
      }
      issued = true;
      issue_program(c, in, s);
      float ms = 0.f;
      for (harmony_ctx* r : R) {
        if (!c->one_device) HM_CUDA(cudaSetDevice(r->cfg.device));
        for (int k = 0; k < S_NUM; ++k) HM_CUDA(cudaEventRecord(r->ev_end[k], r->st[k]));
      }
      for (harmony_ctx* r : R)
        for (int k = 0; k < S_NUM; ++k) {
          HM_CUDA(cudaEventSynchronize(r->ev_end[k]));
          float e = 0.f;
          HM_CUDA(cudaEventElapsedTime(&e, c0->ev_begin, r->ev_end[k]));
          ms = std::max(ms, e);
        }
      HM_CUDA(cudaSetDevice(c0->cfg.device));
      for (auto& x2 : s) x2.step_seconds = ms * 1e-3;
      launches = g_kernel_launches;
    }
    HM_CUDA(cudaGetLastError());
  } catch (...) {
    // nothing of this step may count: t back, and — once work was issued — the context is unusable
    g_prof.on = g_prof.external = false;
    for (harmony_ctx* r : R) r->t = t_next - 1;
    if (issued) {
      sync_all(c);
      cudaGetLastError();
      c->broken = true;
      for (harmony_ctx* r : R) r->broken = true;
    }
    throw;
  }
  c->t = t_next;
  if (c->profiling) {
    std::vector<std::pair<float, float>> iv[PROF_NUM];  // launch intervals per class, ms from the step start
    c->ktimeline.clear();
    for (auto& rc : *recs) {
      float e = 0.f, t0 = 0.f;
      HM_CUDA(cudaEventElapsedTime(&e, g_prof.pool[rc.e0], g_prof.pool[rc.e1]));
      HM_CUDA(cudaEventElapsedTime(&t0, c0->ev_begin, g_prof.pool[rc.e0]));
      c->prof.launches[rc.cat] += 1;
      c->prof.seconds[rc.cat] += e * 1e-3;
      c->prof.work[rc.cat] += rc.work;
      iv[rc.cat].push_back({t0, t0 + e});
      harmony_kernel_rec kr{};
      kr.cat = rc.cat;
      kr.stream = -1;
      for (int k = 0; k < S_NUM; ++k)
        if (rc.st == c0->st[k]) kr.stream = k;
      if (rc.st == c0->side) kr.stream = S_NUM;
      kr.work = rc.work;
      kr.t0 = t0 * 1e-3;
      kr.t1 = (t0 + e) * 1e-3;
      c->ktimeline.push_back(kr);
    }
    for (int k = 0; k < PROF_NUM; ++k) {  // union of the class's intervals
      auto& v = iv[k];
      std::sort(v.begin(), v.end());
      double busy = 0.0;
      float lo = 0.f, hi = -1.f;
      for (auto& x : v) {
        if (x.first > hi) {
          if (hi > lo) busy += hi - lo;
          lo = x.first; hi = x.second;
        } else {
          hi = std::max(hi, x.second);
        }
      }
      if (hi > lo) busy += hi - lo;
      c->prof.busy_seconds[k] += busy * 1e-3;
    }
    c->timeline.clear();
    for (auto& orc : *oprecs) {
      const Op& o = p0.ops[orc.op];
      float t0 = 0.f, t1 = 0.f;
      HM_CUDA(cudaEventElapsedTime(&t0, c0->ev_begin, g_prof.pool[orc.e0]));
      HM_CUDA(cudaEventElapsedTime(&t1, c0->ev_begin, g_prof.pool[orc.e1]));
      harmony_timeline_rec r{};
      r.op = orc.op; r.kind = o.kind; r.stream = o.stream; r.cat = o.cat; r.layer = o.layer; r.micro = o.mb;
      r.bytes = o.bytes; r.t0 = t0 * 1e-3; r.t1 = t1 * 1e-3;
      c->timeline.push_back(r);
    }
    g_prof.on = false;
  }
  double loss = 0.0;  // rank partials summed in rank order, microbatches in order (reading c22)
  if (pp) {  // the last layer's rank computed the loss of every microbatch
    const harmony_ctx* cl = R[c->gplan->layer_rank.back()];
    for (int i = 0; i < p0.m; ++i) loss += cl->h_loss[i];
  } else {
    for (int r = 0; r < p0.N; ++r)
      for (int i = 0; i < p0.m; ++i) loss += c0->h_loss[r * p0.m + i];
  }
  if (loss_out) *loss_out = loss;
  // a rank's ledger, or a group's box totals (bytes summed over ranks)
  harmony_step_stats tot = s[0];
  for (int r = 1; r < NR; ++r) {
    tot.h2d_bytes += s[r].h2d_bytes; tot.d2h_bytes += s[r].d2h_bytes;
    tot.h2d_weight_bytes += s[r].h2d_weight_bytes; tot.d2h_weight_bytes += s[r].d2h_weight_bytes;
    tot.h2d_state_bytes += s[r].h2d_state_bytes; tot.d2h_state_bytes += s[r].d2h_state_bytes;
    tot.h2d_stash_bytes += s[r].h2d_stash_bytes; tot.d2h_stash_bytes += s[r].d2h_stash_bytes;
    tot.h2d_input_bytes += s[r].h2d_input_bytes; tot.d2h_output_bytes += s[r].d2h_output_bytes;
    tot.h2d_grad_bytes += s[r].h2d_grad_bytes; tot.d2h_grad_bytes += s[r].d2h_grad_bytes;
    tot.nvlink_bytes += s[r].nvlink_bytes;
  }
  tot.kernel_launches = launches;
  tot.n_ops = pp ? c->gplan->ops.size() : p0.ops.size() * NR;
  tot.peak_arena_bytes = 0;
  for (harmony_ctx* r : R) tot.peak_arena_bytes = std::max<uint64_t>(tot.peak_arena_bytes, r->plan.arena_bytes);
  tot.graph = use_graph ? 1 : 0;
  for (int r = 0; r < NR; ++r) {
    R[r]->last = s[r];
    R[r]->last.kernel_launches = launches;
  }
  c->last = tot;
  if (out) *out = tot;
}

// Fill one rank's pinned host store and resident HBM tensors from the caller's fp32 parameters.
void register_rank(harmony_ctx* c, Plan&& p_in, const float* const* init_params) {
  Plan p = std::move(p_in);
  const int L = (int)p.layers.size(), m = p.m, N = p.N, r = p.rank;
  const size_t ts = p.dtype ? 2 : 4;
  HM_CUDA(cudaSetDevice(c->cfg.device));
  // arena
  if (c->arena) {
    HM_CHECK(p.arena_bytes <= c->cfg.hbm_cap_bytes, HARMONY_E_CAP_TOO_SMALL, "plan exceeds the adopted arena");
  } else {
    HM_CUDA(cudaMalloc(&c->arena, p.arena_bytes));
    c->own_arena = true;
  }
  // every arena byte starts at zero (the dW padding every rank's reduce-scatter reads among them)
  HM_CUDA(cudaMemset(c->arena, 0, p.arena_bytes));
  // events of the program
  c->events.resize(p.n_events);
  for (auto& e : c->events) HM_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  // pinned host store
  c->h_wc.assign(L, nullptr);
  c->h_state.assign(L, nullptr);
  c->h_stash.assign((size_t)L * m, nullptr);
  c->h_grad.assign(L, nullptr);
  c->h_loss = static_cast<double*>(alloc_host((size_t)N * m * 8));
  if (N > 1) {
    int64_t maxPpad = 0;
    for (auto& lp : p.layers) maxPpad = std::max(maxPpad, lp.Ppad);
    c->h_gather = static_cast<float*>(alloc_host((size_t)maxPpad * 4));
  }
  std::vector<uint8_t> full;  // staging of a full compute copy for resident layers
  for (int l = 0; l < L; ++l) {
    const LayerPlan& lp = p.layers[l];
    const int64_t sh = lp.shard, P = lp.P;
    c->h_wc[l] = static_cast<uint8_t*>(alloc_host((size_t)sh * ts));
    c->h_state[l] = static_cast<float*>(alloc_host((size_t)lp.state_bytes));
    if (p.retain_grads || p.schedule == HARMONY_SCHED_PER_GPU_VIRT) c->h_grad[l] = static_cast<float*>(alloc_host((size_t)sh * 4));
    float* master = c->h_state[l];
    memset(master, 0, lp.state_bytes);  // m = v = 0 (reading c3), padding = 0
    const int64_t lo = (int64_t)r * sh, hi = std::min<int64_t>(P, lo + sh);
    if (hi > lo) memcpy(master, init_params[l] + lo, (size_t)(hi - lo) * 4);
    if (ts == 2) {
      uint16_t* w = reinterpret_cast<uint16_t*>(c->h_wc[l]);
      for (int64_t i = 0; i < sh; ++i) w[i] = f32_to_bf16_rne(master[i]);
    } else {
      memcpy(c->h_wc[l], master, (size_t)sh * 4);
    }
    for (int i = 0; i < m; ++i)
      if (lp.stash_res[i] < 0) c->h_stash[(size_t)l * m + i] = static_cast<uint8_t*>(alloc_host(lp.g.st.total));
    // resident tensors go to HBM now
    if (lp.wc_res >= 0) {
      full.assign((size_t)lp.Ppad * ts, 0);
      if (ts == 2) {
        uint16_t* w = reinterpret_cast<uint16_t*>(full.data());
        for (int64_t i = 0; i < P; ++i) w[i] = f32_to_bf16_rne(init_params[l][i]);
      } else {
        memcpy(full.data(), init_params[l], (size_t)P * 4);
      }
      HM_CUDA(cudaMemcpy(c->arena + lp.wc_res, full.data(), full.size(), cudaMemcpyHostToDevice));
    }
    if (lp.state_res >= 0)
      HM_CUDA(cudaMemcpy(c->arena + lp.state_res, c->h_state[l], lp.state_bytes, cudaMemcpyHostToDevice));
  }
  HM_CUDA(cudaDeviceSynchronize());
  c->plan = std::move(p);
  c->registered = true;
}

// This rank's shard of one fp32 state tensor into host memory (n = shard elements).
void read_shard(harmony_ctx* c, int layer, int which, float* dst) {
  const LayerPlan& lp = c->plan.layers[layer];
  const uint64_t sh = (uint64_t)lp.shard;
  HM_CUDA(cudaSetDevice(c->cfg.device));
  if (which == HARMONY_GRAD) {
    memcpy(dst, c->h_grad[layer], sh * 4);
  } else {
    const uint64_t off = (which == HARMONY_PARAM ? 0 : which == HARMONY_ADAM_M ? 1 : 2) * sh * 4;
    if (lp.state_res >= 0) HM_CUDA(cudaMemcpy(dst, c->arena + lp.state_res + off, sh * 4, cudaMemcpyDeviceToHost));
    else memcpy(dst, reinterpret_cast<uint8_t*>(c->h_state[layer]) + off, sh * 4);
  }
}

}  // namespace

// ============================================================================================ C ABI
extern "C" {

int32_t harmony_abi_version(void) { return HARMONY_ABI_VERSION; }

void harmony_abi_sizes(uint64_t out[6]) {
  out[0] = sizeof(harmony_config);
  out[1] = sizeof(harmony_layer_desc);
  out[2] = sizeof(harmony_step_stats);
  out[3] = sizeof(harmony_plan_summary);
  out[4] = sizeof(hk_gemm_args);
  out[5] = sizeof(harmony_kernel_profile);
}

const char* harmony_last_error(const harmony_ctx* ctx) { return ctx ? ctx->err.c_str() : global_error(); }

harmony_status harmony_get_unique_id(uint8_t out[128]) {
  HM_API_BEGIN
  HM_CHECK(out != nullptr, HARMONY_E_INVALID_ARG, "out is NULL");
  HM_CHECK(nccl().load(), HARMONY_E_NCCL, nccl().err);
  ncclUniqueId id;
  check_nccl(nccl().GetUniqueId(&id), "ncclGetUniqueId");
  static_assert(sizeof(id) == 128, "ncclUniqueId size");
  memcpy(out, &id, 128);
  HM_API_END(nullptr)
}

harmony_status harmony_plan_dry(const harmony_config* cfg, int32_t n_layers, const harmony_layer_desc* descs,
                                harmony_plan_summary* out, char* text, uint64_t text_len) {
  HM_API_BEGIN
  HM_CHECK(cfg && descs && out, HARMONY_E_INVALID_ARG, "NULL argument");
  Plan p = make_plan(*cfg, n_layers, descs);
  *out = p.summary;
  if (text && text_len > 0) {
    std::string d = dump_plan(p);
    size_t n = std::min<size_t>(d.size(), text_len - 1);
    memcpy(text, d.data(), n);
    text[n] = 0;
  }
  HM_API_END(nullptr)
}

harmony_status harmony_plan_dry_group(const harmony_config* cfg, int32_t num_ranks, int32_t n_layers,
                                      const harmony_layer_desc* descs, harmony_plan_summary* out, char* text,
                                      uint64_t text_len) {
  HM_API_BEGIN
  HM_CHECK(cfg && descs && out, HARMONY_E_INVALID_ARG, "NULL argument");
  std::string d;
  if (cfg->schedule == HARMONY_SCHED_HARMONY_PP) {
    GroupPlan g = make_plan_pp(*cfg, num_ranks, n_layers, descs);
    *out = g.summary;
    if (text && text_len > 0) d = dump_group_plan(g);
  } else {  // data parallel: rank 0's program (every rank's has the same shape)
    harmony_config c0 = *cfg;
    c0.rank = 0;
    c0.world_size = num_ranks;
    Plan p = make_plan(c0, n_layers, descs);
    *out = p.summary;
    if (text && text_len > 0) d = dump_plan(p);
  }
  if (text && text_len > 0) {
    size_t n = std::min<size_t>(d.size(), text_len - 1);
    memcpy(text, d.data(), n);
    text[n] = 0;
  }
  HM_API_END(nullptr)
}

harmony_status harmony_init(const harmony_config* cfg, harmony_ctx** out) {
  harmony_ctx* c = nullptr;
  HM_API_BEGIN
  HM_CHECK(cfg && out, HARMONY_E_INVALID_ARG, "NULL argument");
  *out = nullptr;
  validate_config(*cfg);
  c = new harmony_ctx();
  init_rank(c, *cfg, true);
  if (cfg->arena) {
    HM_CHECK(cfg->hbm_cap_bytes > 0, HARMONY_E_INVALID_ARG, "an adopted arena needs hbm_cap_bytes");
    HM_CHECK(is_device_ptr(cfg->arena), HARMONY_E_INVALID_ARG, "cfg.arena is not a device pointer");
    HM_CHECK(reinterpret_cast<uintptr_t>(cfg->arena) % 1024 == 0, HARMONY_E_INVALID_ARG, "cfg.arena must be 1 KiB aligned");
    c->arena = static_cast<uint8_t*>(cfg->arena);
  }
  *out = c;
  c = nullptr;
  }
  catch (const Error& e) {
    harmony_status st = fail(nullptr, e);
    destroy(c);
    return st;
  }
  return HARMONY_OK;
}

harmony_status harmony_init_group(const harmony_config* cfg, int32_t num_ranks, const int32_t* devices,
                                  harmony_ctx** out) {
  harmony_ctx* g = nullptr;
  HM_API_BEGIN
  HM_CHECK(cfg && out, HARMONY_E_INVALID_ARG, "NULL argument");
  *out = nullptr;
  HM_CHECK(num_ranks >= 1 && num_ranks <= HM_MAX_GROUP, HARMONY_E_INVALID_ARG, "num_ranks must be in 1..16");
  HM_CHECK(cfg->arena == nullptr, HARMONY_E_INVALID_ARG, "a group allocates its ranks' arenas (cfg.arena must be NULL)");
  harmony_config gc = *cfg;
  gc.rank = 0;
  gc.world_size = num_ranks;
  gc.device = devices ? devices[0] : 0;
  validate_config(gc);
  g = new harmony_ctx();
  g->cfg = gc;
  for (int r = 0; r < num_ranks; ++r) {
    harmony_config rc = gc;
    rc.rank = r;
    rc.device = devices ? devices[r] : 0;
    if (rc.device != gc.device) g->one_device = false;
    harmony_ctx* m = new harmony_ctx();
    m->group = g;
    g->members.push_back(m);
    init_rank(m, rc, false);
  }
  if (!g->one_device) {  // pulls from peers' HBM over NVLink
    for (int r = 0; r < num_ranks; ++r)
      for (int q = 0; q < num_ranks; ++q) {
        const int a = g->members[r]->cfg.device, b = g->members[q]->cfg.device;
        if (a == b) continue;
        int can = 0;
        HM_CUDA(cudaDeviceCanAccessPeer(&can, a, b));
        HM_CHECK(can, HARMONY_E_UNSUPPORTED, "group ranks on GPUs without peer access");
        HM_CUDA(cudaSetDevice(a));
        cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
        if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
        else HM_CUDA(e);
      }
    HM_CUDA(cudaSetDevice(gc.device));
  }
  *out = g;
  g = nullptr;
  }
  catch (const Error& e) {
    harmony_status st = fail(nullptr, e);
    destroy(g);
    return st;
  }
  return HARMONY_OK;
}

harmony_status harmony_register_layers(harmony_ctx* c, int32_t n_layers, const harmony_layer_desc* descs,
                                       const float* const* init_params) {
  HM_API_BEGIN
  HM_CHECK(c != nullptr, HARMONY_E_INVALID_ARG, "ctx is NULL");
  HM_CHECK(!c->broken, HARMONY_E_BAD_STATE, "context has a sticky CUDA/NCCL error: " + c->err);
  HM_CHECK(!c->registered, HARMONY_E_BAD_STATE, "layers already registered");
  HM_CHECK(c->group == nullptr, HARMONY_E_BAD_STATE, "a group's rank context is not the caller's");
  HM_CHECK(descs && init_params, HARMONY_E_INVALID_ARG, "NULL argument");
  for (int l = 0; l < n_layers; ++l) HM_CHECK(init_params[l] != nullptr, HARMONY_E_INVALID_ARG, "init_params[l] is NULL");
  std::vector<harmony_ctx*> R = ranks_of(c);
  if (c->cfg.schedule == HARMONY_SCHED_HARMONY_PP) {
    HM_CHECK(!c->members.empty(), HARMONY_E_UNSUPPORTED, "Harmony-PP runs in a group (harmony_init_group)");
    auto gp = std::make_unique<GroupPlan>(make_plan_pp(c->cfg, (int)R.size(), n_layers, descs));
    HM_CHECK(gp->summary.hazards == 0, HARMONY_E_INVALID_ARG, "internal: planned program has a hazard: " + gp->hazard_msg);
    for (size_t r = 0; r < R.size(); ++r) {
      std::vector<const float*> mine;
      for (int l = (int)r; l < n_layers; l += (int)R.size()) mine.push_back(init_params[l]);
      register_rank(R[r], Plan(gp->ranks[r]), mine.data());
      HM_CUDA(cudaSetDevice(R[r]->cfg.device));
      for (auto e : R[r]->events) cudaEventDestroy(e);
      R[r]->events.assign(gp->n_events, nullptr);  // slots of the group program's events
      for (auto& e : R[r]->events) HM_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    }
    HM_CUDA(cudaSetDevice(c->cfg.device));
    c->plan = R[0]->plan;
    c->plan.summary = gp->summary;
    c->gplan = std::move(gp);
    c->registered = true;
    return HARMONY_OK;
  }
  std::vector<Plan> plans;
  for (harmony_ctx* r : R) {
    plans.push_back(make_plan(r->cfg, n_layers, descs));
    HM_CHECK(plans.back().summary.hazards == 0, HARMONY_E_INVALID_ARG,
             "internal: planned program has a hazard: " + plans.back().hazard_msg);
  }
  // lock-step issue needs the same program shape on every rank (same ops, kinds, streams, edges)
  for (size_t r = 1; r < plans.size(); ++r) {
    HM_CHECK(plans[r].ops.size() == plans[0].ops.size(), HARMONY_E_INVALID_ARG, "internal: rank programs differ");
    for (size_t i = 0; i < plans[0].ops.size(); ++i)
      HM_CHECK(plans[r].ops[i].kind == plans[0].ops[i].kind && plans[r].ops[i].stream == plans[0].ops[i].stream &&
                   plans[r].ops[i].waits == plans[0].ops[i].waits &&
                   (!is_group_collective(plans[0].ops[i].kind) ||
                    (plans[r].ops[i].dev == plans[0].ops[i].dev && plans[r].ops[i].count == plans[0].ops[i].count)),
               HARMONY_E_INVALID_ARG, "internal: rank programs differ");
  }
  // parameters per task layer: a column panel gets its W[:, panel] and b[panel] (every rank plans the
  // same panels: the split depends on the layer shapes and the cap only)
  std::vector<std::vector<float>> panel_store;
  std::vector<const float*> tparams;
  {
    const Plan& p0 = plans[0];
    for (int u = 0; u < n_layers; ++u) {
      const int cnt = p0.user_count[u];
      if (cnt == 1) { tparams.push_back(init_params[u]); continue; }
      const int din = descs[u].d_in, dout = descs[u].d_out, dp = dout / cnt;
      for (int k = 0; k < cnt; ++k) {
        std::vector<float> w((size_t)din * dp + dp);
        for (int i = 0; i < din; ++i)
          memcpy(w.data() + (size_t)i * dp, init_params[u] + (size_t)i * dout + (size_t)k * dp, (size_t)dp * 4);
        memcpy(w.data() + (size_t)din * dp, init_params[u] + (size_t)din * dout + (size_t)k * dp, (size_t)dp * 4);
        panel_store.push_back(std::move(w));
      }
    }
    size_t q = 0;
    tparams.clear();
    for (int u = 0; u < n_layers; ++u) {
      if (p0.user_count[u] == 1) tparams.push_back(init_params[u]);
      else
        for (int k = 0; k < p0.user_count[u]; ++k) tparams.push_back(panel_store[q++].data());
    }
  }
  for (size_t r = 0; r < R.size(); ++r) register_rank(R[r], std::move(plans[r]), tparams.data());
  HM_CUDA(cudaSetDevice(c->cfg.device));
  if (!c->members.empty()) {
    c->plan = R[0]->plan;  // the group's view: rank 0's plan (summary, geometry)
    c->registered = true;
  }
  HM_API_END(c)
}

harmony_status harmony_step(harmony_ctx* c, const float* x, const float* target, int64_t batch, double* loss_out,
                            harmony_step_stats* stats) {
  HM_API_BEGIN
  HM_CHECK(c != nullptr, HARMONY_E_INVALID_ARG, "ctx is NULL");
  HM_CHECK(!c->broken, HARMONY_E_BAD_STATE, "context has a sticky CUDA/NCCL error: " + c->err);
  HM_CHECK(c->registered, HARMONY_E_BAD_STATE, "harmony_register_layers first");
  HM_CHECK(c->group == nullptr, HARMONY_E_BAD_STATE, "a group's rank context is not the caller's");
  HM_CHECK(x && target, HARMONY_E_INVALID_ARG, "x/target NULL");
  const int64_t ranks = c->gplan ? 1 : (int64_t)ranks_of(c).size();  // Harmony-PP: one batch flows through the ranks
  HM_CHECK(batch == ranks * c->plan.m * c->plan.b, HARMONY_E_INVALID_ARG,
           ranks > 1 ? "batch must equal num_ranks*microbatches*microbatch_size (the global batch)"
                     : "batch must equal microbatches*microbatch_size (this rank's rows)");
  HM_CUDA(cudaSetDevice(c->cfg.device));
  run_step(c, x, target, loss_out, stats);
  HM_API_END(c)
}

static harmony_status read_task_layer(harmony_ctx* c, int32_t layer, int32_t which, float* dst, uint64_t n);

harmony_status harmony_read_state(harmony_ctx* c, int32_t layer, int32_t which, float* dst, uint64_t n) {
  HM_API_BEGIN
  HM_CHECK(c != nullptr, HARMONY_E_INVALID_ARG, "ctx is NULL");
  HM_CHECK(!c->broken, HARMONY_E_BAD_STATE, "context has a sticky CUDA/NCCL error: " + c->err);
  HM_CHECK(c->registered, HARMONY_E_BAD_STATE, "harmony_register_layers first");
  const Plan& p = c->plan;
  if (!c->gplan && !p.user_first.empty() && p.user_count.size() == (size_t)p.n_user &&
      (size_t)p.n_user != p.layers.size()) {  // some layer runs as column panels: reassemble W, b
    HM_CHECK(layer >= 0 && layer < p.n_user, HARMONY_E_INVALID_ARG, "layer out of range");
    const int first = p.user_first[layer], cnt = p.user_count[layer];
    if (cnt == 1) return read_task_layer(c, first, which, dst, n);
    const LayerGeom& g0 = p.layers[first].g;
    const int din = g0.desc.d_in, dp = g0.desc.d_out, dout = g0.ld_out;
    HM_CHECK(dst && n == (uint64_t)din * dout + dout, HARMONY_E_INVALID_ARG,
             "n_floats must equal the layer's parameter count");
    std::vector<float> part((size_t)din * dp + dp);
    for (int k = 0; k < cnt; ++k) {
      const harmony_status st = read_task_layer(c, first + k, which, part.data(), part.size());
      if (st != HARMONY_OK) return st;
      for (int i = 0; i < din; ++i)
        memcpy(dst + (size_t)i * dout + (size_t)k * dp, part.data() + (size_t)i * dp, (size_t)dp * 4);
      memcpy(dst + (size_t)din * dout + (size_t)k * dp, part.data() + (size_t)din * dp, (size_t)dp * 4);
    }
    return HARMONY_OK;
  }
  return read_task_layer(c, layer, which, dst, n);
  HM_API_END(c)
}

static harmony_status read_task_layer(harmony_ctx* c, int32_t layer, int32_t which, float* dst, uint64_t n) {
  HM_API_BEGIN
  if (c->gplan) {  // Harmony-PP: the layer lives, unsharded, on rank layer % N
    const GroupPlan& gp = *c->gplan;
    HM_CHECK(layer >= 0 && layer < (int)gp.layer_rank.size(), HARMONY_E_INVALID_ARG, "layer out of range");
    harmony_ctx* m = c->members[gp.layer_rank[layer]];
    const int k = gp.layer_local[layer];
    const LayerPlan& lq = m->plan.layers[k];
    HM_CHECK(dst && n == (uint64_t)lq.P, HARMONY_E_INVALID_ARG, "n_floats must equal the layer's parameter count");
    HM_CHECK(which >= HARMONY_PARAM && which <= HARMONY_ADAM_V, HARMONY_E_INVALID_ARG, "bad state kind");
    HM_CHECK(which != HARMONY_GRAD || m->plan.retain_grads, HARMONY_E_BAD_STATE, "HARMONY_GRAD needs retain_grads");
    std::vector<float> all((size_t)lq.shard);
    read_shard(m, k, which, all.data());
    memcpy(dst, all.data(), (size_t)lq.P * 4);
    HM_CUDA(cudaSetDevice(c->cfg.device));
    return HARMONY_OK;
  }
  const Plan& p = c->plan;
  HM_CHECK(layer >= 0 && layer < (int)p.layers.size(), HARMONY_E_INVALID_ARG, "layer out of range");
  const LayerPlan& lp = p.layers[layer];
  HM_CHECK(dst && n == (uint64_t)lp.P, HARMONY_E_INVALID_ARG, "n_floats must equal the layer's parameter count");
  HM_CHECK(which >= HARMONY_PARAM && which <= HARMONY_ADAM_V, HARMONY_E_INVALID_ARG, "bad state kind");
  HM_CHECK(which != HARMONY_GRAD || p.retain_grads, HARMONY_E_BAD_STATE, "HARMONY_GRAD needs retain_grads");
  const uint64_t sh = (uint64_t)lp.shard;
  if (!c->members.empty()) {  // a group reads every rank's shard directly
    std::vector<float> all((size_t)lp.Ppad);
    for (size_t r = 0; r < c->members.size(); ++r) read_shard(c->members[r], layer, which, all.data() + r * sh);
    memcpy(dst, all.data(), (size_t)lp.P * 4);
    HM_CUDA(cudaSetDevice(c->cfg.device));
  } else if (p.N == 1) {
    std::vector<float> mine(sh);
    read_shard(c, layer, which, mine.data());
    memcpy(dst, mine.data(), (size_t)lp.P * 4);
  } else {
    // all-gather through the arena: dW buffer 0 (Ppad fp32 elements) is free between steps
    std::vector<float> mine(sh);
    read_shard(c, layer, which, mine.data());
    float* d = reinterpret_cast<float*>(c->arena + p.dw[0]);
    cudaStream_t cs = c->st[S_COMM];
    HM_CUDA(cudaMemcpyAsync(d + (uint64_t)p.rank * sh, mine.data(), sh * 4, cudaMemcpyHostToDevice, cs));
    check_nccl(nccl().AllGather(d + (uint64_t)p.rank * sh, d, sh, ncclFloat32, c->comm, cs), "ncclAllGather(read_state)");
    HM_CUDA(cudaMemcpyAsync(c->h_gather, d, (size_t)lp.Ppad * 4, cudaMemcpyDeviceToHost, cs));
    HM_CUDA(cudaStreamSynchronize(cs));
    memcpy(dst, c->h_gather, (size_t)lp.P * 4);
  }
  HM_API_END(c)
}

harmony_status harmony_read_stats(const harmony_ctx* c, harmony_step_stats* out) {
  if (!c || !out) return HARMONY_E_INVALID_ARG;
  *out = c->last;
  return HARMONY_OK;
}

harmony_status harmony_read_rank_stats(const harmony_ctx* c, int32_t rank, harmony_step_stats* out) {
  if (!c || !out) return HARMONY_E_INVALID_ARG;
  if (c->members.empty()) {
    if (rank != 0) return HARMONY_E_INVALID_ARG;
    *out = c->last;
    return HARMONY_OK;
  }
  if (rank < 0 || rank >= (int32_t)c->members.size()) return HARMONY_E_INVALID_ARG;
  *out = c->members[rank]->last;
  return HARMONY_OK;
}

harmony_status harmony_plan_info(const harmony_ctx* c, harmony_plan_summary* out) {
  if (!c || !out) return HARMONY_E_INVALID_ARG;
  if (!c->registered) return HARMONY_E_BAD_STATE;
  *out = c->plan.summary;
  return HARMONY_OK;
}

harmony_status harmony_set_profiling(harmony_ctx* c, int32_t on) {
  if (!c) return HARMONY_E_INVALID_ARG;
  if (on && !c->members.empty() && c->members.size() > 1) {
    c->err = "per-kernel profiling is per rank context (one process per GPU), not for a group";
    return HARMONY_E_UNSUPPORTED;
  }
  c->profiling = on != 0;
  c->prof = harmony_kernel_profile{};
  return HARMONY_OK;
}

harmony_status harmony_read_timeline(const harmony_ctx* c, harmony_timeline_rec* out, int32_t cap, int32_t* n_out) {
  if (!c || !n_out || cap < 0) return HARMONY_E_INVALID_ARG;
  const int32_t n = (int32_t)c->timeline.size();
  *n_out = n;
  if (out)
    for (int32_t i = 0; i < std::min(n, cap); ++i) out[i] = c->timeline[i];
  return HARMONY_OK;
}

harmony_status harmony_read_kernel_timeline(const harmony_ctx* c, harmony_kernel_rec* out, int32_t cap,
                                           int32_t* n_out) {
  if (!c || !n_out || cap < 0) return HARMONY_E_INVALID_ARG;
  const int32_t n = (int32_t)c->ktimeline.size();
  *n_out = n;
  if (out)
    for (int32_t i = 0; i < std::min(n, cap); ++i) out[i] = c->ktimeline[i];
  return HARMONY_OK;
}

harmony_status harmony_read_profile(const harmony_ctx* c, harmony_kernel_profile* out) {
  if (!c || !out) return HARMONY_E_INVALID_ARG;
  *out = c->prof;
  return HARMONY_OK;
}

harmony_status harmony_finalize(harmony_ctx* c) {
  if (!c) return HARMONY_E_INVALID_ARG;
  if (c->group) return HARMONY_E_BAD_STATE;
  destroy(c);
  return HARMONY_OK;
}

}  // extern "C"
