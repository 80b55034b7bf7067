// split_gemm.cpp — operator decomposition of one GEMM fwd+bwd across GPUs.
//
// Harmony can "further decompose individual operations—such as a matrix
// multiplication—into subtasks that can run on different physical devices".  For
// Y = X.W (X [M,K], W [K,N]; reading c19) the natural axis is K: rank r owns the K-slice
// X[:, K_r], W[K_r, :], computes the fp32 partial X[:,K_r].W[K_r,:], and a reduce-scatter sums the
// partials so rank r ends with rows [r*M/N, (r+1)*M/N) of Y.  The forward is cut into C row-chunk
// tile subtasks: chunk c's GEMM (batched over the N destination row blocks) writes a send buffer
// whose reduce-scatter runs on the comm stream while the GEMM of chunk c+1 runs (event-ordered).
// Backward: all-gather the row-sharded dY (bf16), then dX[:,K_r] = dY.W[K_r,:]^T and
// dW[K_r,:] = X[:,K_r]^T.dY are local (no communication).
//
// The ranks are either one process each (harmony_split_gemm_init: NCCL reduce-scatter / all-gather)
// or one process driving them all (harmony_split_gemm_init_group: the library's own collectives,
// pulls from the peers' buffers — rank i's chunk rows are the sum of every rank's partial in rank
// order, the same on one GPU (loopback) or many).
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "comm.hpp"
#include "common.hpp"
#include "harmony_kernels.h"
#include "kernels/kernels.hpp"

using namespace hm;

namespace {
struct Lane {  // one rank
  int rank = 0, device = 0;
  cudaStream_t comp = nullptr, comm_st = nullptr;
  std::vector<cudaEvent_t> ev_chunk, ev_rs;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev_ag = nullptr;
  float* send = nullptr;             // [2][world][R][N] fp32 partials (double-buffered chunks), world > 1
  __nv_bfloat16* dy_full = nullptr;  // [M][N] gathered dY (world > 1)
};
}  // namespace

struct harmony_split_gemm {
  harmony_config cfg{};
  int64_t M = 0, N = 0, K = 0, Kr = 0, Mr = 0;  // Kr = K/world, Mr = M/world
  int world = 1, chunks = 1;
  bool group = false, one_device = true;
  std::vector<Lane> lanes;  // one (per process) or world (group)
  ncclComm_t comm = nullptr;
  std::string err;
};

namespace {
harmony_status sfail(harmony_split_gemm* g, const Error& e) {
  if (g) g->err = e.msg;
  set_global_error(e.msg);
  return e.code;
}
void destroy(harmony_split_gemm* g) {
  if (!g) return;
  for (auto& l : g->lanes) {
    cudaSetDevice(l.device);
    if (l.comp) cudaStreamSynchronize(l.comp);
    if (l.comm_st) cudaStreamSynchronize(l.comm_st);
  }
  for (auto& l : g->lanes) {
    cudaSetDevice(l.device);
    for (auto e : l.ev_chunk) cudaEventDestroy(e);
    for (auto e : l.ev_rs) cudaEventDestroy(e);
    if (l.ev0) cudaEventDestroy(l.ev0);
    if (l.ev1) cudaEventDestroy(l.ev1);
    if (l.ev_ag) cudaEventDestroy(l.ev_ag);
    if (l.comp) cudaStreamDestroy(l.comp);
    if (l.comm_st) cudaStreamDestroy(l.comm_st);
    if (l.send) cudaFree(l.send);
    if (l.dy_full) cudaFree(l.dy_full);
  }
  if (g->comm && nccl().CommDestroy) nccl().CommDestroy(g->comm);
  delete g;
}
void nccl_ok(ncclResult_t r, const char* what) {
  if (r != ncclSuccess)
    throw Error{HARMONY_E_NCCL, std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "?")};
}

void check_shape(int W, int64_t M, int64_t N, int64_t K, int chunks) {
  HM_CHECK(M > 0 && N > 0 && K > 0 && chunks >= 1, HARMONY_E_INVALID_ARG, "bad shape");
  HM_CHECK(K % (8 * W) == 0, HARMONY_E_UNSUPPORTED, "K must be a multiple of 8*world_size (bf16 TMA strides)");
  HM_CHECK(M % ((int64_t)W * chunks) == 0, HARMONY_E_UNSUPPORTED, "M must be a multiple of world_size*chunks");
  HM_CHECK(N % 8 == 0 && M % 8 == 0, HARMONY_E_UNSUPPORTED, "M and N must be multiples of 8");
}

void init_lane(harmony_split_gemm* g, Lane& l) {
  HM_CUDA(cudaSetDevice(l.device));
  HM_CUDA(cudaStreamCreateWithFlags(&l.comp, cudaStreamNonBlocking));
  HM_CUDA(cudaStreamCreateWithFlags(&l.comm_st, cudaStreamNonBlocking));
  HM_CUDA(cudaEventCreate(&l.ev0));
  HM_CUDA(cudaEventCreate(&l.ev1));
  HM_CUDA(cudaEventCreateWithFlags(&l.ev_ag, cudaEventDisableTiming));
  l.ev_chunk.resize(g->chunks);
  l.ev_rs.resize(g->chunks);
  for (int c = 0; c < g->chunks; ++c) {
    HM_CUDA(cudaEventCreateWithFlags(&l.ev_chunk[c], cudaEventDisableTiming));
    HM_CUDA(cudaEventCreateWithFlags(&l.ev_rs[c], cudaEventDisableTiming));
  }
  if (g->world > 1) {
    const int64_t R = g->M / ((int64_t)g->world * g->chunks);
    HM_CUDA(cudaMalloc(&l.send, sizeof(float) * 2 * (size_t)g->world * R * g->N));
    HM_CUDA(cudaMalloc(&l.dy_full, sizeof(__nv_bfloat16) * (size_t)g->M * g->N));
  }
}

struct RankArgs {
  const void* X;
  const void* W;
  const void* dY;
  float* Y;
  void* dX;
  float* dW;
};

// Forward tile subtasks of chunk c on lane l: rows i*Mr + c*R .. +R of the partial product for every
// destination rank i (world 1: straight into Y).
void fwd_chunk(harmony_split_gemm* g, Lane& l, const RankArgs& a, int64_t c) {
  const int Wn = g->world;
  const int64_t N = g->N, Kr = g->Kr, R = g->M / (Wn * g->chunks);
  const __nv_bfloat16* x = static_cast<const __nv_bfloat16*>(a.X);
  float* sb = Wn == 1 ? nullptr : l.send + (size_t)(c % 2) * Wn * R * N;
  for (int i = 0; i < Wn; ++i) {
    hk_gemm_args ga = gemm_args(1, (int)R, (int)N, (int)Kr);
    ga.A = x + (size_t)(i * g->Mr + c * R) * Kr; ga.a_mn_major = 0; ga.lda = Kr;
    ga.B = a.W; ga.b_mn_major = 1; ga.ldb = N;
    ga.C = Wn == 1 ? a.Y + (size_t)(c * R) * N : sb + (size_t)i * R * N;
    ga.ldc = N;
    ga.epilogue = HK_EPI_STORE_F32;
    gemm(ga, l.comp);
  }
}

void bwd_local(harmony_split_gemm* g, Lane& l, const RankArgs& a, const void* dy) {
  const int64_t M = g->M, N = g->N, Kr = g->Kr;
  {  // dX[:, K_r] = dY . W[K_r,:]^T   (A = dY K-major, B = W K-major)
    hk_gemm_args ga = gemm_args(1, (int)M, (int)Kr, (int)N);
    ga.A = dy; ga.a_mn_major = 0; ga.lda = N;
    ga.B = a.W; ga.b_mn_major = 0; ga.ldb = N;
    ga.C = a.dX; ga.ldc = Kr;
    ga.epilogue = HK_EPI_STORE_T;
    gemm(ga, l.comp);
  }
  {  // dW[K_r,:] = X[:,K_r]^T . dY  (A, B MN-major), fp32
    hk_gemm_args ga = gemm_args(1, (int)Kr, (int)N, (int)M);
    ga.A = a.X; ga.a_mn_major = 1; ga.lda = Kr;
    ga.B = dy; ga.b_mn_major = 1; ga.ldb = N;
    ga.C = a.dW; ga.ldc = N;
    ga.epilogue = HK_EPI_ACC_F32; ga.accumulate = 0;
    gemm(ga, l.comp);
  }
}

// One process, one rank (NCCL between processes when world > 1).
void run_rank(harmony_split_gemm* g, const RankArgs& a, double* seconds) {
  Lane& l = g->lanes[0];
  const int Wn = g->world;
  const int64_t N = g->N, C = g->chunks, R = g->M / (Wn * C);
  HM_CUDA(cudaSetDevice(l.device));
  HM_CUDA(cudaEventRecord(l.ev0, cudaStreamLegacy));  // the caller's default-stream work on the operands
  HM_CUDA(cudaStreamWaitEvent(l.comp, l.ev0, 0));
  HM_CUDA(cudaEventRecord(l.ev0, l.comp));
  HM_CUDA(cudaStreamWaitEvent(l.comm_st, l.ev0, 0));
  for (int64_t c = 0; c < C; ++c) {
    if (Wn > 1 && c >= 2) HM_CUDA(cudaStreamWaitEvent(l.comp, l.ev_rs[c - 2], 0));  // send buffer reuse
    fwd_chunk(g, l, a, c);
    if (Wn > 1) {
      float* sb = l.send + (size_t)(c % 2) * Wn * R * N;
      HM_CUDA(cudaEventRecord(l.ev_chunk[c], l.comp));
      HM_CUDA(cudaStreamWaitEvent(l.comm_st, l.ev_chunk[c], 0));
      nccl_ok(nccl().ReduceScatter(sb, a.Y + (size_t)(c * R) * N, (size_t)R * N, ncclFloat32, ncclSum, g->comm,
                                   l.comm_st),
              "ncclReduceScatter(split gemm)");
      HM_CUDA(cudaEventRecord(l.ev_rs[c], l.comm_st));
    }
  }
  const void* dy = a.dY;
  if (Wn > 1) {
    nccl_ok(nccl().AllGather(a.dY, l.dy_full, (size_t)g->Mr * N, ncclBfloat16, g->comm, l.comm_st), "ncclAllGather(dY)");
    HM_CUDA(cudaEventRecord(l.ev_ag, l.comm_st));
    HM_CUDA(cudaStreamWaitEvent(l.comp, l.ev_ag, 0));
    dy = l.dy_full;
  }
  bwd_local(g, l, a, dy);
  if (Wn > 1) {
    HM_CUDA(cudaEventRecord(l.ev_ag, l.comm_st));  // all reduce-scatters done
    HM_CUDA(cudaStreamWaitEvent(l.comp, l.ev_ag, 0));
  }
  HM_CUDA(cudaEventRecord(l.ev1, l.comp));
  HM_CUDA(cudaEventSynchronize(l.ev1));
  float ms = 0.f;
  HM_CUDA(cudaEventElapsedTime(&ms, l.ev0, l.ev1));
  if (seconds) *seconds = ms * 1e-3;
}

// One process, all ranks: the chunk reduce-scatter is rank i's pull-and-sum of block i of every
// rank's send buffer (rank order), the dY all-gather a copy of every rank's shard.
void run_group(harmony_split_gemm* g, const std::vector<RankArgs>& a, double* seconds) {
  const int Wn = g->world;
  const int64_t N = g->N, C = g->chunks, R = g->M / (Wn * C);
  auto dev = [&](Lane& l) {
    if (!g->one_device) HM_CUDA(cudaSetDevice(l.device));
  };
  Lane& l0 = g->lanes[0];
  HM_CUDA(cudaSetDevice(l0.device));
  HM_CUDA(cudaEventRecord(l0.ev0, cudaStreamLegacy));
  HM_CUDA(cudaStreamWaitEvent(l0.comp, l0.ev0, 0));
  HM_CUDA(cudaEventRecord(l0.ev0, l0.comp));
  for (auto& l : g->lanes) {
    dev(l);
    if (&l != &l0) HM_CUDA(cudaStreamWaitEvent(l.comp, l0.ev0, 0));
    HM_CUDA(cudaStreamWaitEvent(l.comm_st, l0.ev0, 0));
  }
  for (int64_t c = 0; c < C; ++c) {
    for (int r = 0; r < Wn; ++r) {
      Lane& l = g->lanes[r];
      dev(l);
      if (c >= 2)  // this send buffer was last pulled by every rank for chunk c-2
        for (int i = 0; i < Wn; ++i) HM_CUDA(cudaStreamWaitEvent(l.comp, g->lanes[i].ev_rs[c - 2], 0));
      fwd_chunk(g, l, a[r], c);
      HM_CUDA(cudaEventRecord(l.ev_chunk[c], l.comp));
    }
    for (int i = 0; i < Wn; ++i) {
      Lane& l = g->lanes[i];
      dev(l);
      const float* src[HM_MAX_GROUP];
      for (int q = 0; q < Wn; ++q) {
        HM_CUDA(cudaStreamWaitEvent(l.comm_st, g->lanes[q].ev_chunk[c], 0));
        src[q] = g->lanes[q].send + (size_t)(c % 2) * Wn * R * N + (size_t)i * R * N;
      }
      rank_sum(Wn, src, R * N, a[i].Y + (size_t)(c * R) * N, l.comm_st);
      HM_CUDA(cudaEventRecord(l.ev_rs[c], l.comm_st));
    }
  }
  for (int r = 0; r < Wn; ++r) {  // dY all-gather (the shards are caller inputs, ready at ev0)
    Lane& l = g->lanes[r];
    dev(l);
    const size_t sh = (size_t)g->Mr * N;
    for (int q = 0; q < Wn; ++q)
      HM_CUDA(cudaMemcpyAsync(l.dy_full + q * sh, a[q].dY, sh * sizeof(__nv_bfloat16), cudaMemcpyDefault, l.comm_st));
    HM_CUDA(cudaEventRecord(l.ev_ag, l.comm_st));
    HM_CUDA(cudaStreamWaitEvent(l.comp, l.ev_ag, 0));
    bwd_local(g, l, a[r], l.dy_full);
  }
  float ms = 0.f;
  for (int r = 0; r < Wn; ++r) {  // done when every rank's GEMMs and every pull have finished
    Lane& l = g->lanes[r];
    dev(l);
    for (int i = 0; i < Wn; ++i) HM_CUDA(cudaStreamWaitEvent(l.comp, g->lanes[i].ev_rs[C - 1], 0));
    HM_CUDA(cudaEventRecord(l.ev1, l.comp));
  }
  for (int r = 0; r < Wn; ++r) {
    HM_CUDA(cudaEventSynchronize(g->lanes[r].ev1));
    float e = 0.f;
    HM_CUDA(cudaEventElapsedTime(&e, l0.ev0, g->lanes[r].ev1));
    ms = std::max(ms, e);
  }
  HM_CUDA(cudaSetDevice(l0.device));
  if (seconds) *seconds = ms * 1e-3;
}
}  // namespace

extern "C" {

harmony_status harmony_split_gemm_init(const harmony_config* cfg, int64_t M, int64_t N, int64_t K, int32_t chunks,
                                       harmony_split_gemm** out) {
  harmony_split_gemm* g = nullptr;
  try {
    HM_CHECK(cfg && out, HARMONY_E_INVALID_ARG, "NULL argument");
    HM_CHECK(cfg->struct_size == sizeof(harmony_config), HARMONY_E_INVALID_ARG, "harmony_config.struct_size mismatch");
    const int W = cfg->world_size;
    HM_CHECK(W >= 1 && cfg->rank >= 0 && cfg->rank < W, HARMONY_E_INVALID_ARG, "bad rank / world_size");
    check_shape(W, M, N, K, chunks);
    g = new harmony_split_gemm();
    g->cfg = *cfg;
    g->M = M; g->N = N; g->K = K; g->Kr = K / W; g->Mr = M / W; g->chunks = chunks; g->world = W;
    g->lanes.resize(1);
    g->lanes[0].rank = cfg->rank;
    g->lanes[0].device = cfg->device;
    init_lane(g, g->lanes[0]);
    if (W > 1) {
      HM_CHECK(nccl().load(), HARMONY_E_NCCL, nccl().err);
      ncclUniqueId id;
      memcpy(&id, cfg->nccl_id, 128);
      nccl_ok(nccl().CommInitRank(&g->comm, W, id, cfg->rank), "ncclCommInitRank");
    }
    *out = g;
  } catch (const Error& e) {
    harmony_status s = sfail(nullptr, e);
    destroy(g);
    return s;
  }
  return HARMONY_OK;
}

harmony_status harmony_split_gemm_init_group(int32_t num_ranks, const int32_t* devices, int64_t M, int64_t N,
                                             int64_t K, int32_t chunks, harmony_split_gemm** out) {
  harmony_split_gemm* g = nullptr;
  try {
    HM_CHECK(out, HARMONY_E_INVALID_ARG, "NULL argument");
    HM_CHECK(num_ranks >= 1 && num_ranks <= HM_MAX_GROUP, HARMONY_E_INVALID_ARG, "num_ranks must be in 1..16");
    check_shape(num_ranks, M, N, K, chunks);
    g = new harmony_split_gemm();
    g->M = M; g->N = N; g->K = K; g->Kr = K / num_ranks; g->Mr = M / num_ranks; g->chunks = chunks;
    g->world = num_ranks;
    g->group = true;
    g->lanes.resize(num_ranks);
    for (int r = 0; r < num_ranks; ++r) {
      g->lanes[r].rank = r;
      g->lanes[r].device = devices ? devices[r] : 0;
      if (g->lanes[r].device != g->lanes[0].device) g->one_device = false;
    }
    if (!g->one_device)
      for (int r = 0; r < num_ranks; ++r)
        for (int q = 0; q < num_ranks; ++q) {
          const int a = g->lanes[r].device, b = g->lanes[q].device;
          if (a == b) continue;
          int can = 0;
          HM_CUDA(cudaDeviceCanAccessPeer(&can, a, b));
          HM_CHECK(can, HARMONY_E_UNSUPPORTED, "group ranks on GPUs without peer access");
          HM_CUDA(cudaSetDevice(a));
          cudaError_t e = cudaDeviceEnablePeerAccess(b, 0);
          if (e == cudaErrorPeerAccessAlreadyEnabled) cudaGetLastError();
          else HM_CUDA(e);
        }
    for (auto& l : g->lanes) init_lane(g, l);
    HM_CUDA(cudaSetDevice(g->lanes[0].device));
    *out = g;
  } catch (const Error& e) {
    harmony_status s = sfail(nullptr, e);
    destroy(g);
    return s;
  }
  return HARMONY_OK;
}

harmony_status harmony_split_gemm_run(harmony_split_gemm* g, const void* X, const void* W, const void* dY_shard,
                                      float* Y_shard, void* dX, float* dW, double* seconds) {
  try {
    HM_CHECK(g && X && W && dY_shard && Y_shard && dX && dW, HARMONY_E_INVALID_ARG, "NULL argument");
    HM_CHECK(!g->group, HARMONY_E_BAD_STATE, "a group takes per-rank pointer arrays (harmony_split_gemm_run_group)");
    run_rank(g, RankArgs{X, W, dY_shard, Y_shard, dX, dW}, seconds);
  } catch (const Error& e) {
    return sfail(g, e);
  }
  return HARMONY_OK;
}

harmony_status harmony_split_gemm_run_group(harmony_split_gemm* g, const void* const* X, const void* const* W,
                                            const void* const* dY_shard, float* const* Y_shard, void* const* dX,
                                            float* const* dW, double* seconds) {
  try {
    HM_CHECK(g && X && W && dY_shard && Y_shard && dX && dW, HARMONY_E_INVALID_ARG, "NULL argument");
    HM_CHECK(g->group, HARMONY_E_BAD_STATE, "not a group (harmony_split_gemm_run)");
    std::vector<RankArgs> a(g->world);
    for (int r = 0; r < g->world; ++r) {
      HM_CHECK(X[r] && W[r] && dY_shard[r] && Y_shard[r] && dX[r] && dW[r], HARMONY_E_INVALID_ARG, "NULL rank pointer");
      a[r] = RankArgs{X[r], W[r], dY_shard[r], Y_shard[r], dX[r], dW[r]};
    }
    run_group(g, a, seconds);
  } catch (const Error& e) {
    return sfail(g, e);
  }
  return HARMONY_OK;
}

harmony_status harmony_split_gemm_finalize(harmony_split_gemm* g) {
  if (!g) return HARMONY_E_INVALID_ARG;
  destroy(g);
  return HARMONY_OK;
}

}  // extern "C"
