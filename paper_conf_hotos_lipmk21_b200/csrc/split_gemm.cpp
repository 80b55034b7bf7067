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
#include <string.h>

#include <algorithm>
#include <string>
#include <vector>

#include "comm.hpp"
#include "common.hpp"
#include "harmony_kernels.h"
#include "kernels/kernels.hpp"

using namespace hm;

struct harmony_split_gemm {
  harmony_config cfg{};
  int64_t M = 0, N = 0, K = 0, Kr = 0, Mr = 0;  // Kr = K/world, Mr = M/world
  int chunks = 1;
  cudaStream_t comp = nullptr, comm_st = nullptr;
  std::vector<cudaEvent_t> ev_chunk, ev_rs;
  cudaEvent_t ev0 = nullptr, ev1 = nullptr, ev_ag = nullptr;
  ncclComm_t comm = nullptr;
  float* send = nullptr;          // [2][world][R][N] fp32 partials (double-buffered chunks), N>1
  __nv_bfloat16* dy_full = nullptr;  // [M][N] gathered dY (N>1)
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
  cudaSetDevice(g->cfg.device);
  if (g->comp) cudaStreamSynchronize(g->comp);
  if (g->comm_st) cudaStreamSynchronize(g->comm_st);
  for (auto e : g->ev_chunk) cudaEventDestroy(e);
  for (auto e : g->ev_rs) cudaEventDestroy(e);
  if (g->ev0) cudaEventDestroy(g->ev0);
  if (g->ev1) cudaEventDestroy(g->ev1);
  if (g->ev_ag) cudaEventDestroy(g->ev_ag);
  if (g->comp) cudaStreamDestroy(g->comp);
  if (g->comm_st) cudaStreamDestroy(g->comm_st);
  if (g->comm && nccl().CommDestroy) nccl().CommDestroy(g->comm);
  if (g->send) cudaFree(g->send);
  if (g->dy_full) cudaFree(g->dy_full);
  delete g;
}
void nccl_ok(ncclResult_t r, const char* what) {
  if (r != ncclSuccess)
    throw Error{HARMONY_E_NCCL, std::string(what) + ": " + (nccl().GetErrorString ? nccl().GetErrorString(r) : "?")};
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
    HM_CHECK(M > 0 && N > 0 && K > 0 && chunks >= 1, HARMONY_E_INVALID_ARG, "bad shape");
    HM_CHECK(K % (8 * W) == 0, HARMONY_E_UNSUPPORTED, "K must be a multiple of 8*world_size (bf16 TMA strides)");
    HM_CHECK(M % ((int64_t)W * chunks) == 0, HARMONY_E_UNSUPPORTED, "M must be a multiple of world_size*chunks");
    HM_CHECK(N % 8 == 0 && M % 8 == 0, HARMONY_E_UNSUPPORTED, "M and N must be multiples of 8");
    g = new harmony_split_gemm();
    g->cfg = *cfg;
    g->M = M; g->N = N; g->K = K; g->Kr = K / W; g->Mr = M / W; g->chunks = chunks;
    HM_CUDA(cudaSetDevice(cfg->device));
    HM_CUDA(cudaStreamCreateWithFlags(&g->comp, cudaStreamNonBlocking));
    HM_CUDA(cudaStreamCreateWithFlags(&g->comm_st, cudaStreamNonBlocking));
    HM_CUDA(cudaEventCreate(&g->ev0));
    HM_CUDA(cudaEventCreate(&g->ev1));
    HM_CUDA(cudaEventCreateWithFlags(&g->ev_ag, cudaEventDisableTiming));
    g->ev_chunk.resize(chunks);
    g->ev_rs.resize(chunks);
    for (int c = 0; c < chunks; ++c) {
      HM_CUDA(cudaEventCreateWithFlags(&g->ev_chunk[c], cudaEventDisableTiming));
      HM_CUDA(cudaEventCreateWithFlags(&g->ev_rs[c], cudaEventDisableTiming));
    }
    if (W > 1) {
      HM_CHECK(nccl().load(), HARMONY_E_NCCL, nccl().err);
      ncclUniqueId id;
      memcpy(&id, cfg->nccl_id, 128);
      nccl_ok(nccl().CommInitRank(&g->comm, W, id, cfg->rank), "ncclCommInitRank");
      const int64_t R = M / ((int64_t)W * chunks);
      HM_CUDA(cudaMalloc(&g->send, sizeof(float) * 2 * (size_t)W * R * N));
      HM_CUDA(cudaMalloc(&g->dy_full, sizeof(__nv_bfloat16) * (size_t)M * N));
    }
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
    HM_CUDA(cudaSetDevice(g->cfg.device));
    const int Wn = g->cfg.world_size, r = g->cfg.rank;
    const int64_t M = g->M, N = g->N, Kr = g->Kr, C = g->chunks;
    const int64_t R = M / (Wn * C);  // rows per (chunk, destination rank)
    const __nv_bfloat16* x = static_cast<const __nv_bfloat16*>(X);
    HM_CUDA(cudaEventRecord(g->ev0, g->comp));
    HM_CUDA(cudaStreamWaitEvent(g->comm_st, g->ev0, 0));
    // ---- forward: C chunk subtasks, each a GEMM batched over the Wn destination row blocks
    for (int64_t c = 0; c < C; ++c) {
      // tile subtask (c, i): rows i*Mr + c*R .. +R of the partial product, for destination rank i
      float* sb = Wn == 1 ? nullptr : g->send + (size_t)(c % 2) * Wn * R * N;
      if (Wn > 1 && c >= 2) HM_CUDA(cudaStreamWaitEvent(g->comp, g->ev_rs[c - 2], 0));  // send buffer reuse
      for (int i = 0; i < Wn; ++i) {
        hk_gemm_args a = gemm_args(1, (int)R, (int)N, (int)Kr);
        a.A = x + (size_t)(i * g->Mr + c * R) * Kr; a.a_mn_major = 0; a.lda = Kr;
        a.B = W; a.b_mn_major = 1; a.ldb = N;
        a.C = Wn == 1 ? Y_shard + (size_t)(c * R) * N : sb + (size_t)i * R * N;
        a.ldc = N;
        a.epilogue = HK_EPI_STORE_F32;
        gemm(a, g->comp);
      }
      if (Wn > 1) {
        HM_CUDA(cudaEventRecord(g->ev_chunk[c], g->comp));
        HM_CUDA(cudaStreamWaitEvent(g->comm_st, g->ev_chunk[c], 0));
        nccl_ok(nccl().ReduceScatter(sb, Y_shard + (size_t)(c * R) * N, (size_t)R * N, ncclFloat32, ncclSum, g->comm,
                                     g->comm_st),
                "ncclReduceScatter(split gemm)");
        HM_CUDA(cudaEventRecord(g->ev_rs[c], g->comm_st));
      }
    }
    // ---- backward: gather dY, then the K-slice of dX and dW locally
    const void* dy = dY_shard;
    if (Wn > 1) {
      nccl_ok(nccl().AllGather(dY_shard, g->dy_full, (size_t)g->Mr * N, ncclBfloat16, g->comm, g->comm_st),
              "ncclAllGather(dY)");
      HM_CUDA(cudaEventRecord(g->ev_ag, g->comm_st));
      HM_CUDA(cudaStreamWaitEvent(g->comp, g->ev_ag, 0));
      dy = g->dy_full;
    }
    {  // dX[:, K_r] = dY . W[K_r,:]^T   (A = dY K-major, B = W K-major)
      hk_gemm_args a = gemm_args(1, (int)M, (int)Kr, (int)N);
      a.A = dy; a.a_mn_major = 0; a.lda = N;
      a.B = W; a.b_mn_major = 0; a.ldb = N;
      a.C = dX; a.ldc = Kr;
      a.epilogue = HK_EPI_STORE_T;
      gemm(a, g->comp);
    }
    {  // dW[K_r,:] = X[:,K_r]^T . dY  (A, B MN-major), fp32
      hk_gemm_args a = gemm_args(1, (int)Kr, (int)N, (int)M);
      a.A = X; a.a_mn_major = 1; a.lda = Kr;
      a.B = dy; a.b_mn_major = 1; a.ldb = N;
      a.C = dW; a.ldc = N;
      a.epilogue = HK_EPI_ACC_F32; a.accumulate = 0;
      gemm(a, g->comp);
    }
    if (Wn > 1) {
      HM_CUDA(cudaEventRecord(g->ev_ag, g->comm_st));  // all reduce-scatters done
      HM_CUDA(cudaStreamWaitEvent(g->comp, g->ev_ag, 0));
    }
    HM_CUDA(cudaEventRecord(g->ev1, g->comp));
    HM_CUDA(cudaEventSynchronize(g->ev1));
    float ms = 0.f;
    HM_CUDA(cudaEventElapsedTime(&ms, g->ev0, g->ev1));
    if (seconds) *seconds = ms * 1e-3;
    (void)r;
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
