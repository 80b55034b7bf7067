// collective.cu — the library's own collectives for the single-process "one virtual device" mode
// (harmony_init_group; SURVEY §8(b) primary mode, rows a11 / a14).
//
// Every rank's arena is directly addressable from every rank's device: ranks that share a GPU
// (the loopback used to test N > 1 on one B200) address the same HBM, ranks on different GPUs
// read their peers' HBM over NVLink / NVSwitch (cudaDeviceEnablePeerAccess at group init).  So the
// collectives are plain pulls, issued on the receiving rank's stream:
//   reduce-scatter: rank r sums its shard of every rank's fp32 dW, ranks in
//     order 0..N-1 (one fixed summation order: the result is deterministic and identical whether
//     the ranks share a GPU or not);
//   all-gather (weights, loss partials): rank r copies shard q out of rank q's buffer
//     (cudaMemcpyAsync, a copy-engine transfer over NVLink between GPUs).
#include "../common.hpp"
#include "kernels.hpp"

namespace hm {

struct RankPtrs {
  const float* p[HM_MAX_GROUP];
};

// dst[k] = (((src_0[k] + src_1[k]) + src_2[k]) + ...) for k < n, float4-vectorised (n4 = n / 4)
__global__ void __launch_bounds__(256) rank_sum_kernel(int nsrc, int64_t n4, RankPtrs src, float4* __restrict__ dst) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += (int64_t)gridDim.x * blockDim.x) {
    float4 a = reinterpret_cast<const float4*>(src.p[0])[i];
    for (int q = 1; q < nsrc; ++q) {
      const float4 b = reinterpret_cast<const float4*>(src.p[q])[i];
      a.x += b.x; a.y += b.y; a.z += b.z; a.w += b.w;
    }
    dst[i] = a;
  }
}

__global__ void rank_sum_tail_kernel(int nsrc, int64_t lo, int64_t n, RankPtrs src, float* __restrict__ dst) {
  pdl_wait();  // programmatic dependent launch: the previous kernel's results are visible
  const int64_t i = lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  float a = src.p[0][i];
  for (int q = 1; q < nsrc; ++q) a += src.p[q][i];
  dst[i] = a;
}

void rank_sum(int nsrc, const float* const* src, int64_t n, float* dst, cudaStream_t st) {
  HM_CHECK(nsrc >= 1 && nsrc <= HM_MAX_GROUP, HARMONY_E_INVALID_ARG, "rank_sum: bad source count");
  RankPtrs rp{};
  bool aligned = (reinterpret_cast<uintptr_t>(dst) & 15) == 0;
  for (int q = 0; q < nsrc; ++q) {
    rp.p[q] = src[q];
    aligned = aligned && (reinterpret_cast<uintptr_t>(src[q]) & 15) == 0;
  }
  int64_t n4 = aligned ? n / 4 : 0;
  if (n4 > 0) {
    const int grid = (int)std::min<int64_t>(ceil_div(n4, 256), 148 * 8);
    launch_k(rank_sum_kernel, dim3(grid), dim3(256), 0, st, nsrc, n4, rp, reinterpret_cast<float4*>(dst));
    check_launch("rank_sum_kernel");
  }
  const int64_t lo = n4 * 4;
  if (lo < n) {
    launch_k(rank_sum_tail_kernel, dim3((int)ceil_div(n - lo, 256)), dim3(256), 0, st, nsrc, lo, n, rp, dst);
    check_launch("rank_sum_tail_kernel");
  }
}

}  // namespace hm
