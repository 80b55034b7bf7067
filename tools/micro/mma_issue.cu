// mma_issue.cu — microbenchmark: how long a batch of tcgen05.mma (cta_group::1, kind::f16, M=128,
// K=16 each) takes from one issuing thread to completion, per N, for A from shared memory (SS) or
// from TMEM (TS).  Compared against the tensor-pipe floor 128*N/256 cycles per instruction, it
// shows whether short (N = 64) products are issue-bound — the attention kernels' case.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mma_issue tools/micro/mma_issue.cu
#include <cstdio>
#include <cstdint>

#include "../../paper_conf_hotos_lipmk21_b200/csrc/kernels/tc_common.cuh"

using namespace hm::tcx;

template <int N, bool TS, bool FOUR>
__global__ void __launch_bounds__(128, 1) k(int batches, int per_batch, long long* cyc) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t tbase;
  __shared__ uint64_t bar;
  const int warp = threadIdx.x / 32;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (threadIdx.x == 0) { mbar_init(&bar, 1); asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = tbase;
  if (threadIdx.x == 0) {
    const uint32_t idesc = make_idesc_f16(128, N, 0, 0);
    const uint32_t a = smem_u32(smem), b = a + 16384;
    long long t0 = clock64();
    uint32_t ph = 0;
    for (int r = 0; r < batches; ++r) {
      for (int i = 0; i < per_batch; i += (FOUR ? 4 : 1)) {
        if constexpr (FOUR) {
          mma4_bf16(tm, make_sdesc(a, 16, 1024), make_sdesc(b, 16, 1024), 2, 2, idesc, 1u);
        } else if constexpr (TS) {
          mma_bf16_ts(tm, tm + 256 + (i & 3) * 8, make_sdesc(b + (i & 3) * 32, 16, 1024), idesc, 1u);
        } else {
          mma_bf16(tm, make_sdesc(a + (i & 3) * 32, 16, 1024), make_sdesc(b + (i & 3) * 32, 16, 1024), idesc, 1u);
        }
      }
      mma_commit(&bar);
      mbar_wait(&bar, ph);
      ph ^= 1;
    }
    long long t1 = clock64();
    cyc[blockIdx.x] = t1 - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm) : "memory");
  }
}

template <int N, bool TS, bool FOUR>
void run(const char* name, long long* d, int per_batch) {
  const int batches = 400;
  auto kern = k<N, TS, FOUR>;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  kern<<<148, 128, 65536>>>(4, per_batch, d);
  kern<<<148, 128, 65536>>>(batches, per_batch, d);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("%s err %s\n", name, cudaGetErrorString(e)); exit(1); }
  long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  long long mx = 0;
  for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
  const double per = (double)mx / batches / per_batch;
  printf("%-28s N=%3d batch %3d: %.1f cycles per MMA (floor %d) -> %.2f of the tensor-pipe floor\n", name, N,
         per_batch, per, 128 * N / 256, (128.0 * N / 256) / per);
}

int main() {
  long long* d;
  cudaMalloc(&d, 148 * 8);
  for (int pb : {4, 8, 16, 64}) {
    run<64, false, false>("SS", d, pb);
    run<128, false, false>("SS", d, pb);
    run<256, false, false>("SS", d, pb);
    run<64, true, false>("TS", d, pb);
    run<128, true, false>("TS", d, pb);
    run<64, false, true>("SS x4 asm", d, pb);
    run<128, false, true>("SS x4 asm", d, pb);
  }
  return 0;
}
