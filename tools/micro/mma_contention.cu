// mma_contention.cu — microbenchmark: does TMEM-load (or FMA) traffic from other warps slow the
// tcgen05.mma stream of one issuing thread?  Warp 1 lane 0 issues batches of M=128, K=16 UMMAs
// (N = 64 or 128, A from shared memory) with a commit + wait per batch, as the attention kernels
// do; warps 4..11 meanwhile either idle, load TMEM columns the MMAs do not touch (tcgen05.ld
// 32x32b.x32 in a loop), or run an FMA loop.  Prints cycles per UMMA for each combination.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -Iinclude -o /tmp/mma_contention tools/micro/mma_contention.cu
#include <cstdio>
#include <cstdint>

#include "../../paper_conf_hotos_lipmk21_b200/csrc/kernels/tc_common.cuh"

using namespace hm::tcx;

template <int N>
__global__ void __launch_bounds__(384, 1) k(int mode, int batches, int per_batch, long long* cyc, float* sink) {
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ uint32_t tbase;
  __shared__ uint64_t bar;
  __shared__ volatile int done;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tbase)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    done = 0;
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = tbase;
  if (warp == 1) {
    if (lane == 0) {
      const uint32_t idesc = make_idesc_f16(128, N, 0, 0);
      const uint32_t a = smem_u32(smem), b = a + 16384;
      long long t0 = clock64();
      uint32_t ph = 0;
      for (int r = 0; r < batches; ++r) {
        for (int i = 0; i < per_batch; ++i)
          mma_bf16(tm, make_sdesc(a + (i & 3) * 32, 16, 1024), make_sdesc(b + (i & 3) * 32, 16, 1024), idesc, 1u);
        mma_commit(&bar);
        mbar_wait(&bar, ph);
        ph ^= 1;
      }
      cyc[blockIdx.x] = clock64() - t0;
      done = 1;
    }
    __syncwarp();
  } else if (warp >= 4) {
    float acc = 0.f;
    // the other warps' work: TMEM columns 256..511 of their lane quadrant (the MMAs write 0..N-1)
    const uint32_t ta = tm + ((uint32_t)((warp & 3) * 32) << 16) + 256 + ((warp >> 2) - 1) * 64;
    float x = lane * 1e-3f, y = 1.0001f;
    while (!done) {
      if (mode == 1) {
        uint32_t r[32];
        tmem_ld32_nw(ta, r);
        tmem_wait_ld();
#pragma unroll
        for (int i = 0; i < 32; ++i) acc += __uint_as_float(r[i]);
      } else if (mode == 2) {
#pragma unroll
        for (int i = 0; i < 64; ++i) x = fmaf(x, y, 1e-7f);
      } else {
        __nanosleep(100);
      }
    }
    sink[blockIdx.x * 384 + threadIdx.x] = acc + x;
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tm) : "memory");
  }
}

template <int N>
void run(long long* d, float* sink, int mode, int per_batch) {
  const char* names[] = {"idle", "tcgen05.ld", "FMA"};
  const int batches = 400;
  cudaFuncSetAttribute(k<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  k<N><<<148, 384, 65536>>>(mode, 4, per_batch, d, sink);
  k<N><<<148, 384, 65536>>>(mode, batches, per_batch, d, sink);
  cudaError_t e = cudaDeviceSynchronize();
  if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); exit(1); }
  long long h[148];
  cudaMemcpy(h, d, sizeof(h), cudaMemcpyDeviceToHost);
  long long mx = 0;
  for (int i = 0; i < 148; ++i) mx = h[i] > mx ? h[i] : mx;
  printf("N=%3d batch %2d, other warps %-10s: %.1f cycles per UMMA\n", N, per_batch, names[mode],
         (double)mx / batches / per_batch);
}

int main() {
  long long* d;
  float* sink;
  cudaMalloc(&d, 148 * 8);
  cudaMalloc(&sink, 148 * 384 * 4);
  for (int pb : {4, 8, 32})
    for (int mode = 0; mode < 3; ++mode) {
      run<64>(d, sink, mode, pb);
      run<128>(d, sink, mode, pb);
    }
  return 0;
}
