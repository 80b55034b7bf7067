// Per-launch cost of back-to-back kernels in a CUDA graph on B200: empty kernel vs the GEMM's
// launch shape (148 CTAs x 320 threads, clusters of 2, ~200 KB dynamic smem, TMEM alloc/dealloc).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o /tmp/lo tools/micro/launch_overhead.cu && /tmp/lo
#include <cstdio>
#include <cuda_runtime.h>

__global__ void k_empty() {}
__global__ void k_smem() {
  extern __shared__ char s[];
  if (threadIdx.x == 9999) s[0] = 0;
}
__global__ void __cluster_dims__(2, 1, 1) k_cluster() {
  extern __shared__ char s[];
  if (threadIdx.x == 9999) s[0] = 0;
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
__global__ void __cluster_dims__(2, 1, 1) k_tmem() {
  extern __shared__ __align__(16) char s[];
  __shared__ unsigned base;
  if (threadIdx.x / 32 == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
                     (unsigned)__cvta_generic_to_shared(&base))
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (threadIdx.x / 32 == 1)
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(base) : "memory");
  if (threadIdx.x == 9999) s[0] = 0;
}

// the GEMM's launch shape doing ~spin cycles of "work"; PDL variant: prologue (TMEM alloc, barriers)
// before griddepcontrol.wait, dependents released once every CTA has started
template <bool PDL>
__global__ void __cluster_dims__(2, 1, 1) k_work(long long spin) {
  extern __shared__ __align__(16) char s[];
  __shared__ unsigned base;
  if (threadIdx.x / 32 == 1) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
                     (unsigned)__cvta_generic_to_shared(&base))
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (PDL) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    asm volatile("griddepcontrol.launch_dependents;" :::);
  }
  long long t0 = clock64();
  while (clock64() - t0 < spin) {
  }
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (threadIdx.x / 32 == 1)
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(base) : "memory");
  if (threadIdx.x == 9999) s[0] = 0;
}

template <bool PDL>
void launch_work(cudaStream_t st, int smem, long long spin) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(148);
  cfg.blockDim = dim3(320);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = PDL ? 1 : 0;
  cudaLaunchKernelEx(&cfg, k_work<PDL>, spin);
}

template <typename F>
float time_graph(F launch, int reps) {
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaGraph_t g;
  cudaGraphExec_t ge;
  cudaStreamBeginCapture(st, cudaStreamCaptureModeGlobal);
  for (int i = 0; i < reps; ++i) launch(st);
  cudaStreamEndCapture(st, &g);
  cudaGraphInstantiate(&ge, g, 0);
  cudaGraphLaunch(ge, st);
  cudaStreamSynchronize(st);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0, st);
  cudaGraphLaunch(ge, st);
  cudaEventRecord(e1, st);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  return ms * 1e3f / reps;
}

int main() {
  const int smem = 200 * 1024, reps = 200;
  cudaFuncSetAttribute(k_smem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_cluster, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_tmem, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  printf("empty 148x32          %.2f us\n", time_graph([](cudaStream_t s) { k_empty<<<148, 32, 0, s>>>(); }, reps));
  printf("empty 148x320         %.2f us\n", time_graph([](cudaStream_t s) { k_empty<<<148, 320, 0, s>>>(); }, reps));
  printf("smem200K 148x320      %.2f us\n",
         time_graph([&](cudaStream_t s) { k_smem<<<148, 320, smem, s>>>(); }, reps));
  printf("cluster2 smem200K     %.2f us\n",
         time_graph([&](cudaStream_t s) { k_cluster<<<148, 320, smem, s>>>(); }, reps));
  printf("cluster2 smem200K tmem %.2f us\n",
         time_graph([&](cudaStream_t s) { k_tmem<<<148, 320, smem, s>>>(); }, reps));
  cudaFuncSetAttribute(k_work<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k_work<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  for (long long spin : {0LL, 4000LL, 20000LL}) {
    printf("work spin=%lld plain   %.2f us\n", spin, time_graph([&](cudaStream_t s) { launch_work<false>(s, smem, spin); }, reps));
    printf("work spin=%lld PDL     %.2f us\n", spin, time_graph([&](cudaStream_t s) { launch_work<true>(s, smem, spin); }, reps));
  }
  cudaError_t e = cudaGetLastError();
  printf("err %s\n", cudaGetErrorString(e));
  return 0;
}
