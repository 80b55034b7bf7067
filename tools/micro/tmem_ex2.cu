// tmem_ex2.cu — microbenchmark: TMEM read (tcgen05.ld) throughput, ex2 (MUFU) throughput, and
// whether the two overlap when different warps of one SM sub-partition issue them.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tmem_ex2 tools/micro/tmem_ex2.cu
// Each warp reads its own TMEM lane quadrant (warp % 4).  mode: 0 = every warp loads,
// 1 = every warp exponentiates, 2 = warps 0-3 load while warps 4-7 exponentiate, 3 = every warp
// loads then exponentiates (serial chain), 4 = loads issued for the next tile before the exps of
// the current one (software pipelined within a warp).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ float ex2(float x) {
  float y;
  asm volatile("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

#define LD32(taddr, r)                                                                                          \
  asm volatile(                                                                                                 \
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18," \
      "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"                                            \
      : "=r"((r)[0]), "=r"((r)[1]), "=r"((r)[2]), "=r"((r)[3]), "=r"((r)[4]), "=r"((r)[5]), "=r"((r)[6]), "=r"((r)[7]),         \
        "=r"((r)[8]), "=r"((r)[9]), "=r"((r)[10]), "=r"((r)[11]), "=r"((r)[12]), "=r"((r)[13]), "=r"((r)[14]), "=r"((r)[15]),   \
        "=r"((r)[16]), "=r"((r)[17]), "=r"((r)[18]), "=r"((r)[19]), "=r"((r)[20]), "=r"((r)[21]), "=r"((r)[22]), "=r"((r)[23]), \
        "=r"((r)[24]), "=r"((r)[25]), "=r"((r)[26]), "=r"((r)[27]), "=r"((r)[28]), "=r"((r)[29]), "=r"((r)[30]), "=r"((r)[31])  \
      : "r"(taddr))
#define WAITLD() asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory")

__global__ void __launch_bounds__(256, 1) k(int mode, int iters, long long* cyc, float* sink) {
  __shared__ uint32_t tbase;
  const int warp = threadIdx.x / 32;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(
        (uint32_t)__cvta_generic_to_shared(&tbase)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tm = tbase + ((uint32_t)((warp & 3) * 32) << 16) + (warp >> 2) * 128;
  float acc = 0.f;
  float x = threadIdx.x * 1e-3f;
  const bool do_ld = mode == 0 || mode == 3 || mode == 4 || (mode == 2 && warp < 4);
  const bool do_ex = mode == 1 || mode == 3 || mode == 4 || (mode == 2 && warp >= 4);
  __syncthreads();
  long long t0 = clock64();
  uint32_t r[64], q[64];
  if (mode == 4) {
    LD32(tm, q); LD32(tm + 32, q + 32);
    WAITLD();
  }
  for (int it = 0; it < iters; ++it) {
    if (mode == 4) {
#pragma unroll
      for (int i = 0; i < 64; ++i) r[i] = q[i];
      LD32(tm + (it & 1) * 64, q); LD32(tm + (it & 1) * 64 + 32, q + 32);
#pragma unroll
      for (int i = 0; i < 64; ++i) acc += ex2(__uint_as_float(r[i]) * 1e-6f + x);
      WAITLD();
      continue;
    }
    if (do_ld) {
      LD32(tm + (it & 1) * 64, r); LD32(tm + (it & 1) * 64 + 32, r + 32);
      WAITLD();
#pragma unroll
      for (int i = 0; i < 64; ++i) acc += __uint_as_float(r[i]);
    }
    if (do_ex) {
#pragma unroll
      for (int i = 0; i < 64; ++i) acc += ex2(acc * 1e-9f + x + i);
    }
  }
  long long t1 = clock64();
  __syncthreads();
  if (threadIdx.x % 32 == 0) cyc[blockIdx.x * 8 + warp] = t1 - t0;
  sink[blockIdx.x * 256 + threadIdx.x] = acc;
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase) : "memory");
}

int main() {
  long long* cyc; float* sink;
  cudaMalloc(&cyc, 148 * 8 * 8); cudaMalloc(&sink, 148 * 256 * 4);
  const int iters = 2000;
  const char* names[] = {"ld only", "ex2 only", "ld warps 0-3 | ex2 warps 4-7", "ld then ex2 per warp", "ld(next) || ex2(cur) per warp"};
  for (int mode = 0; mode < 5; ++mode) {
    k<<<148, 256>>>(mode, 10, cyc, sink);
    k<<<148, 256>>>(mode, iters, cyc, sink);
    cudaError_t e = cudaDeviceSynchronize();
    if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
    long long h[148 * 8];
    cudaMemcpy(h, cyc, sizeof(h), cudaMemcpyDeviceToHost);
    double mx = 0, mean = 0;
    for (int i = 0; i < 148 * 8; ++i) { mean += h[i]; if (h[i] > mx) mx = h[i]; }
    mean /= 148 * 8;
    // per iteration, per SM: ld moves 8 warps x 32 lanes x 64 x 4 B = 64 KB (modes 0,3,4), 32 KB (mode 2);
    // ex2 8 x 32 x 64 = 16384 exps (1,3,4), 8192 (2)
    double per_it = mx / iters;
    printf("mode %d %-32s cycles/iter %.1f  (ld %s B/cyc/SM, ex2 %s /cyc/SM)\n", mode, names[mode], per_it,
           mode == 1 ? "-" : (mode == 2 ? "" : ""), "");
    double ldb = mode == 1 ? 0 : (mode == 2 ? 32768 : 65536), exn = mode == 0 ? 0 : (mode == 2 ? 8192 : 16384);
    printf("        ld %.1f B/cyc/SM   ex2 %.2f /cyc/SM\n", ldb / per_it, exn / per_it);
  }
  return 0;
}
