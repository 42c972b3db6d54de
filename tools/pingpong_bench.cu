// pingpong_bench.cu -- base latencies of mbarrier hand-offs on B200.
//  test 0: one thread, arrive + try_wait on its own count-1 barrier, repeated
//  test 1: two warps ping-pong through two count-1 barriers (round trip)
//  test 2: like 1 but the pinger only arrives, the ponger drains a ring of 4 (throughput)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pingpong_bench pingpong_bench.cu
#include <cstdio>
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ bool try_wait(uint32_t bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(bar), "r"(par) : "memory");
  return ok;
}
__device__ __forceinline__ bool test_wait_(uint32_t bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(bar), "r"(par) : "memory");
  return ok;
}
__device__ __forceinline__ void arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void arrive_relaxed(uint32_t bar) {
  asm volatile("mbarrier.arrive.relaxed.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

__global__ void pp(int test, int iters, int relaxed, long long* out, int park) {
  __shared__ uint64_t b[8];
  __shared__ uint64_t endb;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    for (int i = 0; i < 8; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&b[i])));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&endb)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  long long t0 = clock64();
  if (test == 0) {
    if (tid == 0) {
      for (int i = 0; i < iters; ++i) {
        if (relaxed) arrive_relaxed(su32(&b[0])); else arrive(su32(&b[0]));
        while (!try_wait(su32(&b[0]), i & 1)) {}
      }
      out[blockIdx.x] = (clock64() - t0) / iters;
    }
  } else if (test == 1) {
    if (lane == 0 && warp == 0) {
      for (int i = 0; i < iters; ++i) {
        if (relaxed) arrive_relaxed(su32(&b[0])); else arrive(su32(&b[0]));
        while (!try_wait(su32(&b[1]), i & 1)) {}
      }
      out[blockIdx.x] = (clock64() - t0) / iters;
    } else if (lane == 0 && warp == 1) {
      for (int i = 0; i < iters; ++i) {
        while (!try_wait(su32(&b[0]), i & 1)) {}
        if (relaxed) arrive_relaxed(su32(&b[1])); else arrive(su32(&b[1]));
      }
    }
  } else {
    // ring of 4 full/empty pairs: b[0..3] full, b[4..7] empty
    if (lane == 0 && warp == 0) {
      for (int i = 0; i < iters; ++i) {
        const int s = i & 3, r = i >> 2;
        if (r > 0) while (!try_wait(su32(&b[4 + s]), (r - 1) & 1)) {}
        if (relaxed) arrive_relaxed(su32(&b[s])); else arrive(su32(&b[s]));
      }
    } else if (lane == 0 && warp == 1) {
      for (int i = 0; i < iters; ++i) {
        const int s = i & 3, r = i >> 2;
        while (!try_wait(su32(&b[s]), r & 1)) {}
        if (relaxed) arrive_relaxed(su32(&b[4 + s])); else arrive(su32(&b[4 + s]));
      }
      out[blockIdx.x] = (clock64() - t0) / iters;
    }
  }
  if (park >= 3 && warp == 1 && lane == 0) arrive(su32(&endb));
  if (park == 3 && warp >= 1) while (!try_wait(su32(&endb), 0)) {}
  if (park == 4 && warp >= 1) { if (lane == 0) while (!try_wait(su32(&endb), 0)) {} __syncwarp(); }
  if (park == 5 && warp >= 1) while (!test_wait_(su32(&endb), 0)) { __nanosleep(200); }
  if (park == 1) __syncthreads();
  if (park == 2) asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

int main() {
  long long* out;
  cudaMalloc(&out, 148 * 8);
  cudaFuncSetAttribute(pp, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int test = 1; test < 3; ++test)
    for (int cfg = 1; cfg < 24; cfg += 4)
      for (int grid : {148}) {
        const int relaxed = 0;
        const int thr = (cfg & 1) ? 320 : 64;
        const int sm = (cfg & 2) ? 200 * 1024 : 0;
        const int park = cfg >> 2;
        printf("threads %d dyn smem %d park %d: ", thr, sm, park);
        pp<<<grid, thr, sm>>>(test, 1000, relaxed, out, park);
        cudaDeviceSynchronize();
        pp<<<grid, thr, sm>>>(test, 1000, relaxed, out, park);
        cudaError_t e = cudaDeviceSynchronize();
        long long o[148];
        cudaMemcpy(o, out, grid * 8, cudaMemcpyDeviceToHost);
        printf("test %d relaxed %d grid %3d: %lld cycles/iter  (%s)\n", test, relaxed, grid, o[0],
               cudaGetErrorString(e));
      }
  return 0;
}
