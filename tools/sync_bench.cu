// sync_bench.cu -- cycle cost of the synchronization primitives in the cell kernel's MMA loop
// (one CTA, one warp issuing): mbarrier try_wait on a completed phase, tcgen05 fences,
// tcgen05.commit, tcgen05.mma (128 x N x 16, SS), __syncwarp.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o sync_bench sync_bench.cu
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
__device__ __forceinline__ bool test_wait(uint32_t bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(bar), "r"(par) : "memory");
  return ok;
}

__global__ void bench(unsigned long long* out, int iters, int N) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar[4];
  __shared__ uint32_t tslot;
  const int lane = threadIdx.x;
  if (lane == 0) {
    for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[i])));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&bar[0])) : "memory");  // phase 0 done
  }
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncwarp();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tslot;
  uint64_t d = 0;
  d |= (uint64_t)((su32(sm) >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)64 << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  const uint64_t db = d + ((16384 >> 4));
  const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24);
  unsigned long long t[8];
  // 0: try_wait on a completed phase
  long long c0 = clock64();
  for (int i = 0; i < iters; ++i) while (!try_wait(su32(&bar[0]), 0)) {}
  long long c1 = clock64();
  // 1: test_wait
  for (int i = 0; i < iters; ++i) while (!test_wait(su32(&bar[0]), 0)) {}
  long long c2 = clock64();
  // 2: tcgen05 fence after + syncwarp
  for (int i = 0; i < iters; ++i) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    __syncwarp();
  }
  long long c3 = clock64();
  // 3: commit only (to bar[1])
  for (int i = 0; i < iters; ++i) {
    if (lane == 0) asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar[1])) : "memory");
    __syncwarp();
  }
  long long c4 = clock64();
  // 4: 4 MMAs (128 x N x 16) + commit
  for (int i = 0; i < iters; ++i) {
    if (lane == 0) {
      for (int k = 0; k < 4; ++k)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" ::"r"(tmem),
                     "l"(d + 2 * k), "l"(db + 2 * k), "r"(idesc), "r"(1) : "memory");
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar[1])) : "memory");
    }
    __syncwarp();
  }
  long long c5 = clock64();
  // 5: same and wait for the commit each iteration (MMA round trip latency)
  uint32_t par = 0;
  // drain outstanding commits on bar[2] phases: use a fresh barrier
  for (int i = 0; i < iters; ++i) {
    if (lane == 0) {
      for (int k = 0; k < 4; ++k)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" ::"r"(tmem),
                     "l"(d + 2 * k), "l"(db + 2 * k), "r"(idesc), "r"(1) : "memory");
      asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar[2])) : "memory");
    }
    __syncwarp();
    while (!try_wait(su32(&bar[2]), par)) {}
    par ^= 1;
  }
  long long c6 = clock64();
  if (lane == 0) {
    out[0] = (c1 - c0) / iters;
    out[1] = (c2 - c1) / iters;
    out[2] = (c3 - c2) / iters;
    out[3] = (c4 - c3) / iters;
    out[4] = (c5 - c4) / iters;
    out[5] = (c6 - c5) / iters;
  }
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem));
}

// The cell kernel's MMA-issuer loop in context: warp 8 waits on pre-completed stage barriers,
// commits, and (optionally) issues MMAs, while warps 0-7 poll another mbarrier (mode 1: all
// lanes poll, mode 2: lane 0 polls, mode 0: warps 0-7 sit in bar.sync).
__global__ void bench_ctx(unsigned long long* out, int iters, int mode, int do_mma) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t full[8], done, sink;
  __shared__ uint32_t tslot;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < 8; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[i])));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&done)));
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&sink)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    for (int i = 0; i < 8; ++i) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[i])) : "memory");
  }
  if (warp == 8) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tslot;
  if (warp == 8) {
    uint64_t d = 0;
    d |= (uint64_t)((su32(sm) >> 4) & 0x3FFF);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)64 << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(64 >> 3) << 17) | (8u << 24);
    long long c0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const int s = i & 7;
      if (lane == 0) while (!try_wait(su32(&full[s]), 0)) {}
      __syncwarp();
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      if (lane == 0) {
        if (do_mma)
          for (int k = 0; k < 4; ++k)
            asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}" ::"r"(tmem),
                         "l"(d + 2 * k), "l"(d + 1024 + 2 * k), "r"(idesc), "r"(1) : "memory");
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&sink)) : "memory");
      }
      __syncwarp();
    }
    long long c1 = clock64();
    if (lane == 0) {
      out[0] = (c1 - c0) / iters;
      asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&done)) : "memory");
    }
  } else if (warp < 8) {
    if (mode == 1) while (!try_wait(su32(&done), 0)) {}
    else if (mode == 2) { if (lane == 0) while (!try_wait(su32(&done), 0)) {} __syncwarp(); }
  }
  __syncthreads();
  if (warp == 8) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem));
}

int main() {
  {
    unsigned long long* d;
    cudaMalloc(&d, 64);
    cudaFuncSetAttribute(bench_ctx, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    for (int mma = 0; mma < 2; ++mma)
      for (int mode = 0; mode < 3; ++mode) {
        bench_ctx<<<1, 320, 64 * 1024>>>(d, 64, mode, mma);
        unsigned long long h = 0;
        cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
        printf("ctx: mma=%d pollers=%s  cycles/iter %llu (%s)\n", mma, mode == 0 ? "none(bar.sync)" : mode == 1 ? "all lanes" : "lane 0",
               h, cudaGetErrorString(cudaGetLastError()));
      }
  }
  unsigned long long* d;
  cudaMalloc(&d, 64);
  cudaFuncSetAttribute(bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
  for (int N : {16, 64, 256}) {
    bench<<<1, 32, 64 * 1024>>>(d, 1000, N);
    unsigned long long h[6];
    cudaMemcpy(h, d, 48, cudaMemcpyDeviceToHost);
    printf("N=%3d cycles/iter: try_wait(done) %llu | test_wait %llu | tc fence+syncwarp %llu | commit %llu | 4 mma + commit %llu | 4 mma + commit + wait %llu  (%s)\n",
           N, h[0], h[1], h[2], h[3], h[4], h[5], cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
