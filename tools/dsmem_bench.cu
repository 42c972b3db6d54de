// dsmem_bench.cu -- split-K partial exchange inside a cluster of S CTAs (one per SM):
// mode 0: every thread pulls its slice with ld.shared::cluster.v4 (the cell kernel's reduction);
// mode 1: one thread per CTA pushes the (S-1) slices with cp.async.bulk shared::cta ->
//         shared::cluster (TMA engine), completion on the receiver's mbarrier (complete_tx).
// Reports median cycles per CTA for moving `slice` bytes to each of the S-1 peers.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o dsmem_bench dsmem_bench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <algorithm>
#include <vector>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t mapa(uint32_t a, uint32_t r) {
  uint32_t o;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"(a), "r"(r));
  return o;
}
__device__ __forceinline__ uint32_t crank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void csync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

__global__ void __launch_bounds__(320, 1) kern(int S, int slice, int mode, long long* out, float* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t rxbar;
  const int tid = threadIdx.x;
  const uint32_t me = crank();
  uint8_t* src = sm;                           // S slices of `slice` bytes (slice s -> rank s)
  uint8_t* rx = sm + S * slice;                // S-1 receive slots
  for (int i = tid * 4; i < S * slice; i += 320 * 4) *(float*)(src + i) = (float)(i + me);
  if (tid == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&rxbar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  float acc = 0.f;
  long long best = 0;
  for (int rep = 0; rep < 8; ++rep) {
    if (tid == 0 && mode == 1)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&rxbar)), "r"((S - 1) * slice) : "memory");
    csync();
    const long long t0 = clock64();
    if (mode == 0) {
      // pull: my slice from each peer's src (as the kernel reduces its column slice)
      for (int s = 0; s < S; ++s) {
        if (s == (int)me) continue;
        const uint32_t base = mapa(su32(src + me * slice), s);
        for (int i = tid * 16; i < slice; i += 320 * 16) {
          float4 v;
          asm volatile("ld.shared::cluster.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(base + i));
          acc += v.x + v.y + v.z + v.w;
        }
      }
      __syncthreads();
    } else {
      if (tid == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        for (int s = 0; s < S; ++s) {
          if (s == (int)me) continue;
          const int slot = (int)me < s ? me : me - 1;   // my slot in the receiver's rx area
          const uint32_t dst = mapa(su32(rx + slot * slice), s);
          const uint32_t bar = mapa(su32(&rxbar), s);
          asm volatile("cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
                       "r"(su32(src + s * slice)), "r"(slice), "r"(bar) : "memory");
        }
      }
      if (tid == 0) {
        uint32_t ok = 0;
        while (!ok)
          asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                       : "=r"(ok) : "r"(su32(&rxbar)), "r"(rep & 1) : "memory");
      }
      __syncthreads();
      acc += *(float*)(rx + tid * 4);
    }
    const long long t1 = clock64();
    if (rep >= 2) best += t1 - t0;
    csync();
  }
  if (tid == 0) out[blockIdx.x] = best / 6;
  if (acc == 1234.5f) sink[0] = acc;
}

int main() {
  long long* d;
  float* sink;
  cudaMalloc(&d, 1024 * 8);
  cudaMalloc(&sink, 4);
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int S : {2, 4}) {
    for (int slice : {16384, 32768}) {
      for (int mode : {0, 1}) {
        const int grid = (148 / S) * S;
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(grid);
        cfg.blockDim = dim3(320);
        cfg.dynamicSmemBytes = 2 * S * slice > 200 * 1024 ? 200 * 1024 : 2 * S * slice;
        cudaLaunchAttribute at[1];
        at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = S;
        at[0].val.clusterDim.y = 1;
        at[0].val.clusterDim.z = 1;
        cfg.attrs = at;
        cfg.numAttrs = 1;
        if (2 * S * slice > 200 * 1024) continue;
        cudaError_t e = cudaLaunchKernelEx(&cfg, kern, S, slice, mode, d, sink);
        if (e == cudaSuccess) e = cudaDeviceSynchronize();
        if (e != cudaSuccess) { printf("S %d slice %d mode %d: %s\n", S, slice, mode, cudaGetErrorString(e)); return 1; }
        std::vector<long long> o(grid);
        cudaMemcpy(o.data(), d, grid * 8, cudaMemcpyDeviceToHost);
        std::sort(o.begin(), o.end());
        const double med = o[grid / 2];
        printf("S %d slice %6d mode %-5s: median %7.0f cyc per CTA for %d KB in -> %.1f B/cyc\n", S, slice,
               mode ? "push" : "pull", med, (S - 1) * slice / 1024, (S - 1) * slice / med);
      }
    }
  }
  return 0;
}
