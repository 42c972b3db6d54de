// ingest_bench.cu -- how fast can N CTAs stream bytes from global memory into shared memory
// with cp.async.bulk (the weight stream of the cell kernel)? Each CTA streams `per_cta` bytes
// in `chunk`-byte bulk copies with `stages` copies in flight (mbarrier ring). Reports GB/s.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o ingest_bench ingest_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// mode 1: 256 threads, cp.async 16 B chunks into a smem ring of `stages` x chunk bytes
// mode 2: 256 threads, ld.global 16 B (v4) into registers, summed
__global__ void ingest_threads(const uint8_t* src, size_t per_cta, int chunk, int stages, int mode,
                               unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  const uint8_t* base = src + (size_t)blockIdx.x * per_cta;
  const int n16 = (int)(per_cta / 16);
  unsigned long long acc = 0;
  if (mode == 1) {
    const int ring16 = chunk * stages / 16;
    int g = 0;
    for (int i = threadIdx.x; i < n16; i += blockDim.x, ++g) {
      const uint32_t dst = (uint32_t)__cvta_generic_to_shared(sm + (size_t)(i % ring16) * 16);
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(base + (size_t)i * 16) : "memory");
      if ((g & 7) == 7) {
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 4;" ::: "memory");
      }
    }
    asm volatile("cp.async.commit_group;\n cp.async.wait_group 0;" ::: "memory");
    acc = sm[threadIdx.x];
  } else {
    const int4* p4 = reinterpret_cast<const int4*>(base);
#pragma unroll 8
    for (int i = threadIdx.x; i < n16; i += blockDim.x) {
      int4 v;
      asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p4 + i));
      acc += v.x ^ v.w;
    }
  }
  if (acc == 0x12345) sink[blockIdx.x] = acc;
}

__global__ void ingest(const uint8_t* src, size_t per_cta, int chunk, int stages, int reuse_mod,
                       unsigned long long* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bars[16];
  const int n_chunks = (int)(per_cta / chunk);
  const uint8_t* base = src + (size_t)(blockIdx.x % reuse_mod) * per_cta;
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bars[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long acc = 0;
    for (int i = 0; i < n_chunks + stages; ++i) {
      if (i >= stages) {  // consume chunk i - stages
        const int s = (i - stages) % stages;
        const uint32_t par = ((i - stages) / stages) & 1;
        uint32_t ok = 0;
        while (!ok) {
          asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
                       : "=r"(ok) : "r"(su32(&bars[s])), "r"(par) : "memory");
        }
        acc += sm[s * chunk];
      }
      if (i < n_chunks) {
        const int s = i % stages;
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bars[s])), "r"(chunk) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(su32(sm + s * chunk)), "l"(base + (size_t)i * chunk), "r"(chunk), "r"(su32(&bars[s])) : "memory");
      }
    }
    sink[blockIdx.x] = acc;
  }
}

int main(int argc, char** argv) {
  const int ctas = argc > 1 ? atoi(argv[1]) : 128;
  const size_t per_cta = argc > 2 ? atol(argv[2]) : 131072;
  const int chunk = argc > 3 ? atoi(argv[3]) : 16384;
  const int stages = argc > 4 ? atoi(argv[4]) : 4;
  const int l2_resident = argc > 5 ? atoi(argv[5]) : 1;  // 1: same bytes every launch
  const int mode = argc > 6 ? atoi(argv[6]) : 0;          // 0 bulk, 1 cp.async, 2 ldg
  const int share = argc > 7 ? atoi(argv[7]) : 1 << 30;   // CTAs i and i+share.. read the same bytes
  const size_t total = per_cta * ctas;
  const size_t buf_bytes = l2_resident ? total : (size_t)2 << 30;
  uint8_t* src;
  cudaMalloc(&src, buf_bytes);
  cudaMemset(src, 1, buf_bytes);
  unsigned long long* sink;
  cudaMalloc(&sink, 8 * 4096);
  const int smem = chunk * stages;
  cudaFuncSetAttribute(ingest, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(ingest_threads, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int iters = 50;
  float best = 1e9;
  for (int rep = 0; rep < 3; ++rep) {
    cudaEventRecord(a);
    for (int it = 0; it < iters; ++it) {
      const uint8_t* s = l2_resident ? src : src + ((size_t)it * total) % (buf_bytes - total);
      if (mode == 0) ingest<<<ctas, 32, smem>>>(s, per_cta, chunk, stages, share, sink);
      else ingest_threads<<<ctas, 256, smem>>>(s, per_cta, chunk, stages, mode, sink);
    }
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (ms < best) best = ms;
  }
  const double us = best * 1e3 / iters;
  printf("{\"share\": %d, \"mode\": %d, \"ctas\": %d, \"per_cta\": %zu, \"chunk\": %d, \"stages\": %d, \"l2\": %d, \"us\": %.2f, \"GBps\": %.1f, \"err\": \"%s\"}\n",
         share, mode, ctas, per_cta, chunk, stages, l2_resident, us, total / us / 1e3, cudaGetErrorString(cudaGetLastError()));
  return 0;
}
