// stream_bench.cu -- how many bytes per SM per cycle can B200 move from L2/HBM into shared
// memory, measured INSIDE one long-running kernel (no launch overhead in the number)?
//
// Every CTA (one per SM) streams `per_cta` bytes through a ring of `depth` slots of `chunk`
// bytes, a single thread issuing the copies and re-arming the slots as they land (the
// weight-stream pattern of the cell kernels). Modes:
//   0  cp.async.bulk (1-D TMA bulk copy), one issuing thread
//   1  cp.async 16 B by 256 threads into the same ring (LSU path), one commit group per slot
//   2  cp.async.bulk ... .multicast::cluster: a cluster of `csz` CTAs, CTA r copies slice r of
//      every chunk to ALL CTAs of the cluster (each SM receives the full chunk; L2 serves it once
//      per cluster)
//   3  cp.async.bulk.tensor.2d tile loads (tensor map: bf16 rows of 64 elements = 128 B, 128B
//      swizzle), one instruction per chunk (box = chunk / 128 rows, <= 256)
//   4  cp.async.bulk.tensor.2d.tile::gather4: 4 random rows x 128 B per instruction, chunk / 512
//      instructions per slot (the activation gather by slot)
//   5  mode 0 with `csz` issuing warps, each with its own ring of `depth` slots
// src: `footprint` bytes, read cyclically (footprint <= L2: L2-resident; >> L2: HBM).
// Output: one JSON line, GB/s received per SM and chip-wide, and B/cycle/SM at the measured SM
// clock (clock64 / globaltimer inside the kernel).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o stream_bench stream_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ unsigned long long gt() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ bool try_wait(uint32_t bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(bar), "r"(par) : "memory");
  return ok;
}
__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

struct Args {
  CUtensorMap tmap;
  const uint8_t* src;
  size_t footprint;
  size_t per_cta;
  int chunk, depth, mode, csz;
  unsigned long long* out;   // [grid][3]: t0, t1, clock cycles
};

__global__ void stream_kernel(const __grid_constant__ Args a) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t full[64], empty[64];
  const int tid = threadIdx.x;
  const uint32_t rank = a.mode == 2 ? cluster_rank() : 0;
  const int csz = a.mode == 2 ? a.csz : 1;   // mode 5: a.csz = issuing warps
  const size_t n_chunks = a.per_cta / a.chunk;
  // each cluster (or CTA) starts at its own offset in the footprint
  const size_t cluster_id = blockIdx.x / csz;
  size_t off = (cluster_id * 7919ull * a.chunk) % a.footprint;
  if (tid == 0) {
    for (int s = 0; s < a.depth * (a.mode == 5 || a.mode == 7 || a.mode == 8 ? a.csz : 1); ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&full[s])),
                   "r"(a.mode == 1 || a.mode == 6 ? 256 : a.mode == 7 ? 256 / a.csz : 1));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(csz));
    }
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (a.mode == 2) asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  const unsigned long long t0 = gt();
  const long long c0 = clock64();
  if (a.mode == 7) {
    // cp.async in G = csz independent groups of 256/G threads; group g streams chunks
    // i = g, g + G, ... through its own `depth` slots (arrive.noinc, as mode 1)
    const int G = a.csz;
    const int gsz = 256 / G;
    const int g = tid / gsz, gt = tid % gsz;
    const size_t mine = (n_chunks + G - 1 - g) / G;
    for (size_t i = 0; i < mine; ++i) {
      const int s = g * a.depth + i % a.depth;
      if (i >= (size_t)a.depth) {
        if ((tid & 31) == 0) while (!try_wait(su32(&full[s]), ((i / a.depth) - 1) & 1)) {}
        __syncwarp();
      }
      const uint8_t* src = a.src + (off + (i * G + g) * a.chunk) % a.footprint;
      for (int k = gt; k < a.chunk / 16; k += gsz)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(sm + s * a.chunk + k * 16)),
                     "l"(src + k * 16) : "memory");
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
    }
    for (int d = 0; d < a.depth && (size_t)d < mine; ++d) {
      const size_t last = ((mine - 1 - d) / a.depth) * a.depth + d;
      if ((tid & 31) == 0) while (!try_wait(su32(&full[g * a.depth + d]), (last / a.depth) & 1)) {}
    }
  } else if (a.mode == 6) {
    // cp.async with commit groups: each thread keeps depth - 1 groups in flight
    // (cp.async.wait_group), then a plain arrive on the oldest slot's barrier
    for (size_t i = 0; i < n_chunks; ++i) {
      const int s = i % a.depth;
      const uint8_t* src = a.src + (off + i * a.chunk) % a.footprint;
      for (int k = tid; k < a.chunk / 16; k += blockDim.x)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(sm + s * a.chunk + k * 16)),
                     "l"(src + k * 16) : "memory");
      asm volatile("cp.async.commit_group;" ::: "memory");
      if (i + 1 >= (size_t)a.depth) {
        asm volatile("cp.async.wait_group %0;" ::"n"(3) : "memory");   // depth 4
        const size_t j = i + 1 - a.depth;
        asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[j % a.depth])) : "memory");
      }
    }
    asm volatile("cp.async.wait_all;" ::: "memory");
  } else if (a.mode == 1) {
    // 256 threads: each slot = chunk bytes = chunk/16 copies; thread t copies 16 B pieces
    for (size_t i = 0; i < n_chunks; ++i) {
      const int s = i % a.depth;
      if (i >= (size_t)a.depth) {  // wait until the slot's previous fill landed (we are the consumer)
        if ((tid & 31) == 0) while (!try_wait(su32(&full[s]), ((i / a.depth) - 1) & 1)) {}
        __syncwarp();
      }
      const uint8_t* src = a.src + (off + i * a.chunk) % a.footprint;
      for (int k = tid; k < a.chunk / 16; k += blockDim.x)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(sm + s * a.chunk + k * 16)),
                     "l"(src + k * 16) : "memory");
      asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
    }
    for (int s = 0; s < a.depth && (size_t)s < n_chunks; ++s) {
      const size_t last = ((n_chunks - 1 - s) / a.depth) * a.depth + s;
      if ((tid & 31) == 0) while (!try_wait(su32(&full[s]), (last / a.depth) & 1)) {}
    }
  } else if ((a.mode == 5 && (tid & 31) == 0) || (a.mode == 8 && tid < a.csz) || tid == 0) {
    const int nw = (a.mode == 5 || a.mode == 8) ? a.csz : 1;
    const int w = a.mode == 8 ? tid : tid >> 5;   // mode 8: issuing LANES of warp 0
    const int slice = a.chunk / csz;
    const int rows = a.footprint / 128;
    uint32_t rng = 12345u + 7919u * blockIdx.x;
    const size_t my_chunks = (n_chunks + nw - 1 - w) / nw;
    for (size_t i = 0; i < my_chunks + a.depth; ++i) {
      if (i >= (size_t)a.depth) {  // consume chunk i - depth: wait for it, then free the slot
        const size_t j = i - a.depth;
        const int s = w * a.depth + j % a.depth;
        while (!try_wait(su32(&full[s]), (j / a.depth) & 1)) {}
        if (a.mode == 2) {   // tell every CTA of the cluster that this CTA's slot s is free
          for (int r = 0; r < csz; ++r) {
            uint32_t remote;
            asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(su32(&empty[s])), "r"(r));
            asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
          }
        }
      }
      if (i < my_chunks) {
        const int s = w * a.depth + i % a.depth;
        if (a.mode == 2 && i >= (size_t)a.depth) {  // every CTA of the cluster freed slot s
          while (!try_wait(su32(&empty[s]), ((i / a.depth) - 1) & 1)) {}
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(a.chunk) : "memory");
        const uint8_t* src = a.src + (off + (i * nw + w) * a.chunk) % a.footprint;
        if (a.mode == 3) {
          const int row0 = (int)(((off + (i * nw + w) * a.chunk) % a.footprint) / 128);
          asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                       ::"r"(su32(sm + s * a.chunk)), "l"(&a.tmap), "r"(0), "r"(row0), "r"(su32(&full[s])) : "memory");
        } else if (a.mode == 4) {
          for (int g = 0; g < a.chunk / 512; ++g) {
            int r4[4];
            for (int k = 0; k < 4; ++k) {
              rng = rng * 1664525u + 1013904223u;
              r4[k] = (int)((rng >> 8) % (uint32_t)rows);
            }
            asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                         ::"r"(su32(sm + s * a.chunk + g * 512)), "l"(&a.tmap), "r"(0), "r"(r4[0]), "r"(r4[1]),
                         "r"(r4[2]), "r"(r4[3]), "r"(su32(&full[s])) : "memory");
          }
        } else if (a.mode == 0 || a.mode == 5 || a.mode == 8) {
          asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                       ::"r"(su32(sm + s * a.chunk)), "l"(src), "r"(a.chunk), "r"(su32(&full[s])) : "memory");
        } else {
          const uint16_t mask = (uint16_t)((1u << csz) - 1);
          asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;"
                       ::"r"(su32(sm + s * a.chunk + rank * slice)), "l"(src + rank * slice), "r"(slice),
                       "r"(su32(&full[s])), "h"(mask) : "memory");
        }
      }
    }
  }
  __syncthreads();
  const long long c1 = clock64();
  const unsigned long long t1 = gt();
  if (a.mode == 2) asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (tid == 0) {
    a.out[blockIdx.x * 3 + 0] = t0;
    a.out[blockIdx.x * 3 + 1] = t1;
    a.out[blockIdx.x * 3 + 2] = (unsigned long long)(c1 - c0);
  }
}

int main(int argc, char** argv) {
  const int mode = argc > 1 ? atoi(argv[1]) : 0;
  const int chunk = argc > 2 ? atoi(argv[2]) : 16384;
  const int depth = argc > 3 ? atoi(argv[3]) : 4;
  const size_t footprint = argc > 4 ? (size_t)atoll(argv[4]) : (size_t)16 << 20;
  const int ctas = argc > 5 ? atoi(argv[5]) : 148;
  const int csz = argc > 6 ? atoi(argv[6]) : 1;
  const size_t per_cta = argc > 7 ? (size_t)atoll(argv[7]) : (size_t)8 << 20;
  uint8_t* src;
  cudaMalloc(&src, footprint + chunk);
  cudaMemset(src, 1, footprint + chunk);
  unsigned long long* out;
  cudaMalloc(&out, ctas * 3 * 8);
  const int smem = chunk * depth * (mode == 5 || mode == 7 || mode == 8 ? csz : 1) + 1024;
  CUtensorMap tmap = {};
  if (mode == 3 || mode == 4) {
    typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                            const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                            CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    cuuint64_t dims[2] = {64, footprint / 128};
    cuuint64_t strides[1] = {128};
    cuuint32_t box[2] = {64, mode == 3 ? (cuuint32_t)(chunk / 128) : 1u};
    cuuint32_t es[2] = {1, 1};
    CUresult r = ((Enc)fn)(&tmap, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, src, dims, strides, box, es,
                           CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                           CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) {
      printf("{\"error\": \"tensor map %d\"}\n", (int)r);
      return 1;
    }
  }
  cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (csz > 8) cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  Args a{tmap, src, footprint, per_cta, chunk, depth, mode, csz, out};
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(ctas);
  cfg.blockDim = dim3(mode == 1 || mode == 6 || mode == 7 ? 256 : mode == 5 ? 32 * csz : 32);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = mode == 2 ? csz : 1;
  if (csz > 8 && mode == 2) cudaFuncSetAttribute(stream_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  double best_us = 1e30, cyc = 0;
  for (int rep = 0; rep < 4; ++rep) {
    cudaError_t e = cudaLaunchKernelEx(&cfg, stream_kernel, a);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
      printf("{\"error\": \"%s\"}\n", cudaGetErrorString(e));
      return 1;
    }
    unsigned long long* h = (unsigned long long*)malloc(ctas * 24);
    cudaMemcpy(h, out, ctas * 24, cudaMemcpyDeviceToHost);
    unsigned long long t0 = ~0ull, t1 = 0;
    double c = 0;
    for (int i = 0; i < ctas; ++i) {
      if (h[3 * i] < t0) t0 = h[3 * i];
      if (h[3 * i + 1] > t1) t1 = h[3 * i + 1];
      c += h[3 * i + 2];
    }
    const double us = (t1 - t0) / 1e3;
    if (us < best_us) best_us = us, cyc = c / ctas;
    free(h);
  }
  const double per_sm = per_cta / best_us / 1e3;   // GB/s received per SM
  const double mhz = cyc / best_us;
  printf("{\"mode\": %d, \"chunk\": %d, \"depth\": %d, \"footprint_MB\": %.1f, \"ctas\": %d, \"csz\": %d, "
         "\"us\": %.1f, \"GBps_per_sm\": %.1f, \"TBps_chip\": %.2f, \"sm_mhz\": %.0f, \"B_per_clk_per_sm\": %.1f, "
         "\"l2_reads_TBps\": %.2f}\n",
         mode, chunk, depth, footprint / 1048576.0, ctas, csz, best_us, per_sm, per_sm * ctas / 1e3, mhz,
         per_cta / cyc, per_sm * ctas / 1e3 / (mode == 2 ? csz : 1));
  return 0;
}
