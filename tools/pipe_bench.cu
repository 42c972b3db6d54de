// pipe_bench.cu -- the cell kernel's producer -> MMA stage hand-off in isolation.
// 148 CTAs x 320 threads: warps 0-7 produce stages into a 4-slot ring, warp 8 lane 0 consumes
// them (waits `full`, optionally issues tcgen05.mma, signals `empty` with tcgen05.commit or a
// plain arrive). Reports cycles per stage seen by the consumer.
//   prod: 0 = 256 mbarrier.arrive per stage (no data)   1 = one arrive per warp (no data)
//         2 = cp.async zero-fill + cp.async.mbarrier.arrive.noinc per thread
//         3 = cp.async from an L2-resident table + arrive.noinc per thread
//         4 = cp.async from the table + commit/wait_group(lag) + per-warp arrive
//   cons: 0 = plain mbarrier.arrive on empty   1 = tcgen05.commit on empty (no MMA)
//         2 = 4 x tcgen05.mma 128xNx16 + commit
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pipe_bench pipe_bench.cu
#include <cstdio>
#include <cstdlib>
#include <cuda_bf16.h>
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
__device__ __forceinline__ bool try_wait_hint(uint32_t bar, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(bar), "r"(par), "r"(20) : "memory");
  return ok;
}
__device__ int g_wmode;
template <int W>
__device__ __forceinline__ void wait_warp(uint32_t bar, uint32_t par) {
  if (W == 1) { while (!try_wait(bar, par)) {} return; }
  if (W == 2) { while (!test_wait(bar, par)) {} return; }
  if ((threadIdx.x & 31) == 0) {
    while (!try_wait(bar, par)) {}
  }
  __syncwarp();
}
__device__ __forceinline__ void arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.release.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

constexpr int kStagesMax = 8;

template <int W>
__global__ void __launch_bounds__(320, 1) pipe(const __nv_bfloat16* table, const int* idx, int npad, int nk,
                                              int kstages, int prod, int cons, long long* out, int wm2) {
  extern __shared__ uint8_t raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t full[kStagesMax], empty[kStagesMax], done;
  __shared__ uint32_t tslot;
  __shared__ int rows_s[256];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int stage_bytes = npad * 128;
  uint8_t* wbuf = sm + kstages * stage_bytes;  // 16 KB of "weights" (zeros)
  if (tid == 0) {
    for (int s = 0; s < kStagesMax; ++s) {
      asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&full[s])),
                   "r"(prod == 1 || prod == 4 ? 8 : prod == 5 ? 1 : 256));
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&empty[s])));
    }
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&done)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  if (tid < npad) rows_s[tid] = idx[blockIdx.x * 256 + tid];
  for (int i = tid; i < 16384 / 16; i += 320) reinterpret_cast<uint4*>(wbuf)[i] = make_uint4(0, 0, 0, 0);
  if (warp == 8) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&tslot)) : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = tslot;
  const long long t0 = clock64();
  if (warp < 8 && (prod != 5 || warp == 0)) {
    const int n_items = (npad * 8 + 255 - tid) / 256;
    int handed = 0;
    const int lag = kstages - 1;
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % kstages, round = kb / kstages;
      if (round > 0) wait_warp<W>(su32(&empty[s]), (round - 1) & 1);
      const uint32_t xs = su32(sm + s * stage_bytes);
      if (prod == 0) {
        arrive(su32(&full[s]));
      } else if (prod == 1) {
        __syncwarp();
        if (lane == 0) arrive(su32(&full[s]));
      } else if (prod == 5) {
        if (warp == 0 && lane == 0) arrive(su32(&full[s]));
      } else {
        for (int i = 0; i < n_items; ++i) {
          const int q = tid + 256 * i, row = q >> 3, ch = q & 7;
          const uint32_t dst = xs + row * 128 + ((ch ^ (row & 7)) << 4);
          const __nv_bfloat16* src = table + (size_t)rows_s[row] * 1024 + kb * 64 + ch * 8;
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src),
                       "r"(prod == 2 ? 0 : 16) : "memory");
        }
        if (prod == 4) {
          asm volatile("cp.async.commit_group;" ::: "memory");
          while (handed <= kb - lag) {
            const int pend = kb - handed;
            if (pend >= 3) asm volatile("cp.async.wait_group 3;" ::: "memory");
            else if (pend == 2) asm volatile("cp.async.wait_group 2;" ::: "memory");
            else if (pend == 1) asm volatile("cp.async.wait_group 1;" ::: "memory");
            else asm volatile("cp.async.wait_group 0;" ::: "memory");
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            __syncwarp();
            if (lane == 0) arrive(su32(&full[handed % kstages]));
            ++handed;
          }
        } else {
          asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
        }
      }
    }
    if (prod == 4) {
      asm volatile("cp.async.wait_group 0;" ::: "memory");
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      while (handed < nk) {
        if (lane == 0) arrive(su32(&full[handed % kstages]));
        ++handed;
      }
    }
  } else if (warp == 8 && wm2) {
    long long tf = 0;
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        const int s = kb % kstages;
        while (!try_wait(su32(&full[s]), (kb / kstages) & 1)) {}
        if (kb == 0) tf = clock64();
        arrive(su32(&empty[s]));
      }
      arrive(su32(&done));
      while (!try_wait(su32(&done), 0)) {}
      out[blockIdx.x * 2] = tf - t0;
      out[blockIdx.x * 2 + 1] = clock64() - t0;
    }
    __syncwarp();
  } else if (warp == 8) {
    long long tf = 0;
    const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(npad >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    for (int kb = 0; kb < nk; ++kb) {
      const int s = kb % kstages;
      wait_warp<W>(su32(&full[s]), (kb / kstages) & 1);
      if (cons != 0) asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      if (kb == 0) tf = clock64();
      if (lane == 0) {
        if (cons == 0) {
          arrive(su32(&empty[s]));
        } else {
          if (cons == 2) {
            const uint64_t a = sdesc(su32(wbuf)), b = sdesc(su32(sm + s * stage_bytes));
            for (int k = 0; k < 4; ++k)
              asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}"
                           ::"r"(tmem), "l"(a + 2 * k), "l"(b + 2 * k), "r"(idesc), "r"((kb | k) != 0 ? 1 : 0) : "memory");
          }
          asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&empty[s])) : "memory");
          if (kb == nk - 1)
            asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&done)) : "memory");
        }
      }
      __syncwarp();
    }
    if (cons == 0 && lane == 0) arrive(su32(&done));
    wait_warp<W>(su32(&done), 0);
    if (lane == 0) {
      out[blockIdx.x * 2] = tf - t0;
      out[blockIdx.x * 2 + 1] = clock64() - t0;
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 8) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem) : "memory");
  }
}

int main() {
  const int R = 8192;
  __nv_bfloat16* table;
  cudaMalloc(&table, (size_t)R * 1024 * 2);
  cudaMemset(table, 0, (size_t)R * 1024 * 2);
  int* idx;
  cudaMalloc(&idx, 148 * 256 * 4);
  int h[148 * 256];
  srand(1);
  for (auto& x : h) x = rand() % R;
  cudaMemcpy(idx, h, sizeof(h), cudaMemcpyHostToDevice);
  long long* out;
  cudaMalloc(&out, 148 * 16);
  cudaFuncSetAttribute(pipe<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);cudaFuncSetAttribute(pipe<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);cudaFuncSetAttribute(pipe<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int wm = 0; wm < 2; ++wm) for (int W3 = 0; W3 < 3; ++W3) {
  cudaMemcpyToSymbol(g_wmode, &wm, 4);
  printf("consumer lane-only %d, wait style %d\n", wm, W3);
  for (int npad : {64}) {
    const int kst = npad == 64 ? 4 : 2; for (int nk : {64}) {
    for (int prod : {5, 1, 3})
      for (int cons : {0}) {
        long long best = 1LL << 60, bf = 0;
        for (int rep = 0; rep < 5; ++rep) {
          (W3 == 0 ? pipe<0> : W3 == 1 ? pipe<1> : pipe<2>)<<<148, 320, 200 * 1024>>>(table, idx, npad, nk, kst, prod, cons, out, wm);
          cudaError_t e = cudaDeviceSynchronize();
          if (e != cudaSuccess) { printf("err %s\n", cudaGetErrorString(e)); return 1; }
          long long o[296];
          cudaMemcpy(o, out, sizeof(o), cudaMemcpyDeviceToHost);
          long long sf = 0, sl = 0;
          for (int i = 0; i < 148; ++i) { sf += o[2 * i]; sl += o[2 * i + 1]; }
          if (sl / 148 < best) { best = sl / 148; bf = sf / 148; }
        }
        printf("npad %3d stages %d nk %d prod %d cons %d: first %5lld cyc, all %6lld cyc, per stage %5lld cyc\n",
               npad, kst, nk, prod, cons, bf, best, (best - bf) / (nk - 1));
      }
    }
  }
  }
  return 0;
}
