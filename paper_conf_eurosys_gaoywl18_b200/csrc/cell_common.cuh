// cell_common.cuh -- device helpers shared by the cell-step kernels (cell_step_sm100.cu,
// cell_pair_sm100.cu): gate nonlinearities, the launch chain (dependency flag, completion
// signal), row sources of the gather (A6), the epilogue's c-state prefetch, cluster / CTA-pair
// barrier and MMA wrappers. Device code only; every TU gets its own internal-linkage copy.
#pragma once
#include <cuda_bf16.h>
#include <stdint.h>

#include "kernels.h"
#include "sm100_ptx.cuh"

namespace bm {
namespace {
using namespace ptx;

__device__ __forceinline__ float sigm(float x) { return __fdividef(1.0f, 1.0f + __expf(-x)); }
__device__ __forceinline__ float tanh_f(float x) { return 1.0f - __fdividef(2.0f, __expf(2.0f * x) + 1.0f); }

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Diagnostics (BM_PHASE_DUMP): %globaltimer of one thread at phase boundaries of each CTA.
__device__ __forceinline__ void phase_mark(const StepArgs& p, int i) {
  if (p.phase != nullptr) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    const int cta = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
    p.phase[cta * 64 + i] = t;
  }
}

// ------------------------------------------------------------------ launch chain
// Consecutive launches on the engine stream form a chain: the last CTA of launch n publishes
// n in *dep_flag (release) once every CTA's writes are done; launch n+1, started early under
// PDL, waits for it with an acquire poll instead of griddepcontrol.wait (grid-completion
// propagation measured ~3.5 us end -> release on B200; a flag hand-off is a few hundred ns).
// A poll that has not succeeded after 10 s traps (sticky launch error) instead of hanging.
__device__ __forceinline__ void dep_wait(const StepArgs& p) {
  if (p.dep_flag == nullptr) {
    pdl_wait();
    return;
  }
  const unsigned int want = p.dep_seq - 1u;
  if ((threadIdx.x & 31) == 0) {
    unsigned long long t0 = 0;
    while (static_cast<int>(ld_acquire_gpu(p.dep_flag) - want) < 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t0 == 0) t0 = t;
      else if (t - t0 > 10000000000ull) __trap();
    }
  }
  __syncwarp();
  (void)ld_acquire_gpu(p.dep_flag);  // every lane acquires the predecessors' writes
}

// End of a launch: count this CTA; the last one resets the counter, publishes the launch in
// the chain flag and, on a task's last launch, bumps the host-mapped completion counter (A12).
__device__ __forceinline__ void launch_done(const StepArgs& p, unsigned int* ctas) {
  if (threadIdx.x != 0) return;
  const unsigned total = gridDim.x * gridDim.y * gridDim.z;
  __threadfence();
  if (atomicAdd(ctas, 1u) == total - 1) {
    *ctas = 0;
    __threadfence();
    if (p.dep_flag != nullptr) st_release_gpu(p.dep_flag, p.dep_seq);
    if (p.signal != nullptr) {  // the task's own slot: no ordering against other tasks needed
      __threadfence_system();
      signal_store(p.signal, p.sig_value);
    }
  }
}

// ------------------------------------------------------------------ row sources (A6)
// The launch's rows travel either inline in the parameter block (RowsParam<true>, direct
// steps) or in the device descriptor ring (RowsParam<false>: a 4-byte dummy, so the launch
// carries ~0.5 KB of parameters instead of ~8.7 KB -- 3.3 vs 6.5-8.9 us of host time per
// launch, tools/launch_bench.cu). Ring rows are published by a copy on the copy stream
// followed by a stream write of rows_seq to *rows_flag; the kernel polls the flag (acquire)
// before its first row read, so no cross-stream event sits between two launches.
template <bool INL>
struct RowsParam {
  RowDesc r[kMaxRowsInline];
};
template <>
struct RowsParam<false> {
  int unused;
};
template <bool INL>
__device__ __forceinline__ RowDesc row_at(const StepArgs& p, const RowsParam<INL>& rr, int i) {
  if constexpr (INL) {
    return rr.r[i];
  } else {
    const int4 v = *(reinterpret_cast<const int4*>(p.rows) + i);
    return RowDesc{v.x, v.y, v.z, v.w};
  }
}
// Ring rows: wait until the copy that carries them has landed (lane 0 polls, 10 s trap).
__device__ __forceinline__ void rows_wait(const StepArgs& p) {
  if (p.rows_flag == nullptr) return;
  if ((threadIdx.x & 31) == 0) {
    unsigned long long t0 = 0;
    while (static_cast<int>(ld_acquire_gpu(p.rows_flag) - p.rows_seq) < 0) {
      unsigned long long t;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
      if (t0 == 0) t0 = t;
      else if (t - t0 > 10000000000ull) __trap();
    }
  }
  __syncwarp();
  (void)ld_acquire_gpu(p.rows_flag);
}

// Pointer to the first element of a row's operand segment `seg`, or nullptr for a zero row.
template <int EPI>
__device__ __forceinline__ const __nv_bfloat16* seg_src(const StepArgs& p, const RowDesc& r,
                                                        int seg) {
  const size_t H = p.H;
  const size_t S = p.n_slots;
  const __nv_bfloat16* hp = static_cast<const __nv_bfloat16*>(p.h_pool);
  if constexpr (EPI == EPI_LSTM) {
    const int par = (r.flags & ROW_PARITY) ? 1 : 0;
    if (seg == 0) {
      if (p.h_lower != nullptr) {  // layer > 0: x = h'(layer-1) just written at parity 1-par
        return static_cast<const __nv_bfloat16*>(p.h_lower) + ((1 - par) * S + r.slot) * H;
      }
      const int tok = r.a >= 0 ? r.a : p.tok[r.slot];
      return static_cast<const __nv_bfloat16*>(p.E) + static_cast<size_t>(tok) * H;
    }
    if (r.flags & ROW_FIRST) return nullptr;  // h_prev = 0
    return hp + (par * S + r.slot) * H;
  } else if constexpr (EPI == EPI_LEAF) {
    return static_cast<const __nv_bfloat16*>(p.E) + static_cast<size_t>(r.a) * H;
  } else if constexpr (EPI == EPI_INTERNAL) {
    return hp + static_cast<size_t>(seg == 0 ? r.a : r.b) * H;  // children h at parity 0
  } else {  // EPI_PROJ: h of the top layer, written at parity 1-par by this step
    const int par = (r.flags & ROW_PARITY) ? 1 : 0;
    return hp + ((1 - par) * S + r.slot) * H;
  }
}


// Epilogue c-state prefetch (A9 inputs): the c rows this CTA's epilogue will read (LSTM: c of
// the row's slot, zero for a first step; internal: c_L and c_R of the children), U units per
// row, copied into shared memory by the producers with the first activation stage, so the
// reduction loop does not wait on global loads. Layout: column cl (relative to c_lo) holds
// nseg x U floats. The copies are covered by the stage's cp.async arrive (and a wait_all
// before the epilogue).
template <int EPI>
__device__ __forceinline__ void prefetch_c(const StepArgs& p, const RowDesc* rtab, int c_lo, int my_cols,
                                           int unit0, uint32_t cbuf, int t, int nthr) {
  if constexpr (EPI == EPI_LSTM || EPI == EPI_INTERNAL) {
    constexpr int nseg = EPI == EPI_INTERNAL ? 2 : 1;
    const int cpc = nseg * p.U / 4;  // 16-byte chunks per column
    const int cps = p.U / 4;         // chunks per segment
    const size_t H = p.H;
    for (int q = t; q < my_cols * cpc; q += nthr) {
      const int cl = q / cpc, ch = q % cpc;
      const RowDesc r = rtab[c_lo + cl];
      const int seg = ch / cps;
      const float* src;
      bool zero = false;
      if constexpr (EPI == EPI_LSTM) {
        src = p.c_pool + static_cast<size_t>(r.slot) * H + unit0 + ch * 4;
        zero = (r.flags & ROW_FIRST) != 0;
      } else {
        src = p.c_pool + static_cast<size_t>(seg ? r.b : r.a) * H + unit0 + (ch % cps) * 4;
      }
      cp_async_16(cbuf + q * 16, zero ? static_cast<const void*>(p.c_pool) : src, zero ? 0u : 16u);
    }
  }
}


__device__ __forceinline__ bool mbar_try_wait_cluster(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
// Bounded spin on an mbarrier phase (traps after ~4 s instead of hanging the GPU).
template <bool CLUSTER>
__device__ __forceinline__ void wait_bounded(uint32_t bar, uint32_t parity) {
  unsigned long long t0 = 0;
  for (int it = 0;; ++it) {
    if (CLUSTER ? mbar_try_wait_cluster(bar, parity) : mbar_try_wait(bar, parity)) return;
    if ((it & 1023) == 1023) {
      const unsigned long long t = gtimer();
      if (t0 == 0) t0 = t;
      else if (t - t0 > 4000000000ull) __trap();
    }
  }
}
__device__ __forceinline__ void wait_bounded_warp(uint32_t bar, uint32_t parity) {
  if ((threadIdx.x & 31) == 0) wait_bounded<false>(bar, parity);
  __syncwarp();
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t cluster_addr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_addr) : "memory");
}
__device__ __forceinline__ void mma_bf16_pair(uint32_t tmem_d, uint64_t a, uint64_t b, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(a), "l"(b), "r"(idesc), "r"(accumulate)
      : "memory");
}
__device__ __forceinline__ void mma_commit_pair(uint32_t bar, uint16_t mask) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          bar),
      "h"(mask)
      : "memory");
}
__device__ __forceinline__ void cluster_arrive() {
  asm volatile("barrier.cluster.arrive.release.aligned;" ::: "memory");
}
__device__ __forceinline__ void cluster_wait() {
  asm volatile("barrier.cluster.wait.acquire.aligned;" ::: "memory");
}

}  // namespace
}  // namespace bm
