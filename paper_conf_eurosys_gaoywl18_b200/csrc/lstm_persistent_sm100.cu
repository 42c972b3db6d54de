// lstm_persistent_sm100.cu -- weight-stationary persistent LSTM cell engine (SURVEY §8f N3,
// "persistent RNN ... complementary", §8).
//
// One launch serves a whole bm_run: the grid (S K-slices x h/32 unit tiles = 128 CTAs for
// h = 1024, clusters of S) stays resident, each CTA keeps ITS slice of the packed bf16 LSTM
// weights (128 gate rows x 512 K = 128 KB) in shared memory for the lifetime of the kernel, and
// tasks are fed through a device ring (row descriptors + headers copied by the host on a copy
// stream). Per task every CTA gathers its K-slice of [x ; h] for the task's rows, runs tcgen05
// MMAs against the resident weights into TMEM (up to 4 column chunks of 128 = 512 TMEM
// columns), reduces the S split-K partials through DSMEM in fixed order, applies the fused LSTM
// gates and scatters h'/c' by slot; a grid-wide barrier (global counter) separates consecutive
// tasks (the next step of a request reads this step's h'), and the last CTA to arrive bumps the
// host-mapped completion counter (A12). No weight bytes cross the memory system per step and
// no kernel is launched per step; what is left per step is the gather, the MMAs and the
// epilogue. Spin loops carry timeouts so a host that stops feeding cannot hang the GPU.
#include <cuda_bf16.h>
#include <stdint.h>

#include "kernels.h"
#include "sm100_ptx.cuh"

namespace bm {
namespace {
using namespace ptx;

constexpr int kThreads = 320;           // warps 0-7 gather + epilogue, 8 MMA, 9 control
constexpr int kProducers = 256;
constexpr int kMmaWarp = 8;
constexpr int kCtlWarp = 9;
constexpr int kBK = 64;
constexpr int kChunk = 128;             // batch columns per MMA (N) chunk
constexpr int kMaxChunks = 4;           // 512 TMEM columns
constexpr int kXStages = 4;
constexpr int kXStageBytes = kChunk * 128;      // 16 KB: 128 rows x 64 K bf16
constexpr int kWBlk = 128 * 128;                // one K block of the 128-row weight tile
constexpr int kMaxKB = 8;                       // K blocks per CTA slice (<= 512 wide)
constexpr int kTail = 10 * 1024;                // row sources [2][512] (8 KB) + barriers
constexpr int kMaxS = 4;
constexpr unsigned long long kTimeoutNs = 20ull * 1000 * 1000 * 1000;  // 20 s

__device__ __forceinline__ unsigned long long now_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ unsigned int ld_acquire_u32(const unsigned int* p) {
  unsigned int v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ int ld_volatile_i32(const int* p) {
  int v;
  asm volatile("ld.volatile.global.s32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + __expf(-x)); }

// diagnostics: %globaltimer at phase i of task kPhaseTask, per CTA (BM_PHASE_DUMP)
constexpr int kPhaseTask = 20;
__device__ __forceinline__ void pmark(const PersistArgs& p, int t, int i) {
  if (p.phase != nullptr && t == kPhaseTask)
    p.phase[(blockIdx.x + gridDim.x * blockIdx.y) * 16 + i] = now_ns();
}

__device__ __forceinline__ const __nv_bfloat16* seg_src(const PersistArgs& p, const RowDesc& r, int seg) {
  const size_t H = p.H;
  const size_t S = p.n_slots;
  const int par = (r.flags & ROW_PARITY) ? 1 : 0;
  if (seg == 0) {
    const int tok = r.a >= 0 ? r.a : p.tok[r.slot];
    return static_cast<const __nv_bfloat16*>(p.E) + static_cast<size_t>(tok) * H;
  }
  if (r.flags & ROW_FIRST) return nullptr;
  return static_cast<const __nv_bfloat16*>(p.h_pool) + (par * S + r.slot) * H;
}

__global__ void __launch_bounds__(kThreads, 1) lstm_persistent_kernel(const __grid_constant__ PersistArgs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const uint32_t rank = cluster_rank();
  const int S = p.S;
  const int nk = p.kslice / kBK;
  const int k_begin = static_cast<int>(rank) * p.kslice;
  const int ncta = gridDim.x * gridDim.y;

  // ---- shared memory: [tail][resident weights nk x 16 KB][activation ring 4 x 16 KB]
  const __nv_bfloat16** src_tab = reinterpret_cast<const __nv_bfloat16**>(base);  // [2][512]
  uint64_t* bars = reinterpret_cast<uint64_t*>(base + 2 * 512 * sizeof(void*));
  const uint32_t xfull0 = smem_u32(bars);
  const uint32_t xempty0 = smem_u32(bars + kXStages);
  const uint32_t wready = smem_u32(bars + 2 * kXStages);
  const uint32_t task_ready = smem_u32(bars + 2 * kXStages + 1);
  const uint32_t done_bar = smem_u32(bars + 2 * kXStages + 2);
  const uint32_t grid_ready = smem_u32(bars + 2 * kXStages + 3);
  volatile int* s_task = reinterpret_cast<volatile int*>(bars + 2 * kXStages + 4);  // b, row_off
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * kXStages + 6);
  uint8_t* w_res = base + kTail;
  uint8_t* x_ring = w_res + kMaxKB * kWBlk;
  float* P = reinterpret_cast<float*>(x_ring);  // epilogue partial tile [128 cols][128 rows]

  if (tid == 0) {
    for (int s = 0; s < kXStages; ++s) {
      mbar_init(xfull0 + 8 * s, 1);
      mbar_init(xempty0 + 8 * s, 1);
    }
    mbar_init(wready, 1);
    mbar_init(task_ready, 1);
    mbar_init(done_bar, 1);
    mbar_init(grid_ready, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"(512)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  // ---- resident weights: this CTA's tile (128 packed rows) x K slice, loaded once (A7)
  if (warp == kCtlWarp && lane == 0) {
    const int kblocks = p.K / kBK;
    const uint8_t* wsrc = static_cast<const uint8_t*>(p.W) +
                          (static_cast<size_t>(blockIdx.y) * kblocks + k_begin / kBK) * kWBlk;
    const uint32_t bytes = static_cast<uint32_t>(nk * kWBlk);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(wready), "r"(bytes) : "memory");
    for (uint32_t off = 0; off < bytes; off += 64 * 1024) {
      const uint32_t n = bytes - off < 64 * 1024 ? bytes - off : 64 * 1024;
      bulk_load(smem_u32(w_res + off), wsrc + off, n, wready);
    }
  }

  const int lag = kXStages - 1;
  uint32_t kbg = 0;  // activation stages consumed so far (ring position / phase across tasks)
  for (int t = 0;; ++t) {
    // ================================================================ next task (control warp)
    if (warp == kCtlWarp) {
      if (lane == 0) {
        pmark(p, t, 0);
        const TaskHdr* h = p.hdr + (t % p.hdr_ring);
        const unsigned long long t0 = now_ns();
        int seq;
        while ((seq = ld_volatile_i32(&h->seq)) != t) {
          if (now_ns() - t0 > kTimeoutNs) break;
        }
        int b = -2;  // -2: abort (host stopped feeding)
        int off = 0;
        if (seq == t) {
          b = ld_volatile_i32(&h->b);
          off = ld_volatile_i32(&h->row_off);
        }
        if (b == -2) atomicExch(p.err, 1);
        s_task[0] = b;
        s_task[1] = off;
        mbar_arrive(task_ready);  // rows can be read now (they precede the header in the ring)
        if (b >= 0) {
          // grid barrier: every CTA finished task t-1 (its h'/c' writes are visible)
          const unsigned int target = static_cast<unsigned int>(ncta) * static_cast<unsigned int>(t);
          const unsigned long long t1 = now_ns();
          while (ld_acquire_u32(p.gbar) < target) {
            if (now_ns() - t1 > kTimeoutNs) {
              atomicExch(p.err, 1);  // a peer CTA is gone: finish this task's protocol anyway
              break;
            }
          }
          if (p.span != nullptr) atomicMin(p.span + 2 * (t & 63), now_ns());
        }
        pmark(p, t, 1);
        mbar_arrive(grid_ready);
      }
      __syncwarp();
    }
    mbar_wait_warp(task_ready, t & 1);
    const int b = s_task[0];
    const int row_off = s_task[1];
    if (b < 0) break;  // stop (-1) or abort (-2): every CTA reads the same header
    const RowDesc* rows = p.rows + row_off;
    const int npad = (b + 15) & ~15;
    const int nch = (npad + kChunk - 1) / kChunk;
    // a stage holds kpb consecutive K blocks of one column chunk (16 KB slots): narrow tasks
    // move the whole K slice in 1-2 hand-offs instead of 8
    const int cw = npad < kChunk ? npad : kChunk;  // widest chunk
    const int kpb = min(nk, kXStageBytes / (cw * 128));
    const int spc = (nk + kpb - 1) / kpb;           // stages per chunk
    const int nstage = nch * spc;

    if (warp < 8) {
      // ============================================================ gather (A6)
      for (int c = tid; c < npad; c += kProducers) {
        const __nv_bfloat16* s0 = nullptr;
        const __nv_bfloat16* s1 = nullptr;
        if (c < b) {
          const RowDesc r = rows[c];
          s0 = seg_src(p, r, 0);
          s1 = seg_src(p, r, 1);
        }
        src_tab[c] = s0;
        src_tab[512 + c] = s1;
      }
      named_bar(1, kProducers);
      if (tid == 0) pmark(p, t, 2);
      mbar_wait_warp(grid_ready, t & 1);  // h of the previous task is complete everywhere
      const __nv_bfloat16* dummy = static_cast<const __nv_bfloat16*>(p.E);
      for (int j = 0; j < nstage; ++j) {
        const uint32_t g = kbg + j;
        const int s = g % kXStages;
        const uint32_t round = g / kXStages;
        if (round > 0) mbar_wait_warp(xempty0 + 8 * s, (round - 1) & 1);
        const int ch = j / spc;
        const int c0 = ch * kChunk;
        const int ncol = min(kChunk, npad - c0);
        const int kb0 = (j % spc) * kpb;
        const int nkb = min(kpb, nk - kb0);
        const uint32_t xs0 = smem_u32(x_ring + s * kXStageBytes);
        for (int q = tid; q < nkb * ncol * 8; q += kProducers) {
          const int blk = q / (ncol * 8);
          const int rem = q - blk * ncol * 8;
          const int row = rem >> 3;
          const int chk = rem & 7;
          const int k = k_begin + (kb0 + blk) * kBK;
          const int seg = k >= p.K0 ? 1 : 0;
          const int kk = k - seg * p.K0;
          const __nv_bfloat16* src = src_tab[seg * 512 + c0 + row];
          const uint32_t dst = xs0 + blk * (ncol * 128) + row * 128 + ((chk ^ (row & 7)) << 4);
          if (src != nullptr) cp_async_16(dst, src + kk + chk * 8, 16);
          else cp_async_16(dst, dummy, 0);
        }
        cp_async_commit();
        if (j >= lag) {
          cp_async_wait<kXStages - 1>();
          fence_proxy_async();
          named_bar(1, kProducers);
          if (tid == 0) mbar_arrive(xfull0 + 8 * ((g - lag) % kXStages));
          if (tid == 0 && j == lag) pmark(p, t, 3);
        }
      }
      cp_async_wait<0>();
      fence_proxy_async();
      named_bar(1, kProducers);
      if (tid == 0)
        for (int j = max(0, nstage - lag); j < nstage; ++j) mbar_arrive(xfull0 + 8 * ((kbg + j) % kXStages));
    } else if (warp == kMmaWarp) {
      // ============================================================ MMA (A8)
      if (t == 0) mbar_wait_warp(wready, 0);
      for (int j = 0; j < nstage; ++j) {
        const uint32_t g = kbg + j;
        const int s = g % kXStages;
        mbar_wait_warp(xfull0 + 8 * s, (g / kXStages) & 1);
        tc_fence_after();
        const int ch = j / spc;
        const int ncol = min(kChunk, npad - ch * kChunk);
        const int kb0 = (j % spc) * kpb;
        const int nkb = min(kpb, nk - kb0);
        if (lane == 0) {
          const uint32_t idesc = idesc_bf16(128, ncol);
          for (int blk = 0; blk < nkb; ++blk) {
            const int kb = kb0 + blk;
            const uint64_t a = sdesc_sw128(smem_u32(w_res + kb * kWBlk));
            const uint64_t bd = sdesc_sw128(smem_u32(x_ring + s * kXStageBytes + blk * ncol * 128));
#pragma unroll
            for (int k = 0; k < kBK / 16; ++k)
              mma_bf16(tmem + ch * kChunk, a + 2 * k, bd + 2 * k, idesc, (kb | k) != 0 ? 1u : 0u);
          }
          mma_commit(xempty0 + 8 * s);
          if (j == nstage - 1) mma_commit(done_bar);
        }
        __syncwarp();
      }
    }
    kbg += nstage;

    // ================================================================ epilogue (A9)
    if (warp < 8) {
      mbar_wait_warp(done_bar, t & 1);
      tc_fence_after();
      if (tid == 0) pmark(p, t, 4);
    }
    const int q = warp & 3;
    const int trow = 32 * q + lane;
    const int unit0 = blockIdx.y * 32;
    const int prow0 = blockIdx.y * 128;
    const size_t H = p.H;
    const size_t NS = p.n_slots;
    for (int ch = 0; ch < nch; ++ch) {
      const int c0 = ch * kChunk;
      const int ncol = min(kChunk, npad - c0);
      const int nvalid = min(kChunk, b - c0);
      if (warp < 8) {  // TMEM -> P[col][row]
        for (int cc = (warp >> 2) * 32; cc < ncol; cc += 64) {
          float v[32];
          tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0 + cc, v);
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (cc + i < ncol) P[(cc + i) * 128 + trow] = v[i];
        }
      }
      tc_fence_before();
      if (tid == 0 && ch == 0) pmark(p, t, 5);
      cluster_sync();  // A: partials of this chunk are in every CTA's smem
      if (tid == 0 && ch == 0) pmark(p, t, 6);
      if (warp < 8) {
        uint32_t peer[kMaxS];
#pragma unroll
        for (int s = 0; s < kMaxS; ++s) peer[s] = mapa(smem_u32(P), s < S ? s : 0);
        const int cper = (nvalid + S - 1) / S;
        const int c_lo = static_cast<int>(rank) * cper;
        const int my_cols = max(0, min(nvalid, c_lo + cper) - c_lo);
        const int j = tid % 32;
        const float4 bias = *reinterpret_cast<const float4*>(p.bias + prow0 + j * 4);
        for (int cl = tid / 32; cl < my_cols; cl += kProducers / 32) {
          const uint32_t off = static_cast<uint32_t>(((c_lo + cl) * 128 + j * 4) * 4);
          float4 v[kMaxS];
#pragma unroll
          for (int s = 0; s < kMaxS; ++s)
            if (s < S) v[s] = ld_cluster_v4(peer[s] + off);
          float z0 = bias.x, z1 = bias.y, z2 = bias.z, z3 = bias.w;
#pragma unroll
          for (int s = 0; s < kMaxS; ++s)  // fixed order s = 0..S-1
            if (s < S) {
              z0 += v[s].x;
              z1 += v[s].y;
              z2 += v[s].z;
              z3 += v[s].w;
            }
          const RowDesc r = rows[c0 + c_lo + cl];
          const int u = unit0 + j;
          const float cp = (r.flags & ROW_FIRST) ? 0.f : p.c_pool[r.slot * H + u];
          const float cn = sigm(z1) * cp + sigm(z0) * tanhf(z2);
          const float hn = sigm(z3) * tanhf(cn);
          p.c_pool[r.slot * H + u] = cn;
          const int par_out = (r.flags & ROW_PARITY) ? 0 : 1;
          static_cast<__half*>(p.h_pool)[(par_out * NS + r.slot) * H + u] = act_from_float(hn);
          if (r.flags & ROW_LAST) {
            const size_t ro = static_cast<size_t>(r.flags >> 8) * p.res_layers * H + u;
            p.res_h[ro] = hn;
            p.res_c[ro] = cn;
          }
        }
      }
      if (tid == 0 && ch == 0) pmark(p, t, 7);
      cluster_sync();  // B: P may be overwritten (next chunk / next task's gather)
      if (tid == 0 && ch == 0) pmark(p, t, 8);
    }
    // ================================================================ task done
    __threadfence();
    __syncthreads();
    if (tid == 0) {
      pmark(p, t, 9);
      const unsigned int prev = atomicAdd(p.gbar, 1u);
      if (prev == static_cast<unsigned int>(ncta) * static_cast<unsigned int>(t + 1) - 1u) {
        if (p.span != nullptr) {  // device-side task span: first CTA ready .. last CTA done
          const unsigned long long t0 = atomicExch(p.span + 2 * (t & 63), ~0ull);
          atomicAdd(p.span_acc, now_ns() - t0);
          atomicAdd(p.span_acc + 1, 1ull);
        }
        __threadfence_system();
        const unsigned long long seq = p.sig_base + static_cast<unsigned long long>(t);
        signal_store(p.signal + seq % kSignalSlots, seq + 1ull);  // completion signal (A12)
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512) : "memory");
  }
}

}  // namespace

int persistent_smem_bytes() { return 1024 + kTail + kMaxKB * kWBlk + kXStages * kXStageBytes; }

cudaError_t launch_lstm_persistent(const PersistArgs& a, cudaStream_t st) {
  static bool configured = false;
  const int smem = persistent_smem_bytes();
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(lstm_persistent_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(a.S, a.H / 32, 1);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = a.S;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  // every CTA must be resident at once (grid barrier): check before launching
  int clusters = 0;
  cudaError_t e = cudaOccupancyMaxActiveClusters(&clusters, lstm_persistent_kernel, &cfg);
  if (e != cudaSuccess) return e;
  if (clusters < static_cast<int>(cfg.gridDim.y)) return cudaErrorCooperativeLaunchTooLarge;
  return cudaLaunchKernelEx(&cfg, lstm_persistent_kernel, a);
}

}  // namespace bm
