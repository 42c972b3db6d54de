// cell_pair_sm100.cu -- the LSTM cell step (A6-A9) on CTA pairs, second design, EXPERIMENTAL
// (BM_PAIR2=1; the default remains cell_pair_kernel in cell_step_sm100.cu). Results are bitwise
// equal to the first design (tools/pair_cmp.py), but it measured slower (b = 512: 37.2 vs
// 24.7 us, profiles/round2/): the L2 round trip of the split-K partials costs more than the
// DSMEM exchange it replaces, and two 32 KB activation stages keep fewer bytes in flight than
// the first design's three 64 KB (activation + weight) stages.
//
// Same tiling as cell_pair_kernel: tcgen05.mma.cta_group::2, M = 256 weight rows per pair
// (each CTA holds its own 128-row tile = 32 units x 4 gates, the A operand), N = the column
// block's rows with each CTA gathering half of them (B operand), K split over S clusters ranks
// (S = 2: 1024-wide slices). What changed, from measurements on the pool's B200s
// (tools/stream_bench.cu, profiles/round2/):
//  * Weight stream. A single thread's bulk copies complete one at a time (~0.6 us each, any
//    size <= 64 KB: 32 KB copies = 55 GB/s per SM); copies issued by different warps overlap
//    (4 warps x 16-32 KB reach ~88 GB/s per SM, the chip's L2 limit with every SM streaming).
//    So the weights move by 1-D bulk copies (pre-swizzled tiles, as before) issued by kNW = 4
//    warps, each owning ring slots, starting at kernel entry -- before the dependency wait,
//    since weights never depend on the previous launch (the PDL overlap). The producer warps'
//    cp.async carry only the activation gather.
//  * Epilogue. The fp32 split-K partials no longer cross DSMEM (9-21 B/cycle/SM; 6 us at 512
//    rows): every CTA writes the partial columns OTHER K slices own straight from TMEM to a
//    global (L2-resident) scratch region, one cluster barrier, and each owner adds them to its
//    own partial read straight from TMEM, in the fixed order s = 0..S-1 (batch invariance,
//    P10). A per-warp 32 x 33 shared tile turns the TMEM lane layout (lane = gate row) into
//    unit-major (unit, column) work items for the fused gates + state update + scatter (A9).
// The split of work, the fixed summation order and the gate arithmetic are unchanged, so
// results equal the first design's bit for bit.
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include <algorithm>

#include "cell_common.cuh"
#include "kernels.h"
#include "sm100_ptx.cuh"

namespace bm {
namespace {
using namespace ptx;

namespace p2 {
constexpr int kProd = 256;                    // warps 0-7: activation gather, then epilogue
constexpr int kMma = 8;                       // warp 8: TMEM alloc; MMA issue (leader) / forwarder (peer)
constexpr int kW0 = 9;                        // warps 9 .. 9 + kNW - 1: weight stream
constexpr int kNW = 4;
constexpr int kThreads = (kW0 + kNW) * 32;    // 416
constexpr int kWSlotsMax = 4;
constexpr int kXMax = 4;
constexpr int kTail = 5120;                   // barriers (1 KB) + row table [256] (4 KB)
constexpr int kBK = 64;
constexpr int kWBlk = 128 * 128;              // one K block of a 128-row weight tile (16 KB)
constexpr int kScrCols = 256;                 // scratch row pitch (columns)
constexpr int kTilePitch = 33;                // epilogue transpose tile [32 rows][33]
}  // namespace p2

__device__ __forceinline__ float4 ldcg4(const float* p) { return __ldcg(reinterpret_cast<const float4*>(p)); }

template <bool INL>
__global__ void __launch_bounds__(p2::kThreads, 1)
    cell_pair2_kernel(const __grid_constant__ StepArgs p, const __grid_constant__ RowsParam<INL> rr) {
  using namespace p2;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int U = p.U;                                      // 32 units per 128-row tile
  const uint32_t crank = cluster_rank();
  const int pm = static_cast<int>(crank & 1u);            // pair member (0 = leader: MMA issue)
  const int ks = static_cast<int>(crank >> 1);            // K slice
  const int S = p.S;
  const int tile = 2 * blockIdx.y + pm;
  const int cpb = p.cpb;
  const int col0 = blockIdx.z * cpb;
  const int ncols = min(cpb, p.b - col0);
  const int npad = (ncols + 31) & ~31;                    // MMA N (both halves)
  const int nhalf = npad >> 1;                            // rows gathered by this CTA
  const int h0 = pm * nhalf;
  const int nk = p.kslice / kBK;
  const int k_begin = ks * p.kslice;
  const int xkb = p.xkb;
  const int nst = nk / xkb;
  const int x_blk = nhalf * 128;
  const int x_stage = x_blk * xkb;
  const int kStages = min(kXMax, p.xring / x_stage);     // the last column block may be narrower
  const int wcb = p.wcb;                                  // K blocks per weight chunk
  const int wslots = p.wslots;                            // weight ring slots (launcher)
  const int n_chunks = nk / wcb;
  // epilogue ownership: K slice s owns columns [s * cper, (s + 1) * cper), cper a multiple of 32
  const int cper = (((npad + S - 1) / S) + 31) & ~31;
  const int c_lo = ks * cper;
  const int my_cols = max(0, min(ncols, c_lo + cper) - c_lo);
  const uint16_t pair_mask = static_cast<uint16_t>(3u << (crank & ~1u));

  uint64_t* bars = reinterpret_cast<uint64_t*>(base);
  const uint32_t full0 = smem_u32(bars);                  // local producers landed stage s
  const uint32_t empty0 = smem_u32(bars + kXMax);         // leader's commit (multicast)
  const uint32_t pfull0 = smem_u32(bars + 2 * kXMax);     // peer's stage s landed (forwarded)
  const uint32_t wfull0 = smem_u32(bars + 3 * kXMax);     // local weight chunk landed
  const uint32_t wempty0 = smem_u32(bars + 3 * kXMax + kWSlotsMax);
  const uint32_t pwfull0 = smem_u32(bars + 3 * kXMax + 2 * kWSlotsMax);
  const uint32_t done_bar = smem_u32(bars + 3 * kXMax + 3 * kWSlotsMax);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * kXMax + 3 * kWSlotsMax + 1);
  RowDesc* rtab = reinterpret_cast<RowDesc*>(base + 1024);
  uint8_t* w_ring = base + kTail;
  uint8_t* x_ring = w_ring + wslots * wcb * kWBlk;
  const float* cbuf = reinterpret_cast<const float*>(base + p.cbuf_off);

  if (tid == 0) phase_mark(p, 0);
  if (tid == 0) {
    for (int s = 0; s < kXMax; ++s) {
      mbar_init(full0 + 8 * s, kProd);
      mbar_init(empty0 + 8 * s, 1);
      mbar_init(pfull0 + 8 * s, 1);
    }
    for (int s = 0; s < kWSlotsMax; ++s) {
      mbar_init(wfull0 + 8 * s, 1);
      mbar_init(wempty0 + 8 * s, 1);
      mbar_init(pwfull0 + 8 * s, 1);
    }
    mbar_init(done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMma) {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(256)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  cluster_arrive();  // barrier inits of every CTA visible before any remote arrive / multicast
  const uint32_t tmem = *tmem_slot;
  pdl_launch_dependents();
  if (tid == 0) phase_mark(p, 1);

  if (warp >= kW0) {
    // ================================================================ weight stream (A7)
    // warp w issues chunks c = w, w + kNW, ... into slot c % wslots; weights never depend on
    // the previous launch, so this starts at kernel entry (overlapping the PDL wait)
    if (lane == 0) {
      const int w = warp - kW0;
      const int kblocks = (p.K0 + p.K1) / kBK;
      const uint8_t* wsrc = static_cast<const uint8_t*>(p.W) +
                            (static_cast<size_t>(tile) * kblocks + k_begin / kBK) * kWBlk;
      const uint32_t bytes = static_cast<uint32_t>(wcb * kWBlk);
      for (int c = w; c < n_chunks; c += kNW) {
        const int s = c % wslots;
        const int round = c / wslots;
        if (round > 0) wait_bounded<false>(wempty0 + 8 * s, (round - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(wfull0 + 8 * s), "r"(bytes)
                     : "memory");
        bulk_load(smem_u32(w_ring + s * wcb * kWBlk), wsrc + static_cast<size_t>(c) * wcb * kWBlk, bytes,
                  wfull0 + 8 * s);
      }
    }
    __syncwarp();
  } else if (warp < 8) {
    // ================================================================ activation gather (A6)
    constexpr int kItems = 4;  // nhalf <= 128 rows x 8 chunks / 256 threads
    const int n_items = (nhalf * 8 + kProd - 1 - tid) / kProd;
    if constexpr (!INL) rows_wait(p);
    if (tid < ncols) rtab[tid] = row_at(p, rr, col0 + tid);
    named_bar(1, kProd);
    RowDesc rd[kItems];
#pragma unroll
    for (int i = 0; i < kItems; ++i) rd[i] = rtab[min(h0 + ((tid + i * kProd) >> 3), ncols - 1)];
    dep_wait(p);
    if (tid == 0 && p.span != nullptr) atomicMin(p.span, gtimer());
    if (tid == 0) phase_mark(p, 8);
    const __nv_bfloat16* src0[kItems];
    const __nv_bfloat16* src1[kItems];
    uint32_t dst_off[kItems];
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
      const int q = tid + i * kProd;
      const int row = q >> 3;
      const int ch = q & 7;
      dst_off[i] = row * 128 + ((ch ^ (row & 7)) << 4);
      src0[i] = nullptr;
      src1[i] = nullptr;
      if (i < n_items && h0 + row < ncols) {
        const __nv_bfloat16* a0 = seg_src<EPI_LSTM>(p, rd[i], 0);
        const __nv_bfloat16* a1 = seg_src<EPI_LSTM>(p, rd[i], 1);
        src0[i] = a0 != nullptr ? a0 + ch * 8 : nullptr;
        src1[i] = a1 != nullptr ? a1 + ch * 8 : nullptr;
      }
    }
    const __nv_bfloat16* dummy = static_cast<const __nv_bfloat16*>(p.E != nullptr ? p.E : p.h_pool);
    for (int st = 0; st < nst; ++st) {
      const int s = st % kStages;
      const int round = st / kStages;
      if (round > 0) wait_bounded_warp(empty0 + 8 * s, (round - 1) & 1);
      for (int j = 0; j < xkb; ++j) {
        const int k = k_begin + (st * xkb + j) * kBK;
        const int seg = k >= p.K0 ? 1 : 0;
        const int kk = k - seg * p.K0;
        const uint32_t xs = smem_u32(x_ring + s * x_stage + j * x_blk);
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
          if (i < n_items) {
            const __nv_bfloat16* src = seg ? src1[i] : src0[i];
            if (src != nullptr) cp_async_16(xs + dst_off[i], src + kk, 16);
            else cp_async_16(xs + dst_off[i], dummy, 0);  // zero fill (h0 = 0, padding)
          }
        }
      }
      if (st == 0)  // the epilogue's c rows, with the first stage
        prefetch_c<EPI_LSTM>(p, rtab, c_lo, my_cols, tile * U, smem_u32(base + p.cbuf_off), tid, kProd);
      cp_async_arrive_noinc(full0 + 8 * s);
      if (tid == 0 && st == 0) phase_mark(p, 10);
    }
  } else if (pm == 0) {
    // ================================================================ MMA issuer (leader, A8)
    cluster_wait();
    const uint32_t idesc = idesc_bf16(256, npad);
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        const int j = kb % xkb;
        const int st = kb / xkb;
        const int s = st % kStages;
        if (j == 0) {
          const uint32_t par = (st / kStages) & 1;
          wait_bounded<false>(full0 + 8 * s, par);
          wait_bounded<true>(pfull0 + 8 * s, par);
          if (st < 4) phase_mark(p, 40 + st);
        }
        const int c = kb / wcb;
        const int ws = c % wslots;
        if (kb % wcb == 0) {
          const uint32_t wpar = (c / wslots) & 1;
          wait_bounded<false>(wfull0 + 8 * ws, wpar);
          wait_bounded<true>(pwfull0 + 8 * ws, wpar);
          if (c < 4) phase_mark(p, 48 + c);
        }
        tc_fence_after();
        const uint64_t a = sdesc_sw128(smem_u32(w_ring + ws * wcb * kWBlk + (kb % wcb) * kWBlk));
        const uint64_t b = sdesc_sw128(smem_u32(x_ring + s * x_stage + j * x_blk));
#pragma unroll
        for (int k = 0; k < kBK / 16; ++k) mma_bf16_pair(tmem, a + 2 * k, b + 2 * k, idesc, (kb | k) != 0 ? 1u : 0u);
        if (kb % wcb == wcb - 1) mma_commit_pair(wempty0 + 8 * ws, pair_mask);
        if (j == xkb - 1) mma_commit_pair(empty0 + 8 * s, pair_mask);
      }
      mma_commit_pair(done_bar, pair_mask);
    }
    __syncwarp();
  } else {
    // ================================================================ forwarder (peer)
    cluster_wait();
    const uint32_t lead = crank & ~1u;
    const uint32_t pfull_l = mapa(pfull0, lead);
    const uint32_t pwfull_l = mapa(pwfull0, lead);
    if (lane == 0) {
      for (int kb = 0; kb < nk; ++kb) {
        if (kb % xkb == 0) {
          const int st = kb / xkb;
          const int s = st % kStages;
          wait_bounded<false>(full0 + 8 * s, (st / kStages) & 1);
          fence_proxy_async();
          mbar_arrive_remote(pfull_l + 8 * s);
        }
        if (kb % wcb == 0) {
          const int c = kb / wcb;
          const int ws = c % wslots;
          wait_bounded<false>(wfull0 + 8 * ws, (c / wslots) & 1);
          mbar_arrive_remote(pwfull_l + 8 * ws);
        }
      }
    }
    __syncwarp();
  }
  if (warp != kMma) cluster_wait();

  // ================================================================ epilogue (A9)
  // scratch: this CTA's region [128 rows][kScrCols] fp32; CTA (y, z, rank r) at index
  // ((z * gridDim.y + y) * gridDim.x + r)
  const size_t cta_lin = (static_cast<size_t>(blockIdx.z) * gridDim.y + blockIdx.y) * gridDim.x;
  float* scr = p.scratch + (cta_lin + crank) * 128 * kScrCols;
  const int q = warp & 3;
  const int wg = warp >> 2;
  const int trow = 32 * q + lane;                         // TMEM lane = this CTA's tile row (u*4 + g)
  if (warp < 8) {
    wait_bounded_warp(done_bar, 0);
    asm volatile("cp.async.wait_all;" ::: "memory");      // own c-prefetch copies
    tc_fence_after();
    if (tid == 0) phase_mark(p, 2);
    // (1) export: partial columns owned by the other K slices -> scratch (rows = TMEM lanes)
    for (int c0 = wg * 32; c0 < npad; c0 += 64) {
      if (c0 / cper == ks) continue;
      float v[32];
      tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0, v);
      float4* dst = reinterpret_cast<float4*>(scr + trow * kScrCols + c0);
#pragma unroll
      for (int i = 0; i < 8; ++i) dst[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
    }
  }
  tc_fence_before();
  cluster_sync();  // A: every CTA's exported partials are visible to its cluster
  if (tid == 0) phase_mark(p, 3);
  if (warp < 8) {
    tc_fence_after();
    // (2) own columns: own partial from TMEM + the other slices' from their scratch, summed in
    // the fixed order s = 0..S-1; a per-warp 32 x 33 tile turns lane-major gate rows into
    // (unit, column) items: lane = (unit ul = lane & 7 of this warp's 8 units, column group)
    float* T = reinterpret_cast<float*>(w_ring) + warp * 32 * kTilePitch;   // drained weight ring
    const float bias = p.bias[tile * 128 + trow];
    const int unit0 = tile * U;
    const size_t H = p.H;
    const size_t NS = p.n_slots;
    const int cu = lane & 7;                              // unit (within this warp's 8)
    const int cg = lane >> 3;                             // column group: columns cg + 4t
    const int ul = 8 * q + cu;                            // unit within the tile
    const int u = unit0 + ul;
    const int my_end = min(npad, c_lo + cper);
    for (int c0 = c_lo + wg * 32; c0 < my_end; c0 += 64) {
      float own[32];
      tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0, own);
      float z[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) z[i] = bias;
      for (int s = 0; s < S; ++s) {  // fixed order (batch invariance)
        if (s == ks) {
#pragma unroll
          for (int i = 0; i < 32; ++i) z[i] += own[i];
        } else {
          const float* src = p.scratch + (cta_lin + 2 * s + pm) * 128 * kScrCols + trow * kScrCols + c0;
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const float4 t = ldcg4(src + 4 * i);
            z[4 * i] += t.x;
            z[4 * i + 1] += t.y;
            z[4 * i + 2] += t.z;
            z[4 * i + 3] += t.w;
          }
        }
      }
#pragma unroll
      for (int i = 0; i < 32; ++i) T[lane * kTilePitch + i] = z[i];
      __syncwarp();
#pragma unroll
      for (int t = 0; t < 8; ++t) {
        const int ci = cg + 4 * t;                        // column within the chunk
        const int col = c0 + ci;
        if (col >= ncols || col >= c_lo + my_cols) continue;
        const float zi = T[(4 * cu + 0) * kTilePitch + ci];
        const float zf = T[(4 * cu + 1) * kTilePitch + ci];
        const float zg = T[(4 * cu + 2) * kTilePitch + ci];
        const float zo = T[(4 * cu + 3) * kTilePitch + ci];
        const RowDesc rw = rtab[col];
        if (p.dead != nullptr) {  // N1: rows of a request that emitted <eos> are no-ops
          if ((rw.flags & ROW_EOS) && p.dead[rw.slot]) continue;
          if (p.layer == 0 && (rw.flags & ROW_FIRST) && u == 0) p.dead[rw.slot] = 0;
        }
        const float cin = cbuf[(col - c_lo) * U + ul];
        const float cn = sigm(zf) * cin + sigm(zi) * tanh_f(zg);
        const float hn = sigm(zo) * tanh_f(cn);
        p.c_pool[rw.slot * H + u] = cn;
        const int par_out = (rw.flags & ROW_PARITY) ? 0 : 1;
        static_cast<__half*>(p.h_pool)[(par_out * NS + rw.slot) * H + u] = act_from_float(hn);
        if (rw.flags & ROW_LAST) {
          const size_t ro = (static_cast<size_t>(rw.flags >> 8) * p.res_layers + p.layer) * H + u;
          p.res_h[ro] = hn;
          p.res_c[ro] = cn;
        }
      }
      __syncwarp();
    }
  }
  if (tid == 0) phase_mark(p, 4);
  tc_fence_before();
  cluster_sync();  // B: both pair TMEMs drained before the cta_group::2 dealloc
  if (tid == 0) phase_mark(p, 5);
  if (p.dep_flag != nullptr || p.signal != nullptr) {
    __threadfence();
    __syncthreads();
    launch_done(p, p.sig_ctas);
  }
  if (warp == kMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256) : "memory");
  }
  if (p.span != nullptr) {
    __syncthreads();
    if (tid == 0) {
      __threadfence();
      const unsigned long long total = gridDim.x * gridDim.y * gridDim.z;
      if (atomicAdd(p.span + 1, 1ull) == total - 1) {
        const unsigned long long t0 = atomicExch(p.span, ~0ull);
        atomicExch(p.span + 1, 0ull);
        const unsigned long long dt = gtimer() - t0;
        atomicAdd(p.span_acc, dt);
        atomicAdd(p.span_acc + 1, 1ull);
        if (p.span_log != nullptr) *p.span_log = dt;
      }
    }
  }
}

}  // namespace

// Launch plan of the second CTA-pair design; *done = false if the task is not eligible.
cudaError_t launch_pair2(StepArgs a, const RowDesc* rows_host, cudaStream_t st, bool* done) {
  using namespace p2;
  *done = false;
  static int state = 0;
  const int smem_max = 227 * 1024;
  if (state == 0) {
    cudaError_t e = cudaFuncSetAttribute(cell_pair2_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_max);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(cell_pair2_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_max);
    if (e != cudaSuccess) {
      state = -1;
      cudaGetLastError();
      return cudaSuccess;
    }
    state = 1;
  }
  if (state < 0 || a.scratch == nullptr) return cudaSuccess;
  const int K = a.K0 + a.K1;
  const int tiles = a.H / a.U;
  static const int min_b = getenv("BM_PAIR_MIN") ? atoi(getenv("BM_PAIR_MIN")) : 129;
  if (a.epi != EPI_LSTM || a.U != 32 || tiles % 2 != 0 || K % 1024 != 0 || a.b > 512 || a.b < min_b) return cudaSuccess;
  const int S = 2;
  a.S = S;
  a.kslice = K / S;
  const int ctas1 = (tiles / 2) * 2 * S;
  int nblk = (ctas1 * 2 <= 148 && a.b > 32) ? 2 : 1;
  if (a.b > 256) nblk = 2;
  const int cpb = ((a.b + nblk - 1) / nblk + 31) & ~31;
  if (cpb > kScrCols) return cudaSuccess;
  nblk = (a.b + cpb - 1) / cpb;
  if (ctas1 * nblk > 148) return cudaSuccess;
  a.cpb = cpb;
  const int nhalf = cpb / 2;
  const int nk = a.kslice / kBK;
  static const int env_wcb = getenv("BM_P2_WCB") ? atoi(getenv("BM_P2_WCB")) : 2;
  static const int env_ws = getenv("BM_P2_WSLOTS") ? atoi(getenv("BM_P2_WSLOTS")) : 4;
  static const int env_xkb = getenv("BM_P2_XKB") ? atoi(getenv("BM_P2_XKB")) : 2;
  a.wcb = env_wcb;
  while (a.wcb > 1 && nk % a.wcb != 0) a.wcb >>= 1;
  a.xkb = env_xkb;
  while (a.xkb > 1 && nk % a.xkb != 0) a.xkb >>= 1;
  const int npad = cpb;  // cpb is a multiple of 32
  const int cper = (((npad + S - 1) / S) + 31) & ~31;
  const int cbuf_bytes = (cper * a.U * 4 + 1023) & ~1023;
  const int budget = smem_max - 1024 - kTail - cbuf_bytes;
  const int x_stage = nhalf * 128 * a.xkb;
  int wslots = std::min(env_ws, kWSlotsMax);
  int stages = 0;
  for (; wslots >= 2; --wslots) {
    stages = std::min(kXMax, (budget - wslots * a.wcb * kWBlk) / x_stage);
    if (stages >= 2) break;
  }
  if (stages < 2 || wslots < 2) return cudaSuccess;
  a.wslots = wslots;
  a.xring = stages * x_stage;
  const int region = wslots * a.wcb * kWBlk + a.xring;
  if (region < 8 * 32 * kTilePitch * 4) return cudaSuccess;   // epilogue tiles reuse the rings
  a.cbuf_off = kTail + region;
  const size_t need = 1024 + a.cbuf_off + cbuf_bytes;
  if (need > static_cast<size_t>(smem_max)) return cudaSuccess;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(2 * S, tiles / 2, nblk);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = need;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2 * S;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = a.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  *done = true;
  if (rows_host != nullptr) {
    static thread_local RowsParam<true> inline_rows;
    if (a.b > kMaxRowsInline) return cudaErrorInvalidValue;
    memcpy(inline_rows.r, rows_host, sizeof(RowDesc) * a.b);
    a.rows = nullptr;
    a.rows_flag = nullptr;
    return cudaLaunchKernelEx(&cfg, cell_pair2_kernel<true>, a, inline_rows);
  }
  if (a.rows == nullptr) return cudaErrorInvalidValue;
  return cudaLaunchKernelEx(&cfg, cell_pair2_kernel<false>, a, RowsParam<false>{0});
}

}  // namespace bm
