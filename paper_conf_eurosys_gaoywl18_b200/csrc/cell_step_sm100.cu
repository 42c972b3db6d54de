// cell_step_sm100.cu -- the hot path of cellular batching on B200 (sm_100a).
//
// ONE kernel = one batched cell step (one layer of an LSTM stack, a TreeLSTM leaf or internal
// step, or the Seq2Seq output projection + argmax) over a dynamically assembled set of rows
// that sit at different steps of different requests (§3.1-§3.2):
//
//   gather by slot (A6)  ->  [x ; h] . W^T on tcgen05 (A8)  ->  fused gates + state update
//   + scatter back to the pool by slot (A9)           (projection: + argmax, A10)
//
// The paper copies the batch into contiguous buffers ("gather", §4.3) and runs MXNet
// operators (cuBLAS GEMM + elementwise kernels) per cell. Here the gather is the operand load
// of the GEMM itself and the elementwise work is the GEMM's epilogue.
//
// Orientation ("swap-AB"): the tensor-core M dimension is the weight rows (gate outputs), the
// N dimension is the batch. A = packed weights (TMA, 128B swizzle), B = gathered activations
// (cp.async, 128B swizzle written by hand), D = fp32 accumulators in TMEM (lane = weight row,
// column = batch row).
//
// Grid = (S, H/U, ceil(b/256)); cluster = (S, 1, 1). The S CTAs of a cluster split K (the
// [x ; h] width 2h) into S slices of `kslice` and reduce their fp32 partial tiles through
// distributed shared memory in a FIXED order (s = 0..S-1), so the result of a row does not
// depend on which other rows share the task (batch invariance, P10).
//
// Roles: warps 0-7 gather the activation tile (and lane 0 of warp 0 issues the weight TMA);
// warp 8 allocates TMEM and issues tcgen05.mma from one lane. After the main loop warps 0-7
// move the accumulators TMEM -> smem, the cluster reduces, and warps 0-7 run the epilogue.
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "cell_common.cuh"
#include "kernels.h"
#include "sm100_ptx.cuh"

namespace bm {
namespace {
using namespace ptx;

constexpr int kMaxStages = 8;           // pipeline depth cap
constexpr int kTailBytes = 5120;        // barriers + TMEM slot (1 KB), row table [256] (4 KB)
constexpr int kBK = 64;                 // K elements per stage (128 B of bf16 = one SW128 atom)
constexpr int kProducerThreads = 256;   // warps 0-7: activation gather (cp.async)
constexpr int kMmaWarp = 8;             // warp 8: TMEM alloc + tcgen05.mma issue
constexpr int kTmaWarp = 9;             // warp 9: weight TMA stream
constexpr int kThreads = kProducerThreads + 64;
constexpr int kMaxCols = 256;           // batch columns per CTA (MMA N <= 256)
constexpr int kWStageBytes = 128 * 128; // 128 weight rows x 128 B
constexpr int kMaxS = 4;                // max split-K cluster size (K = 2h = 2048 -> 4 x 512)
// split-K partial tiles in shared memory: [column][gate row] fp32 with a 132-float pitch, so the
// epilogue's quad items (4 consecutive units = 16 floats of one column, 8 per column in a warp)
// hit 8 distinct 16-B bank groups per wavefront (a 128-float pitch puts every column of a warp
// on the same banks: 16-way conflicts)
constexpr int kPPitch = 132;

// Shared-memory plan (identical on host and device).
// The weight stream and the activation gather use separate rings:
//  * weights: contiguous pre-swizzled tiles, moved by the TMA engine in chunks of kWChunkKB
//    K-blocks (64 KB for 128-row tiles). The per-SM TMA engine completes bulk copies one at a
//    time, so its throughput grows with the chunk size (8 KB: 23 GB/s/SM, 16 KB: 42, 32 KB: 64,
//    64 KB: 85, tools/ingest_bench.cu) and not with the number in flight; a 2-chunk ring covers
//    the whole 512-wide K slice of a split-K CTA.
//  * activations: one 64-wide K block per stage, gathered by 256 threads with cp.async (the
//    LSU path runs beside the TMA engine).
constexpr int kWChunkMax = 4;           // K blocks per weight chunk, large tasks (64 KB chunks)
constexpr int kWRing = 2;               // weight chunks in the CTA-pair kernel's ring
constexpr int kWRingMax = 4;            // single-CTA kernel: up to 4 slots (StepArgs::wslots)
// Small tasks (npad <= 128) use 32 KB weight chunks and a 32 KB activation ring so the CTA fits
// in ~100 KB and two CTAs share an SM: under PDL the next launch's weight stream and gather
// overlap this launch's split-K epilogue. Larger tasks use 64 KB chunks and a 64 KB ring.
// Default plan; the launcher passes the chosen chunk size / ring size in StepArgs.
__host__ __device__ __forceinline__ int w_chunk_blocks(int) { return kWChunkMax; }
__host__ __device__ __forceinline__ int x_ring_bytes(int npad) { return npad <= 128 ? 32 * 1024 : 64 * 1024; }
__host__ __device__ __forceinline__ int x_stages_for(int npad, int xring) {
  const int n = xring / (npad * 128);
  return n < 2 ? 2 : (n > kMaxStages ? kMaxStages : n);
}
// weight ring + activation ring, reused after the main loop for the partial / logits tile
// wblk = one K block of the CTA's weight tile (tile rows x 128 B: 16 KB LSTM / projection,
// 12 KB leaf, 10 KB internal)
// xkb = K blocks per activation stage (one hand-off per stage)
__host__ __device__ __forceinline__ int region_bytes(int pcols, int wcb, int xring, int wblk, int xkb, int npad,
                                                     int wslots) {
  const int a = wslots * wcb * wblk + x_stages_for(npad * xkb, xring) * npad * xkb * 128;
  const int b = 129 * pcols * 4 + 4 * 128 * 4;  // partial / logits tile of pcols columns
  return a > b ? a : b;
}

// Gate nonlinearities: ex2/rcp approximations (MUFU), absolute error ~1e-7 -- far inside the
// bf16 path's 5e-3 bound -- without the IEEE-division / tanhf slow paths.
// ------------------------------------------------------------------ the kernel
template <int EPI, bool INL>
__global__ void __launch_bounds__(kThreads, 2)
    cell_step_sm100_kernel(const __grid_constant__ StepArgs p, const __grid_constant__ RowsParam<INL> rr) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int G = EPI == EPI_PROJ ? 1 : gates_of(EPI);
  const int U = p.U;
  const int tile_rows = EPI == EPI_PROJ ? 128 : G * U;
  const uint32_t rank = (EPI == EPI_PROJ) ? 0u : cluster_rank();
  const int col0 = blockIdx.z * kMaxCols;
  const int ncols = min(kMaxCols, p.b - col0);
  const int npad = (ncols + 15) & ~15;
  const int nk = p.kslice / kBK;
  const int k_begin = static_cast<int>(rank) * p.kslice;
  // activation stages: xkb consecutive K blocks each, ONE producer -> MMA hand-off per stage
  // (every mbarrier hand-off costs ~0.15-0.3 us of latency on the MMA's path, tools/pipe_bench.cu)
  const int xkb = p.xkb > 0 ? p.xkb : 1;
  const int nst = nk / xkb;
  // wcpa (LSTM): the stage also carries the weight K blocks (loaded by the producers)
  const bool wcpa = (EPI == EPI_LSTM || EPI == EPI_PROJ) && p.wcpa != 0;
  const int wblk_ = (EPI == EPI_PROJ ? 128 : G * U) * 128;
  const int kStages = wcpa ? max(2, min(kMaxStages, p.xring / ((npad * 128 + wblk_) * xkb)))
                    : p.max_stages > 0 ? min(p.max_stages, x_stages_for(npad * xkb, p.xring))
                                       : x_stages_for(npad * xkb, p.xring);
  const int wcb = p.wcb;                                  // ring slot capacity in K blocks
  const int kpc = min(wcb, nk);                           // K blocks per weight chunk
  const int n_chunks = (nk + kpc - 1) / kpc;
  const int wblk_bytes = tile_rows * 128;                 // one K block of this CTA's weight tile

  // shared memory: [tail: row sources + barriers][weight ring | activation ring]
  uint64_t* bars = reinterpret_cast<uint64_t*>(base);
  const uint32_t full0 = smem_u32(bars);                            // activation stage full
  const uint32_t empty0 = smem_u32(bars + kMaxStages);              // activation stage free
  const uint32_t wfull0 = smem_u32(bars + 2 * kMaxStages);          // weight chunk landed
  const uint32_t wempty0 = smem_u32(bars + 2 * kMaxStages + kWRingMax);  // weight chunk free
  const uint32_t done_bar = smem_u32(bars + 2 * kMaxStages + 2 * kWRingMax);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 2 * kMaxStages + 2 * kWRingMax + 1);
  // weight ring slots: slot w is filled by lane w of the TMA warp -- one thread's bulk copies
  // complete one after another (~0.6 us each), copies of different threads overlap
  // (tools/stream_bench.cu mode 8)
  const int wr = p.wslots > 0 ? p.wslots : kWRing;
  int* flag_last = reinterpret_cast<int*>(tmem_slot + 1);
  RowDesc* rtab = reinterpret_cast<RowDesc*>(base + 1024);  // this CTA's rows (col0 + c)
  uint8_t* smem = base + kTailBytes;                      // 1024-aligned (kTailBytes = 5 KB)
  uint8_t* w_ring = smem;                                 // wr x wcb x wblk
  uint8_t* x_st = smem + (wcpa ? 0 : wr * wcb * wblk_bytes);  // kStages x stage
  const int x_blk_bytes = npad * 128;                     // one K block of the activation tile
  const int x_stage_bytes = x_blk_bytes * xkb + (wcpa ? wblk_bytes * xkb : 0);

  // ---- setup (overlaps the previous launch's tail under PDL: touches no dependent data)
  if (tid == 0) phase_mark(p, 0);
  if (tid == 0 && p.tl != nullptr) atomicMax(p.tl, ~gtimer());
  if (tid == 0 && p.phase != nullptr) p.phase[(blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z)) * 64 + 14] = clock64();
  if (tid == 0) {
    for (int s = 0; s < kMaxStages; ++s) {
      mbar_init(full0 + 8 * s, kProducerThreads);  // every gather thread's cp.async arrive
      mbar_init(empty0 + 8 * s, 1);
    }
    for (int s = 0; s < kWRingMax; ++s) {
      mbar_init(wfull0 + 8 * s, 1);   // the TMA lane's arrive.expect_tx
      mbar_init(wempty0 + 8 * s, 1);
    }
    mbar_init(done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(tmem_slot)),
                 "r"(256)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  pdl_launch_dependents();  // the next launch may start its own setup + weight stream now
  if (tid == 0) phase_mark(p, 1);

  if (warp < 8) {
    // ================================================================ activation gather (A6)

    // Each producer thread owns fixed (row, 16-B chunk) items of every stage: item q = tid +
    // 256 i, row = q / 8, chunk = q % 8 (8 threads cover a row's 128-B K block, coalesced).
    // Row sources are resolved once into registers (no per-stage table lookups).
    constexpr int kItems = kMaxCols * 8 / kProducerThreads;  // 8
    const int n_items = (npad * 8 + kProducerThreads - 1 - tid) / kProducerThreads;
    const __nv_bfloat16* src0[kItems];
    const __nv_bfloat16* src1[kItems];
    uint32_t dst_off[kItems];
    RowDesc rd[kItems];
    // the launch's own rows (independent of earlier launches) into the smem table: one 16-byte
    // parameter load per thread (parameter loads miss the constant cache and serialise per
    // address: each row is read once and then shared through shared memory)
    // row load and dependency poll overlap: the row's global load is in flight while the chain
    // flag is polled (one round trip less on the launch's critical path)
    if constexpr (!INL) rows_wait(p);
    RowDesc r0{};
    if (tid < ncols) r0 = row_at(p, rr, col0 + tid);
    dep_wait(p);  // pool h/c and feed tokens are written by earlier launches
    if (tid < ncols) rtab[tid] = r0;
    named_bar(1, kProducerThreads);
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
      const int row = min((tid + i * kProducerThreads) >> 3, ncols - 1);
      rd[i] = rtab[row];
    }
    // device span starts when the launch's dependent work may begin (after the PDL wait)
    if (tid == 0 && p.span != nullptr) atomicMin(p.span, gtimer());
    if (tid == 0 && p.tl != nullptr) atomicMax(p.tl + 1, ~gtimer());
    if (tid == 0) phase_mark(p, 8);
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
      const int q = tid + i * kProducerThreads;
      const int row = q >> 3;
      const int ch = q & 7;
      dst_off[i] = row * 128 + ((ch ^ (row & 7)) << 4);
      src0[i] = nullptr;
      src1[i] = nullptr;
      if (i < n_items && row < ncols) {
        const __nv_bfloat16* a0 = seg_src<EPI>(p, rd[i], 0);
        const __nv_bfloat16* a1 = p.K1 > 0 ? seg_src<EPI>(p, rd[i], 1) : nullptr;
        src0[i] = a0 != nullptr ? a0 + ch * 8 : nullptr;
        src1[i] = a1 != nullptr ? a1 + ch * 8 : nullptr;
      }
    }
    if (tid == 0) phase_mark(p, 9);
    // A stage is handed to the MMA by the hardware: every producer thread's
    // cp.async.mbarrier.arrive.noinc fires once that thread's copies of the stage have landed
    // (full barrier count = 256), so no producer waits on its own copies.
    const __nv_bfloat16* dummy = static_cast<const __nv_bfloat16*>(p.E != nullptr ? p.E : p.h_pool);
    const bool no_reads = (p.experiment & 1) != 0;
    for (int st = 0; st < nst; ++st) {
      const int s = st % kStages;
      const int round = st / kStages;
      if (round > 0) mbar_wait_warp(empty0 + 8 * s, (round - 1) & 1);
      if (p.experiment & 4) {  // diagnostics: no gather at all, hand the stage over at once
        mbar_arrive(full0 + 8 * s);
        continue;
      }
      for (int j = 0; j < xkb; ++j) {
        const int k = k_begin + (st * xkb + j) * kBK;
        const int seg = k >= p.K0 ? 1 : 0;
        const int kk = k - seg * p.K0;
        const uint32_t xs = smem_u32(x_st + s * x_stage_bytes + j * x_blk_bytes);
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
          if (i < n_items) {
            const __nv_bfloat16* src = seg ? src1[i] : src0[i];
            if (src != nullptr && !no_reads) {
              cp_async_16(xs + dst_off[i], src + kk, 16);
            } else {
              cp_async_16(xs + dst_off[i], dummy, 0);  // zero fill
            }
          }
        }
        if (wcpa) {  // this K block's pre-swizzled weight tile (16 KB), 4 x 16 B per thread
          const uint8_t* wsrc = static_cast<const uint8_t*>(p.W) +
                                (static_cast<size_t>(blockIdx.y) * ((p.K0 + p.K1) / kBK) + k / kBK) * wblk_bytes;
          const uint32_t wdst = smem_u32(x_st + s * x_stage_bytes + xkb * x_blk_bytes + j * wblk_bytes);
          for (int i = tid; i < wblk_bytes / 16; i += kProducerThreads)
            cp_async_16(wdst + i * 16, wsrc + i * 16, 16);
        }
      }
      cp_async_arrive_noinc(full0 + 8 * s);
      if (tid == 0 && st == 0) phase_mark(p, 10);
      if (st == 0 && EPI != EPI_PROJ && p.pchunk == 0) {  // c rows after stage 0's hand-off
        const int cper_ = (ncols + p.S - 1) / p.S;        // (covered by the next arrive and
        const int clo_ = static_cast<int>(rank) * cper_;  // the epilogue's wait_all)
        prefetch_c<EPI>(p, rtab, clo_, max(0, min(ncols, clo_ + cper_) - clo_), blockIdx.y * U,
                        smem_u32(base + p.cbuf_off), tid, kProducerThreads);
      }
    }
  } else if (warp == kTmaWarp) {
    // ================================================================ weight stream (A7)
    // Weights are read-only: streaming starts before griddepcontrol.wait (PDL overlap).
    if (!wcpa && lane < wr) {
      const int kblocks = (p.K0 + p.K1) / kBK;
      const uint8_t* wsrc = static_cast<const uint8_t*>(p.W) +
                            (static_cast<size_t>(blockIdx.y) * kblocks + k_begin / kBK) * wblk_bytes;
      for (int c = lane; c < n_chunks; c += wr) {
        const int s = c % wr;
        const int round = c / wr;
        if (round > 0) mbar_wait(wempty0 + 8 * s, (round - 1) & 1);
        const int nblk = min(kpc, nk - c * kpc);
        const uint32_t bytes = static_cast<uint32_t>(nblk * wblk_bytes);
        if (p.experiment & 2) {  // diagnostics: no weight traffic
          mbar_arrive(wfull0 + 8 * s);
          continue;
        }
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(wfull0 + 8 * s),
                     "r"(bytes)
                     : "memory");
        // one chunk = nblk consecutive K blocks (contiguous in the stage-tile layout); block i
        // lands at i * wblk_bytes (a multiple of 1024: the 128B-swizzle atom stays aligned)
        bulk_load(smem_u32(w_ring + s * wcb * wblk_bytes),
                  wsrc + static_cast<size_t>(c) * kpc * wblk_bytes, bytes, wfull0 + 8 * s);
      }
    }
    __syncwarp();
  } else {
    // ================================================================ MMA issuer (A8)
    const uint32_t idesc = idesc_bf16(128, npad);
    for (int st = 0; st < nst; ++st) {
      const int s = st % kStages;
      mbar_wait_warp(full0 + 8 * s, (st / kStages) & 1);
      tc_fence_after();
      if (lane == 0 && st < 12) phase_mark(p, 16 + st);   // stage st at the MMA
      if (lane == 0 && st == 0) phase_mark(p, 6);
      if (lane == 0 && st == nst - 1) phase_mark(p, 7);
      if (lane == 0 && st == 1) phase_mark(p, 12);
      for (int j = 0; j < xkb; ++j) {
        const int kb = st * xkb + j;
        const int c = kb / kpc;
        const int ws = c % wr;
        if (!wcpa && kb % kpc == 0) {
          mbar_wait_warp(wfull0 + 8 * ws, (c / wr) & 1);
          tc_fence_after();
          if (lane == 0 && c < 4) phase_mark(p, 28 + c);  // weight chunk c at the MMA
          if (lane == 0 && kb == 0) phase_mark(p, 13);
        }
        if (lane == 0) {
          const uint64_t a =
              sdesc_sw128(wcpa ? smem_u32(x_st + s * x_stage_bytes + xkb * x_blk_bytes + j * wblk_bytes)
                               : smem_u32(w_ring + ws * wcb * wblk_bytes + (kb % kpc) * wblk_bytes));
          const uint64_t b = sdesc_sw128(smem_u32(x_st + s * x_stage_bytes + j * x_blk_bytes));
          if (!(p.experiment & 8)) {  // diagnostics bit 8: no MMA instructions
#pragma unroll
            for (int k = 0; k < kBK / 16; ++k) {
              mma_bf16(tmem, a + 2 * k, b + 2 * k, idesc, (kb | k) != 0 ? 1u : 0u);
            }
          }
          if (!wcpa && (kb % kpc == kpc - 1 || kb == nk - 1)) mma_commit(wempty0 + 8 * ws);
        }
        __syncwarp();
      }
      if (lane == 0) {
        mma_commit(empty0 + 8 * s);
        if (st == nst - 1) mma_commit(done_bar);
      }
      __syncwarp();
    }
  }
  if (warp < 8) {
    mbar_wait_warp(done_bar, 0);
    asm volatile("cp.async.wait_all;" ::: "memory");  // own c-prefetch copies (already landed)
    tc_fence_after();
    if (tid == 0) phase_mark(p, 2);
  }
  const int q = warp & 3;
  const int trow = 32 * q + lane;  // TMEM lane = tile (weight / vocab) row of this thread

  if constexpr (EPI == EPI_PROJ) {
    // ============================================================ projection + argmax (A10)
    float* P = reinterpret_cast<float*>(smem);  // [col][129]: reuses the drained stage ring
    constexpr int pitch = 129;
    // p.pchunk > 0: the logits tile goes through shared memory pchunk columns at a time (a
    // smaller footprint lets two CTAs share an SM, so all vocab tiles run in one wave)
    const int PC = p.pchunk > 0 ? min(p.pchunk, npad) : npad;
    const int v0 = blockIdx.y * 128;
    float pbias[4];  // this lane's vocab rows of the tile (lane + 32 k)
#pragma unroll
    for (int k = 0; k < 4; ++k) pbias[k] = p.bias[v0 + lane + 32 * k];
    for (int cc0 = 0; cc0 < npad; cc0 += PC) {
    if (cc0 > 0) __syncthreads();  // the previous chunk's column scans are done
    if (warp < 8) {
      for (int c0 = cc0 + (warp >> 2) * 32; c0 < cc0 + PC && c0 < npad; c0 += 64) {
        float v[32];
        tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0, v);
        const uint32_t Ps = smem_u32(P) + trow * 4;  // shared-space stores (not generic ST.E)
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (c0 + i < npad) st_shared_f32(Ps + (c0 - cc0 + i) * pitch * 4, v[i]);
      }
    }
    tc_fence_before();
    __syncthreads();
    if (tid == 0 && cc0 == 0) phase_mark(p, 3);
    const int chunk_cols = min(ncols, cc0 + PC) - cc0;
    if (chunk_cols >= 96) {
      // one thread per column: a serial scan of the tile's 128 vocab rows (strict '>' keeps
      // the lowest index among equal maxima, S9); every thread has a column at this width
      for (int c = cc0 + tid; c < min(ncols, cc0 + PC); c += kThreads) {
        const RowDesc r = rtab[c];
        float best = -INFINITY;
        int besti = 0;
        float* lg = nullptr;
        const bool masked = (r.flags & ROW_EOS) && p.dead != nullptr && p.dead[r.slot];
        if (p.logits != nullptr && !masked) {
          const int step = (r.flags & ROW_EOS) ? row_step(r.b) : r.b;
          lg = p.logits + (static_cast<size_t>(r.flags >> 8) * p.max_decode + step) * p.V + v0;
        }
        for (int i = 0; i < 128; ++i) {
          const float z = P[(c - cc0) * pitch + i] + p.bias[v0 + i];
          if (lg != nullptr) lg[i] = z;
          if (z > best) {
            best = z;
            besti = i;
          }
        }
        uint32_t ob = __float_as_uint(best);
        ob = (ob & 0x80000000u) ? ~ob : (ob | 0x80000000u);
        const unsigned long long key =
            (static_cast<unsigned long long>(ob) << 32) | (0xFFFFFFFFu - static_cast<uint32_t>(v0 + besti));
        atomicMax(p.amax + col0 + c, key);
      }
    } else {
      // narrow chunks: one warp per column: lane l scans vocab rows l, l + 32, l + 64, l + 96 (increasing, strict
      // '>' keeps its lowest index), then a shuffle reduction takes the larger value and, on equal
      // values, the lower index -- the same argmax (and lowest-index tie-break, S9) as a serial
      // scan over the 128 rows, with 4 instead of 128 dependent steps per column
      for (int c = cc0 + warp; c < min(ncols, cc0 + PC); c += kThreads / 32) {
        const RowDesc r = rtab[c];
        float* lg = nullptr;
        const bool masked = (r.flags & ROW_EOS) && p.dead != nullptr && p.dead[r.slot];
        if (p.logits != nullptr && !masked) {
          const int step = (r.flags & ROW_EOS) ? row_step(r.b) : r.b;
          lg = p.logits + (static_cast<size_t>(r.flags >> 8) * p.max_decode + step) * p.V + v0;
        }
        float best = -INFINITY;
        int besti = 0;
  #pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int i = lane + 32 * k;
          const float z = P[(c - cc0) * pitch + i] + pbias[k];
          if (lg != nullptr) lg[i] = z;
          if (z > best) {  // strict: keeps the lowest index among equal maxima
            best = z;
            besti = i;
          }
        }
  #pragma unroll
        for (int off = 16; off > 0; off >>= 1) {
          const float ob_ = __shfl_xor_sync(0xffffffffu, best, off);
          const int oi = __shfl_xor_sync(0xffffffffu, besti, off);
          if (ob_ > best || (ob_ == best && oi < besti)) {
            best = ob_;
            besti = oi;
          }
        }
        if (lane == 0) {
          uint32_t ob = __float_as_uint(best);
          ob = (ob & 0x80000000u) ? ~ob : (ob | 0x80000000u);
          const unsigned long long key =
              (static_cast<unsigned long long>(ob) << 32) | (0xFFFFFFFFu - static_cast<uint32_t>(v0 + besti));
          atomicMax(p.amax + col0 + c, key);
        }
      }
    }
    }  // column chunks
    __threadfence();
    __syncthreads();
    if (tid == 0) {
      const unsigned total = gridDim.x * gridDim.y * gridDim.z;
      const unsigned prev = atomicAdd(p.done_ctas, 1u);
      *flag_last = (prev == total - 1) ? 1 : 0;
    }
    __syncthreads();
    if (*flag_last) {  // last CTA: publish argmax -> feed token + emitted token, reset keys
      __threadfence();
      for (int c = tid; c < p.b; c += kThreads) {
        const RowDesc r = row_at(p, rr, c);
        const unsigned long long key = atomicExch(p.amax + c, 0ull);
        const int y = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(key & 0xFFFFFFFFull));
        const bool eos_row = (r.flags & ROW_EOS) && p.dead != nullptr;
        if (eos_row && p.dead[r.slot]) continue;  // N1: masked step after the request's <eos>
        const int step = (r.flags & ROW_EOS) ? row_step(r.b) : r.b;
        p.tok[r.slot] = y;
        p.res_tok[static_cast<size_t>(r.flags >> 8) * p.max_decode + step] = y;
        if (eos_row && y == row_eos(r.b)) {  // <eos> emitted: later steps of the request are no-ops
          p.dead[r.slot] = 1;
          p.eos_host[r.flags >> 8] = step + 1;
          __threadfence_system();
        }
      }
      __threadfence();
      __syncthreads();
      if (tid == 0) {
        *p.done_ctas = 0;
        __threadfence();
        if (p.dep_flag != nullptr) st_release_gpu(p.dep_flag, p.dep_seq);
        if (p.signal != nullptr) {  // completion signal (A12) fused into the last CTA
          __threadfence_system();
          signal_store(p.signal, p.sig_value);
        }
      }
    }
    if (tid == 0) phase_mark(p, 4);
    if (tid == 0) phase_mark(p, 5);
  } else {
    // ============================================================ split-K reduction + gates (A9)
    // Each CTA writes its fp32 partial tile into its own smem (P[col][row], fast local stores);
    // after the cluster barrier each CTA owns a 1/S slice of the batch columns and sums the S
    // partials of its slice with 16-byte DSMEM loads in the fixed order s = 0..S-1
    // (deterministic, independent of the batch's other rows). Posted scalar DSMEM stores
    // measured ~3x slower than these loads on B200.
    const int S = p.S;
    // exchange chunks (p.pchunk columns at a time; 0 = the whole tile): a chunk bounds the
    // partial tile's shared memory so two CTAs fit on an SM (BM_PCHUNK experiments)
    const bool chunked = p.pchunk > 0;  // launch-wide (the launcher then allocates no c prefetch)
    const int CW = chunked ? min(p.pchunk, npad) : npad;
    float* P = reinterpret_cast<float*>(smem);
    constexpr int pitch = 128;
    // P row of tile row n = u * G + g: gates padded to Gp = 4 (G <= 4) or 8 (G = 5) floats per
    // unit, so a unit's gate values are one (or two) aligned 16-byte vector(s) for the reduction
    constexpr int Gp = (EPI == EPI_INTERNAL) ? 8 : 4;
    const int prow = (trow / G) * Gp + trow % G;
    uint32_t peer[kMaxS];
#pragma unroll
    for (int s = 0; s < kMaxS; ++s) peer[s] = mapa(smem_u32(P), s < S ? s : 0);
    const int unit0 = blockIdx.y * U;
    const int prow0 = blockIdx.y * tile_rows;
    const size_t H = p.H;
    const size_t NS = p.n_slots;
    for (int cc0 = 0; cc0 < npad; cc0 += CW) {
    const int ccols = max(0, min(CW, ncols - cc0));
    if (cc0 > 0) cluster_sync();  // peers are done reading the previous chunk's partials
    if (warp < 8) {
      for (int c0 = cc0 + (warp >> 2) * 32; c0 < cc0 + CW && c0 < npad; c0 += 64) {
        float v[32];
        tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0, v);
        if (trow < tile_rows) {
          const uint32_t Ps = smem_u32(P) + prow * 4;  // shared-space stores (not generic ST.E)
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (c0 + i < npad) st_shared_f32(Ps + (c0 - cc0 + i) * pitch * 4, v[i]);
        }
      }
    }
    tc_fence_before();
    cluster_sync();  // A: every CTA's partial tile (chunk) is in its smem
    if (tid == 0 && cc0 == 0) phase_mark(p, 3);
    const int cper = (ccols + S - 1) / S;
    const int c_lo = static_cast<int>(rank) * cper;   // relative to the chunk
    const int my_cols = max(0, min(ccols, c_lo + cper) - c_lo);
    {
      // every warp takes part; each thread owns unit j of columns cl0, cl0 + step, ... and
      // handles two columns per iteration with all their loads issued up front (ILP: the
      // DSMEM round trip, not the arithmetic, bounds an iteration)
      const int ew = kThreads / U;  // columns per pass (LSTM/leaf U = 32: 10, internal U = 16: 20)
      const int j = tid % U;
      const int u = unit0 + j;
      float bias[5];
#pragma unroll
      for (int g = 0; g < 5; ++g) bias[g] = g < G ? p.bias[prow0 + j * G + g] : 0.f;
      const bool no_dsmem = (p.experiment & 32) != 0;  // diagnostics: own partial only
      const float* cbuf = reinterpret_cast<const float*>(base + p.cbuf_off);
      for (int cl = tid / U; cl < my_cols; cl += 2 * ew) {
        if (tid == 0 && cl / (2 * ew) < 16) phase_mark(p, 32 + cl / (2 * ew));
        const int nit = (cl + ew < my_cols) ? 2 : 1;
        float4 v[2][kMaxS], w[2][kMaxS];
        RowDesc r[2];
        float cin[2][2];
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (h < nit) {
            const uint32_t off = static_cast<uint32_t>(((c_lo + cl + h * ew) * pitch + j * Gp) * 4);
#pragma unroll
            for (int s = 0; s < kMaxS; ++s)
              if (s < S) {
                const uint32_t a = no_dsmem ? smem_u32(P) + off : peer[s] + off;
                v[h][s] = ld_cluster_v4(a);
                if (G == 5) w[h][s] = ld_cluster_v4(a + 16);
              }
            r[h] = (p.experiment & 16) ? RowDesc{0, 0, (c_lo + cl + h * ew) & 1023, 0}
                                       : rtab[cc0 + c_lo + cl + h * ew];
            cin[h][0] = cin[h][1] = 0.f;
            if (chunked) {  // no prefetch in chunked mode: c straight from the pool
              if constexpr (EPI == EPI_LSTM) {
                if (!(r[h].flags & ROW_FIRST)) cin[h][0] = p.c_pool[r[h].slot * H + u];
              } else if constexpr (EPI == EPI_INTERNAL) {
                cin[h][0] = p.c_pool[static_cast<size_t>(r[h].a) * H + u];
                cin[h][1] = p.c_pool[static_cast<size_t>(r[h].b) * H + u];
              }
            } else if constexpr (EPI == EPI_LSTM) {
              cin[h][0] = cbuf[(cl + h * ew) * U + j];
            } else if constexpr (EPI == EPI_INTERNAL) {
              cin[h][0] = cbuf[(cl + h * ew) * 2 * U + j];
              cin[h][1] = cbuf[(cl + h * ew) * 2 * U + U + j];
            }
          }
        }
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          if (h < nit) {
            float z[5];
#pragma unroll
            for (int g = 0; g < 5; ++g) z[g] = bias[g];
#pragma unroll
            for (int s = 0; s < kMaxS; ++s)  // fixed order s = 0..S-1 (batch invariance)
              if (s < S) {
                z[0] += v[h][s].x;
                z[1] += v[h][s].y;
                z[2] += v[h][s].z;
                if (G >= 4) z[3] += v[h][s].w;
                if (G == 5) z[4] += w[h][s].x;
              }
            float hn, cn;
            if constexpr (EPI == EPI_LSTM) {
              cn = sigm(z[1]) * cin[h][0] + sigm(z[0]) * tanh_f(z[2]);
              hn = sigm(z[3]) * tanh_f(cn);
            } else if constexpr (EPI == EPI_LEAF) {
              cn = sigm(z[0]) * tanh_f(z[2]);
              hn = sigm(z[1]) * tanh_f(cn);
            } else {
              cn = sigm(z[0]) * tanh_f(z[4]) + sigm(z[1]) * cin[h][0] + sigm(z[2]) * cin[h][1];
              hn = sigm(z[3]) * tanh_f(cn);
            }
            if (p.experiment & 256) {  // diagnostics: no gate math
              cn = z[0] + z[1];
              hn = z[2] + z[3];
            }
            if (p.experiment & 128) {  // diagnostics: no stores (keep the values live)
              if (cn == 12345.f && hn == 54321.f) p.c_pool[0] = cn;
              continue;
            }
            const RowDesc& rr_ = r[h];
            if constexpr (EPI == EPI_LSTM) {  // N1: rows of a request that emitted <eos> are no-ops
              if (p.dead != nullptr) {
                if ((rr_.flags & ROW_EOS) && p.dead[rr_.slot]) continue;
                if (p.layer == 0 && (rr_.flags & ROW_FIRST) && u == 0) p.dead[rr_.slot] = 0;
              }
            }
            p.c_pool[rr_.slot * H + u] = cn;
            const int par_out = (EPI == EPI_LSTM) ? ((rr_.flags & ROW_PARITY) ? 0 : 1) : 0;
            static_cast<__half*>(p.h_pool)[(par_out * NS + rr_.slot) * H + u] = act_from_float(hn);
            if (rr_.flags & ROW_LAST) {
              const size_t ro = (static_cast<size_t>(rr_.flags >> 8) * p.res_layers + p.layer) * H + u;
              p.res_h[ro] = hn;
              p.res_c[ro] = cn;
            }
          }
        }
      }
    }
    }  // chunk loop
    if (tid == 0) phase_mark(p, 4);
    cluster_sync();  // B: peers may read this CTA's partials until here
    if (tid == 0) phase_mark(p, 5);
    if (tid == 0 && p.phase != nullptr) p.phase[(blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z)) * 64 + 15] = clock64();
    if (p.dep_flag != nullptr || p.signal != nullptr) {
      __threadfence();
      __syncthreads();
      launch_done(p, p.sig_ctas);
    }
  }

  if (warp == kMmaWarp) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256)
                 : "memory");
  }
  if (p.tl != nullptr) {
    __syncthreads();
    if (tid == 0) {
      atomicMax(p.tl + 2, gtimer());
      atomicAdd(p.tl + 3, 1ull);
    }
  }
  if (p.span != nullptr) {  // device-side span: first CTA start .. last CTA end
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

template <int EPI>
cudaError_t launch_impl(StepArgs a, const RowDesc* rows_host, cudaStream_t st) {
  static bool configured = false;
  if (!configured) {
    cudaError_t e = cudaFuncSetAttribute(cell_step_sm100_kernel<EPI, true>,
                                         cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(cell_step_sm100_kernel<EPI, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                               227 * 1024);
    if (e != cudaSuccess) return e;
    configured = true;
  }
  const int cols = a.b < kMaxCols ? a.b : kMaxCols;
  const int npad = (cols + 15) & ~15;
  // ring plan (BM_WCB = K blocks per weight chunk, BM_XRING = activation ring KB: experiments)
  static const int env_wcb = getenv("BM_WCB") ? atoi(getenv("BM_WCB")) : 0;
  static const int env_xring = getenv("BM_XRING") ? atoi(getenv("BM_XRING")) : 0;
  // internal cells launch 64 tiles x 4 = 256 CTAs: their plan keeps two CTAs per SM (one
  // wave) -- the whole 80 KB slice + a 24 KB activation ring up to 64 rows, half the slice above
  const bool internal = EPI == EPI_INTERNAL;
  a.wcb = env_wcb > 0 ? env_wcb : (internal && npad > 64 ? 2 : w_chunk_blocks(npad));
  a.xring = env_xring > 0 ? env_xring * 1024 : (internal && npad <= 64 ? 24 * 1024 : x_ring_bytes(npad));
  // K blocks per activation stage: fewer, larger hand-offs where shared memory allows (the
  // 128-row LSTM / projection tiles keep a 128 KB weight slice + a 64 KB activation ring)
  static const int env_xkb = getenv("BM_XKB") ? atoi(getenv("BM_XKB")) : 0;
  a.xkb = 1;
  // two workers share the SMs (small_plan): 2 x 16 KB weight chunks, a <= 64 KB activation
  // ring and 128-column exchange chunks keep a CTA under half an SM's shared memory
  // (measured with two engines, tools/dual_bench.py)
  const bool small = a.small_plan && EPI == EPI_LSTM && env_wcb == 0;
  if (small) a.wcb = 1;
  if (!internal && EPI != EPI_LEAF) {
    if (npad <= 64) a.xkb = 4, a.xring = 2 * 4 * npad * 128;
    else if (npad <= 128) a.xkb = 2, a.xring = 2 * 2 * npad * 128;
    else if (small) a.xring = 32 * 1024;
    else if (env_wcb == 0) a.xkb = 2, a.wcb = 2, a.xring = 2 * 2 * npad * 128;  // 64 KB weight ring
  }
  // internal cells up to 32 rows: 2 K blocks per hand-off still leave 3 stages in the 24 KB
  // ring (span 15.3 -> 13.6 us at b = 1, 16.4 -> 14.8 at b = 32; at 64 rows the 2-stage
  // minimum would overflow the two-CTAs-per-SM budget: profiles/round1/internal_plans_r1l.txt)
  if (internal && npad <= 32 && env_wcb == 0 && env_xring == 0) a.xkb = 2;
  // leaf cells (256-wide K slice = 4 K blocks): the whole slice's activations in one hand-off up
  // to 64 rows, two up to 128 (span -8% at b <= 64, -5% at 128:
  // profiles/round1/leaf_plans_r1o.txt); a two-stage ring next to the 96 KB weight ring
  if (EPI == EPI_LEAF && npad <= 128 && env_wcb == 0 && env_xring == 0) {
    a.xkb = npad <= 64 ? 4 : 2;
    a.xring = 2 * a.xkb * npad * 128;
  }
  if (env_xkb > 0) a.xkb = env_xkb;
  // BM_WCPA=1: LSTM weights by cp.async inside the activation stages (as the CTA-pair kernel),
  // stages of xkb K blocks of (activations + 16 KB weights). Off by default here: this kernel's
  // 128 KB K slice already moves in two 64 KB bulk copies and the two plans measure the same
  // (tools/kbench.py, b = 16..256, within +-2%); the pair kernel's 32 KB chunks gain 10%.
  static const int env_wcpa = getenv("BM_WCPA") ? atoi(getenv("BM_WCPA")) : 0;
  a.wcpa = (EPI == EPI_LSTM && env_wcpa && !a.small_plan && env_wcb == 0) ? 1 : 0;
  if (a.wcpa) {
    a.xkb = npad <= 64 ? 4 : 2;
    if (env_xkb > 0) a.xkb = env_xkb;
  }
  // projection (BM_PROJ_SMALL, default on): cp.async weights in <= 107 KB of stages and the
  // logits tile through shared memory 128 columns at a time, so two CTAs share an SM and all
  // V/128 vocab tiles run in one wave instead of two
  static const int env_proj_small = getenv("BM_PROJ_SMALL") ? atoi(getenv("BM_PROJ_SMALL")) : 1;
  const bool proj_small = EPI == EPI_PROJ && env_proj_small && env_wcb == 0;
  if (proj_small) {
    a.wcpa = 1;
    a.xkb = 1;
  }
  // weight ring slots, one TMA lane each (bulk copies of one thread complete one at a time)
  a.wslots = kWRing;
  static const int env_wslots = getenv("BM_WSLOTS") ? atoi(getenv("BM_WSLOTS")) : 0;
  // projection up to 64 rows (BM_PROJ_TMA, default on): the 256 KB vocab tile through a
  // 4 x 16 KB TMA ring filled by four lanes (instead of the producers' cp.async, which fills
  // one stage at a time), two CTAs per SM (<= 113 KB); -1 us per launch at b <= 64, +1.7 us at
  // 128 (profiles/round2/kbench_wslots_r2o.log), so larger tasks keep the cp.async plan
  static const int env_proj_tma = getenv("BM_PROJ_TMA") ? atoi(getenv("BM_PROJ_TMA")) : 1;
  if (proj_small && env_proj_tma && npad <= 64) {
    a.wcpa = 0;
    a.wcb = 1;
    a.wslots = 4;
    a.xkb = npad <= 64 ? 2 : 1;
    a.xring = 2 * a.xkb * npad * 128;
  }
  if (env_wslots >= 1 && env_wslots <= kWRingMax) a.wslots = env_wslots;
  const int nk_all = a.kslice / kBK;
  if (EPI == EPI_PROJ) {
    if (a.xkb > 1 && (a.H / kBK) % a.xkb != 0) a.xkb = 1;
  } else if (nk_all % a.xkb != 0) {
    a.xkb = 1;
  }
  const int wblk = (EPI == EPI_PROJ ? 128 : gates_of(EPI) * a.U) * 128;
  const int S = EPI == EPI_PROJ ? 1 : a.S;
  // epilogue c-state prefetch: ceil(cols / S) columns x 128 B (LSTM 32 units, internal 2 x 16)
  static const int env_pchunk = getenv("BM_PCHUNK") ? atoi(getenv("BM_PCHUNK")) : 0;
  const int pchunk = env_pchunk > 0 ? env_pchunk : (a.small_plan && EPI == EPI_LSTM ? 128 : 0);
  a.pchunk = (EPI != EPI_PROJ && pchunk > 0 && pchunk % 64 == 0 && pchunk < npad) ? pchunk : 0;
  const int cbuf_bytes = (EPI == EPI_LSTM || EPI == EPI_INTERNAL) && a.pchunk == 0
                             ? (((cols + S - 1) / S) * (EPI == EPI_INTERNAL ? 2 : 1) * a.U * 4 + 1023) & ~1023
                             : 0;
  if (proj_small) a.pchunk = npad > 128 ? 128 : 0;
  if (a.wcpa) {
    const int stage = (npad * 128 + wblk) * a.xkb;
    const int budget = (proj_small ? 113 * 1024 : 227 * 1024) - 1024 - kTailBytes - cbuf_bytes;
    const int stages = std::min(kMaxStages, budget / stage);
    if (stages < 2) {
      a.wcpa = 0;  // does not fit: keep the TMA ring plan computed above
    } else {
      a.xring = stages * stage;
      const int ptile = 129 * (a.pchunk > 0 ? a.pchunk : npad) * 4 + 4 * 128 * 4;
      a.cbuf_off = kTailBytes + std::max(a.xring, ptile);
    }
  }
  if (!a.wcpa)
    a.cbuf_off = kTailBytes + region_bytes(a.pchunk > 0 ? a.pchunk : npad, a.wcb, a.xring, wblk, a.xkb, npad,
                                           a.wslots);
  const size_t smem = 1024 + a.cbuf_off + cbuf_bytes;
  if (smem > 227 * 1024) return cudaErrorInvalidConfiguration;
  const int tiles = EPI == EPI_PROJ ? a.W_rows / 128 : a.H / a.U;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(S, tiles, (a.b + kMaxCols - 1) / kMaxCols);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = S;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = a.pdl ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 2;
  if (rows_host != nullptr) {
    static thread_local RowsParam<true> inline_rows;
    if (a.b > kMaxRowsInline) return cudaErrorInvalidValue;
    memcpy(inline_rows.r, rows_host, sizeof(RowDesc) * a.b);
    a.rows = nullptr;
    a.rows_flag = nullptr;
    return cudaLaunchKernelEx(&cfg, cell_step_sm100_kernel<EPI, true>, a, inline_rows);
  }
  if (a.rows == nullptr) return cudaErrorInvalidValue;
  return cudaLaunchKernelEx(&cfg, cell_step_sm100_kernel<EPI, false>, a, RowsParam<false>{0});
}

// ================================================================== CTA-pair LSTM kernel
// cell_pair_kernel: the LSTM cell step (A6-A9) with tcgen05.mma.cta_group::2 -- two SMs of a
// TPC share one M = 256 MMA (each holds its own 128-row weight tile, A operand) and each
// gathers only HALF of the task's activation rows (B operand, N/2 rows per CTA; the MMA reads
// both halves), so the per-CTA gather -- the cp.async issue rate bounds it (tools/
// ldgsts_bench.cu, exp bits of cell_step_sm100_kernel) -- halves for the same weight tile.
//
// Grid (2S, tiles/2, column blocks), cluster (2S, 1, 1): cluster rank r = 2s + m, m = pair
// member (0 = leader: issues the MMAs), s = K slice. Each CTA's TMEM receives its own 128 rows
// x all N columns, so the epilogue (split-K DSMEM reduction over the S CTAs with the same m,
// fixed order -> batch invariant) is the single-CTA kernel's.
//
// Hand-offs: producers of each CTA arrive on their local `full` barrier; in the peer CTA the
// (otherwise idle) MMA warp forwards each completed local stage / weight chunk to the leader's
// pfull / pwfull barriers (remote mbarrier arrive, release.cluster). The leader's commits
// multicast to both CTAs' `empty` / `wempty` / `done` barriers.
namespace pairk {
constexpr int kStagesMax = 4;
}

template <bool INL, bool WCPA>
__global__ void __launch_bounds__(kThreads, 1)
    cell_pair_kernel(const __grid_constant__ StepArgs p, const __grid_constant__ RowsParam<INL> rr) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) &
                                             ~static_cast<uintptr_t>(1023));
  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  constexpr int G = 4;
  const int U = p.U;                                      // 32 units per 128-row tile
  const uint32_t crank = cluster_rank();
  const int pm = static_cast<int>(crank & 1u);            // pair member (0 = leader)
  const int ks = static_cast<int>(crank >> 1);            // K slice
  const int tile = 2 * blockIdx.y + pm;
  const int cpb = p.cpb;                                  // columns per block
  const int col0 = blockIdx.z * cpb;
  const int ncols = min(cpb, p.b - col0);
  const int npad = (ncols + 31) & ~31;                    // MMA N (both halves)
  const int nhalf = npad >> 1;                            // rows gathered by this CTA
  const int h0 = pm * nhalf;
  const int nk = p.kslice / kBK;
  const int k_begin = ks * p.kslice;
  const int xkb = p.xkb > 0 ? p.xkb : 1;
  const int nst = nk / xkb;
  const int x_blk_bytes = nhalf * 128;
  // WCPA: each stage also carries this CTA's xkb weight K blocks (16 KB each), loaded by the
  // producers' cp.async next to the activations (LSU path) instead of the TMA weight ring
  const int x_stage_bytes = x_blk_bytes * xkb + (WCPA ? xkb * 16384 : 0);
  const int kStages = min(pairk::kStagesMax, max(2, p.xring / x_stage_bytes));
  const int wcb = p.wcb;
  const int kpc = min(wcb, nk);
  const int n_chunks = (nk + kpc - 1) / kpc;
  constexpr int wblk_bytes = 128 * 128;
  const uint16_t pair_mask = static_cast<uint16_t>(3u << (crank & ~1u));
  // WCPA with p.wcpa == 2: the weight K blocks of a stage (contiguous in the packed layout) move
  // by ONE bulk copy of the otherwise idle TMA warp, issued as soon as the stage is free -- for
  // the first ring's worth before the dependency wait -- while the producers' cp.async carry only
  // the activation gather; the copy completes on the stage's full barrier (one more arrival +
  // its bytes)
  const bool wtma = WCPA && p.wcpa == 2;

  uint64_t* bars = reinterpret_cast<uint64_t*>(base);
  const uint32_t full0 = smem_u32(bars);                              // local producers
  const uint32_t empty0 = smem_u32(bars + pairk::kStagesMax);         // leader commit (multicast)
  const uint32_t pfull0 = smem_u32(bars + 2 * pairk::kStagesMax);     // peer stage forwarded
  const uint32_t wfull0 = smem_u32(bars + 3 * pairk::kStagesMax);     // local weight chunk
  const uint32_t wempty0 = smem_u32(bars + 3 * pairk::kStagesMax + kWRing);
  const uint32_t pwfull0 = smem_u32(bars + 3 * pairk::kStagesMax + 2 * kWRing);
  const uint32_t done_bar = smem_u32(bars + 3 * pairk::kStagesMax + 3 * kWRing);
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 3 * pairk::kStagesMax + 3 * kWRing + 1);
  RowDesc* rtab = reinterpret_cast<RowDesc*>(base + 1024);
  uint8_t* smem = base + kTailBytes;
  uint8_t* w_ring = smem;
  uint8_t* x_st = smem + (WCPA ? 0 : kWRing * wcb * wblk_bytes);

  if (tid == 0) phase_mark(p, 0);
  if (tid == 0) {
    for (int s = 0; s < pairk::kStagesMax; ++s) {
      mbar_init(full0 + 8 * s, kProducerThreads + (wtma ? 1 : 0));
      mbar_init(empty0 + 8 * s, 1);
      mbar_init(pfull0 + 8 * s, 1);
    }
    for (int s = 0; s < kWRing; ++s) {
      mbar_init(wfull0 + 8 * s, 1);
      mbar_init(wempty0 + 8 * s, 1);
      mbar_init(pwfull0 + 8 * s, 1);
    }
    mbar_init(done_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
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

  if (warp < 8) {
    // ================================================================ activation gather (A6)
    constexpr int kItems = 4;  // nhalf <= 128 rows x 8 chunks / 256 threads
    const int n_items = (nhalf * 8 + kProducerThreads - 1 - tid) / kProducerThreads;
    // row load and dependency poll overlap (one round trip less on the critical path)
    if constexpr (!INL) rows_wait(p);
    RowDesc r0{};
    if (tid < ncols) r0 = row_at(p, rr, col0 + tid);
    dep_wait(p);
    if (tid < ncols) rtab[tid] = r0;
    named_bar(1, kProducerThreads);
    const __nv_bfloat16* src0[kItems];
    const __nv_bfloat16* src1[kItems];
    uint32_t dst_off[kItems];
    RowDesc rd[kItems];
#pragma unroll
    for (int i = 0; i < kItems; ++i) rd[i] = rtab[min(h0 + ((tid + i * kProducerThreads) >> 3), ncols - 1)];
    if (tid == 0 && p.span != nullptr) atomicMin(p.span, gtimer());
    if (tid == 0) phase_mark(p, 8);
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
      const int q = tid + i * kProducerThreads;
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
        const uint32_t xs = smem_u32(x_st + s * x_stage_bytes + j * x_blk_bytes);
#pragma unroll
        for (int i = 0; i < kItems; ++i) {
          if (i < n_items) {
            const __nv_bfloat16* src = seg ? src1[i] : src0[i];
            if (src != nullptr) cp_async_16(xs + dst_off[i], src + kk, 16);
            else cp_async_16(xs + dst_off[i], dummy, 0);  // zero fill (h0 = 0, padding)
          }
        }
        if (WCPA && !wtma) {  // this CTA's pre-swizzled 16 KB weight tile of K block k
          const uint8_t* wsrc = static_cast<const uint8_t*>(p.W) +
                                (static_cast<size_t>(tile) * ((p.K0 + p.K1) / kBK) + k / kBK) * wblk_bytes;
          const uint32_t wdst = smem_u32(x_st + s * x_stage_bytes + xkb * x_blk_bytes + j * wblk_bytes);
#pragma unroll
          for (int i = 0; i < wblk_bytes / 16 / kProducerThreads; ++i)
            cp_async_16(wdst + (tid + i * kProducerThreads) * 16, wsrc + (tid + i * kProducerThreads) * 16, 16);
        }
      }
      cp_async_arrive_noinc(full0 + 8 * s);
      if (tid == 0 && st == 0) phase_mark(p, 10);
      if (st == 0) {  // the epilogue's c rows, after stage 0's hand-off (off the first MMA's
                      // path; covered by the next stage's arrive and the epilogue's wait_all):
                      // -0.6 us per launch at b = 256..512 against issuing them with stage 0
        const int cper_ = (ncols + p.S - 1) / p.S;
        const int clo_ = ks * cper_;
        prefetch_c<EPI_LSTM>(p, rtab, clo_, max(0, min(ncols, clo_ + cper_) - clo_), tile * U,
                             smem_u32(base + p.cbuf_off), tid, kProducerThreads);
      }
    }
  } else if (warp == kTmaWarp) {
    // ================================================================ weight stream (A7)
    if (wtma && lane == 0) {
      const int kblocks = (p.K0 + p.K1) / kBK;
      const uint8_t* wsrc =
          static_cast<const uint8_t*>(p.W) + (static_cast<size_t>(tile) * kblocks + k_begin / kBK) * wblk_bytes;
      const uint32_t bytes = static_cast<uint32_t>(xkb * wblk_bytes);
      for (int st = 0; st < nst; ++st) {
        const int s = st % kStages;
        const int round = st / kStages;
        if (round > 0) wait_bounded<false>(empty0 + 8 * s, (round - 1) & 1);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(full0 + 8 * s), "r"(bytes)
                     : "memory");
        bulk_load(smem_u32(x_st + s * x_stage_bytes + xkb * x_blk_bytes), wsrc + static_cast<size_t>(st) * bytes,
                  bytes, full0 + 8 * s);
      }
    }
    if (!WCPA && lane == 0) {
      const int kblocks = (p.K0 + p.K1) / kBK;
      const uint8_t* wsrc =
          static_cast<const uint8_t*>(p.W) + (static_cast<size_t>(tile) * kblocks + k_begin / kBK) * wblk_bytes;
      for (int c = 0; c < n_chunks; ++c) {
        const int s = c % kWRing;
        const int round = c / kWRing;
        if (round > 0) wait_bounded<false>(wempty0 + 8 * s, (round - 1) & 1);
        const int nblk = min(kpc, nk - c * kpc);
        const uint32_t bytes = static_cast<uint32_t>(nblk * wblk_bytes);
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(wfull0 + 8 * s), "r"(bytes)
                     : "memory");
        bulk_load(smem_u32(w_ring + s * wcb * wblk_bytes), wsrc + static_cast<size_t>(c) * kpc * wblk_bytes, bytes,
                  wfull0 + 8 * s);
      }
    }
    __syncwarp();
  } else if (pm == 0) {
    // ================================================================ MMA issuer (leader, A8)
    cluster_wait();
    const uint32_t idesc = idesc_bf16(256, npad);
    for (int st = 0; st < nst; ++st) {
      const int s = st % kStages;
      const uint32_t par = (st / kStages) & 1;
      if (lane == 0) {
        wait_bounded<false>(full0 + 8 * s, par);
        if (st < 4) phase_mark(p, 40 + st);
        wait_bounded<true>(pfull0 + 8 * s, par);
        if (st < 4) phase_mark(p, 44 + st);
      }
      __syncwarp();
      tc_fence_after();
      if (lane == 0 && st < 12) phase_mark(p, 16 + st);
      if (lane == 0 && st == 0) phase_mark(p, 6);
      if (lane == 0 && st == nst - 1) phase_mark(p, 7);
      for (int j = 0; j < xkb; ++j) {
        const int kb = st * xkb + j;
        const int c = kb / kpc;
        const int ws = c % kWRing;
        if (!WCPA && kb % kpc == 0) {
          const uint32_t wpar = (c / kWRing) & 1;
          if (lane == 0) {
            wait_bounded<false>(wfull0 + 8 * ws, wpar);
            if (c < 4) phase_mark(p, 48 + c);
            wait_bounded<true>(pwfull0 + 8 * ws, wpar);
            if (c < 4) phase_mark(p, 52 + c);
          }
          __syncwarp();
          tc_fence_after();
        }
        if (lane == 0) {
          const uint64_t a = sdesc_sw128(WCPA ? smem_u32(x_st + s * x_stage_bytes + xkb * x_blk_bytes + j * wblk_bytes)
                                              : smem_u32(w_ring + ws * wcb * wblk_bytes + (kb % kpc) * wblk_bytes));
          const uint64_t b = sdesc_sw128(smem_u32(x_st + s * x_stage_bytes + j * x_blk_bytes));
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k) mma_bf16_pair(tmem, a + 2 * k, b + 2 * k, idesc, (kb | k) != 0 ? 1u : 0u);
          if (!WCPA && (kb % kpc == kpc - 1 || kb == nk - 1)) mma_commit_pair(wempty0 + 8 * ws, pair_mask);
        }
        __syncwarp();
      }
      if (lane == 0) {
        mma_commit_pair(empty0 + 8 * s, pair_mask);
        if (st == nst - 1) mma_commit_pair(done_bar, pair_mask);
      }
      __syncwarp();
    }
  } else {
    // ================================================================ forwarder (peer)
    cluster_wait();
    const uint32_t lead = crank & ~1u;
    const uint32_t pfull_l = mapa(pfull0, lead);
    const uint32_t pwfull_l = mapa(pwfull0, lead);
    if (lane == 0) {
      for (int st = 0; st < nst; ++st) {
        const int s = st % kStages;
        wait_bounded<false>(full0 + 8 * s, (st / kStages) & 1);
        if (st < 4) phase_mark(p, 40 + st);
        fence_proxy_async();
        mbar_arrive_remote(pfull_l + 8 * s);
        for (int j = 0; j < xkb; ++j) {
          const int kb = st * xkb + j;
          if (!WCPA && kb % kpc == 0) {
            const int c = kb / kpc;
            const int ws = c % kWRing;
            wait_bounded<false>(wfull0 + 8 * ws, (c / kWRing) & 1);
            if (c < 4) phase_mark(p, 48 + c);
            mbar_arrive_remote(pwfull_l + 8 * ws);
          }
        }
      }
    }
    __syncwarp();
  }
  if (warp != kMmaWarp) cluster_wait();

  // ================================================================ epilogue (A9)
  wait_bounded_warp(done_bar, 0);
  if (warp < 8) asm volatile("cp.async.wait_all;" ::: "memory");  // own c-prefetch copies
  tc_fence_after();
  if (tid == 0) phase_mark(p, 2);
  const int q = warp & 3;
  const int trow = 32 * q + lane;
  const int S = p.S;
  const int cper = (ncols + S - 1) / S;
  float* P = reinterpret_cast<float*>(smem);
  constexpr int pitch = kPPitch;
  if (warp < 8) {  // shared-space stores (a generic pointer into smem compiles to ST.E)
    const uint32_t Ps = smem_u32(P) + trow * 4;
    for (int c0 = (warp >> 2) * 32; c0 < npad; c0 += 64) {
      float v[32];
      tmem_ld32(tmem + (static_cast<uint32_t>(32 * q) << 16) + c0, v);
#pragma unroll
      for (int i = 0; i < 32; ++i)
        if (c0 + i < npad) st_shared_f32(Ps + (c0 + i) * pitch * 4, v[i]);
    }
  }
  tc_fence_before();
  cluster_sync();  // A: every CTA's partial tile is in its smem
  if (tid == 0) phase_mark(p, 3);
  uint32_t peer[kMaxS];
#pragma unroll
  for (int s = 0; s < kMaxS; ++s) peer[s] = mapa(smem_u32(P), static_cast<uint32_t>(2 * (s < S ? s : 0) + pm));
  const int c_lo = ks * cper;
  const int my_cols = max(0, min(ncols, c_lo + cper) - c_lo);
  const int unit0 = tile * U;
  const int prow0 = tile * 128;
  const size_t H = p.H;
  const size_t NS = p.n_slots;
  {
    const int ew = kThreads / U;
    const int j = tid % U;
    const int u = unit0 + j;
    const float4 bias = *reinterpret_cast<const float4*>(p.bias + prow0 + j * G);
    const float* cbuf = reinterpret_cast<const float*>(base + p.cbuf_off);
    for (int cl = tid / U; cl < my_cols; cl += 2 * ew) {
      const int nit = (cl + ew < my_cols) ? 2 : 1;
      float4 v[2][kMaxS];
      RowDesc r[2];
      float cin[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (h < nit) {
          const uint32_t off = static_cast<uint32_t>(((c_lo + cl + h * ew) * pitch + j * G) * 4);
#pragma unroll
          for (int s = 0; s < kMaxS; ++s)  // own partial through the local shared-memory path
            if (s < S) v[h][s] = s == ks ? ld_shared_v4(smem_u32(P) + off) : ld_cluster_v4(peer[s] + off);
          r[h] = rtab[c_lo + cl + h * ew];
          cin[h] = cbuf[(cl + h * ew) * U + j];
        }
      }
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        if (h < nit) {
          float z0 = bias.x, z1 = bias.y, z2 = bias.z, z3 = bias.w;
#pragma unroll
          for (int s = 0; s < kMaxS; ++s)  // fixed order s = 0..S-1 (batch invariance)
            if (s < S) {
              z0 += v[h][s].x;
              z1 += v[h][s].y;
              z2 += v[h][s].z;
              z3 += v[h][s].w;
            }
          const float cn = sigm(z1) * cin[h] + sigm(z0) * tanh_f(z2);
          const float hn = sigm(z3) * tanh_f(cn);
          const RowDesc& rw = r[h];
          if (p.dead != nullptr) {  // N1: rows of a request that emitted <eos> are no-ops
            if ((rw.flags & ROW_EOS) && p.dead[rw.slot]) continue;
            if (p.layer == 0 && (rw.flags & ROW_FIRST) && u == 0) p.dead[rw.slot] = 0;
          }
          p.c_pool[rw.slot * H + u] = cn;
          const int par_out = (rw.flags & ROW_PARITY) ? 0 : 1;
          static_cast<__half*>(p.h_pool)[(par_out * NS + rw.slot) * H + u] = act_from_float(hn);
          if (rw.flags & ROW_LAST) {
            const size_t ro = (static_cast<size_t>(rw.flags >> 8) * p.res_layers + p.layer) * H + u;
            p.res_h[ro] = hn;
            p.res_c[ro] = cn;
          }
        }
      }
    }
  }
  if (tid == 0) phase_mark(p, 4);
  tc_fence_before();
  cluster_sync();  // B: peers may read this CTA's partials until here; both pair TMEMs drained
  if (tid == 0) phase_mark(p, 5);
  if (p.dep_flag != nullptr || p.signal != nullptr) {
    __threadfence();
    __syncthreads();
    launch_done(p, p.sig_ctas);
  }
  if (warp == kMmaWarp) {
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

// Launch plan of the pair kernel; returns false if the task is not eligible (caller falls back).
// S = 4 (512-wide K slices, clusters of 8) for small tasks when 16 such clusters are
// co-resident, else S = 2 (1024-wide slices, clusters of 4); column blocks of <= 256 so a
// task runs as <= 2 blocks (<= 128 CTAs, one wave).
template <bool INL>
cudaError_t launch_pair(StepArgs a, const RowDesc* rows_host, cudaStream_t st, bool* done) {
  *done = false;
  static int state = 0;  // 0 unknown, 1 usable, -1 not usable
  static int max_clusters8 = 0;
  const int smem = 227 * 1024;
  if (state == 0) {
    cudaError_t e = cudaFuncSetAttribute(cell_pair_kernel<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(cell_pair_kernel<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(cell_pair_kernel<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e == cudaSuccess)
      e = cudaFuncSetAttribute(cell_pair_kernel<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    if (e != cudaSuccess) {
      state = -1;
      cudaGetLastError();
      return cudaSuccess;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(8, 16, 1);
    cfg.blockDim = dim3(kThreads);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 8;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    if (cudaOccupancyMaxActiveClusters(&max_clusters8, cell_pair_kernel<false, false>, &cfg) != cudaSuccess) {
      max_clusters8 = 0;
      cudaGetLastError();
    }
    state = 1;
  }
  if (state < 0) return cudaSuccess;
  const int K = a.K0 + a.K1;
  const int tiles = a.H / a.U;
  // measured (tools/kbench.py, cp.async weights): the pair kernel wins from 129 rows up (b =
  // 160 / 192 / 256: 19.4 / 19.9 / 21.0 vs 20.1 / 21.2 / 23.5 us), ties at 128 and loses below
  // (b = 64: 17.9 vs 16.4 us) -- BM_PAIR_MIN overrides the cut
  static const int min_b = getenv("BM_PAIR_MIN") ? atoi(getenv("BM_PAIR_MIN")) : 129;
  if (a.epi != EPI_LSTM || a.U != 32 || tiles % 2 != 0 || K % 1024 != 0 || a.b > 512 || a.b < min_b)
    return cudaSuccess;
  static const int env_s = getenv("BM_PAIR_S") ? atoi(getenv("BM_PAIR_S")) : 0;
  int S = (a.b <= 128 && max_clusters8 >= tiles / 2) ? 4 : 2;
  if (env_s == 2 || env_s == 4) S = env_s;
  if (S == 4 && max_clusters8 < tiles / 2) S = 2;
  if (K / S > 1024 || (K / S) % 256 != 0) return cudaSuccess;
  a.S = S;
  a.kslice = K / S;
  // column blocks: two blocks when that keeps one wave (tiles/2 x 2S x blocks <= 148 CTAs)
  const int ctas1 = (tiles / 2) * 2 * S;
  int nblk = (ctas1 * 2 <= 148 && a.b > 32) ? 2 : 1;
  if (a.b > 256) nblk = 2;
  int cpb = ((a.b + nblk - 1) / nblk + 31) & ~31;
  if (cpb > 256) return cudaSuccess;
  nblk = (a.b + cpb - 1) / cpb;
  if (ctas1 * nblk > 148) return cudaSuccess;
  a.cpb = cpb;
  const int nhalf = cpb / 2;
  const int nk = a.kslice / kBK;
  // rings: weights 2 x 32 KB (or the whole 128 KB slice when it fits), activations up to 4
  // stages of xkb K blocks
  static const int env_wcb = getenv("BM_PAIR_WCB") ? atoi(getenv("BM_PAIR_WCB")) : 0;
  static const int env_xkb = getenv("BM_PAIR_XKB") ? atoi(getenv("BM_PAIR_XKB")) : 0;
  // weights by cp.async in the activation stages (default): the per-SM TMA engine completes
  // bulk copies one at a time, the LSU path keeps more bytes in flight (-10% per step at
  // b = 288..512, tools/kbench.py); BM_PAIR_WCPA=0 restores the TMA weight ring
  static const int wcpa = getenv("BM_PAIR_WCPA") ? atoi(getenv("BM_PAIR_WCPA")) : 1;
  a.wcb = 2;
  a.xkb = env_xkb > 0 ? env_xkb : (wcpa ? 2 : 4);
  while (a.xkb > 1 && nk % a.xkb != 0) a.xkb >>= 1;
  int xstage = nhalf * 128 * a.xkb + (wcpa ? 16384 * a.xkb : 0);
  if (wcpa) a.wcb = 0;  // no TMA weight ring
  // the stage's weight part by one bulk copy of the TMA warp (a.wcpa = 2; BM_PAIR_WTMA=0: by the
  // producers' cp.async): -0.1..-0.2 us per launch at b = 192..512 (profiles/round2/wtma_r2.log)
  static const int wtma = getenv("BM_PAIR_WTMA") ? atoi(getenv("BM_PAIR_WTMA")) : 1;
  a.wcpa = wcpa ? (wtma ? 2 : 1) : 0;
  const int budget = smem - 1024 - kTailBytes - ((((cpb + S - 1) / S) * a.U * 4 + 1023) & ~1023);
  if (!wcpa && nk * 16 * 1024 + 2 * xstage <= budget && nk <= 8) a.wcb = nk / 2;  // whole slice resident
  if (!wcpa && env_wcb > 0) a.wcb = env_wcb;
  int stages = (budget - kWRing * a.wcb * 16 * 1024) / xstage;
  stages = stages > pairk::kStagesMax ? pairk::kStagesMax : stages;
  if (stages < 2) return cudaSuccess;
  a.xring = stages * xstage;
  const int region = kWRing * a.wcb * 16 * 1024 + a.xring;
  const int pbytes = cpb * kPPitch * 4;
  a.cbuf_off = kTailBytes + (region > pbytes ? region : pbytes);
  const size_t need = 1024 + a.cbuf_off + ((((cpb + S - 1) / S) * a.U * 4 + 1023) & ~1023);
  if (need > static_cast<size_t>(smem)) return cudaSuccess;
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
  if constexpr (INL) {
    static thread_local RowsParam<true> inline_rows;
    memcpy(inline_rows.r, rows_host, sizeof(RowDesc) * a.b);
    a.rows = nullptr;
    a.rows_flag = nullptr;
    return wcpa ? cudaLaunchKernelEx(&cfg, cell_pair_kernel<true, true>, a, inline_rows)
                : cudaLaunchKernelEx(&cfg, cell_pair_kernel<true, false>, a, inline_rows);
  } else {
    return wcpa ? cudaLaunchKernelEx(&cfg, cell_pair_kernel<false, true>, a, RowsParam<false>{0})
                : cudaLaunchKernelEx(&cfg, cell_pair_kernel<false, false>, a, RowsParam<false>{0});
  }
}

}  // namespace

cudaError_t launch_cell_step_sm100(const StepArgs& a0, const RowDesc* rows_host, cudaStream_t st, int* kclass) {
  if (a0.b <= 0) return cudaSuccess;
  StepArgs a = a0;
  // kernel classes (include/bm.h BM_K_*): 0 pair LSTM, 1 LSTM, 2 leaf, 3 internal, 4 projection
  auto cls = [&](int k) {
    if (kclass != nullptr) *kclass = k;
    a.span_acc = a0.span_acc != nullptr ? a0.span_acc + 2 * k : nullptr;
  };
  static const int use_pair = getenv("BM_PAIR") ? atoi(getenv("BM_PAIR")) : 1;
  // second pair design (cell_pair_sm100.cu): bitwise equal, slower as measured (BM_PAIR2=1)
  static const int use_pair2 = getenv("BM_PAIR2") ? atoi(getenv("BM_PAIR2")) : 0;
  if (use_pair && use_pair2 && a.epi == EPI_LSTM && !a.small_plan) {  // second CTA-pair design
    bool done = false;
    cls(0);
    cudaError_t e = (rows_host != nullptr && a.b > kMaxRowsInline) ? cudaSuccess : launch_pair2(a, rows_host, st, &done);
    if (done || e != cudaSuccess) return e;
  }
  if (use_pair && a.epi == EPI_LSTM && !a.small_plan) {  // CTA-pair path (falls through if not eligible)
    bool done = false;
    cls(0);
    cudaError_t e = rows_host != nullptr ? (a.b <= kMaxRowsInline ? launch_pair<true>(a, rows_host, st, &done)
                                                                   : cudaSuccess)
                                         : launch_pair<false>(a, rows_host, st, &done);
    if (done || e != cudaSuccess) return e;
  }
  switch (a.epi) {
    case EPI_LSTM: cls(1); return launch_impl<EPI_LSTM>(a, rows_host, st);
    case EPI_LEAF: cls(2); return launch_impl<EPI_LEAF>(a, rows_host, st);
    case EPI_INTERNAL: cls(3); return launch_impl<EPI_INTERNAL>(a, rows_host, st);
    case EPI_PROJ: cls(4); return launch_impl<EPI_PROJ>(a, rows_host, st);
  }
  return cudaErrorInvalidValue;
}

}  // namespace bm
