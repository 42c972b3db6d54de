// cell_step_simt.cu -- fp32 parity path of the batched cell step (north_star: "1e-5 for an
// fp32 path"), plus load-time weight packing, the completion signal and pool I/O kernels.
//
// The fp32 path computes exactly what cell_step_sm100.cu computes (same packed layout, same
// row descriptors, same fused epilogue) with fp32 FFMA on the SIMT cores: the tensor cores
// have no fp32 x fp32 mode, and TF32 would not meet 1e-5 after hundreds of recurrent steps.
#include <cuda_bf16.h>
#include <stdint.h>

#include "kernels.h"
#include "sm100_ptx.cuh"

namespace bm {
namespace {

constexpr int kTU = 32;   // hidden units per CTA
constexpr int kTC = 32;   // batch columns per CTA
constexpr int kTK = 32;   // K chunk
constexpr int kThreads = 256;

__device__ __forceinline__ float sigm(float x) { return 1.0f / (1.0f + expf(-x)); }

template <int EPI>
__device__ __forceinline__ const float* seg_src(const StepArgs& p, const RowDesc& r, int seg) {
  const size_t H = p.H;
  const size_t S = p.n_slots;
  const float* hp = static_cast<const float*>(p.h_pool);
  if constexpr (EPI == EPI_LSTM) {
    const int par = (r.flags & ROW_PARITY) ? 1 : 0;
    if (seg == 0) {
      if (p.h_lower != nullptr) return static_cast<const float*>(p.h_lower) + ((1 - par) * S + r.slot) * H;
      const int tok = r.a >= 0 ? r.a : p.tok[r.slot];
      return static_cast<const float*>(p.E) + static_cast<size_t>(tok) * H;
    }
    if (r.flags & ROW_FIRST) return nullptr;
    return hp + (par * S + r.slot) * H;
  } else if constexpr (EPI == EPI_LEAF) {
    return static_cast<const float*>(p.E) + static_cast<size_t>(r.a) * H;
  } else if constexpr (EPI == EPI_INTERNAL) {
    return hp + static_cast<size_t>(seg == 0 ? r.a : r.b) * H;
  } else {
    const int par = (r.flags & ROW_PARITY) ? 1 : 0;
    return hp + ((1 - par) * S + r.slot) * H;
  }
}

// Gate GEMM + fused epilogue. CTA tile: 32 units (all G gates of each) x 32 batch columns.
// Thread t: unit j = t % 32, columns 4 * (t / 32) .. +3.
// Device span of a launch (time_kernels, include/bm.h BM_K_SIMT): first CTA start .. last CTA
// done (%globaltimer), accumulated by the last CTA.
__device__ __forceinline__ unsigned long long simt_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ void span_begin(const StepArgs& p) {
  if (p.span != nullptr && threadIdx.x == 0) atomicMin(p.span, simt_now());
}
__device__ __forceinline__ void span_end(const StepArgs& p) {
  if (p.span == nullptr) return;
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned long long total = gridDim.x * gridDim.y * gridDim.z;
    if (atomicAdd(p.span + 1, 1ull) == total - 1) {
      const unsigned long long t0 = atomicExch(p.span, ~0ull);
      atomicExch(p.span + 1, 0ull);
      const unsigned long long dt = simt_now() - t0;
      atomicAdd(p.span_acc, dt);
      atomicAdd(p.span_acc + 1, 1ull);
      if (p.span_log != nullptr) *p.span_log = dt;
    }
  }
}

template <int EPI>
__device__ __forceinline__ void cell_step_simt_body(const StepArgs& p) {
  constexpr int G = EPI == EPI_LSTM ? 4 : EPI == EPI_LEAF ? 3 : 5;
  __shared__ float Ws[G * kTU][kTK + 1];
  __shared__ float Xs[kTC][kTK + 1];
  __shared__ const float* src[2][kTC];
  const int tid = threadIdx.x;
  const int j = tid % kTU;
  const int cg = tid / kTU;
  const int unit0 = blockIdx.x * kTU;
  const int col0 = blockIdx.y * kTC;
  const int K = p.K0 + p.K1;
  const float* W = static_cast<const float*>(p.W);
  if (tid < kTC) {
    const int c = col0 + tid;
    const float* s0 = nullptr;
    const float* s1 = nullptr;
    if (c < p.b) {
      const RowDesc r = p.rows[c];
      s0 = seg_src<EPI>(p, r, 0);
      if (p.K1 > 0) s1 = seg_src<EPI>(p, r, 1);
    }
    src[0][tid] = s0;
    src[1][tid] = s1;
  }
  float acc[G][4];
#pragma unroll
  for (int g = 0; g < G; ++g)
#pragma unroll
    for (int c = 0; c < 4; ++c) acc[g][c] = 0.f;
  __syncthreads();
  for (int k0 = 0; k0 < K; k0 += kTK) {
    const int seg = k0 >= p.K0 ? 1 : 0;
    const int kk = k0 - seg * p.K0;
    for (int e = tid; e < G * kTU * kTK; e += kThreads) {
      const int r = e / kTK, k = e % kTK;
      Ws[r][k] = W[static_cast<size_t>(unit0 * G + r) * K + k0 + k];
    }
    for (int e = tid; e < kTC * kTK; e += kThreads) {
      const int c = e / kTK, k = e % kTK;
      const float* s = src[seg][c];
      Xs[c][k] = s != nullptr ? s[kk + k] : 0.f;
    }
    __syncthreads();
#pragma unroll 8
    for (int k = 0; k < kTK; ++k) {
      float w[G];
#pragma unroll
      for (int g = 0; g < G; ++g) w[g] = Ws[j * G + g][k];
#pragma unroll
      for (int c = 0; c < 4; ++c) {
        const float x = Xs[cg * 4 + c][k];
#pragma unroll
        for (int g = 0; g < G; ++g) acc[g][c] = fmaf(w[g], x, acc[g][c]);
      }
    }
    __syncthreads();
  }
  const size_t H = p.H;
  const size_t NS = p.n_slots;
  const int u = unit0 + j;
  float* hp = static_cast<float*>(p.h_pool);
#pragma unroll
  for (int c = 0; c < 4; ++c) {
    const int col = col0 + cg * 4 + c;
    if (col >= p.b) continue;
    const RowDesc r = p.rows[col];
    float z[G];
#pragma unroll
    for (int g = 0; g < G; ++g) z[g] = acc[g][c] + p.bias[u * G + g];
    float hn, cn;
    if constexpr (EPI == EPI_LSTM) {
      const float cp = (r.flags & ROW_FIRST) ? 0.f : p.c_pool[r.slot * H + u];
      cn = sigm(z[1]) * cp + sigm(z[0]) * tanhf(z[2]);
      hn = sigm(z[3]) * tanhf(cn);
    } else if constexpr (EPI == EPI_LEAF) {
      cn = sigm(z[0]) * tanhf(z[2]);
      hn = sigm(z[1]) * tanhf(cn);
    } else {
      const float cl = p.c_pool[static_cast<size_t>(r.a) * H + u];
      const float cr = p.c_pool[static_cast<size_t>(r.b) * H + u];
      cn = sigm(z[0]) * tanhf(z[4]) + sigm(z[1]) * cl + sigm(z[2]) * cr;
      hn = sigm(z[3]) * tanhf(cn);
    }
    if constexpr (EPI == EPI_LSTM) {  // N1: rows of a request that emitted <eos> are no-ops
      if (p.dead != nullptr) {
        if ((r.flags & ROW_EOS) && p.dead[r.slot]) continue;
        if (p.layer == 0 && (r.flags & ROW_FIRST) && u == 0) p.dead[r.slot] = 0;  // slot's new owner
      }
    }
    p.c_pool[r.slot * H + u] = cn;
    const int par_out = (EPI == EPI_LSTM) ? ((r.flags & ROW_PARITY) ? 0 : 1) : 0;
    hp[(par_out * NS + r.slot) * H + u] = hn;
    if (r.flags & ROW_LAST) {
      const size_t ro = (static_cast<size_t>(r.flags >> 8) * p.res_layers + p.layer) * H + u;
      p.res_h[ro] = hn;
      p.res_c[ro] = cn;
    }
  }
}

// Projection + argmax, fp32. CTA: 128 vocab rows x 32 columns; per-column argmax packed into a
// 64-bit key (ordered value, inverted index) and reduced across CTAs with atomicMax; the last CTA
// publishes the tokens (same protocol as the tcgen05 kernel).
template <int EPI>
__global__ void __launch_bounds__(kThreads) cell_step_simt_kernel(const __grid_constant__ StepArgs p) {
  span_begin(p);
  cell_step_simt_body<EPI>(p);
  span_end(p);
}

__device__ __forceinline__ void proj_simt_body(const StepArgs& p) {
  __shared__ float Ws[128][kTK + 1];
  __shared__ float Xs[kTC][kTK + 1];
  __shared__ const float* src[kTC];
  __shared__ float best_v[8][kTC];
  __shared__ int best_i[8][kTC];
  __shared__ int is_last;
  const int tid = threadIdx.x;
  const int v0 = blockIdx.x * 128;
  const int col0 = blockIdx.y * kTC;
  const int K = p.H;
  const float* W = static_cast<const float*>(p.W);
  if (tid < kTC) {
    const int c = col0 + tid;
    src[tid] = c < p.b ? seg_src<EPI_PROJ>(p, p.rows[c], 0) : nullptr;
  }
  // thread: rows r = tid % 128 (this thread's vocab row), columns half = tid / 128 (16 cols)
  const int r = tid % 128;
  const int ch = tid / 128;
  float acc[16];
#pragma unroll
  for (int c = 0; c < 16; ++c) acc[c] = 0.f;
  __syncthreads();
  for (int k0 = 0; k0 < K; k0 += kTK) {
    for (int e = tid; e < 128 * kTK; e += kThreads) {
      const int rr = e / kTK, k = e % kTK;
      Ws[rr][k] = W[static_cast<size_t>(v0 + rr) * K + k0 + k];
    }
    for (int e = tid; e < kTC * kTK; e += kThreads) {
      const int c = e / kTK, k = e % kTK;
      Xs[c][k] = src[c] != nullptr ? src[c][k0 + k] : 0.f;
    }
    __syncthreads();
    for (int k = 0; k < kTK; ++k) {
      const float w = Ws[r][k];
#pragma unroll
      for (int c = 0; c < 16; ++c) acc[c] = fmaf(w, Xs[ch * 16 + c][k], acc[c]);
    }
    __syncthreads();
  }
  const float bias = p.bias[v0 + r];
  const int warp = tid / 32;
#pragma unroll
  for (int c = 0; c < 16; ++c) {
    const int col = col0 + ch * 16 + c;
    float z = acc[c] + bias;
    if (p.logits != nullptr && col < p.b) {
      const RowDesc rd = p.rows[col];
      const bool skip = (rd.flags & ROW_EOS) && p.dead != nullptr && p.dead[rd.slot];
      const int step = (rd.flags & ROW_EOS) ? row_step(rd.b) : rd.b;
      if (!skip) p.logits[(static_cast<size_t>(rd.flags >> 8) * p.max_decode + step) * p.V + v0 + r] = z;
    }
    int zi = v0 + r;
    for (int o = 16; o > 0; o >>= 1) {  // warp argmax, lowest index on ties
      const float ov = __shfl_xor_sync(0xffffffffu, z, o);
      const int oi = __shfl_xor_sync(0xffffffffu, zi, o);
      if (ov > z || (ov == z && oi < zi)) {
        z = ov;
        zi = oi;
      }
    }
    if ((tid & 31) == 0) {
      best_v[warp % 4][ch * 16 + c] = z;
      best_i[warp % 4][ch * 16 + c] = zi;
    }
  }
  __syncthreads();
  if (tid < kTC && col0 + tid < p.b) {
    float z = best_v[0][tid];
    int zi = best_i[0][tid];
    for (int w = 1; w < 4; ++w) {
      if (best_v[w][tid] > z || (best_v[w][tid] == z && best_i[w][tid] < zi)) {
        z = best_v[w][tid];
        zi = best_i[w][tid];
      }
    }
    uint32_t ob = __float_as_uint(z);
    ob = (ob & 0x80000000u) ? ~ob : (ob | 0x80000000u);
    atomicMax(p.amax + col0 + tid,
              (static_cast<unsigned long long>(ob) << 32) | (0xFFFFFFFFu - static_cast<uint32_t>(zi)));
  }
  __threadfence();
  __syncthreads();
  if (tid == 0) {
    const unsigned total = gridDim.x * gridDim.y;
    is_last = atomicAdd(p.done_ctas, 1u) == total - 1;
  }
  __syncthreads();
  if (is_last) {
    __threadfence();
    for (int c = tid; c < p.b; c += kThreads) {
      const RowDesc rd = p.rows[c];
      const unsigned long long key = atomicExch(p.amax + c, 0ull);
      const int y = static_cast<int>(0xFFFFFFFFu - static_cast<uint32_t>(key & 0xFFFFFFFFull));
      const bool eos_row = (rd.flags & ROW_EOS) && p.dead != nullptr;
      if (eos_row && p.dead[rd.slot]) continue;  // N1: masked step after the request's <eos>
      const int step = (rd.flags & ROW_EOS) ? row_step(rd.b) : rd.b;
      p.tok[rd.slot] = y;
      p.res_tok[static_cast<size_t>(rd.flags >> 8) * p.max_decode + step] = y;
      if (eos_row && y == row_eos(rd.b)) {  // <eos> emitted: later steps of the request are no-ops
        p.dead[rd.slot] = 1;
        p.eos_host[rd.flags >> 8] = step + 1;
        __threadfence_system();
      }
    }
    if (tid == 0) *p.done_ctas = 0;
  }
}

__global__ void __launch_bounds__(kThreads) proj_simt_kernel(const __grid_constant__ StepArgs p) {
  span_begin(p);
  proj_simt_body(p);
  span_end(p);
}

// fp32 paper layout [G*H][K] (row g*H + u) -> packed [H*G][K] (row u*G + g), bf16 or fp32.
__global__ void pack_rows_kernel(const float* __restrict__ src, void* dst, float* bias_dst,
                                 const float* __restrict__ bias_src, int G, int H, int K, int bf16) {
  const size_t n = static_cast<size_t>(G) * H * K;
  for (size_t e = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; e < n;
       e += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const size_t row = e / K, k = e % K;
    const int u = static_cast<int>(row / G), g = static_cast<int>(row % G);
    const float v = src[(static_cast<size_t>(g) * H + u) * K + k];
    if (bf16) static_cast<__nv_bfloat16*>(dst)[e] = __float2bfloat16_rn(v);
    else static_cast<float*>(dst)[e] = v;
    if (k == 0 && bias_dst != nullptr) bias_dst[row] = bias_src[static_cast<size_t>(g) * H + u];
  }
}

// fp32 paper layout -> bf16 "stage tiles" for the tcgen05 kernel: tile t of tile_rows packed
// rows (packed row n = u * G + g <-> paper row g * H + u; G = 1: identity, the projection), and
// 64-column K block kc, stored contiguously (tile_rows x 128 B) in the 128B-swizzled K-major
// layout the UMMA shared-memory descriptor expects: 16-byte chunk j of row r sits at chunk
// position j ^ (r % 8). One pipeline stage of the kernel is then ONE contiguous bulk copy.
// Tensor-core weight tiles: each weight is rounded to its bf16 value (the bf16-weight path) and
// stored as fp16 (exact for |w| >= 2^-17; see act_from_float in sm100_ptx.cuh).
__global__ void pack_tiles_kernel(const float* __restrict__ src, __half* __restrict__ dst,
                                  int G, int H, int K, int tile_rows, int n_rows) {
  const size_t n = static_cast<size_t>(n_rows) * K;
  const int kblocks = K / 64;
  for (size_t e = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; e < n;
       e += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const int row = static_cast<int>(e / K);   // packed row
    const int k = static_cast<int>(e % K);
    const int src_row = G == 1 ? row : (row % G) * H + row / G;
    const int t = row / tile_rows, r = row % tile_rows;
    const int kc = k / 64, j = (k % 64) / 8, el = k % 8;
    const size_t off = ((static_cast<size_t>(t) * kblocks + kc) * tile_rows + r) * 64 +
                       ((j ^ (r & 7)) * 8) + el;
    dst[off] = __float2half_rn(__bfloat162float(__float2bfloat16_rn(src[static_cast<size_t>(src_row) * K + k])));
  }
}

// fp32 -> the tensor-core path's activation type (fp16, act_from_float) or a plain fp32 copy.
__global__ void convert_kernel(const float* __restrict__ src, void* dst, size_t n, int act16) {
  for (size_t e = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; e < n;
       e += static_cast<size_t>(gridDim.x) * blockDim.x) {
    if (act16) static_cast<__half*>(dst)[e] = act_from_float(src[e]);
    else static_cast<float*>(dst)[e] = src[e];
  }
}

// Completion signal (§5): one thread bumps the counter that the host polls through
// zero-copy pinned memory; system-scope release so the host sees everything before it.
__global__ void signal_kernel(unsigned long long* counter, unsigned long long value) {
  __threadfence_system();
  ptx::signal_store(counter, value);
}

__global__ void pool_io_kernel(void* h_pool, float* c_pool, const int32_t* slots, int n, int H,
                               float* h_buf, float* c_buf, int write, int bf16) {
  const size_t total = static_cast<size_t>(n) * H;
  for (size_t e = blockIdx.x * static_cast<size_t>(blockDim.x) + threadIdx.x; e < total;
       e += static_cast<size_t>(gridDim.x) * blockDim.x) {
    const size_t i = e / H, u = e % H;
    const size_t at = static_cast<size_t>(slots[i]) * H + u;
    if (write) {
      if (h_buf) {
        if (bf16) static_cast<__half*>(h_pool)[at] = act_from_float(h_buf[e]);
        else static_cast<float*>(h_pool)[at] = h_buf[e];
      }
      if (c_buf) c_pool[at] = c_buf[e];
    } else {
      if (h_buf) h_buf[e] = bf16 ? __half2float(static_cast<__half*>(h_pool)[at])
                                 : static_cast<float*>(h_pool)[at];
      if (c_buf) c_buf[e] = c_pool[at];
    }
  }
}

}  // namespace

cudaError_t launch_cell_step_simt(const StepArgs& a, cudaStream_t st) {
  if (a.b <= 0) return cudaSuccess;
  if (a.epi == EPI_PROJ) {
    dim3 grid(a.W_rows / 128, (a.b + kTC - 1) / kTC);
    proj_simt_kernel<<<grid, kThreads, 0, st>>>(a);
    return cudaGetLastError();
  }
  dim3 grid(a.H / kTU, (a.b + kTC - 1) / kTC);
  switch (a.epi) {
    case EPI_LSTM: cell_step_simt_kernel<EPI_LSTM><<<grid, kThreads, 0, st>>>(a); break;
    case EPI_LEAF: cell_step_simt_kernel<EPI_LEAF><<<grid, kThreads, 0, st>>>(a); break;
    case EPI_INTERNAL: cell_step_simt_kernel<EPI_INTERNAL><<<grid, kThreads, 0, st>>>(a); break;
    default: return cudaErrorInvalidValue;
  }
  return cudaGetLastError();
}

cudaError_t launch_pack_rows(const float* src, void* dst, float* bias_dst, const float* bias_src,
                             int G, int H, int K, int bf16, cudaStream_t st) {
  pack_rows_kernel<<<1184, 256, 0, st>>>(src, dst, bias_dst, bias_src, G, H, K, bf16);
  return cudaGetLastError();
}

cudaError_t launch_pack_tiles(const float* src, void* dst, int G, int H, int K, int tile_rows,
                              int n_rows, cudaStream_t st) {
  pack_tiles_kernel<<<1184, 256, 0, st>>>(src, static_cast<__half*>(dst), G, H, K, tile_rows, n_rows);
  return cudaGetLastError();
}

cudaError_t launch_convert(const float* src, void* dst, size_t n, int bf16, cudaStream_t st) {
  convert_kernel<<<1184, 256, 0, st>>>(src, dst, n, bf16);
  return cudaGetLastError();
}

cudaError_t launch_signal(unsigned long long* counter, unsigned long long value, cudaStream_t st) {
  signal_kernel<<<1, 1, 0, st>>>(counter, value);
  return cudaGetLastError();
}

cudaError_t launch_pool_io(void* h_pool, float* c_pool, const int32_t* slots, int n, int H,
                           float* h_buf, float* c_buf, int write, int bf16, cudaStream_t st) {
  pool_io_kernel<<<296, 256, 0, st>>>(h_pool, c_pool, slots, n, H, h_buf, c_buf, write, bf16);
  return cudaGetLastError();
}

}  // namespace bm
