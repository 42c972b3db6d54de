// gather_bench.cu -- TMA row gather (cp.async.bulk.tensor.2d ... tile::gather4) vs cp.async
// gather of activation rows into a 128B-swizzled K-major stage, as the cell kernel needs it:
// npad rows (random row indices into a [R][H] bf16 table), nk K blocks of 64 columns.
// Checks the smem image against the expected SW128 layout and reports per-CTA cycles until
// the first stage landed and until all stages landed, with 148 CTAs (one per SM) running.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gather_bench gather_bench.cu
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <cudaTypedefs.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>

#include <vector>

#define CK(x)                                                                         \
  do {                                                                                \
    cudaError_t e_ = (x);                                                             \
    if (e_ != cudaSuccess) {                                                          \
      printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      exit(1);                                                                        \
    }                                                                                 \
  } while (0)

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint32_t b, int n) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(n));
}
__device__ __forceinline__ void expect_tx(uint32_t b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
}
__device__ __forceinline__ bool try_wait(uint32_t b, uint32_t par) {
  uint32_t ok;
  asm volatile("{\n.reg .pred p;\nmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\nselp.u32 %0,1,0,p;\n}"
               : "=r"(ok) : "r"(b), "r"(par) : "memory");
  return ok;
}
__device__ __forceinline__ void gather4(uint32_t dst, const CUtensorMap* map, int col, int r0, int r1, int r2,
                                        int r3, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(dst),
      "l"(map), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(bar)
      : "memory");
}

constexpr int kMaxStages = 8;

// mode 0: TMA gather4 issued by warp 0 (each lane one group of 4 rows); mode 1: cp.async by 256
// threads, one commit group per stage, hand-off after wait_group (lag = stages - 1) as in the
// cell kernel. out: per CTA {cycles to first stage, cycles to last stage}; img: CTA 0's stages.
__global__ void __launch_bounds__(256) gather_kernel(const __grid_constant__ CUtensorMap map,
                                                     const __nv_bfloat16* table, int H, const int* idx,
                                                     int npad, int nk, int mode, long long* out, int rot,
                                                     uint8_t* img, int reps) {
  extern __shared__ __align__(1024) uint8_t sm_raw[];
  uint8_t* sm = (uint8_t*)(((uintptr_t)sm_raw + 1023) & ~(uintptr_t)1023);
  __shared__ uint64_t full[kMaxStages];
  __shared__ int rows_s[256];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int* myidx = idx + blockIdx.x * npad;
  const int stage_bytes = npad * 128;
  long long t_first = 0, t_last = 0;
  for (int rep = 0; rep < reps; ++rep) {
    if (tid == 0) {
      for (int s = 0; s < nk; ++s) mbar_init(su32(&full[s]), (mode == 3 || mode == 4) ? 256 : 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const long long t0 = clock64();
    if (mode == 0) {
      if (warp == 0) {
        // row indices: one group of 4 per lane (npad <= 128 rows per pass of the warp)
        for (int s = 0; s < nk; ++s) {
          if (lane == 0) expect_tx(su32(&full[s]), stage_bytes);
          __syncwarp();
          for (int g = lane; g < npad / 4; g += 32) {
            const int4 r = reinterpret_cast<const int4*>(myidx)[g];
            gather4(su32(sm + s * stage_bytes + g * 512), &map, s * 64, r.x, r.y, r.z, r.w, su32(&full[s]));
          }
        }
      }
    } else if (mode == 2) {
      // LDG.128 into registers (a batch of stages per thread in flight), STS into the swizzled
      // stage, proxy fence, block barrier, one arrive per stage
      if (tid < npad) rows_s[tid] = max(myidx[tid], 0);
      __syncthreads();
      const int per = npad * 8 / 256 > 0 ? npad * 8 / 256 : 1;   // items per thread per stage
      const int batch = per >= 8 ? 2 : (per >= 4 ? 4 : 8);         // stages per batch (<= 16 items)
      for (int s0 = 0; s0 < nk; s0 += batch) {
        uint4 v[16];
        uint32_t dst[16];
#pragma unroll
        for (int j = 0; j < 16; ++j) {
          const int s = s0 + j / per, i = j % per;
          const int q = tid + 256 * i;
          v[j] = make_uint4(0, 0, 0, 0);
          dst[j] = 0xFFFFFFFFu;
          if (j < batch * per && s < nk && q < npad * 8) {
            const int row = q >> 3, ch = q & 7;
            const uint4* src = reinterpret_cast<const uint4*>(table + (size_t)rows_s[row] * H + s * 64 + ch * 8);
            asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v[j].x), "=r"(v[j].y), "=r"(v[j].z), "=r"(v[j].w) : "l"(src));
            dst[j] = su32(sm + s * stage_bytes) + row * 128 + ((ch ^ (row & 7)) << 4);
          }
        }
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if (dst[j] != 0xFFFFFFFFu)
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(dst[j]), "r"(v[j].x), "r"(v[j].y), "r"(v[j].z), "r"(v[j].w) : "memory");
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        asm volatile("bar.sync 1, 256;" ::: "memory");
        if (tid == 0)
          for (int s = s0; s < min(nk, s0 + batch); ++s)
            asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[s])) : "memory");
      }
    } else if (mode == 5 || mode == 6) {
      // mode 5: every stage's copies issued back to back, ONE commit group, wait_group 0,
      // then the hand-offs (no arrive.noinc between the copies)
      // mode 6: per-stage commit groups, hand-off of stage s after wait_group(nk-1-s)
      if (tid < npad) rows_s[tid] = max(myidx[tid], 0);
      __syncthreads();
      for (int s = 0; s < nk; ++s) {
        const uint32_t xs = su32(sm + s * stage_bytes);
        for (int q = tid; q < npad * 8; q += 256) {
          const int row = q >> 3, ch = q & 7;
          const __nv_bfloat16* src = table + (size_t)rows_s[row] * H + s * 64 + ch * 8;
          const uint32_t dst = xs + row * 128 + ((ch ^ (row & 7)) << 4);
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
        }
        if (mode == 6) asm volatile("cp.async.commit_group;" ::: "memory");
      }
      if (mode == 5) {
        asm volatile("cp.async.commit_group;" ::: "memory");
        asm volatile("cp.async.wait_group 0;" ::: "memory");
        asm volatile("bar.sync 1, 256;" ::: "memory");
        if (tid == 0)
          for (int s = 0; s < nk; ++s) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[s])) : "memory");
      } else {
        for (int d = 0; d < nk; ++d) {
          switch (nk - 1 - d) {
            case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
            case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
            case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
            case 3: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
            case 4: asm volatile("cp.async.wait_group 4;" ::: "memory"); break;
            case 5: asm volatile("cp.async.wait_group 5;" ::: "memory"); break;
            case 6: asm volatile("cp.async.wait_group 6;" ::: "memory"); break;
            default: asm volatile("cp.async.wait_group 7;" ::: "memory"); break;
          }
          asm volatile("bar.sync 1, 256;" ::: "memory");
          if (tid == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[d])) : "memory");
        }
      }
    } else if (mode == 4) {
      // one warp op = one row x 4 consecutive K blocks (512 contiguous bytes); stages in
      // groups of 4 K blocks, one arrive.noinc per group on each of its 4 barriers
      if (tid < npad) rows_s[tid] = max(myidx[tid], 0);
      __syncthreads();
      for (int s0 = 0; s0 < nk; s0 += 4) {
        const int g = min(4, nk - s0);
        for (int q = tid; q < npad * 8 * g; q += 256) {
          const int row = q / (8 * g), j = q % (8 * g), blk = j >> 3, ch = j & 7;
          const __nv_bfloat16* src = table + (size_t)rows_s[row] * H + (s0 + blk) * 64 + ch * 8;
          const uint32_t dst = su32(sm + (s0 + blk) * stage_bytes) + row * 128 + ((ch ^ (row & 7)) << 4);
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
        }
        for (int b = 0; b < g; ++b)
          asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s0 + b])) : "memory");
      }
    } else if (mode == 3) {
      // cp.async with one cp.async.mbarrier.arrive.noinc per thread per stage (count 256)
      if (tid < npad) rows_s[tid] = max(myidx[tid], 0);
      __syncthreads();
      for (int s = 0; s < nk; ++s) {
        const uint32_t xs = su32(sm + s * stage_bytes);
        for (int q = tid; q < npad * 8; q += 256) {
          const int row = ((q >> 3) + (rot ? (blockIdx.x / 4) * 8 : 0)) % npad, ch = q & 7;
          const __nv_bfloat16* src = table + (size_t)rows_s[row] * H + s * 64 + ch * 8;
          const uint32_t dst = xs + row * 128 + ((ch ^ (row & 7)) << 4);
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
        }
        asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
      }
    } else {
      if (tid < npad) rows_s[tid] = max(myidx[tid], 0);
      __syncthreads();
      const int lag = nk - 1;
      for (int s = 0; s < nk; ++s) {
        const uint32_t xs = su32(sm + s * stage_bytes);
        for (int q = tid; q < npad * 8; q += 256) {
          const int row = q >> 3, ch = q & 7;
          const __nv_bfloat16* src = table + (size_t)rows_s[row] * H + s * 64 + ch * 8;
          const uint32_t dst = xs + row * 128 + ((ch ^ (row & 7)) << 4);
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
        }
        asm volatile("cp.async.commit_group;" ::: "memory");
        if (s == lag) {
          for (int d = 0; d < nk; ++d) {
            // hand-off of stage d once its group landed (groups complete in order)
            const int pending = nk - 1 - d;
            switch (pending) {
              case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
              case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
              case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
              case 3: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
              case 4: asm volatile("cp.async.wait_group 4;" ::: "memory"); break;
              case 5: asm volatile("cp.async.wait_group 5;" ::: "memory"); break;
              case 6: asm volatile("cp.async.wait_group 6;" ::: "memory"); break;
              default: asm volatile("cp.async.wait_group 7;" ::: "memory"); break;
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
            asm volatile("bar.sync 1, 256;" ::: "memory");
            if (tid == 0) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&full[d])) : "memory");
          }
        }
      }
    }
    // consumer view: one thread waits the stages in order
    if (tid == 255) {
      for (int s = 0; s < nk; ++s) {
        while (!try_wait(su32(&full[s]), 0)) {
        }
        if (s == 0) t_first += clock64() - t0;
      }
      t_last += clock64() - t0;
    }
    __syncthreads();
    if (tid == 0)
      for (int s = 0; s < nk; ++s) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(su32(&full[s])));
    __syncthreads();
  }
  if (tid == 255) {
    out[2 * blockIdx.x] = t_first / reps;
    out[2 * blockIdx.x + 1] = t_last / reps;
  }
  if (blockIdx.x == 0)
    for (int i = tid; i < nk * stage_bytes; i += 256) img[i] = sm[i];
}

int main(int argc, char** argv) {
  const int R = argc > 2 ? atoi(argv[2]) : 65536, H = 1024;
  const int share = argc > 3 ? atoi(argv[3]) : 0;
  std::vector<__nv_bfloat16> h((size_t)R * H);
  for (size_t r = 0; r < (size_t)R; ++r)
    for (int c = 0; c < H; ++c) h[r * H + c] = __float2bfloat16((float)((r * 7 + c) % 251));
  __nv_bfloat16* d;
  CK(cudaMalloc(&d, h.size() * 2));
  CK(cudaMemcpy(d, h.data(), h.size() * 2, cudaMemcpyHostToDevice));
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q));
  const int box_rows = argc > 1 ? atoi(argv[1]) : 1;
  CUtensorMap map;
  cuuint64_t dims[2] = {(cuuint64_t)H, (cuuint64_t)R};
  cuuint64_t strides[1] = {(cuuint64_t)H * 2};
  cuuint32_t box[2] = {64, (cuuint32_t)box_rows};
  cuuint32_t es[2] = {1, 1};
  CUresult cr = enc(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, strides, box, es,
                    CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode (box rows %d): %d\n", box_rows, (int)cr);
  const int nsm = 148;
  int* didx;
  CK(cudaMalloc(&didx, nsm * 256 * 4));
  long long* dout;
  CK(cudaMalloc(&dout, nsm * 16));
  uint8_t* dimg;
  CK(cudaMalloc(&dimg, 8 * 256 * 128));
  CK(cudaFuncSetAttribute(gather_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  srand(1);
  for (int npad : {16, 64, 128, 256}) {
    std::vector<int> idx(nsm * 256);
    for (auto& x : idx) x = rand() % R;
    if (share) for (int c = 0; c < nsm; ++c) for (int r = 0; r < 256; ++r) idx[c * 256 + r] = idx[(c % 4) * 256 + r];
    for (int i = 0; i < 4; ++i) idx[i] = (i == 1) ? -1 : idx[i];  // a negative row: OOB -> zero fill?
    CK(cudaMemcpy(didx, idx.data(), idx.size() * 4, cudaMemcpyHostToDevice));
    const int nk = npad <= 64 ? 8 : (npad == 128 ? 8 : 6);
    for (int mode : {0, 1, 2, 3, 5}) {
      gather_kernel<<<nsm, 256, 200 * 1024>>>(map, d, H, didx, npad, nk, mode, dout, share == 2, dimg, 20);
      CK(cudaGetLastError());
      CK(cudaDeviceSynchronize());
      std::vector<long long> o(nsm * 2);
      CK(cudaMemcpy(o.data(), dout, o.size() * 8, cudaMemcpyDeviceToHost));
      std::vector<uint8_t> img(nk * npad * 128);
      CK(cudaMemcpy(img.data(), dimg, img.size(), cudaMemcpyDeviceToHost));
      // verify CTA 0: stage s, row r, 16-B chunk ch at r*128 + ((ch ^ (r&7))*16)
      int bad = 0, zero_ok = 1;
      for (int s = 0; s < nk; ++s)
        for (int r = 0; r < npad; ++r)
          for (int c = 0; c < 64; ++c) {
            const int ch = c / 8, w = c % 8;
            const size_t off = (size_t)s * npad * 128 + r * 128 + ((ch ^ (r & 7)) * 16) + w * 2;
            __nv_bfloat16 v;
            memcpy(&v, &img[off], 2);
            const int row = idx[r];
            if (row < 0) {
              if (__bfloat162float(v) != 0.f) zero_ok = 0;
              if (mode == 1) continue;
              continue;
            }
            const float want = (float)(((size_t)row * 7 + s * 64 + c) % 251);
            if (__bfloat162float(v) != want) ++bad;
          }
      double f = 0, l = 0;
      for (int i = 0; i < nsm; ++i) f += o[2 * i], l += o[2 * i + 1];
      printf("%-8s npad %3d nk %d: first stage %6.0f cyc, all %6.0f cyc (%.2f us @1.9GHz, %.1f GB/s/SM)  bad %d zero-fill %s\n",
             mode == 0 ? "gather4" : mode == 1 ? "cp.async" : mode == 2 ? "ldg+sts" : mode == 3 ? "cpa+arrv" : mode == 4 ? "cpa-row4" : mode == 5 ? "cpa-1grp" : "cpa-grps", npad, nk, f / nsm, l / nsm, l / nsm / 1900.0,
             (double)nk * npad * 128 / (l / nsm / 1.9), bad, mode == 0 ? (zero_ok ? "ok" : "NO") : "n/a");
    }
  }
  return 0;
}
