// latency_bench.cu -- dependent global-load latency (pointer chase, one thread) for a working
// set that fits L1/L2 or spills to HBM; cycles per load (clock64) and ns (globaltimer).
#include <cstdio>
#include <cuda_runtime.h>
#include <vector>
__global__ void chase(const unsigned* __restrict__ next, int steps, unsigned long long* out, int volatile_ld) {
  unsigned i = 0;
  for (int s = 0; s < 2048; ++s) i = next[i];  // warm
  unsigned long long t0, t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  long long c0 = clock64();
  if (volatile_ld) {
    for (int s = 0; s < steps; ++s) asm volatile("ld.volatile.global.u32 %0, [%1];" : "=r"(i) : "l"(next + i));
  } else {
    for (int s = 0; s < steps; ++s) asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(i) : "l"(next + i));
  }
  long long c1 = clock64();
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  out[0] = (c1 - c0) / steps;
  out[1] = (t1 - t0) * 1000 / steps;  // ps per load
  out[2] = i;
}
int main() {
  unsigned long long* d;
  cudaMalloc(&d, 64);
  for (size_t bytes : {size_t(64) << 10, size_t(8) << 20, size_t(64) << 20, size_t(1) << 30}) {
    const size_t n = bytes / 4;
    std::vector<unsigned> h(n);
    // random cycle with 128 B stride granularity (each hop a new line)
    const size_t lines = n / 32;
    std::vector<unsigned> perm(lines);
    for (size_t i = 0; i < lines; ++i) perm[i] = i;
    unsigned long long s = 88172645463325252ull;
    for (size_t i = lines - 1; i > 0; --i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; size_t j = s % (i + 1); unsigned t = perm[i]; perm[i] = perm[j]; perm[j] = t; }
    for (size_t i = 0; i < lines; ++i) h[perm[i] * 32] = perm[(i + 1) % lines] * 32;
    unsigned* g;
    cudaMalloc(&g, bytes);
    cudaMemcpy(g, h.data(), bytes, cudaMemcpyHostToDevice);
    for (int vol = 0; vol < 2; ++vol) {
      chase<<<1, 1>>>(g, 4096, d, vol);
      unsigned long long o[3];
      cudaMemcpy(o, d, 24, cudaMemcpyDeviceToHost);
      printf("working set %8zu KB  %s: %4llu cycles/load  %7.1f ns/load\n", bytes >> 10, vol ? "ld.volatile" : "ld.cg      ", o[0], o[1] / 1000.0);
    }
    cudaFree(g);
  }
  return 0;
}
