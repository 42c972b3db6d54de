// launch_bench.cu -- host cost of cudaLaunchKernelEx for the cell kernel's launch shapes:
// grid (4, 32, 1) x 320 threads, with / without a cluster dimension (4, 1, 1), with / without
// programmatic stream serialization, with a small (512 B) or large (8.5 KB) parameter block,
// with / without 200 KB of dynamic shared memory.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o launch_bench launch_bench.cu
#include <chrono>
#include <cstdio>
#include <cuda_runtime.h>

struct Small { char b[512]; };
struct Big { char b[8704]; };

template <class P>
__global__ void k(const __grid_constant__ P p) {
  if (threadIdx.x == 0 && p.b[blockIdx.x] == 123) printf("x");
}

template <class P>
double run(int cluster, int pdl, int smem, int n) {
  P p{};
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(4, 32, 1);
  cfg.blockDim = dim3(320);
  cfg.dynamicSmemBytes = smem;
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (cluster) {
    attr[na].id = cudaLaunchAttributeClusterDimension;
    attr[na].val.clusterDim.x = 4;
    attr[na].val.clusterDim.y = 1;
    attr[na].val.clusterDim.z = 1;
    ++na;
  }
  if (pdl) {
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na].val.programmaticStreamSerializationAllowed = 1;
    ++na;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  cudaFuncSetAttribute(k<P>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  for (int i = 0; i < 20; ++i) cudaLaunchKernelEx(&cfg, k<P>, p);
  cudaStreamSynchronize(st);
  const auto t0 = std::chrono::steady_clock::now();
  for (int i = 0; i < n; ++i) cudaLaunchKernelEx(&cfg, k<P>, p);
  const auto t1 = std::chrono::steady_clock::now();
  cudaStreamSynchronize(st);
  const auto t2 = std::chrono::steady_clock::now();
  cudaStreamDestroy(st);
  const double host = std::chrono::duration<double, std::micro>(t1 - t0).count() / n;
  const double all = std::chrono::duration<double, std::micro>(t2 - t0).count() / n;
  printf("cluster %d pdl %d smem %6d param %5zu: host %.2f us/launch, host+drain %.2f us/launch (%s)\n", cluster,
         pdl, smem, sizeof(P), host, all, cudaGetErrorString(cudaGetLastError()));
  return host;
}

int main() {
  cudaFree(0);
  for (int cluster = 0; cluster < 2; ++cluster)
    for (int pdl = 0; pdl < 2; ++pdl)
      for (int smem : {0, 200 * 1024}) {
        run<Small>(cluster, pdl, smem, 200);
        run<Big>(cluster, pdl, smem, 200);
      }
  return 0;
}
