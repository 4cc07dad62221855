// Cluster placement probe: for cluster sizes 1..8 (2 CTAs/SM worth of smem),
// how many clusters are co-resident (occupancy API) and how many SMs do they
// actually cover (each CTA records %smid while all spin together).
#include <cstdio>
#include <cuda_runtime.h>
#include <set>
#include <vector>
__global__ void k(int* smid, unsigned long long* t0, int spin_us) {
  extern __shared__ char s[];
  if (threadIdx.x == 0) {
    int id; asm volatile("mov.u32 %0, %%smid;" : "=r"(id));
    unsigned long long a; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(a));
    smid[blockIdx.x] = id; t0[blockIdx.x] = a;
    unsigned long long b = a;
    while (b - a < (unsigned long long)spin_us * 1000) asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(b));
    s[0] = 1;
  }
}
int main(int argc, char** argv) {
  const int smem = argc > 1 ? atoi(argv[1]) : 95360, threads = argc > 2 ? atoi(argv[2]) : 384;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  int *d; unsigned long long* t; cudaMalloc(&d, 4096 * 4); cudaMalloc(&t, 4096 * 8);
  for (int cl = 1; cl <= 8; ++cl) {
    cudaLaunchConfig_t cfg = {};
    cfg.blockDim = dim3(threads); cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute a; a.id = cudaLaunchAttributeClusterDimension; a.val.clusterDim.x = cl; a.val.clusterDim.y = 1; a.val.clusterDim.z = 1;
    cfg.attrs = &a; cfg.numAttrs = 1;
    cfg.gridDim = dim3(cl * 64);
    int n = 0; cudaError_t e = cudaOccupancyMaxActiveClusters(&n, k, &cfg);
    // launch n + 4 clusters; count those that started within 20 us of the first
    const int nl = n + 4;
    cfg.gridDim = dim3(cl * nl);
    e = cudaLaunchKernelEx(&cfg, k, d, t, 200);
    cudaDeviceSynchronize();
    std::vector<int> sm(cl * nl); std::vector<unsigned long long> ts(cl * nl);
    cudaMemcpy(sm.data(), d, 4 * cl * nl, cudaMemcpyDeviceToHost);
    cudaMemcpy(ts.data(), t, 8 * cl * nl, cudaMemcpyDeviceToHost);
    unsigned long long mn = ~0ull; for (auto v : ts) mn = v < mn ? v : mn;
    std::set<int> sms; int early = 0;
    for (int i = 0; i < cl * nl; ++i) if (ts[i] - mn < 20000) { ++early; sms.insert(sm[i]); }
    printf("cluster %d: occupancy API %d clusters (%d CTAs); co-started CTAs %d on %zu SMs (%s)\n", cl, n, n * cl, early, sms.size(), cudaGetErrorString(e));
  }
}
