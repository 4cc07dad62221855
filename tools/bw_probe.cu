// bw_probe.cu -- streaming-bandwidth ceilings for the SAT traffic mixes
// (development tool, not the product).  Measures, on the 16384^2 workload:
//   read-only 1 B/px, write-only 4 B/px, widening copy 8u->32u (1 B in + 4 B out,
//   the 8u32s traffic mix), and a 32f copy (4 B in + 4 B out), with different
//   store flavours and grid sizes.  The SAT kernel cannot beat the widening copy
//   of its own traffic mix; this gives the 8u roofline that actually binds.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bw_probe tools/bw_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)

__device__ __forceinline__ void st_cs(void* p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ void st_na(void* p, uint4 v) {
  asm volatile("st.global.L1::no_allocate.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
__device__ __forceinline__ void st_plain(void* p, uint4 v) { *reinterpret_cast<uint4*>(p) = v; }
__device__ __forceinline__ uint4 ld_nc(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

// widen: n16 = number of 16-byte input vectors; out has 4x.
template <int MODE>
__global__ void widen(const uint4* __restrict__ in, uint4* __restrict__ out, int64_t n16) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 v = ld_nc(in + i);
    uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      uint4 o = make_uint4(w[k] & 255, (w[k] >> 8) & 255, (w[k] >> 16) & 255, w[k] >> 24);
      // out index: keep each warp's stores contiguous: 4 consecutive 512 B segments
      const int64_t base = (i / 32) * 128 + k * 32 + (i % 32);
      if (MODE == 0) st_cs(out + base, o);
      else if (MODE == 1) st_na(out + base, o);
      else st_plain(out + base, o);
    }
  }
}

template <int MODE>
__global__ void writeonly(uint4* __restrict__ out, int64_t n16) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 o = make_uint4((uint32_t)i, 1, 2, 3);
    if (MODE == 0) st_cs(out + i, o);
    else if (MODE == 1) st_na(out + i, o);
    else st_plain(out + i, o);
  }
}

__global__ void readonly(const uint4* __restrict__ in, int64_t n16, uint32_t* sink) {
  uint32_t acc = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 v = ld_nc(in + i);
    acc ^= v.x ^ v.y ^ v.z ^ v.w;
  }
  if (acc == 0x12345678u) *sink = acc;
}

template <int MODE>
__global__ void copy(const uint4* __restrict__ in, uint4* __restrict__ out, int64_t n16) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n16; i += (int64_t)gridDim.x * blockDim.x) {
    uint4 v = ld_nc(in + i);
    if (MODE == 0) st_cs(out + i, v);
    else st_plain(out + i, v);
  }
}

template <class F>
float timeit(F f, int iters = 20) {
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) f();
  cudaDeviceSynchronize();
  std::vector<float> ts;
  for (int i = 0; i < iters; ++i) {
    cudaEventRecord(a); f(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); ts.push_back(ms);
  }
  std::sort(ts.begin(), ts.end());
  return ts[ts.size() / 2];
}

int main() {
  const int64_t px = 16384LL * 16384LL;
  uint8_t* in; uint32_t* out; uint32_t* sink;
  CK(cudaMalloc(&in, px * 4)); CK(cudaMalloc(&out, px * 4)); CK(cudaMalloc(&sink, 4));
  CK(cudaMemset(in, 1, px * 4)); CK(cudaMemset(out, 0, px * 4));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const int64_t n16 = px / 16;
  for (int bpsm : {2, 4, 8, 16}) for (int thr : {256, 512}) {
    const int grid = sms * bpsm;
    float t;
    t = timeit([&] { readonly<<<grid, thr>>>((const uint4*)in, n16, sink); });
    printf("grid %4d x %3d  read  1B/px  : %.4f ms %7.1f GB/s\n", grid, thr, t, px * 1.0 / t / 1e6);
    t = timeit([&] { writeonly<0><<<grid, thr>>>((uint4*)out, n16 * 4); });
    printf("grid %4d x %3d  write 4B/px cs: %.4f ms %7.1f GB/s\n", grid, thr, t, px * 4.0 / t / 1e6);
    t = timeit([&] { writeonly<2><<<grid, thr>>>((uint4*)out, n16 * 4); });
    printf("grid %4d x %3d  write 4B/px wb: %.4f ms %7.1f GB/s\n", grid, thr, t, px * 4.0 / t / 1e6);
    for (int m = 0; m < 3; ++m) {
      if (m == 0) t = timeit([&] { widen<0><<<grid, thr>>>((const uint4*)in, (uint4*)out, n16); });
      if (m == 1) t = timeit([&] { widen<1><<<grid, thr>>>((const uint4*)in, (uint4*)out, n16); });
      if (m == 2) t = timeit([&] { widen<2><<<grid, thr>>>((const uint4*)in, (uint4*)out, n16); });
      printf("grid %4d x %3d  widen 8u->32u st%d: %.4f ms %7.1f GB/s  %6.1f Gpx/s\n", grid, thr, m, t, px * 5.0 / t / 1e6, px / t / 1e6);
    }
    t = timeit([&] { copy<0><<<grid, thr>>>((const uint4*)in, (uint4*)out, n16 * 4); });
    printf("grid %4d x %3d  copy 32f cs   : %.4f ms %7.1f GB/s\n", grid, thr, t, px * 8.0 / t / 1e6);
    t = timeit([&] { copy<2><<<grid, thr>>>((const uint4*)in, (uint4*)out, n16 * 4); });
    printf("grid %4d x %3d  copy 32f wb   : %.4f ms %7.1f GB/s\n", grid, thr, t, px * 8.0 / t / 1e6);
  }
  float t = timeit([&] { cudaMemcpyAsync(out, in, px * 4, cudaMemcpyDeviceToDevice); });
  printf("cudaMemcpy D2D 4B/px: %.4f ms %7.1f GB/s (r+w)\n", t, px * 8.0 / t / 1e6);
  t = timeit([&] { cudaMemsetAsync(out, 7, px * 4); });
  printf("cudaMemset 4B/px: %.4f ms %7.1f GB/s\n", t, px * 4.0 / t / 1e6);
  return 0;
}
