// pattern_probe.cu -- HBM ceiling of the band-walk access pattern of the 8u
// SAT kernel as a function of the chunk width TW and the band height TH
// (development tool).  Persistent CTAs walk TH-row bands of a 16384^2 u8 image
// left to right in TH x TW chunks: a producer warp TMA-loads each chunk (TW/256
// boxes of 256 x TH bytes) into an NST-deep smem ring, NW worker warps widen it
// to u32 and store it with st.global.cs.v4.  No scan: the data movement only.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o pp tools/pattern_probe.cu
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <vector>

#define CK(x)                                                                  \
  do {                                                                         \
    cudaError_t e = (x);                                                       \
    if (e != cudaSuccess) {                                                    \
      printf("%s: %s\n", #x, cudaGetErrorString(e));                           \
      exit(1);                                                                 \
    }                                                                          \
  } while (0)

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("{.reg .b64 st; mbarrier.arrive.shared::cta.b64 st, [%0];}" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t n) {
  asm volatile("{.reg .b64 st; mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;}" ::"r"(smem_u32(b)), "r"(n)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t ph) {
  asm volatile(
      "{.reg .pred p; W_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2; @!p bra W_%=;}" ::"r"(
          smem_u32(b)),
      "r"(ph), "r"(0x100000u)
      : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* m, uint64_t* bar, int x, int y) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"((uint64_t)m), "r"(x), "r"(y), "r"(smem_u32(bar))
      : "memory");
}
// store flavour: 0 st.global.cs (evict-first), 1 st.global (write-back default)
template <int STK>
__device__ __forceinline__ void st_out(void* p, uint4 v) {
  if (STK == 0)
    asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
  else
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
                 : "memory");
}

constexpr int64_t H = 16384, W = 16384;

template <int TW, int TH, int NST>
struct Sm {
  uint8_t in[NST][TW / 256][TH][256];
  uint64_t full[NST], empty[NST];
  int band[NST], chunk[NST];
};

template <int TW, int TH, int NW, int NST, int STK>
__global__ void __launch_bounds__((NW + 1) * 32) skel(const __grid_constant__ CUtensorMap min, uint32_t* out) {
  extern __shared__ __align__(128) unsigned char raw[];
  auto& s = *reinterpret_cast<Sm<TW, TH, NST>*>(raw);
  constexpr int RW = TH / NW, NB = TW / 256, NCH = W / TW, NBANDS = H / TH;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NST; ++i) {
      mbar_init(&s.full[i], 1);
      mbar_init(&s.empty[i], NW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == NW) {
    uint32_t q = 0;
    for (int b = blockIdx.x;; b += gridDim.x) {
      const bool done = b >= NBANDS;
      const int nch = done ? 1 : NCH;
      for (int c = 0; c < nch; ++c, ++q) {
        const int st = q % NST;
        mbar_wait(&s.empty[st], ((q / NST) & 1) ^ 1);
        if (lane == 0) {
          s.band[st] = done ? -1 : b;
          s.chunk[st] = c;
          if (done) {
            mbar_arrive(&s.full[st]);
          } else {
            mbar_arrive_tx(&s.full[st], TH * TW);
            for (int k = 0; k < NB; ++k) tma_load_2d(&s.in[st][k][0][0], &min, &s.full[st], c * TW + k * 256, b * TH);
          }
        }
        __syncwarp();
      }
      if (done) break;
    }
    return;
  }
  for (uint32_t q = 0;; ++q) {
    const int st = q % NST;
    mbar_wait(&s.full[st], (q / NST) & 1);
    const int band = s.band[st], chunk = s.chunk[st];
    if (band < 0) break;
    uint32_t w[RW][2 * NB];
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < 2 * NB; ++g)
        w[i][g] = *reinterpret_cast<const uint32_t*>(&s.in[st][g / 2][warp * RW + i][(g & 1) * 128 + 4 * lane]);
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.empty[st]);
    const int64_t y0 = (int64_t)band * TH + warp * RW, x0 = (int64_t)chunk * TW;
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < 2 * NB; ++g) {
        const uint32_t v = w[i][g];
        st_out<STK>(out + (y0 + i) * W + x0 + g * 128 + 4 * lane,
              make_uint4(v & 255, (v >> 8) & 255, (v >> 16) & 255, v >> 24));
      }
  }
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

uint8_t* g_in;
uint32_t* g_out;
Enc g_enc;
int g_sms;

template <int TW, int TH, int NW, int NST, int STK = 0>
void run(std::vector<int> grids = {}) {
  auto kern = skel<TW, TH, NW, NST, STK>;
  CUtensorMap mi;
  cuuint64_t d[2] = {(cuuint64_t)W, (cuuint64_t)H};
  cuuint64_t st[1] = {(cuuint64_t)W};
  cuuint32_t box[2] = {256, TH};
  cuuint32_t es[2] = {1, 1};
  g_enc(&mi, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, g_in, d, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  const size_t smem = sizeof(Sm<TW, TH, NST>);
  CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, (NW + 1) * 32, smem));
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  if (grids.empty())
    for (int per = 1; per <= std::min(occ, 3); ++per) grids.push_back(g_sms * per);
  for (int grid : grids) {
    std::vector<float> ts;
    for (int it = 0; it < 13; ++it) {
      cudaEventRecord(a);
      kern<<<grid, (NW + 1) * 32, smem>>>(mi, g_out);
      cudaEventRecord(b);
      CK(cudaEventSynchronize(b));
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (it >= 3) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    const double ms = ts[ts.size() / 2];
    printf("STK=%d TW=%4d TH=%3d NW=%2d NST=%d smem=%6zu occ=%d grid=%4d: %.4f ms %7.1f GB/s %.3f of 6543.7\n", STK, TW, TH, NW,
           NST, smem, occ, grid, ms, H * W * 5.0 / ms / 1e6, H * W * 5.0 / ms / 1e6 / 6543.7);
    fflush(stdout);
  }
}

int main() {
  CK(cudaMalloc(&g_in, H * W));
  CK(cudaMalloc(&g_out, H * W * 4));
  CK(cudaMemset(g_in, 3, H * W));
  void* fp;
  cudaDriverEntryPointQueryResult qr;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &qr));
  g_enc = (Enc)fp;
  cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, 0);
  run<256, 32, 8, 4>({296, 280});
  run<256, 32, 8, 4, 1>({296, 280});
  run<256, 16, 8, 6>({148, 144, 140, 136, 128});
  run<256, 16, 8, 6, 1>({148, 144});
  run<256, 16, 8, 10>({148, 144});
  run<256, 16, 8, 4>({148, 144});
  run<256, 16, 16, 8>({148, 144});
  run<512, 16, 8, 6>({148, 144});
  run<256, 8, 8, 12>({148, 296});
  run<512, 8, 8, 8>({148, 296});
  run<256, 32, 8, 4>({148, 296});
  return 0;
}
