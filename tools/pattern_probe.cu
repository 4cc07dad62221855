// pattern_probe.cu -- which tile shape lets band-walking persistent CTAs stream
// at the widening-copy bandwidth? (development tool)  Each CTA walks a row band
// of TH rows left to right in chunks of TW input bytes (u8 -> u32, 1 B in + 4 B
// out per px), TMA loads into a smem ring, NW worker warps widen and store with
// st.global.cs.v4.  BPC consecutive bands per "cluster ticket" are assigned to
// consecutive CTAs (as the SAT kernel does).
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(c)); }
__device__ __forceinline__ void mbar_arrive(uint64_t* b) { asm volatile("{.reg .b64 st; mbarrier.arrive.shared::cta.b64 st, [%0];}" ::"r"(smem_u32(b)) : "memory"); }
__device__ __forceinline__ void mbar_arrive_tx(uint64_t* b, uint32_t n) { asm volatile("{.reg .b64 st; mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;}" ::"r"(smem_u32(b)), "r"(n) : "memory"); }
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t ph) {
  asm volatile("{.reg .pred p; W_%=: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2; @!p bra W_%=;}" ::"r"(smem_u32(b)), "r"(ph), "r"(0x100000u) : "memory");
}
__device__ __forceinline__ void tma_load_2d(void* dst, const CUtensorMap* m, uint64_t* bar, int x, int y) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
               ::"r"(smem_u32(dst)), "l"((uint64_t)m), "r"(x), "r"(y), "r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void st_cs(void* p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}
struct P { uint32_t* out; int64_t H, W, nb, nch; };
constexpr int NW = 8;
template <int TH, int TW> struct Cfg { static constexpr int NST = (32768 / (TH * TW)) < 2 ? 2 : (32768 / (TH * TW)) > 8 ? 8 : (32768 / (TH * TW)); };
template <int TH, int TW, int MODE = 0, int SPREAD = 0>
__global__ void __launch_bounds__((NW + 1) * 32) skel(const __grid_constant__ CUtensorMap min, P p) {
  constexpr int NST = Cfg<TH, TW>::NST;
  constexpr int RW = TH / NW;
  constexpr int GR = TW / 128;  // 4-byte groups per lane per row
  extern __shared__ __align__(128) unsigned char raw[];
  uint8_t (*in)[TH][TW] = reinterpret_cast<uint8_t (*)[TH][TW]>(raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(raw + NST * TH * TW);
  uint64_t* empty = full + NST;
  int* bandv = reinterpret_cast<int*>(empty + NST);
  int* chv = bandv + NST;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NST; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == NW) {
    uint32_t q = 0;
    for (int64_t bi = blockIdx.x;; bi += gridDim.x) {
      const bool done = bi >= p.nb;
      int64_t b = bi;
      if (SPREAD && !done) { const int64_t per = p.nb / 8; b = (bi % 8) * per + bi / 8; }
      const int64_t nch = done ? 1 : p.nch;
      for (int64_t c = 0; c < nch; ++c, ++q) {
        const int st = q % NST;
        mbar_wait(&empty[st], ((q / NST) & 1) ^ 1);
        if (lane == 0) {
          bandv[st] = done ? -1 : (int)b; chv[st] = (int)c;
          if (done) mbar_arrive(&full[st]);
          else if (MODE == 2) mbar_arrive(&full[st]);
          else { mbar_arrive_tx(&full[st], TH * TW); for (int k = 0; k < (TW + 255) / 256; ++k) tma_load_2d(&in[st][0][0] + k * TH * 256, &min, &full[st], (int)(c * TW + k * 256), (int)(b * TH)); }
        }
        __syncwarp();
      }
      if (done) break;
    }
    return;
  }
  for (uint32_t q = 0;; ++q) {
    const int st = q % NST;
    mbar_wait(&full[st], (q / NST) & 1);
    const int band = bandv[st], chunk = chv[st];
    if (band < 0) break;
    uint32_t w[RW][GR];
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < GR; ++g) { const int x = g * 128 + 4 * lane; constexpr int BW = TW < 256 ? TW : 256; w[i][g] = *reinterpret_cast<const uint32_t*>(&in[st][0][0] + (x / BW) * TH * BW + (warp * RW + i) * BW + x % BW); }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[st]);
    const int64_t y0 = (int64_t)band * TH + warp * RW, x0 = (int64_t)chunk * TW;
    if (MODE == 1) { if (w[0][0] == 0x12345u) p.out[0] = 1; continue; }
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < GR; ++g) {
        const uint32_t v = w[i][g];
        st_cs(p.out + (y0 + i) * p.W + x0 + g * 128 + 4 * lane, make_uint4(v & 255, (v >> 8) & 255, (v >> 16) & 255, v >> 24));
      }
  }
}
typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
  const int64_t H = 16384, W = 16384, px = H * W;
  uint8_t* in; uint32_t* out;
  CK(cudaMalloc(&in, px)); CK(cudaMalloc(&out, px * 4)); CK(cudaMemset(in, 3, px));
  void* fp; cudaDriverEntryPointQueryResult qr;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &qr));
  Enc enc = (Enc)fp;
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto run = [&](auto kern, int TH, int TW, const char* tag = "") {
    CUtensorMap mi;
    cuuint64_t d[2] = {(cuuint64_t)W, (cuuint64_t)H}; cuuint64_t st[1] = {(cuuint64_t)W};
    cuuint32_t box[2] = {(cuuint32_t)(TW < 256 ? TW : 256), (cuuint32_t)TH}; cuuint32_t es[2] = {1, 1};
    if (enc(&mi, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, in, d, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE)) { printf("enc fail\n"); return; }
    int nst = 32768 / (TH * TW); nst = nst < 2 ? 2 : nst > 8 ? 8 : nst;
    size_t smem = nst * TH * TW + 2 * nst * 8 + 2 * nst * 4 + 64;
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, (NW + 1) * 32, smem));
    P p{out, H, W, H / TH, W / TW};
    for (int per : {1, 2, 4, 6}) {
      if (per > occ) break;
      const int grid = sms * per;
      std::vector<float> ts;
      for (int it = 0; it < 13; ++it) {
        cudaEventRecord(a); kern<<<grid, (NW + 1) * 32, smem>>>(mi, p); cudaEventRecord(b); CK(cudaEventSynchronize(b));
        float ms; cudaEventElapsedTime(&ms, a, b); if (it >= 3) ts.push_back(ms);
      }
      std::sort(ts.begin(), ts.end());
      printf("%-10s TH=%3d TW=%5d (out row seg %5d B) nst=%d grid=%4d: %.4f ms %7.1f GB/s\n", tag, TH, TW, TW * 4, nst, grid, ts[ts.size() / 2], px * 5.0 / ts[ts.size() / 2] / 1e6);
    }
  };
  run(skel<32, 256>, 32, 256, "normal");
  run(skel<32, 256, 1>, 32, 256, "readonly");
  run(skel<32, 256, 2>, 32, 256, "writeonly");
  run(skel<32, 256, 0, 1>, 32, 256, "spread");
  run(skel<8, 2048>, 8, 2048, "normal");
  run(skel<8, 2048, 1>, 8, 2048, "readonly");
  run(skel<8, 2048, 2>, 8, 2048, "writeonly");
  run(skel<8, 2048, 0, 1>, 8, 2048, "spread");
  run(skel<8, 256>, 8, 256, "normal");
  run(skel<16, 256>, 16, 256, "normal");
  return 0;
}
