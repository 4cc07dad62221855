// store_probe.cu -- data-movement skeleton of the 8u SAT kernel (development
// tool).  Persistent CTAs walk row bands of a u8 image in 32 x 256 chunks:
// a producer warp TMA-loads each chunk into a smem ring, NW worker warps widen
// it to u32 and write it out, either with direct st.global.cs.v4 from registers
// (MODE 0, what sat_tile_kernel does) or through a per-warp smem staging buffer
// and bulk (TMA) stores (MODE 1: one 1D bulk copy per row; MODE 2: one 2D
// tensor store per warp).  No scan: this is the ceiling of the traffic pattern.
#include <cstdio>
#include <cstdint>
#include <cstring>
#include <vector>
#include <algorithm>
#include <cuda.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); exit(1); } } while (0)

constexpr int TW = 256, NST = 4;

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
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* m, const void* src, int x, int y) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
               ::"l"((uint64_t)m), "r"(x), "r"(y), "r"(smem_u32(src)) : "memory");
}
__device__ __forceinline__ void bulk_store(void* g, const void* s, uint32_t n) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(g), "r"(smem_u32(s)), "r"(n) : "memory");
}
__device__ __forceinline__ void st_cs8(void* p, uint4 a, uint4 b) {
  asm volatile("st.global.cs.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(a.x), "r"(a.y), "r"(a.z), "r"(a.w),
               "r"(b.x), "r"(b.y), "r"(b.z), "r"(b.w) : "memory");
}
__device__ __forceinline__ void st_cs(void* p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

template <int NW>
struct Sm {
  uint8_t in[NST][32][TW];
  uint32_t stage[NW][2][32 / NW][TW];  // per-warp double-buffered staging
  uint64_t full[NST], empty[NST];
  int band[NST], chunk[NST];
};

struct P {
  uint32_t* out; int64_t H, W, nb, nch;
};

template <int NW, int MODE>
__global__ void __launch_bounds__((NW + 1) * 32) skel(const __grid_constant__ CUtensorMap min, const __grid_constant__ CUtensorMap mout, P p) {
  extern __shared__ __align__(128) unsigned char raw[];
  Sm<NW>& s = *reinterpret_cast<Sm<NW>*>(raw);
  constexpr int RW = 32 / NW;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NST; ++i) { mbar_init(&s.full[i], 1); mbar_init(&s.empty[i], NW); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  if (warp == NW) {
    uint32_t q = 0;
    for (int64_t b = blockIdx.x;; b += gridDim.x) {
      const bool done = b >= p.nb;
      const int64_t nch = done ? 1 : p.nch;
      for (int64_t c = 0; c < nch; ++c, ++q) {
        const int st = q % NST;
        mbar_wait(&s.empty[st], ((q / NST) & 1) ^ 1);
        if (lane == 0) {
          s.band[st] = done ? -1 : (int)b; s.chunk[st] = (int)c;
          if (done) mbar_arrive(&s.full[st]);
          else { mbar_arrive_tx(&s.full[st], 32 * TW); tma_load_2d(&s.in[st][0][0], &min, &s.full[st], (int)(c * TW), (int)(b * 32)); }
        }
        __syncwarp();
      }
      if (done) break;
    }
    return;
  }
  uint32_t q = 0;
  for (;; ++q) {
    const int st = q % NST;
    mbar_wait(&s.full[st], (q / NST) & 1);
    const int band = s.band[st], chunk = s.chunk[st];
    if (band < 0) break;
    uint32_t w[RW][2];
    if (MODE == 3) {
#pragma unroll
      for (int i = 0; i < RW; ++i) {
        const uint2 v = *reinterpret_cast<const uint2*>(&s.in[st][warp * RW + i][8 * lane]);
        w[i][0] = v.x; w[i][1] = v.y;
      }
    } else
#pragma unroll
    for (int i = 0; i < RW; ++i) {
      w[i][0] = *reinterpret_cast<const uint32_t*>(&s.in[st][warp * RW + i][4 * lane]);
      w[i][1] = *reinterpret_cast<const uint32_t*>(&s.in[st][warp * RW + i][128 + 4 * lane]);
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&s.empty[st]);
    const int64_t y0 = (int64_t)band * 32 + warp * RW, x0 = (int64_t)chunk * TW;
    if (MODE == 3) {
#pragma unroll
      for (int i = 0; i < RW; ++i) {
        const uint32_t u = w[i][0], v = w[i][1];
        st_cs8(p.out + (y0 + i) * p.W + x0 + 8 * lane, make_uint4(u & 255, (u >> 8) & 255, (u >> 16) & 255, u >> 24),
               make_uint4(v & 255, (v >> 8) & 255, (v >> 16) & 255, v >> 24));
      }
    } else if (MODE == 0) {
#pragma unroll
      for (int i = 0; i < RW; ++i)
#pragma unroll
        for (int g = 0; g < 2; ++g) {
          const uint32_t v = w[i][g];
          st_cs(p.out + (y0 + i) * p.W + x0 + g * 128 + 4 * lane, make_uint4(v & 255, (v >> 8) & 255, (v >> 16) & 255, v >> 24));
        }
    } else {
      const int buf = q & 1;
      if (lane == 0) asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      __syncwarp();
#pragma unroll
      for (int i = 0; i < RW; ++i)
#pragma unroll
        for (int g = 0; g < 2; ++g) {
          const uint32_t v = w[i][g];
          *reinterpret_cast<uint4*>(&s.stage[warp][buf][i][g * 128 + 4 * lane]) = make_uint4(v & 255, (v >> 8) & 255, (v >> 16) & 255, v >> 24);
        }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      __syncwarp();
      if (lane == 0) {
        if (MODE == 1) {
          for (int i = 0; i < RW; ++i) bulk_store(p.out + (y0 + i) * p.W + x0, &s.stage[warp][buf][i][0], TW * 4);
        } else {
          tma_store_2d(&mout, &s.stage[warp][buf][0][0], (int)x0, (int)y0);
        }
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      }
    }
  }
  if (MODE != 0 && MODE != 3 && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int64_t H = 16384, W = 16384, px = H * W;
  uint8_t* in; uint32_t* out;
  CK(cudaMalloc(&in, px)); CK(cudaMalloc(&out, px * 4));
  CK(cudaMemset(in, 3, px));
  void* fp; cudaDriverEntryPointQueryResult qr;
  CK(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fp, cudaEnableDefault, &qr));
  Enc enc = (Enc)fp;
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  P p{out, H, W, H / 32, W / TW};
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  auto run = [&](auto kern, int nw, int rw, const char* name) {
    CUtensorMap mi, mo;
    { cuuint64_t d[2] = {(cuuint64_t)W, (cuuint64_t)H}; cuuint64_t st[1] = {(cuuint64_t)W}; cuuint32_t box[2] = {TW, 32}; cuuint32_t es[2] = {1, 1};
      enc(&mi, CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, in, d, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE); }
    { cuuint64_t d[2] = {(cuuint64_t)W, (cuuint64_t)H}; cuuint64_t st[1] = {(cuuint64_t)W * 4}; cuuint32_t box[2] = {TW, (cuuint32_t)rw}; cuuint32_t es[2] = {1, 1};
      CUresult r = enc(&mo, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, out, d, st, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (r) printf("enc out %d\n", (int)r); }
    size_t smem = nw == 8 ? sizeof(Sm<8>) : (nw == 16 ? sizeof(Sm<16>) : sizeof(Sm<4>));
    CK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    int occ = 0; CK(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, (nw + 1) * 32, smem));
    for (int per : {1, 2, 3, 4}) {
      if (per > occ) break;
      const int grid = sms * per;
      std::vector<float> ts;
      for (int it = 0; it < 13; ++it) {
        CK(cudaMemset(out, 0xff, 64));
        cudaEventRecord(a);
        kern<<<grid, (nw + 1) * 32, smem>>>(mi, mo, p);
        cudaEventRecord(b); CK(cudaEventSynchronize(b));
        float ms; cudaEventElapsedTime(&ms, a, b); if (it >= 3) ts.push_back(ms);
      }
      std::sort(ts.begin(), ts.end());
      // check a few values
      uint32_t h[4]; CK(cudaMemcpy(h, out + (H - 1) * W + W - 4, 16, cudaMemcpyDeviceToHost));
      printf("%-26s NW=%2d smem=%6zu occ=%d grid=%4d: %.4f ms %7.1f GB/s  chk=%u\n", name, nw, smem, occ, grid, ts[ts.size() / 2], px * 5.0 / ts[ts.size() / 2] / 1e6, h[3]);
    }
  };
  run(skel<8, 0>, 8, 4, "direct st.cs.v4");
  run(skel<8, 3>, 8, 4, "direct st.cs.v8 (256-bit)");
  run(skel<8, 0>, 8, 4, "direct st.cs.v4");
  run(skel<8, 3>, 8, 4, "direct st.cs.v8 (256-bit)");
  run(skel<8, 1>, 8, 4, "bulk 1D per row");
  run(skel<8, 2>, 8, 4, "tensor 2D per warp");
  run(skel<16, 0>, 16, 2, "direct st.cs.v4");
  run(skel<16, 3>, 16, 2, "direct st.cs.v8 (256-bit)");
  run(skel<16, 1>, 16, 2, "bulk 1D per row");
  run(skel<16, 2>, 16, 2, "tensor 2D per warp");
  run(skel<4, 0>, 4, 8, "direct st.cs.v4");
  run(skel<4, 2>, 4, 8, "tensor 2D per warp");
  return 0;
}
