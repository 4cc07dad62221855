// sat_brlt.cu -- ABLATION: a B200 port of the
// paper's fastest method, Register-based BRLT-ScanRow run twice (PAPER.md:
// 248-254, Sec. IV-B; Alg. 5 at PAPER.md:201-244; "fastest ... called twice"
// at PAPER.md:441), kept beside the single-pass kernel to measure what the
// single pass saves on the same box.  Not on the product path: sat_compute
// never calls it.
//
// One BRLT-ScanRow pass (a CTA per 32-row strip, Fig. 3a):
//   1. each warp caches a 32 x 32 block in registers (lane l holds column
//      c0 + l of the strip's 32 rows: data[j] = A(r0 + j, c0 + l), coalesced);
//   2. BRLT (Alg. 5): the block is transposed through a [32][33] shared-memory
//      matrix per warp (stride 33: no bank conflicts), so lane l now holds row
//      r0 + l's 32 values;
//   3. serial scan of the 32 registers (Alg. 2) -- the row prefix inside the
//      warp's 32 columns;
//   4. block partial-sum scan over the warps (Fig. 3c) plus the
//      row carry of the previous 32 x WarpCount-column segments;
//   5. the row prefixes are stored TRANSPOSED: out(c, r) = rowprefix(r, c)
//      (lanes write consecutive r: coalesced).
// Two passes, BRLT-ScanRow(BRLT-ScanRow(A)) = SAT(A): traffic per pixel is
// sizeof(T_A) + 3 sizeof(T_B) (13 / 16 / 32 B for 8u / 32f / 64f) against the
// single pass's sizeof(T_A) + sizeof(T_B) (5 / 8 / 16 B).
//
// Readings: Alg. 5 as printed puts __syncthreads under the warp-dependent
// `if i <= warpId` (a divergent barrier, SURVEY reading 14); here every warp
// owns its own [32][33] buffer (S = WarpCount fits B200's 227 KB of shared
// memory: 1024 threads for 4-byte T, 512 for 8-byte T as the paper does for
// double), so the transpose needs only warp-level synchronisation.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/libsat.h"
#include "sat_internal.h"

namespace {

template <typename T>
struct BAcc {
  using type = T;
};
template <>
struct BAcc<int32_t> {
  using type = uint32_t;
};

// One BRLT-ScanRow pass: in is h x w (TA, pitch ip bytes), out is w x h (TB,
// pitch op bytes) = transpose(rowprefix(in)), accumulated in TB (u32 wraps).
template <typename TB, int NW>
struct BrltSmem {
  TB sm[NW][32][33];  // Alg. 5 line 2 (one buffer per warp)
  TB tot[NW][32];     // Fig. 3c: each warp's row totals
  TB carry[32];       // row totals of the previous segments
};

template <typename TA, typename TB, int NW>
__global__ void __launch_bounds__(NW * 32)
    brlt_scanrow_kernel(const char* __restrict__ in, int64_t ip, char* __restrict__ out, int64_t op,
                        int64_t h, int64_t w) {
  extern __shared__ __align__(16) unsigned char brlt_raw[];
  BrltSmem<TB, NW>& S = *reinterpret_cast<BrltSmem<TB, NW>*>(brlt_raw);
  auto& sm = S.sm;
  auto& tot = S.tot;
  auto& carry = S.carry;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int64_t r0 = (int64_t)blockIdx.x * 32;
  if (threadIdx.x < 32) carry[threadIdx.x] = TB(0);
  __syncthreads();
  for (int64_t seg = 0; seg * NW * 32 < w; ++seg) {
    const int64_t c0 = seg * NW * 32 + wid * 32;
    TB data[32];  // Alg. 5 line 1: 32 registers per thread
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      const int64_t r = r0 + j, c = c0 + lane;
      data[j] = (r < h && c < w) ? (TB)reinterpret_cast<const TA*>(in + r * ip)[c] : TB(0);
    }
    // BRLT (Alg. 5 lines 7-12): write rows, read columns
#pragma unroll
    for (int j = 0; j < 32; ++j) sm[wid][j][lane] = data[j];
    __syncwarp();
#pragma unroll
    for (int j = 0; j < 32; ++j) data[j] = sm[wid][lane][j];
    __syncwarp();
    // serial scan (Alg. 2): lane = row r0 + lane, j = column c0 + j
#pragma unroll
    for (int j = 1; j < 32; ++j) data[j] = data[j] + data[j - 1];
    tot[wid][lane] = data[31];
    __syncthreads();
    // partial sums of the warps to the left (Fig. 3c step 2-3) + earlier segments
    TB off = carry[lane];
    for (int k = 0; k < wid; ++k) off = off + tot[k][lane];
#pragma unroll
    for (int j = 0; j < 32; ++j) data[j] = data[j] + off;
    __syncthreads();  // every warp has read carry and tot
    if (wid == NW - 1) carry[lane] = data[31];
    // transposed store: out(c0 + j, r0 + lane)
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      const int64_t c = c0 + j, r = r0 + lane;
      if (c < w && r < h) reinterpret_cast<TB*>(out + c * op)[r] = data[j];
    }
    __syncthreads();  // carry is updated before the next segment reads it
  }
}

template <typename TA, typename TB, int NW>
sat_status brlt_pass(const void* in, int64_t ip, void* out, int64_t op, int64_t h, int64_t w,
                     cudaStream_t s) {
  const unsigned grid = (unsigned)((h + 31) / 32);
  const int smem = (int)sizeof(BrltSmem<TB, NW>);
  cudaError_t e = cudaFuncSetAttribute(brlt_scanrow_kernel<TA, TB, NW>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return sat::cuda_fail(e, "cudaFuncSetAttribute(brlt)");
  brlt_scanrow_kernel<TA, TB, NW><<<grid, NW * 32, smem, s>>>(static_cast<const char*>(in), ip,
                                                              static_cast<char*>(out), op, h, w);
  e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "brlt_scanrow_kernel launch");
}

template <typename TA, typename TB, int NW>
sat_status brlt_sat(const void* in, int64_t ip, void* out, int64_t op, void* tmp, int64_t tp,
                    int64_t h, int64_t w, cudaStream_t s) {
  sat_status st = brlt_pass<TA, TB, NW>(in, ip, tmp, tp, h, w, s);  // tmp: w x h
  if (st != SAT_OK) return st;
  return brlt_pass<TB, TB, NW>(tmp, tp, out, op, w, h, s);          // out: h x w
}

}  // namespace

extern "C" {

sat_status sat_compute_brlt(sat_pair pair, const void* in, void* out, void* tmp, int64_t h,
                            int64_t w, int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                            int64_t tmp_pitch_bytes, void* stream) {
  if (pair != SAT_8U_32S && pair != SAT_32F_32F && pair != SAT_64F_64F)
    return sat::fail(SAT_ERR_UNSUPPORTED, "the BRLT ablation covers 8u->32s, 32f, 64f");
  if (h < 0 || w < 0) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "negative extent");
  if (h == 0 || w == 0) return SAT_OK;
  if (!in || !out || !tmp) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "NULL pointer");
  const int64_t sa = (int64_t)sat::in_size(pair), sb = (int64_t)sat::out_size(pair);
  if (in_pitch_bytes < w * sa || out_pitch_bytes < w * sb || tmp_pitch_bytes < h * sb ||
      in_pitch_bytes % sa || out_pitch_bytes % sb || tmp_pitch_bytes % sb)
    return sat::fail(SAT_ERR_INVALID_ARGUMENT, "pitch too small or misaligned (tmp is w x h)");
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  switch (pair) {
    case SAT_8U_32S:
      return brlt_sat<uint8_t, uint32_t, 32>(in, in_pitch_bytes, out, out_pitch_bytes, tmp,
                                             tmp_pitch_bytes, h, w, s);
    case SAT_32F_32F:
      return brlt_sat<float, float, 32>(in, in_pitch_bytes, out, out_pitch_bytes, tmp,
                                        tmp_pitch_bytes, h, w, s);
    default:
      return brlt_sat<double, double, 16>(in, in_pitch_bytes, out, out_pitch_bytes, tmp,
                                          tmp_pitch_bytes, h, w, s);
  }
}

}  // extern "C"
