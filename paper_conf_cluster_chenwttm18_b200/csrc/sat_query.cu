// sat_query.cu -- consumers of an inclusive SAT:
// rectangle sums and the box filter, the O(1)-per-query use that motivates
// the primitive (four-corner identity PAPER.md:95).
//
// For a half-open rectangle [y0, y1) x [x0, x1) of the image,
//   sum = S(y1-1, x1-1) - S(y0-1, x1-1) - S(y1-1, x0-1) + S(y0-1, x0-1),
// with S(-1, .) = S(., -1) = 0.  8u->32s SATs are the exact sums mod 2^32
// (reading R2), and the identity holds mod 2^32, so every rectangle whose
// true sum is below 2^32 comes out exact even where the SAT itself wrapped.
//
// Both kernels are HBM/L2-bound gathers: the box filter reads the SAT with
// coalesced row segments (each SAT row is needed by two output rows, 2r+1
// apart; the L2 serves the second read) and writes the output once.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "../../include/libsat.h"
#include "sat_internal.h"

namespace {

template <typename T>
struct Acc {
  using type = T;
};
template <>
struct Acc<int32_t> {
  using type = uint32_t;  // wrap arithmetic (signed overflow is UB)
};

template <typename T>
__device__ __forceinline__ typename Acc<T>::type at(const char* sat, int64_t pitch, int64_t y,
                                                    int64_t x) {
  using A = typename Acc<T>::type;
  if (y < 0 || x < 0) return A(0);
  return (A)__ldg(reinterpret_cast<const T*>(sat + y * pitch) + x);
}

template <typename T>
__device__ __forceinline__ T rect(const char* sat, int64_t pitch, int64_t y0, int64_t x0,
                                  int64_t y1, int64_t x1) {
  using A = typename Acc<T>::type;
  if (y1 <= y0 || x1 <= x0) return T(0);
  const A d = at<T>(sat, pitch, y1 - 1, x1 - 1);
  const A b = at<T>(sat, pitch, y0 - 1, x1 - 1);
  const A c = at<T>(sat, pitch, y1 - 1, x0 - 1);
  const A a = at<T>(sat, pitch, y0 - 1, x0 - 1);
  return (T)((d - b) - (c - a));
}

// One thread per query; rects[i] = {y0, x0, y1, x1}, clamped to the image.
template <typename T>
__global__ void rect_sums_kernel(const char* sat, int64_t pitch, int64_t h, int64_t w,
                                 const int4* rects, int64_t n, T* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int4 r = rects[i];
    const int64_t y0 = std::min<int64_t>(std::max<int64_t>(r.x, 0), h);
    const int64_t x0 = std::min<int64_t>(std::max<int64_t>(r.y, 0), w);
    const int64_t y1 = std::min<int64_t>(std::max<int64_t>(r.z, 0), h);
    const int64_t x1 = std::min<int64_t>(std::max<int64_t>(r.w, 0), w);
    out[i] = rect<T>(sat, pitch, y0, x0, y1, x1);
  }
}

// Box filter: out(y, x) = sum of A over [y-ry, y+ry] x [x-rx, x+rx] clipped to
// the image.  Block = 32 x 8 threads walking a 32-column strip down ROWS rows
// per block (coalesced 128-byte row segments of the SAT and of the output).
template <typename T, int ROWS>
__global__ void __launch_bounds__(256) box_kernel(const char* sat, int64_t sp, char* out,
                                                  int64_t op, int64_t h, int64_t w, int64_t ry,
                                                  int64_t rx) {
  const int64_t x = blockIdx.x * 32 + threadIdx.x;
  if (x >= w) return;
  const int64_t x0 = std::max<int64_t>(x - rx, 0), x1 = std::min<int64_t>(x + rx + 1, w);
  const int64_t ybase = (int64_t)blockIdx.y * ROWS;
  for (int r = threadIdx.y; r < ROWS; r += 8) {
    const int64_t y = ybase + r;
    if (y >= h) break;
    const int64_t y0 = std::max<int64_t>(y - ry, 0), y1 = std::min<int64_t>(y + ry + 1, h);
    reinterpret_cast<T*>(out + y * op)[x] = rect<T>(sat, sp, y0, x0, y1, x1);
  }
}

// Tiled box filter: a block stages the SAT window its 32 x 256 output tile
// needs -- (32 + 2ry + 1) x (256 + 2rx + 1) elements, read once with
// coalesced rows -- in shared memory, then every thread walks one output
// column down the tile with four shared-memory corner reads per output.
// Staged element (r, c) is S(min(ya + r, h - 1), min(xa + c, w - 1)) with
// ya = y_tile - ry - 1, xa = x_tile - rx - 1, and 0 where ya + r < 0 or
// xa + c < 0: exactly the clipped corners of the four-corner identity.
constexpr int kBoxRows = 32, kBoxCols = 256;

template <typename T>
__global__ void __launch_bounds__(kBoxCols) box_tiled_kernel(const char* sat, int64_t sp, char* out,
                                                             int64_t op, int64_t h, int64_t w,
                                                             int ry, int rx) {
  using A = typename Acc<T>::type;
  extern __shared__ __align__(16) unsigned char box_smem[];
  A* tile = reinterpret_cast<A*>(box_smem);
  const int R = kBoxRows + 2 * ry + 1, C = kBoxCols + 2 * rx + 1;
  const int64_t yt = (int64_t)blockIdx.y * kBoxRows, xt = (int64_t)blockIdx.x * kBoxCols;
  const int64_t ya = yt - ry - 1, xa = xt - rx - 1;
  // staging: 8 independent row loads in flight per thread before the smem stores
  for (int c = threadIdx.x; c < C; c += kBoxCols) {
    const int64_t x = xa + c;
    const int64_t xc = std::min<int64_t>(x, w - 1);
    for (int r0 = 0; r0 < R; r0 += 8) {
      A v[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int64_t y = ya + r0 + k;
        v[k] = (r0 + k >= R || y < 0 || x < 0)
                   ? A(0)
                   : (A)__ldg(reinterpret_cast<const T*>(sat + std::min<int64_t>(y, h - 1) * sp) + xc);
      }
#pragma unroll
      for (int k = 0; k < 8; ++k)
        if (r0 + k < R) tile[(r0 + k) * C + c] = v[k];
    }
  }
  __syncthreads();
  const int tx = threadIdx.x;
  const int64_t x = xt + tx;
  if (x >= w) return;
  const int dy = 2 * ry + 1, dx = 2 * rx + 1;
  for (int ty = 0; ty < kBoxRows; ++ty) {
    const int64_t y = yt + ty;
    if (y >= h) break;
    const A* top = tile + ty * C + tx;
    const A* bot = top + dy * C;
    reinterpret_cast<T*>(out + y * op)[x] = (T)((bot[dx] - top[dx]) - (bot[0] - top[0]));
  }
}

template <typename T>
sat_status launch_box(const void* sat, void* out, int64_t h, int64_t w, int64_t sp, int64_t op,
                      int64_t ry, int64_t rx, cudaStream_t s) {
  const int64_t smem = (kBoxRows + 2 * ry + 1) * (kBoxCols + 2 * rx + 1) * (int64_t)sizeof(T);
  if (smem <= 200 * 1024) {
    // per device and cheap: set on every launch (a process may drive several GPUs)
    cudaError_t ea = cudaFuncSetAttribute(box_tiled_kernel<T>,
                                          cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (ea != cudaSuccess) return sat::cuda_fail(ea, "cudaFuncSetAttribute(box_tiled_kernel)");
    dim3 grid((unsigned)((w + kBoxCols - 1) / kBoxCols), (unsigned)((h + kBoxRows - 1) / kBoxRows));
    box_tiled_kernel<T><<<grid, kBoxCols, (size_t)smem, s>>>(
        static_cast<const char*>(sat), sp, static_cast<char*>(out), op, h, w, (int)ry, (int)rx);
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "box_tiled_kernel launch");
  }
  constexpr int ROWS = 64;
  dim3 grid((unsigned)((w + 31) / 32), (unsigned)((h + ROWS - 1) / ROWS));
  box_kernel<T, ROWS><<<grid, dim3(32, 8), 0, s>>>(static_cast<const char*>(sat), sp,
                                                   static_cast<char*>(out), op, h, w, ry, rx);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "box_kernel launch");
}

// Multi-channel SATs (SAT_8U_SQ: K = 2, SAT_8U_HIST4: K = 4): the same
// four-corner identity per channel, mod 2^32; out is [n][K] uint32.
template <int K>
__global__ void rect_sums_chan_kernel(const char* sat, int64_t pitch, int64_t h, int64_t w,
                                      const int4* rects, int64_t n, uint32_t* out) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int4 r = rects[i];
    const int64_t y0 = std::min<int64_t>(std::max<int64_t>(r.x, 0), h);
    const int64_t x0 = std::min<int64_t>(std::max<int64_t>(r.y, 0), w);
    const int64_t y1 = std::min<int64_t>(std::max<int64_t>(r.z, 0), h);
    const int64_t x1 = std::min<int64_t>(std::max<int64_t>(r.w, 0), w);
#pragma unroll
    for (int c = 0; c < K; ++c) {
      uint32_t v = 0;
      if (y1 > y0 && x1 > x0) {
        const uint32_t d = at<int32_t>(sat, pitch, y1 - 1, (x1 - 1) * K + c);
        const uint32_t b = y0 > 0 ? at<int32_t>(sat, pitch, y0 - 1, (x1 - 1) * K + c) : 0u;
        const uint32_t cc = x0 > 0 ? at<int32_t>(sat, pitch, y1 - 1, (x0 - 1) * K + c) : 0u;
        const uint32_t a = (y0 > 0 && x0 > 0) ? at<int32_t>(sat, pitch, y0 - 1, (x0 - 1) * K + c) : 0u;
        v = (d - b) - (cc - a);
      }
      out[i * K + c] = v;
    }
  }
}

template <int K>
sat_status launch_rects_chan(const void* sat, int64_t sp, int64_t h, int64_t w, const void* rects,
                             int64_t n, void* out, cudaStream_t s) {
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 16);
  rect_sums_chan_kernel<K><<<grid, 256, 0, s>>>(static_cast<const char*>(sat), sp, h, w,
                                                static_cast<const int4*>(rects), n,
                                                static_cast<uint32_t*>(out));
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "rect_sums_chan_kernel launch");
}

template <typename T>
sat_status launch_rects(const void* sat, int64_t sp, int64_t h, int64_t w, const void* rects,
                        int64_t n, void* out, cudaStream_t s) {
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 16);
  rect_sums_kernel<T><<<grid, 256, 0, s>>>(static_cast<const char*>(sat), sp, h, w,
                                            static_cast<const int4*>(rects), n,
                                            static_cast<T*>(out));
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "rect_sums_kernel launch");
}

sat_status check_sat_args(sat_plan plan, const void* sat, int64_t h, int64_t w, int64_t sp,
                          sat_pair pair) {
  if (!plan) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (pair != plan->pair)
    return sat::fail(SAT_ERR_INVALID_ARGUMENT, "pair %d does not match the plan's pair %d",
                     (int)pair, (int)plan->pair);
  if (h < 0 || w < 0) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "negative extent");
  const int64_t sb = (int64_t)sat::out_size(pair);
  if (h > 0 && w > 0) {
    if (!sat) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "NULL SAT pointer");
    if (sp < w * sb || sp % sb != 0 || (uintptr_t)sat % sb != 0)
      return sat::fail(SAT_ERR_INVALID_ARGUMENT, "SAT pitch %lld / alignment invalid",
                       (long long)sp);
  }
  return SAT_OK;
}

}  // namespace

extern "C" {

sat_status sat_rect_sums(sat_plan plan, const void* sat, int64_t h, int64_t w,
                         int64_t sat_pitch_bytes, const void* rects, int64_t n, void* out,
                         sat_pair pair, void* stream) {
  sat_status st = check_sat_args(plan, sat, h, w, sat_pitch_bytes, pair);
  if (st != SAT_OK) return st;
  if (n < 0) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "negative query count");
  if (n == 0) return SAT_OK;
  if (!rects || !out) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "NULL rects or out");
  if ((uintptr_t)rects % 16 != 0)
    return sat::fail(SAT_ERR_INVALID_ARGUMENT, "rects must be 16-byte aligned int32[n][4]");
  const size_t ob = sat::multi_channel(pair) ? 4 : sat::out_size(pair);  // channels are u32
  if ((uintptr_t)out % ob != 0) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "out misaligned");
  sat::DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (h == 0 || w == 0) {  // every rectangle is empty
    cudaError_t e = cudaMemsetAsync(out, 0, (size_t)n * sat::out_size(pair), s);
    return e == cudaSuccess ? SAT_OK : sat::cuda_fail(e, "cudaMemsetAsync");
  }
  switch (pair) {
    case SAT_8U_SQ:
      return launch_rects_chan<2>(sat, sat_pitch_bytes, h, w, rects, n, out, s);
    case SAT_8U_HIST4:
      return launch_rects_chan<4>(sat, sat_pitch_bytes, h, w, rects, n, out, s);
    case SAT_8U_32S:
    case SAT_32S_32S:
      return launch_rects<int32_t>(sat, sat_pitch_bytes, h, w, rects, n, out, s);
    case SAT_32F_32F:
    case SAT_8U_32F:
      return launch_rects<float>(sat, sat_pitch_bytes, h, w, rects, n, out, s);
    case SAT_64F_64F:
      return launch_rects<double>(sat, sat_pitch_bytes, h, w, rects, n, out, s);
  }
  return sat::fail(SAT_ERR_INVALID_ARGUMENT, "bad pair");
}

sat_status sat_box_filter(sat_plan plan, const void* sat, void* out, int64_t h, int64_t w,
                          int64_t sat_pitch_bytes, int64_t out_pitch_bytes, int64_t ry,
                          int64_t rx, sat_pair pair, void* stream) {
  sat_status st = check_sat_args(plan, sat, h, w, sat_pitch_bytes, pair);
  if (st != SAT_OK) return st;
  if (ry < 0 || rx < 0) return sat::fail(SAT_ERR_INVALID_ARGUMENT, "negative radius");
  if (sat::multi_channel(pair))
    return sat::fail(SAT_ERR_UNSUPPORTED, "box filter: single-channel SATs only");
  if (h == 0 || w == 0) return SAT_OK;
  const int64_t sb = (int64_t)sat::out_size(pair);
  if (!out || out_pitch_bytes < w * sb || out_pitch_bytes % sb != 0 || (uintptr_t)out % sb != 0)
    return sat::fail(SAT_ERR_INVALID_ARGUMENT, "output pointer / pitch invalid");
  const char* a = static_cast<const char*>(sat);
  const char* b = static_cast<const char*>(out);
  const int64_t sn = (h - 1) * sat_pitch_bytes + w * sb, on = (h - 1) * out_pitch_bytes + w * sb;
  if (a < b + on && b < a + sn)
    return sat::fail(SAT_ERR_UNSUPPORTED, "SAT and output overlap");
  sat::DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  switch (pair) {
    case SAT_8U_32S:
    case SAT_32S_32S:
      return launch_box<int32_t>(sat, out, h, w, sat_pitch_bytes, out_pitch_bytes, ry, rx, s);
    case SAT_32F_32F:
    case SAT_8U_32F:
      return launch_box<float>(sat, out, h, w, sat_pitch_bytes, out_pitch_bytes, ry, rx, s);
    case SAT_64F_64F:
      return launch_box<double>(sat, out, h, w, sat_pitch_bytes, out_pitch_bytes, ry, rx, s);
  }
  return sat::fail(SAT_ERR_INVALID_ARGUMENT, "bad pair");
}

}  // extern "C"
