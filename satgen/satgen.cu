// satgen.cu -- device and host fill entry points of the seeded input generator
// (libsatgen.so).  Test/bench infrastructure: no summed-area-table arithmetic
// lives here, only coordinate -> value mapping from satgen.h.
#include <cuda_runtime.h>
#include <stdint.h>
#include <string.h>

#include "satgen.h"

namespace {

template <typename T>
__host__ __device__ inline T gen_value(int kind, uint64_t seed, uint64_t img, uint64_t y,
                                       uint64_t x, int mode, double value);

template <>
__host__ __device__ inline uint8_t gen_value<uint8_t>(int, uint64_t s, uint64_t n, uint64_t y,
                                                      uint64_t x, int m, double v) {
  return satgen_u8(s, n, y, x, m, v);
}
template <>
__host__ __device__ inline float gen_value<float>(int, uint64_t s, uint64_t n, uint64_t y,
                                                  uint64_t x, int m, double v) {
  return satgen_f32(s, n, y, x, m, v);
}
template <>
__host__ __device__ inline double gen_value<double>(int, uint64_t s, uint64_t n, uint64_t y,
                                                    uint64_t x, int m, double v) {
  return satgen_f64(s, n, y, x, m, v);
}

template <typename T>
__global__ void fill_kernel(int mode, uint64_t seed, double value, char* dst, int64_t H, int64_t W,
                            int64_t pitch, int64_t batch, int64_t img_stride, int64_t img0,
                            int64_t y0) {
  const int64_t rows = H * batch;
  for (int64_t r = blockIdx.y; r < rows; r += gridDim.y) {
    const int64_t n = r / H, y = r % H;
    T* row = reinterpret_cast<T*>(dst + n * img_stride + y * pitch);
    for (int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; x < W;
         x += (int64_t)gridDim.x * blockDim.x)
      row[x] = gen_value<T>(0, seed, (uint64_t)(img0 + n), (uint64_t)(y0 + y), (uint64_t)x, mode,
                            value);
  }
}

template <typename T>
void fill_host(int mode, uint64_t seed, double value, char* dst, int64_t H, int64_t W, int64_t pitch,
               int64_t batch, int64_t img_stride, int64_t img0, int64_t y0) {
  for (int64_t n = 0; n < batch; ++n)
    for (int64_t y = 0; y < H; ++y) {
      T* row = reinterpret_cast<T*>(dst + n * img_stride + y * pitch);
      for (int64_t x = 0; x < W; ++x)
        row[x] = gen_value<T>(0, seed, (uint64_t)(img0 + n), (uint64_t)(y0 + y), (uint64_t)x, mode,
                              value);
    }
}

}  // namespace

extern "C" {

// kind: 0 = u8, 1 = f32, 2 = f64 (enum satgen_kind); mode: enum satgen_mode.
// Fills batch images of H rows x W elements at dst (pitched, bytes), using
// global coordinates (img0 + n, y0 + y, x).  Returns a cudaError_t value.
int satgen_fill_device(int kind, int mode, uint64_t seed, double value, void* dst, int64_t H,
                       int64_t W, int64_t pitch_bytes, int64_t batch, int64_t image_stride_bytes,
                       int64_t img0, int64_t y0, void* stream) {
  if (H <= 0 || W <= 0 || batch <= 0) return 0;
  const int64_t rows = H * batch;
  dim3 block(256);
  dim3 grid((unsigned)((W + 255) / 256 < 64 ? (W + 255) / 256 : 64),
            (unsigned)(rows < 65535 ? rows : 65535));
  cudaStream_t s = (cudaStream_t)stream;
  char* d = (char*)dst;
  switch (kind) {
    case SATGEN_U8:
      fill_kernel<uint8_t><<<grid, block, 0, s>>>(mode, seed, value, d, H, W, pitch_bytes, batch,
                                                  image_stride_bytes, img0, y0);
      break;
    case SATGEN_F32:
      fill_kernel<float><<<grid, block, 0, s>>>(mode, seed, value, d, H, W, pitch_bytes, batch,
                                                image_stride_bytes, img0, y0);
      break;
    case SATGEN_F64:
      fill_kernel<double><<<grid, block, 0, s>>>(mode, seed, value, d, H, W, pitch_bytes, batch,
                                                 image_stride_bytes, img0, y0);
      break;
    default:
      return (int)cudaErrorInvalidValue;
  }
  return (int)cudaGetLastError();
}

int satgen_fill_host(int kind, int mode, uint64_t seed, double value, void* dst, int64_t H,
                     int64_t W, int64_t pitch_bytes, int64_t batch, int64_t image_stride_bytes,
                     int64_t img0, int64_t y0) {
  char* d = (char*)dst;
  switch (kind) {
    case SATGEN_U8:
      fill_host<uint8_t>(mode, seed, value, d, H, W, pitch_bytes, batch, image_stride_bytes, img0,
                         y0);
      return 0;
    case SATGEN_F32:
      fill_host<float>(mode, seed, value, d, H, W, pitch_bytes, batch, image_stride_bytes, img0,
                       y0);
      return 0;
    case SATGEN_F64:
      fill_host<double>(mode, seed, value, d, H, W, pitch_bytes, batch, image_stride_bytes, img0,
                        y0);
      return 0;
  }
  return 1;
}

}  // extern "C"
