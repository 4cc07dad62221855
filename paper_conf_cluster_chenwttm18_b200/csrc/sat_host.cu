// sat_host.cu -- streamed end-to-end path for HOST images (sat_compute_host).
//
// The image is cut into row bands; band i is copied host->device on an
// internal stream, its SAT is computed on the caller's stream with the last
// output row of band i-1 as carry-in (sat_compute_band semantics: the band's
// S(r0-1, .) row is exactly that row), and the result is copied device->host
// on a second internal stream.  Three buffer sets let the H2D of band i+1, the
// SAT of band i and the D2H of band i-1 overlap, so the call runs at the
// PCIe/C2C copy rate rather than copy + compute.
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "sat_internal.h"

namespace sat {

constexpr int kHostBufs = 3;

struct HostPath {
  int64_t band_rows = 0, w = 0;
  size_t in_bytes = 0, out_bytes = 0;
  void* din[kHostBufs] = {};
  void* dout[kHostBufs] = {};
  cudaStream_t s_in = nullptr, s_out = nullptr;
  cudaEvent_t ev_start = nullptr;
  cudaEvent_t ev_in[kHostBufs] = {}, ev_comp[kHostBufs] = {}, ev_out[kHostBufs] = {};
};

void host_path_release(sat_plan_st* pl) {
  HostPath* hp = pl->host;
  if (!hp) return;
  if (hp->s_in) cudaStreamSynchronize(hp->s_in);
  if (hp->s_out) cudaStreamSynchronize(hp->s_out);
  for (int j = 0; j < kHostBufs; ++j) {
    if (hp->din[j]) cudaFree(hp->din[j]);
    if (hp->dout[j]) cudaFree(hp->dout[j]);
    if (hp->ev_in[j]) cudaEventDestroy(hp->ev_in[j]);
    if (hp->ev_comp[j]) cudaEventDestroy(hp->ev_comp[j]);
    if (hp->ev_out[j]) cudaEventDestroy(hp->ev_out[j]);
  }
  if (hp->ev_start) cudaEventDestroy(hp->ev_start);
  if (hp->s_in) cudaStreamDestroy(hp->s_in);
  if (hp->s_out) cudaStreamDestroy(hp->s_out);
  delete hp;
  pl->host = nullptr;
}

static sat_status host_path_ensure(sat_plan_st* pl, int64_t h, int64_t w) {
  const size_t sa = in_size(pl->pair), sb = out_size(pl->pair);
  const int64_t TH = tile_h(pl->pair);
  // ~48 MiB of input+output per band, a multiple of the tile height.
  int64_t rows = (int64_t)((48ull << 20) / ((size_t)w * (sa + sb)));
  rows = std::max<int64_t>(TH, rows / TH * TH);
  rows = std::min<int64_t>(rows, (h + TH - 1) / TH * TH);
  rows = std::min<int64_t>(rows, pl->max_h);
  HostPath* hp = pl->host;
  if (hp && hp->w >= w && hp->band_rows >= rows) return SAT_OK;
  if (hp) host_path_release(pl);
  hp = new HostPath();
  pl->host = hp;
  hp->band_rows = rows;
  hp->w = w;
  hp->in_bytes = (size_t)rows * w * sa;
  hp->out_bytes = (size_t)rows * w * sb;
  cudaError_t e = cudaSuccess;
  for (int j = 0; j < kHostBufs && e == cudaSuccess; ++j) {
    e = cudaMalloc(&hp->din[j], hp->in_bytes);
    if (e == cudaSuccess) e = cudaMalloc(&hp->dout[j], hp->out_bytes);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&hp->ev_in[j], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&hp->ev_comp[j], cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&hp->ev_out[j], cudaEventDisableTiming);
  }
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&hp->ev_start, cudaEventDisableTiming);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&hp->s_in, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&hp->s_out, cudaStreamNonBlocking);
  if (e != cudaSuccess) {
    host_path_release(pl);
    return cuda_fail(e, "host path staging allocation");
  }
  return SAT_OK;
}

}  // namespace sat

using namespace sat;

extern "C" sat_status sat_compute_host(sat_plan plan, const void* in_host, void* out_host,
                                       int64_t h, int64_t w, int64_t in_pitch_bytes,
                                       int64_t out_pitch_bytes, sat_pair pair, void* stream) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (pair != plan->pair) return fail(SAT_ERR_INVALID_ARGUMENT, "pair does not match the plan");
  if (h < 0 || w < 0) return fail(SAT_ERR_INVALID_ARGUMENT, "negative extent");
  if (h == 0 || w == 0) return SAT_OK;
  if (!in_host || !out_host) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL host pointer");
  if (w > plan->max_w) return fail(SAT_ERR_INVALID_ARGUMENT, "w exceeds the plan limit");
  const int64_t sa = (int64_t)in_size(pair), sb = (int64_t)out_size(pair);
  if (in_pitch_bytes < w * sa || out_pitch_bytes < w * sb)
    return fail(SAT_ERR_INVALID_ARGUMENT, "pitch smaller than a row");
  DeviceGuard g(plan->device);
  sat_status st = host_path_ensure(plan, h, w);
  if (st != SAT_OK) return st;
  HostPath* hp = plan->host;
  cudaStream_t cs = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaEventRecord(hp->ev_start, cs);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(hp->s_in, hp->ev_start, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(hp->s_out, hp->ev_start, 0);
  if (e != cudaSuccess) return cuda_fail(e, "host path ordering");
  const int64_t nb = (h + hp->band_rows - 1) / hp->band_rows;
  for (int64_t i = 0; i < nb; ++i) {
    const int j = (int)(i % kHostBufs);
    const int64_t r0 = i * hp->band_rows;
    const int64_t rows = std::min(hp->band_rows, h - r0);
    // H2D: buffer j's previous band must have finished computing.
    if (i >= kHostBufs) e = cudaStreamWaitEvent(hp->s_in, hp->ev_comp[j], 0);
    if (e == cudaSuccess)
      e = cudaMemcpy2DAsync(hp->din[j], (size_t)(w * sa),
                            static_cast<const char*>(in_host) + r0 * in_pitch_bytes,
                            (size_t)in_pitch_bytes, (size_t)(w * sa), (size_t)rows,
                            cudaMemcpyHostToDevice, hp->s_in);
    if (e == cudaSuccess) e = cudaEventRecord(hp->ev_in[j], hp->s_in);
    // SAT on the caller's stream; output buffer j must have been drained.
    if (e == cudaSuccess) e = cudaStreamWaitEvent(cs, hp->ev_in[j], 0);
    if (e == cudaSuccess && i >= kHostBufs) e = cudaStreamWaitEvent(cs, hp->ev_out[j], 0);
    if (e != cudaSuccess) return cuda_fail(e, "host path H2D");
    const void* carry = nullptr;
    if (i > 0) {
      const int jp = (int)((i - 1) % kHostBufs);
      carry = static_cast<const char*>(hp->dout[jp]) + (size_t)(hp->band_rows - 1) * w * sb;
    }
    st = launch(plan, hp->din[j], hp->dout[j], rows, w, w * sa, w * sb, rows * w * sa,
                rows * w * sb, 1, carry, cs);
    if (st != SAT_OK) return st;
    e = cudaEventRecord(hp->ev_comp[j], cs);
    // D2H
    if (e == cudaSuccess) e = cudaStreamWaitEvent(hp->s_out, hp->ev_comp[j], 0);
    if (e == cudaSuccess)
      e = cudaMemcpy2DAsync(static_cast<char*>(out_host) + r0 * out_pitch_bytes,
                            (size_t)out_pitch_bytes, hp->dout[j], (size_t)(w * sb),
                            (size_t)(w * sb), (size_t)rows, cudaMemcpyDeviceToHost, hp->s_out);
    if (e == cudaSuccess) e = cudaEventRecord(hp->ev_out[j], hp->s_out);
    if (e != cudaSuccess) return cuda_fail(e, "host path D2H");
  }
  // The caller's stream waits for the last copies.
  e = cudaStreamWaitEvent(cs, hp->ev_out[(nb - 1) % kHostBufs], 0);
  if (e != cudaSuccess) return cuda_fail(e, "host path completion");
  return SAT_OK;
}
