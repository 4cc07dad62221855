// sat_dist.cu -- row-banded multi-GPU SAT (one process per GPU, NCCL).
//
// Rank r holds rows [r0, r1) of one image.  Its output needs the carry row
// S(r0-1, x) = sum_{x' <= x} sum_{y < r0} A(y, x')  (Eq. 1).
// Plan ("reduce-first"):
//   1. sat_colsum_kernel    : raw column totals of the local band (accumulated
//                              in u32 for 8u, compensated fp64 for 32f/64f);
//   2. ncclAllGather         : every rank receives all ranks' W-vectors over
//                              NVLink/NVSwitch (the one data exchange);
//   3. sat_carry_*_kernels   : exclusive prefix over lower ranks, then the
//                              horizontal inclusive prefix over x, rounded
//                              once to T_B -> the carry-in row;
//   4. sat_tile_kernel       : the band's SAT with that carry-in on its top
//                              tile row (fused carry-add: no extra pass).
// The paper itself is single-node; this path is the build's
// horizontal-scaling extension.
#include <cuda_runtime.h>
#include <dlfcn.h>
#include <stdint.h>
#include <string.h>

#include <algorithm>
#include <vector>
#include <mutex>

#include "nccl.h"
#include "sat_internal.h"

namespace sat {

// ---------------------------------------------------------------------------
// NCCL, loaded at run time (reuses the libnccl.so.2 torch already loaded).
struct NcclApi {
  bool ok = false;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t,
                            cudaStream_t) = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

static NcclApi& nccl() {
  static NcclApi api;
  static std::once_flag once;
  std::call_once(once, [] {
    const char* env = getenv("SAT_NCCL_LIBRARY");
    void* h = env ? dlopen(env, RTLD_NOW | RTLD_GLOBAL) : nullptr;
    if (!h) h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
    if (!h) return;
    api.GetUniqueId = (decltype(api.GetUniqueId))dlsym(h, "ncclGetUniqueId");
    api.CommInitRank = (decltype(api.CommInitRank))dlsym(h, "ncclCommInitRank");
    api.CommDestroy = (decltype(api.CommDestroy))dlsym(h, "ncclCommDestroy");
    api.AllGather = (decltype(api.AllGather))dlsym(h, "ncclAllGather");
    api.GetErrorString = (decltype(api.GetErrorString))dlsym(h, "ncclGetErrorString");
    api.ok = api.GetUniqueId && api.CommInitRank && api.CommDestroy && api.AllGather &&
             api.GetErrorString;
  });
  return api;
}

static sat_status nccl_fail(ncclResult_t r, const char* what) {
  return fail(SAT_ERR_NCCL, "%s: %s", what, nccl().GetErrorString ? nccl().GetErrorString(r) : "?");
}

// ---------------------------------------------------------------------------
// Kernels

constexpr int kColsumThreads = 256;

template <typename TA, typename ACC>
__global__ void sat_colsum_kernel(const char* __restrict__ in, int64_t h, int64_t w, int64_t pitch,
                                  int64_t rows_per_split, ACC* __restrict__ partial) {
  const int64_t x = (int64_t)blockIdx.x * kColsumThreads + threadIdx.x;
  const int64_t y0 = (int64_t)blockIdx.y * rows_per_split;
  const int64_t y1 = min(h, y0 + rows_per_split);
  if (x >= w) return;
  ACC s = ACC(0), comp = ACC(0);
  for (int64_t y = y0; y < y1; ++y) {
    const ACC v = (ACC)reinterpret_cast<const TA*>(in + y * pitch)[x];
    if constexpr (sizeof(ACC) == 8) {  // Kahan-Babuska (Neumaier) compensated sum
      const ACC t = s + v;
      comp += (fabs(s) >= fabs(v)) ? ((s - t) + v) : ((v - t) + s);
      s = t;
    } else {
      s += v;  // u32, exact mod 2^32
    }
  }
  partial[(int64_t)blockIdx.y * w + x] = s + comp;
}

// Vectorised variant: each thread sums V adjacent columns with one 4/16-byte
// load per row (the scalar kernel issues 4-byte loads; this halves the pass).
template <typename TA, typename ACC, int V>
__global__ void sat_colsum_vec_kernel(const char* __restrict__ in, int64_t h, int64_t w,
                                      int64_t pitch, int64_t rows_per_split, ACC* __restrict__ partial) {
  const int64_t x = ((int64_t)blockIdx.x * kColsumThreads + threadIdx.x) * V;
  const int64_t y0 = (int64_t)blockIdx.y * rows_per_split;
  const int64_t y1 = min(h, y0 + rows_per_split);
  if (x >= w) return;
  ACC s[V], comp[V];
#pragma unroll
  for (int v = 0; v < V; ++v) s[v] = comp[v] = ACC(0);
  for (int64_t y = y0; y < y1; ++y) {
    TA a[V];
    const TA* src = reinterpret_cast<const TA*>(in + y * pitch) + x;
    if constexpr (sizeof(TA) * V == 16) {
      *reinterpret_cast<uint4*>(a) = __ldg(reinterpret_cast<const uint4*>(src));
    } else {
      static_assert(sizeof(TA) * V == 4, "4- or 16-byte vectors");
      *reinterpret_cast<uint32_t*>(a) = __ldg(reinterpret_cast<const uint32_t*>(src));
    }
#pragma unroll
    for (int v = 0; v < V; ++v) {
      const ACC val = (ACC)a[v];
      if constexpr (sizeof(ACC) == 8) {
        const ACC t = s[v] + val;
        comp[v] += (fabs(s[v]) >= fabs(val)) ? ((s[v] - t) + val) : ((val - t) + s[v]);
        s[v] = t;
      } else {
        s[v] += val;
      }
    }
  }
#pragma unroll
  for (int v = 0; v < V; ++v) partial[(int64_t)blockIdx.y * w + x + v] = s[v] + comp[v];
}

template <typename ACC>
__global__ void sat_colsum_reduce_kernel(const ACC* __restrict__ partial, int splits, int64_t w,
                                         ACC* __restrict__ out) {
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= w) return;
  ACC s = ACC(0), comp = ACC(0);
  for (int k = 0; k < splits; ++k) {
    const ACC v = partial[(int64_t)k * w + x];
    if constexpr (sizeof(ACC) == 8) {
      const ACC t = s + v;
      comp += (fabs(s) >= fabs(v)) ? ((s - t) + v) : ((v - t) + s);
      s = t;
    } else {
      s += v;
    }
  }
  out[x] = s + comp;
}

// Carry row, three coalesced phases (was one CTA walking strided segments):
//   c(x) = sum_{r' < rank} gathered[r'][x],   carry(x) = sum_{x' <= x} c(x').
// Phase 1: each CTA scans kCarryItems * kCarryThreads consecutive x (thread-
// serial over kCarryItems, then warp shuffles and a shared-memory pass over
// the warps) and writes local prefixes + its total; phase 2 (one thread):
// compensated exclusive scan of the CTA totals; phase 3: add and round once
// to T_B.
constexpr int kCarryThreads = 1024, kCarryItems = 4;
constexpr int kCarryTile = kCarryThreads * kCarryItems;

template <typename ACC>
__device__ __forceinline__ ACC warp_incl_scan(ACC v, int lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const ACC o = __shfl_up_sync(0xffffffffu, v, d);
    if (lane >= d) v += o;
  }
  return v;
}

template <typename ACC>
__global__ void __launch_bounds__(kCarryThreads)
    sat_carry_scan_kernel(const ACC* __restrict__ gathered, int rank, int64_t w,
                          ACC* __restrict__ local, ACC* __restrict__ tile_tot) {
  __shared__ ACC wsum[kCarryThreads / 32];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t base = (int64_t)blockIdx.x * kCarryTile + (int64_t)tid * kCarryItems;
  ACC v[kCarryItems];
  ACC run = ACC(0);
#pragma unroll
  for (int k = 0; k < kCarryItems; ++k) {
    const int64_t x = base + k;
    ACC c = ACC(0);
    if (x < w)
      for (int r = 0; r < rank; ++r) c += gathered[(int64_t)r * w + x];
    run += c;
    v[k] = run;
  }
  const ACC incl = warp_incl_scan(run, lane);
  if (lane == 31) wsum[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    const ACC ws = warp_incl_scan(wsum[lane], lane);
    wsum[lane] = ws;
  }
  __syncthreads();
  const ACC off = (incl - run) + (wid > 0 ? wsum[wid - 1] : ACC(0));
#pragma unroll
  for (int k = 0; k < kCarryItems; ++k)
    if (base + k < w) local[base + k] = off + v[k];
  if (tid == kCarryThreads - 1) tile_tot[blockIdx.x] = wsum[kCarryThreads / 32 - 1];
}

// Phase 2: exclusive scan of the CTA totals by ONE WARP (ntiles = W / 4096,
// e.g. 16 at W = 65536): lane l sums a contiguous segment serially
// (compensated for doubles), the 32 segment totals are scanned with
// shuffles in double-double arithmetic (TwoSum), and each lane writes its
// segment's exclusive offsets.
__device__ __forceinline__ void two_sum(double a, double b, double& s, double& e) {
  s = a + b;
  const double bb = s - a;
  e = (a - (s - bb)) + (b - bb);
}

template <typename ACC>
__global__ void sat_carry_offsets_kernel(ACC* __restrict__ tile_tot, int64_t ntiles) {
  const int lane = threadIdx.x;
  const int64_t per = (ntiles + 31) / 32;
  const int64_t i0 = ntiles < lane * per ? ntiles : lane * per;
  const int64_t i1 = ntiles < i0 + per ? ntiles : i0 + per;
  ACC hi = ACC(0), lo = ACC(0);  // segment total (hi + lo)
  for (int64_t i = i0; i < i1; ++i) {
    if constexpr (sizeof(ACC) == 8) {
      double s, e;
      two_sum(hi, tile_tot[i], s, e);
      hi = s;
      lo += e;
    } else {
      hi += tile_tot[i];
    }
  }
  // inclusive warp scan of (hi, lo)
  ACC ih = hi, il = lo;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const ACC oh = __shfl_up_sync(0xffffffffu, ih, d), ol = __shfl_up_sync(0xffffffffu, il, d);
    if (lane >= d) {
      if constexpr (sizeof(ACC) == 8) {
        double s, e;
        two_sum(ih, oh, s, e);
        ih = s;
        il = il + ol + e;
      } else {
        ih += oh;
      }
    }
  }
  ACC rh = ih - hi, rl = il - lo;  // exclusive: running offset of this segment
  if constexpr (sizeof(ACC) == 8) {
    double s, e;  // (ih, il) - (hi, lo) exactly enough: re-split the high part
    two_sum(ih, -hi, s, e);
    rh = s;
    rl = il - lo + e;
  }
  for (int64_t i = i0; i < i1; ++i) {
    const ACC v = tile_tot[i];
    tile_tot[i] = rh + rl;
    if constexpr (sizeof(ACC) == 8) {
      double s, e;
      two_sum(rh, v, s, e);
      rh = s;
      rl += e;
    } else {
      rh += v;
    }
  }
}

template <typename ACC, typename TB>
__global__ void sat_carry_finish_kernel(const ACC* __restrict__ local, const ACC* __restrict__ tile_off,
                                        int64_t w, TB* __restrict__ carry) {
  const int64_t x = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (x < w) carry[x] = (TB)(tile_off[x / kCarryTile] + local[x]);
}

size_t acc_size(sat_pair p) { return (p == SAT_8U_32S || p == SAT_32S_32S) ? 4 : 8; }

// ---------------------------------------------------------------------------

struct DistBufs {
  int64_t w = 0;
  int nranks = 0;
  int splits = 0;
  void* partial = nullptr;   // [splits][w] ACC
  void* local = nullptr;     // [w] ACC
  void* gathered = nullptr;  // [nranks][w] ACC
  void* carry = nullptr;     // [w] TB
  void* scratch = nullptr;   // band_carry scratch (zeroed once)
  uint32_t epoch = 0;        // band_carry call counter (tile-flag epoch)
};

sat_status colsum(sat_pair pair, const void* in, int64_t h, int64_t w, int64_t pitch,
                  void* partial, int splits, void* out, cudaStream_t s) {
  if (h <= 0) {
    cudaError_t e = cudaMemsetAsync(out, 0, (size_t)w * acc_size(pair), s);
    return e == cudaSuccess ? SAT_OK : cuda_fail(e, "cudaMemsetAsync(colsum)");
  }
  const int64_t rps = (h + splits - 1) / splits;
  const int used = (int)((h + rps - 1) / rps);
  dim3 grid((unsigned)((w + kColsumThreads - 1) / kColsumThreads), (unsigned)used);
  const char* p = static_cast<const char*>(in);
  const int vw = pair == SAT_64F_64F ? 2 : 4;  // elements per vector load
  const int vb = (pair == SAT_8U_32S || pair == SAT_8U_32F) ? 4 : 16;  // bytes per vector load
  if (w % vw == 0 && pitch % vb == 0 && (uintptr_t)in % vb == 0) {
    dim3 gv((unsigned)((w / vw + kColsumThreads - 1) / kColsumThreads), (unsigned)used);
    switch (pair) {
      case SAT_8U_32S:
        sat_colsum_vec_kernel<uint8_t, uint32_t, 4><<<gv, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (uint32_t*)partial);
        sat_colsum_reduce_kernel<uint32_t><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((uint32_t*)partial, used, w, (uint32_t*)out);
        break;
      case SAT_32F_32F:
        sat_colsum_vec_kernel<float, double, 4><<<gv, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
        sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
        break;
      case SAT_8U_32F:
        sat_colsum_vec_kernel<uint8_t, double, 4><<<gv, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
        sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
        break;
      case SAT_32S_32S:
        sat_colsum_vec_kernel<uint32_t, uint32_t, 4><<<gv, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (uint32_t*)partial);
        sat_colsum_reduce_kernel<uint32_t><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((uint32_t*)partial, used, w, (uint32_t*)out);
        break;
      case SAT_64F_64F:
        sat_colsum_vec_kernel<double, double, 2><<<gv, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
        sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
        break;
    }
    cudaError_t e = cudaGetLastError();
    return e == cudaSuccess ? SAT_OK : cuda_fail(e, "sat_colsum_vec_kernel launch");
  }
  switch (pair) {
    case SAT_8U_32S:
      sat_colsum_kernel<uint8_t, uint32_t><<<grid, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (uint32_t*)partial);
      sat_colsum_reduce_kernel<uint32_t><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((uint32_t*)partial, used, w, (uint32_t*)out);
      break;
    case SAT_32F_32F:
      sat_colsum_kernel<float, double><<<grid, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
      sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
      break;
    case SAT_8U_32F:
      sat_colsum_kernel<uint8_t, double><<<grid, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
      sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
      break;
    case SAT_32S_32S:
      sat_colsum_kernel<uint32_t, uint32_t><<<grid, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (uint32_t*)partial);
      sat_colsum_reduce_kernel<uint32_t><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((uint32_t*)partial, used, w, (uint32_t*)out);
      break;
    case SAT_64F_64F:
      sat_colsum_kernel<double, double><<<grid, kColsumThreads, 0, s>>>(p, h, w, pitch, rps, (double*)partial);
      sat_colsum_reduce_kernel<double><<<(unsigned)((w + 255) / 256), 256, 0, s>>>((double*)partial, used, w, (double*)out);
      break;
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "sat_colsum_kernel launch");
}

// One-kernel carry row (ntiles <= kCarryFusedMaxTiles, all CTAs co-resident):
// phase 1 as sat_carry_scan_kernel; each CTA publishes its tile total with an
// epoch flag (release), warp 0 then sums the totals of the tiles to its left
// (acquire; double-double for the float pairs, the same compensated sum as
// the offsets kernel) and every thread adds that offset and rounds once to
// T_B.  Same arithmetic as the three-kernel path, one launch instead of three.
// Small tiles (1024 x) spread the gathered-vector reads over many CTAs.
constexpr int kFusedThreads = 256;
constexpr int64_t kFusedTile = kFusedThreads * kCarryItems;
constexpr int64_t kCarryFusedMaxTiles = 512;  // <= co-resident 256-thread CTAs on 148 SMs

template <typename ACC, typename TB>
__global__ void __launch_bounds__(kFusedThreads)
    sat_carry_fused_kernel(const ACC* __restrict__ gathered, int rank, int64_t w,
                           TB* __restrict__ carry, ACC* tile_tot, uint32_t* flags, uint32_t epoch) {
  __shared__ ACC wsum[32];
  __shared__ ACC toff;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  constexpr int kW = kFusedThreads / 32;
  const int64_t base = (int64_t)blockIdx.x * kFusedTile + (int64_t)tid * kCarryItems;
  ACC v[kCarryItems];
  ACC run = ACC(0);
#pragma unroll
  for (int k = 0; k < kCarryItems; ++k) {
    const int64_t x = base + k;
    ACC c = ACC(0);
    if (x < w)
      for (int r = 0; r < rank; ++r) c += gathered[(int64_t)r * w + x];
    run += c;
    v[k] = run;
  }
  const ACC incl = warp_incl_scan(run, lane);
  if (lane == 31) wsum[wid] = incl;
  __syncthreads();
  if (wid == 0) {
    const ACC ws = warp_incl_scan(lane < kW ? wsum[lane] : ACC(0), lane);
    wsum[lane] = ws;
  }
  __syncthreads();
  const ACC off = (incl - run) + (wid > 0 ? wsum[wid - 1] : ACC(0));
  if (tid == 0) {
    tile_tot[blockIdx.x] = wsum[kW - 1];
    __threadfence();
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flags + blockIdx.x), "r"(epoch) : "memory");
  }
  if (wid == 0) {
    ACC hi = ACC(0), lo = ACC(0);
    for (int64_t i = lane; i < (int64_t)blockIdx.x; i += 32) {
      uint32_t f;
      do {
        asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(f) : "l"(flags + i) : "memory");
      } while (f != epoch);
      const ACC t = *reinterpret_cast<volatile ACC*>(tile_tot + i);
      if constexpr (sizeof(ACC) == 8) {
        double a, e;
        two_sum(hi, t, a, e);
        hi = a;
        lo += e;
      } else {
        hi += t;
      }
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
      const ACC oh = __shfl_down_sync(0xffffffffu, hi, d), ol = __shfl_down_sync(0xffffffffu, lo, d);
      if constexpr (sizeof(ACC) == 8) {
        double a, e;
        two_sum(hi, oh, a, e);
        hi = a;
        lo = lo + ol + e;
      } else {
        hi += oh;
      }
    }
    if (lane == 0) toff = hi + lo;
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kCarryItems; ++k)
    if (base + k < w) carry[base + k] = (TB)(toff + (off + v[k]));
}

// Scratch of band_carry: local prefixes [w] + tile totals (8 bytes each) + tile flags.
size_t carry_scratch_bytes(int64_t w) {
  const int64_t nt = (w + kFusedTile - 1) / kFusedTile;  // >= the 3-kernel path's tile count
  return (size_t)(w + nt) * 8 + (size_t)nt * 4;
}

sat_status band_carry(sat_pair pair, const void* gathered, int rank, int64_t w, void* carry,
                      void* scratch, uint32_t epoch, cudaStream_t s) {
  const int64_t ntiles = (w + kCarryTile - 1) / kCarryTile;
  cudaError_t e = cudaSuccess;
  const unsigned fin = (unsigned)((w + 255) / 256);
  const int64_t nfused = (w + kFusedTile - 1) / kFusedTile;
  if (nfused <= kCarryFusedMaxTiles) {
    const unsigned ntiles = (unsigned)nfused;
    uint32_t* flags = reinterpret_cast<uint32_t*>(static_cast<char*>(scratch) + (size_t)(w + nfused) * 8);
    switch (pair) {
      case SAT_8U_32S:
      case SAT_32S_32S:
        sat_carry_fused_kernel<uint32_t, uint32_t><<<ntiles, kFusedThreads, 0, s>>>(
            (const uint32_t*)gathered, rank, w, (uint32_t*)carry, (uint32_t*)scratch, flags, epoch);
        break;
      case SAT_32F_32F:
      case SAT_8U_32F:
        sat_carry_fused_kernel<double, float><<<ntiles, kFusedThreads, 0, s>>>(
            (const double*)gathered, rank, w, (float*)carry, (double*)scratch, flags, epoch);
        break;
      case SAT_64F_64F:
        sat_carry_fused_kernel<double, double><<<ntiles, kFusedThreads, 0, s>>>(
            (const double*)gathered, rank, w, (double*)carry, (double*)scratch, flags, epoch);
        break;
    }
    e = cudaGetLastError();
    return e == cudaSuccess ? SAT_OK : cuda_fail(e, "sat_carry_fused_kernel launch");
  }
  switch (pair) {
    case SAT_8U_32S:
    case SAT_32S_32S: {
      uint32_t* loc = (uint32_t*)scratch;
      uint32_t* tt = loc + w;
      sat_carry_scan_kernel<uint32_t><<<(unsigned)ntiles, kCarryThreads, 0, s>>>((const uint32_t*)gathered, rank, w, loc, tt);
      sat_carry_offsets_kernel<uint32_t><<<1, 32, 0, s>>>(tt, ntiles);
      sat_carry_finish_kernel<uint32_t, uint32_t><<<fin, 256, 0, s>>>(loc, tt, w, (uint32_t*)carry);
      break;
    }
    case SAT_32F_32F:
    case SAT_8U_32F:
    case SAT_64F_64F: {
      double* loc = (double*)scratch;
      double* tt = loc + w;
      sat_carry_scan_kernel<double><<<(unsigned)ntiles, kCarryThreads, 0, s>>>((const double*)gathered, rank, w, loc, tt);
      sat_carry_offsets_kernel<double><<<1, 32, 0, s>>>(tt, ntiles);
      if (pair != SAT_64F_64F)
        sat_carry_finish_kernel<double, float><<<fin, 256, 0, s>>>(loc, tt, w, (float*)carry);
      else
        sat_carry_finish_kernel<double, double><<<fin, 256, 0, s>>>(loc, tt, w, (double*)carry);
      break;
    }
  }
  e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "carry kernels launch");
}

}  // namespace sat

using namespace sat;

// Chained-band state (sat_compute_dist_chained): this rank's link and the
// peer-mapped links of the ranks above and below (CUDA IPC over NVLink),
// exchanged once per width; calls then need no collective at all (the links'
// ack words give device-side flow control, see KParams).
struct ChainBufs {
  int64_t w = 0;
  size_t bytes = 0;
  void* link = nullptr;        // own link (ack words + 2 receive slots)
  void* peer_above = nullptr;  // rank - 1's link
  void* peer_below = nullptr;  // rank + 1's link
  void* hdl_dev = nullptr;     // [nranks] IPC handles (allgather staging)
  uint32_t epoch = 0;
};

struct sat_comm_st {
  ncclComm_t comm = nullptr;
  int nranks = 0, rank = 0, device = 0;
  DistBufs bufs;
  ChainBufs chain;
};

static void free_chain(ChainBufs& c) {
  if (c.peer_above) cudaIpcCloseMemHandle(c.peer_above);
  if (c.peer_below) cudaIpcCloseMemHandle(c.peer_below);
  if (c.link) cudaFree(c.link);
  if (c.hdl_dev) cudaFree(c.hdl_dev);
  c = ChainBufs();
}

static void free_bufs(DistBufs& b) {
  if (b.partial) cudaFree(b.partial);
  if (b.local) cudaFree(b.local);
  if (b.gathered) cudaFree(b.gathered);
  if (b.carry) cudaFree(b.carry);
  if (b.scratch) cudaFree(b.scratch);
  b = DistBufs();
}

static sat_status ensure_bufs(DistBufs& b, int64_t w, int nranks) {
  if (b.w >= w && b.nranks >= nranks) return SAT_OK;
  free_bufs(b);
  b.w = w;
  b.nranks = nranks;
  b.splits = 64;
  cudaError_t e = cudaMalloc(&b.partial, (size_t)b.splits * w * 8);
  if (e == cudaSuccess) e = cudaMalloc(&b.local, (size_t)w * 8);
  if (e == cudaSuccess) e = cudaMalloc(&b.gathered, (size_t)nranks * w * 8);
  if (e == cudaSuccess) e = cudaMalloc(&b.carry, (size_t)w * 8);
  if (e == cudaSuccess) e = cudaMalloc(&b.scratch, carry_scratch_bytes(w));
  if (e == cudaSuccess) e = cudaMemset(b.scratch, 0, carry_scratch_bytes(w));
  if (e != cudaSuccess) {
    free_bufs(b);
    return cuda_fail(e, "dist buffers");
  }
  return SAT_OK;
}

extern "C" {

sat_status sat_band_partition(int64_t h, int nranks, int rank, int64_t* r0, int64_t* r1) {
  if (!r0 || !r1 || h < 0 || nranks < 1 || rank < 0 || rank >= nranks)
    return fail(SAT_ERR_INVALID_ARGUMENT, "bad partition request (h=%lld, rank %d of %d)",
                (long long)h, rank, nranks);
  const int64_t base = h / nranks, extra = h % nranks;
  *r0 = rank * base + std::min<int64_t>(rank, extra);
  *r1 = *r0 + base + (rank < extra ? 1 : 0);
  return SAT_OK;
}

sat_status sat_comm_unique_id(void* id_out) {
  if (!id_out) return fail(SAT_ERR_INVALID_ARGUMENT, "id_out is NULL");
  if (!nccl().ok) return fail(SAT_ERR_NCCL, "libnccl.so.2 could not be loaded");
  ncclUniqueId id;
  ncclResult_t r = nccl().GetUniqueId(&id);
  if (r != ncclSuccess) return nccl_fail(r, "ncclGetUniqueId");
  static_assert(sizeof(id) == SAT_COMM_ID_BYTES, "unique id size");
  memcpy(id_out, &id, sizeof(id));
  return SAT_OK;
}

sat_status sat_comm_create(sat_comm* comm, const void* id, int nranks, int rank, int device) {
  if (!comm || !id) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  *comm = nullptr;
  if (nranks < 1 || rank < 0 || rank >= nranks)
    return fail(SAT_ERR_INVALID_ARGUMENT, "bad rank %d of %d", rank, nranks);
  if (!nccl().ok) return fail(SAT_ERR_NCCL, "libnccl.so.2 could not be loaded");
  DeviceGuard g(device);
  ncclUniqueId uid;
  memcpy(&uid, id, sizeof(uid));
  sat_comm_st* c = new sat_comm_st();
  c->nranks = nranks;
  c->rank = rank;
  c->device = device;
  ncclResult_t r = nccl().CommInitRank(&c->comm, nranks, uid, rank);
  if (r != ncclSuccess) {
    delete c;
    return nccl_fail(r, "ncclCommInitRank");
  }
  *comm = c;
  return SAT_OK;
}

sat_status sat_comm_destroy(sat_comm comm) {
  if (!comm) return SAT_OK;
  DeviceGuard g(comm->device);
  cudaDeviceSynchronize();
  free_bufs(comm->bufs);
  free_chain(comm->chain);
  if (comm->comm) nccl().CommDestroy(comm->comm);
  delete comm;
  return SAT_OK;
}

// Plan-owned scratch of the exported building blocks: grown (synchronously,
// after draining the plan's last stream) only when a wider call needs more.
static sat_status plan_dist_scratch(sat_plan plan, size_t bytes) {
  if (plan->dist_scratch_bytes >= bytes) return SAT_OK;
  cudaDeviceSynchronize();
  if (plan->dist_scratch) cudaFree(plan->dist_scratch);
  plan->dist_scratch = nullptr;
  plan->dist_scratch_bytes = 0;
  cudaError_t e = cudaMalloc(&plan->dist_scratch, bytes);
  if (e == cudaSuccess) e = cudaMemset(plan->dist_scratch, 0, bytes);
  if (e != cudaSuccess) return cuda_fail(e, "dist scratch");
  plan->dist_epoch = 0;
  plan->dist_scratch_bytes = bytes;
  return SAT_OK;
}

// Building blocks of sat_compute_dist, exported so that the carry algebra can
// be exercised on one GPU with "virtual ranks" (tests/test_dist_gpu.py).
size_t sat_dist_acc_bytes(sat_pair pair) { return acc_size(pair); }

sat_status sat_dist_colsum(sat_plan plan, const void* in_band, int64_t band_h, int64_t w,
                           int64_t in_pitch_bytes, void* acc_out, void* stream) {
  if (plan && multi_channel(plan->pair))
    return fail(SAT_ERR_UNSUPPORTED, "row-banded building blocks: single-channel pairs only");
  if (!plan || !acc_out || (band_h > 0 && !in_band))
    return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  if (band_h < 0 || w <= 0 || w > plan->max_w)
    return fail(SAT_ERR_INVALID_ARGUMENT, "bad extent");
  if (in_pitch_bytes < w * (int64_t)in_size(plan->pair))
    return fail(SAT_ERR_INVALID_ARGUMENT, "bad pitch");
  DeviceGuard g(plan->device);
  sat_status st = plan_dist_scratch(plan, (size_t)64 * w * 8);
  if (st != SAT_OK) return st;
  return colsum(plan->pair, in_band, band_h, w, in_pitch_bytes, plan->dist_scratch, 64, acc_out,
                (cudaStream_t)stream);
}

sat_status sat_dist_carry(sat_plan plan, const void* gathered, int nranks, int rank, int64_t w,
                          void* carry_out, void* stream) {
  if (plan && multi_channel(plan->pair))
    return fail(SAT_ERR_UNSUPPORTED, "row-banded building blocks: single-channel pairs only");
  if (!plan || !gathered || !carry_out) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  if (nranks < 1 || rank < 0 || rank >= nranks || w <= 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "bad rank/extent");
  DeviceGuard g(plan->device);
  sat_status st = plan_dist_scratch(plan, carry_scratch_bytes(w));
  if (st != SAT_OK) return st;
  if (++plan->dist_epoch == 0) ++plan->dist_epoch;
  return band_carry(plan->pair, gathered, rank, w, carry_out, plan->dist_scratch, plan->dist_epoch,
                    (cudaStream_t)stream);
}

sat_status sat_compute_dist(sat_plan plan, sat_comm comm, const void* in_band, void* out_band,
                            int64_t band_h, int64_t w, int64_t in_pitch_bytes,
                            int64_t out_pitch_bytes, sat_pair pair, void* stream) {
  if (!comm) return fail(SAT_ERR_INVALID_ARGUMENT, "comm is NULL");
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (multi_channel(plan->pair))
    return fail(SAT_ERR_UNSUPPORTED, "row-banded SAT: single-channel pairs only");
  if (w <= 0) return fail(SAT_ERR_INVALID_ARGUMENT, "w must be positive for a collective call");
  bool empty = false;
  if (band_h > 0) {
    sat_status st = validate(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                             band_h * in_pitch_bytes, band_h * out_pitch_bytes, 1, pair, &empty);
    if (st != SAT_OK) return st;
  } else if (band_h < 0) {
    return fail(SAT_ERR_INVALID_ARGUMENT, "negative band height");
  } else if (pair != plan->pair || w > plan->max_w) {
    return fail(SAT_ERR_INVALID_ARGUMENT, "pair/extent does not match the plan");
  }
  DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (comm->nranks == 1) {  // one band = the whole image: no carry to exchange
    if (band_h == 0) return SAT_OK;
    return launch(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                  band_h * in_pitch_bytes, band_h * out_pitch_bytes, 1, nullptr, s);
  }
  DistBufs& b = comm->bufs;
  sat_status st = ensure_bufs(b, w, comm->nranks);
  if (st != SAT_OK) return st;
  st = colsum(pair, in_band, band_h, w, in_pitch_bytes, b.partial, b.splits, b.local, s);
  if (st != SAT_OK) return st;
  const ncclDataType_t dt = acc_size(pair) == 4 ? ncclUint32 : ncclFloat64;
  ncclResult_t r = nccl().AllGather(b.local, b.gathered, (size_t)w, dt, comm->comm, s);
  if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather");
  if (++b.epoch == 0) ++b.epoch;  // tile flags: epoch-tagged, never re-zeroed
  st = band_carry(pair, b.gathered, comm->rank, w, b.carry, b.scratch, b.epoch, s);
  if (st != SAT_OK) return st;
  if (band_h == 0) return SAT_OK;
  return launch(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                band_h * in_pitch_bytes, band_h * out_pitch_bytes, 1,
                comm->rank > 0 ? b.carry : nullptr, s);
}


static bool valid_pair(sat_pair pair) {
  return pair == SAT_8U_32S || pair == SAT_32F_32F || pair == SAT_64F_64F || pair == SAT_8U_32F ||
         pair == SAT_32S_32S;
}

// Link layout: [ack words: nchunks u32, padded to 256 B][slot 0][slot 1], a
// slot = one tagged 64-bit word per 32-bit half of each output element, per chunk.
static size_t chain_ack_bytes(sat_pair pair, int64_t w) {
  const int64_t nch = (w + tile_w(pair) - 1) / tile_w(pair);
  return (size_t)((nch * 4 + 255) / 256 * 256);
}
static size_t chain_slot_bytes(sat_pair pair, int64_t w) {
  const int64_t tw = tile_w(pair);
  return (size_t)((w + tw - 1) / tw) * (size_t)tw * out_size(pair) * 2;
}

size_t sat_chain_bytes(sat_pair pair, int64_t w) {
  if (w <= 0 || !valid_pair(pair)) return 0;
  return chain_ack_bytes(pair, w) + 2 * chain_slot_bytes(pair, w);
}

sat_status sat_chain_link_create(int device, sat_pair pair, int64_t w, void** link) {
  if (!link) return fail(SAT_ERR_INVALID_ARGUMENT, "link out-pointer is NULL");
  *link = nullptr;
  if (w <= 0 || !valid_pair(pair)) return fail(SAT_ERR_INVALID_ARGUMENT, "bad pair or width");
  DeviceGuard g(device);
  void* p = nullptr;
  cudaError_t e = cudaMalloc(&p, sat_chain_bytes(pair, w));
  if (e == cudaSuccess) e = cudaMemset(p, 0, sat_chain_bytes(pair, w));
  if (e != cudaSuccess) {
    if (p) cudaFree(p);
    return cuda_fail(e, "sat_chain_link_create");
  }
  *link = p;
  return SAT_OK;
}

sat_status sat_chain_link_destroy(void* link) {
  if (!link) return SAT_OK;
  cudaError_t e = cudaFree(link);
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "sat_chain_link_destroy");
}

sat_status sat_chain_ipc_handle(const void* link, void* handle_out) {
  if (!link || !handle_out) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  static_assert(sizeof(cudaIpcMemHandle_t) == SAT_IPC_HANDLE_BYTES, "IPC handle size");
  cudaIpcMemHandle_t h;
  cudaError_t e = cudaIpcGetMemHandle(&h, const_cast<void*>(link));
  if (e != cudaSuccess) return cuda_fail(e, "cudaIpcGetMemHandle");
  memcpy(handle_out, &h, sizeof(h));
  return SAT_OK;
}

sat_status sat_chain_open_peer(int device, const void* handle, void** peer_link) {
  if (!handle || !peer_link) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  *peer_link = nullptr;
  DeviceGuard g(device);
  cudaIpcMemHandle_t h;
  memcpy(&h, handle, sizeof(h));
  cudaError_t e = cudaIpcOpenMemHandle(peer_link, h, cudaIpcMemLazyEnablePeerAccess);
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "cudaIpcOpenMemHandle");
}

sat_status sat_chain_close_peer(void* peer_link) {
  if (!peer_link) return SAT_OK;
  cudaError_t e = cudaIpcCloseMemHandle(peer_link);
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "cudaIpcCloseMemHandle");
}

sat_status sat_compute_band_chained(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                                    int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                                    void* link_self, void* link_above, void* link_below,
                                    uint32_t epoch, sat_pair pair, void* stream) {
  if (h <= 0 || w <= 0) return fail(SAT_ERR_INVALID_ARGUMENT, "a chained band needs h, w >= 1");
  if (epoch == 0 || epoch >= (1u << 30))
    return fail(SAT_ERR_INVALID_ARGUMENT, "epoch must be in [1, 2^30)");
  if ((link_above || link_below) && !link_self)
    return fail(SAT_ERR_INVALID_ARGUMENT, "a band with a neighbour needs its own link");
  if (((uintptr_t)link_self | (uintptr_t)link_above | (uintptr_t)link_below) % 256 != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "chain links must be 256-byte aligned");
  bool empty = false;
  sat_status st = validate(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                           h * in_pitch_bytes, h * out_pitch_bytes, 1, pair, &empty);
  if (st != SAT_OK || empty) return st;
  DeviceGuard g(plan->device);
  const size_t ab = chain_ack_bytes(pair, w), sb = chain_slot_bytes(pair, w);
  const size_t slot = ab + (size_t)(epoch & 1u) * sb;
  ChainSpec chain;
  chain.in = link_above ? static_cast<const char*>(link_self) + slot : nullptr;
  chain.ack_out = link_above ? static_cast<uint32_t*>(link_above) : nullptr;
  chain.out = link_below ? static_cast<char*>(link_below) + slot : nullptr;
  chain.ack_in = link_below ? static_cast<const uint32_t*>(link_self) : nullptr;
  chain.epoch = epoch;
  return launch(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes, h * in_pitch_bytes,
                h * out_pitch_bytes, 1, nullptr, static_cast<cudaStream_t>(stream), nullptr, &chain);
}

sat_status sat_compute_dist_chained(sat_plan plan, sat_comm comm, const void* in_band,
                                    void* out_band, int64_t band_h, int64_t w,
                                    int64_t in_pitch_bytes, int64_t out_pitch_bytes, sat_pair pair,
                                    void* stream) {
  if (!comm) return fail(SAT_ERR_INVALID_ARGUMENT, "comm is NULL");
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (band_h <= 0 || w <= 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "every rank needs a band of >= 1 row (H >= nranks)");
  bool empty = false;
  sat_status st = validate(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                           band_h * in_pitch_bytes, band_h * out_pitch_bytes, 1, pair, &empty);
  if (st != SAT_OK) return st;
  DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (comm->nranks == 1)
    return launch(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                  band_h * in_pitch_bytes, band_h * out_pitch_bytes, 1, nullptr, s);
  ChainBufs& c = comm->chain;
  const size_t bytes = sat_chain_bytes(pair, w);
  if (c.bytes != bytes || c.w != w) {  // (re)build: collective, every rank calls with the same w
    cudaStreamSynchronize(s);
    free_chain(c);
    const size_t hb = sizeof(cudaIpcMemHandle_t);
    st = sat_chain_link_create(comm->device, pair, w, &c.link);
    if (st != SAT_OK) return st;
    cudaError_t e = cudaMalloc(&c.hdl_dev, (size_t)comm->nranks * hb);
    unsigned char mine[SAT_IPC_HANDLE_BYTES];
    if (e == cudaSuccess) {
      st = sat_chain_ipc_handle(c.link, mine);
      if (st != SAT_OK) {
        free_chain(c);
        return st;
      }
      e = cudaMemcpyAsync(static_cast<char*>(c.hdl_dev) + comm->rank * hb, mine, hb,
                          cudaMemcpyHostToDevice, s);
    }
    if (e != cudaSuccess) {
      free_chain(c);
      return cuda_fail(e, "chain handle staging");
    }
    ncclResult_t r = nccl().AllGather(static_cast<char*>(c.hdl_dev) + comm->rank * hb, c.hdl_dev, hb,
                                      ncclUint8, comm->comm, s);
    if (r != ncclSuccess) return nccl_fail(r, "ncclAllGather(ipc handles)");
    std::vector<unsigned char> all((size_t)comm->nranks * hb);
    e = cudaMemcpyAsync(all.data(), c.hdl_dev, all.size(), cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    if (e != cudaSuccess) {
      free_chain(c);
      return cuda_fail(e, "chain handle exchange");
    }
    if (comm->rank > 0) st = sat_chain_open_peer(comm->device, &all[(comm->rank - 1) * hb], &c.peer_above);
    if (st == SAT_OK && comm->rank + 1 < comm->nranks)
      st = sat_chain_open_peer(comm->device, &all[(comm->rank + 1) * hb], &c.peer_below);
    if (st != SAT_OK) {
      free_chain(c);
      return st;
    }
    c.bytes = bytes;
    c.w = w;
    c.epoch = 0;
  }
  if (++c.epoch >= (1u << 30)) return fail(SAT_ERR_UNSUPPORTED, "chain epochs exhausted: recreate the comm");
  return sat_compute_band_chained(plan, in_band, out_band, band_h, w, in_pitch_bytes, out_pitch_bytes,
                                  c.link, c.peer_above, c.peer_below, c.epoch, pair, stream);
}

}  // extern "C"
