// sat_kernel.cuh -- single-pass summed-area-table kernel for sm_100a.
//
// What it computes: the inclusive SAT S(i,j) = sum_{y<=i, x<=j} A(y,x)
// (Eq. 1) of pitched row-major images, in one HBM pass.
//
// Decomposition: the image is cut into
// row BANDS of TH rows; a band is walked left-to-right in CHUNKS of TW columns
// by one persistent CTA.  For tile (band k, chunk c) with rows [r0, r1):
//   R(y, x)  = rowcarry(y) + rowprefix_tile(y, x)        (horizontal carry is
//              the CTA's own running row total: the paper's ScanRow chunk
//              carry, PAPER.md:258 / Fig. 4, kept in registers)
//   S'(i, x) = sum_{r0 <= y <= i} R(y, x)                (per-thread serial
//              column scan down the tile, PAPER.md:260 ScanColumn / Alg. 2)
//   S(i, x)  = V_up(x) + S'(i, x),  V_up(x) = S(r0 - 1, x)
// The vertical carry V_up is the only cross-CTA quantity.  It is obtained by
// a decoupled look-back up the tile column: each tile publishes its vertical
// aggregate S'(r1 - 1, .) and then its inclusive prefix V_up + S'(r1 - 1, .).
//
// Inside a tile (Alg. 2 and Alg. 3; PAPER.md:191 block
// partial-sum scan):
//   a2  each lane serially scans its E consecutive elements (Alg. 2);
//   a3  a Kogge-Stone shfl.up scan over the 32 lanes combines the per-lane
//       totals (Alg. 3, condition read as lane >= d, reading R10);
//   a5  each compute warp owns RW consecutive rows and keeps a per-thread
//       running column sum (serial scan down the rows, Alg. 2);
//   a4  the compute warps' column totals are combined in shared memory by
//       the look-back warps (block partial-sum scan, Fig. 3c).
//
// Warp roles (one CTA = 8 compute warps + 1 producer warp + kNLB look-back
// warps):
//   producer : draws band tickets (atomic counter => forward progress), late
//              enough that a drawn band is active, and streams the band's
//              tiles into an NSTAGE-deep shared-memory ring with TMA
//              (cp.async.bulk.tensor.3d + mbarrier complete_tx), or with plain
//              loads on the generic (unaligned) path;
//   compute  : pass A of chunk q (row + column scans -> the warp's column
//              totals, row carries advanced), and, LOOK chunks later, pass B
//              of chunk q: the same scans re-run from the still-resident smem
//              tile plus the fix-up offset, stored straight to HBM.  Re-running
//              the scans costs ALU but lets LOOK look-backs overlap;
//   look-back: warp i handles chunks q = i (mod kNLB): aggregate publication,
//              decoupled look-back (32 predecessors probed per round),
//              inclusive publication, per-warp fix-up offsets.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace sat {

enum Pair : int { P8U32S = 0, P32F32F = 1, P64F64F = 2 };

constexpr int kNCW = 8;                          // compute warps
#ifndef SAT_NLB
#define SAT_NLB 2
#endif
constexpr int kNLB = SAT_NLB;                    // look-back warps
constexpr int kProducerWarp = kNCW;
constexpr int kFirstLbWarp = kNCW + 1;
constexpr int kThreads = (kNCW + 1 + kNLB) * 32;
constexpr uint32_t kFull = 0xffffffffu;

// Status word: (epoch << 2) | st,  st: 0 none, 1 aggregate, 2 inclusive.
constexpr uint32_t kStAgg = 1u, kStIncl = 2u;

template <int P>
struct Cfg;
template <>
struct Cfg<P8U32S> {
  using TA = uint8_t;
  using TB = uint32_t;  // wrap arithmetic mod 2^32, reinterpreted as int32 (R2)
  static constexpr int E = 4;   // consecutive elements per lane-group (16 B out)
  static constexpr int G = 2;   // groups per lane: cols {4l..4l+3} and {128+4l..}
  static constexpr int TW = 32 * E * G;  // 256
  static constexpr int TH = 32;
  static constexpr int LOOK = 3;         // pass B runs LOOK chunks behind pass A
  static constexpr int NSTAGE = 8;       // LOOK + 1 resident + prefetch
};
template <>
struct Cfg<P32F32F> {
  using TA = float;
  using TB = float;
  static constexpr int E = 4;
  static constexpr int G = 1;
  static constexpr int TW = 128;
  static constexpr int TH = 32;
  static constexpr int LOOK = 2;
  static constexpr int NSTAGE = 6;
};
template <>
struct Cfg<P64F64F> {
  using TA = double;
  using TB = double;
  static constexpr int E = 2;
  static constexpr int G = 1;
  static constexpr int TW = 64;
  static constexpr int TH = 32;
  static constexpr int LOOK = 2;
  static constexpr int NSTAGE = 6;
};

template <int P>
constexpr int kNTot = (Cfg<P>::LOOK + 1 > kNLB) ? Cfg<P>::LOOK + 1 : kNLB;  // >= kNLB (phase safety)

struct KParams {
  const char* in;       // generic-path input base (TMA path uses the tensor map)
  char* out;
  int64_t H, W;
  int64_t in_pitch, out_pitch;           // bytes
  int64_t in_img_stride, out_img_stride; // bytes
  int64_t bands_per_image;               // ceil(H / TH)
  int64_t total_bands;                   // batch * bands_per_image
  int32_t nchunks;                       // ceil(W / TW)
  uint32_t epoch;                        // status-word epoch of this launch
  uint64_t ticket_base;                  // counter value at launch
  unsigned long long* counter;           // ticket counter (workspace)
  uint32_t* flags;                       // [total_bands][nchunks] status words (hints)
  void* payload;                         // [total_bands][nchunks][2][kVecWords] tagged carries
  const void* carry_in;                  // optional S(r0-1, .) row (W elems of TB) for band 0
};

// Optional phase profiling (debug builds with -DSAT_PROFILE): per-CTA shared
// counters, each written by one warp's lane 0, summed into g_sat_prof at exit.
#ifdef SAT_PROFILE
__device__ unsigned long long g_sat_prof[16];
__device__ __forceinline__ uint64_t gtime() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#define SAT_PT(v) const uint64_t v = gtime()
#define SAT_PADD(sm_, slot_, val_) \
  if ((threadIdx.x & 31) == 0) atomicAdd(&(sm_).prof[slot_], (unsigned long long)(val_))
#else
#define SAT_PT(v)
#define SAT_PADD(sm_, slot_, val_)
#endif
enum ProfSlot {
  kPfComputeWaitFull = 0,   // warp 0: waiting for TMA data
  kPfComputeWaitCarry = 1,  // warp 0: waiting for the look-back result
  kPfComputeLocal = 2,      // warp 0: pass A
  kPfComputeFixup = 3,      // warp 0: pass B (after the wait)
  kPfLbWaitTot = 4,         // look-back warps: waiting for the column totals
  kPfLbPublishAgg = 5,      // look-back warps: aggregate publication
  kPfLbLookback = 6,        // look-back warps: probe + payload reads
  kPfLbDepth = 7,           // vectors summed
  kPfLbRetries = 8,         // probe rounds that found a missing predecessor
  kPfLbChunks = 9,          // chunks handled
  kPfLbRest = 10,           // offsets + inclusive publication
  kPfProdWaitTicket = 11,   // producer: holding the next ticket back
};

template <int P>
struct __align__(128) Smem {
  using C = Cfg<P>;
  typename C::TA in[C::NSTAGE][C::TH][C::TW];   // TMA destination ring
  typename C::TB tot[kNTot<P>][kNCW][C::TW];    // per-warp column totals -> fix-up offsets
  typename C::TB rc_in[C::NSTAGE][C::TH];       // row carries entering each resident tile
  uint64_t full[C::NSTAGE];
  uint64_t empty[C::NSTAGE];
  uint64_t tot_full[kNTot<P>];
  uint64_t carry_full[kNTot<P>];
  int64_t stage_band[C::NSTAGE];   // ticket (global band index), -1 = end
  int32_t stage_img[C::NSTAGE];    // image index n
  int32_t stage_k[C::NSTAGE];      // band index within the image
  int32_t stage_chunk[C::NSTAGE];
  int64_t tot_band[kNTot<P>];
  int32_t tot_img[kNTot<P>];
  int32_t tot_k[kNTot<P>];
  int32_t tot_chunk[kNTot<P>];
  volatile uint32_t passA_done;                 // chunks through pass A (ticket pacing)
#ifdef SAT_PROFILE
  unsigned long long prof[16];
#endif
};

// ---------------------------------------------------------------------------
// PTX helpers (mbarrier, TMA, memory-model loads/stores)

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile(
      "{\n\t.reg .b64 st;\n\t"
      "mbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile(
      "{\n\t.reg .b64 st;\n\t"
      "mbarrier.arrive.expect_tx.shared::cta.b64 st, [%0], %1;\n\t}" ::"r"(smem_u32(bar)),
      "r"(bytes)
      : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  // try_wait with a suspend-time hint: the warp sleeps in hardware until the
  // phase completes (or the hint expires) instead of spinning on issue slots.
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(addr),
      "r"(parity), "r"(0x100000u)
      : "memory");
}

__device__ __forceinline__ void tma_load_3d(void* dst, const CUtensorMap* map, uint64_t* bar,
                                            int32_t x, int32_t y, int32_t z, uint64_t policy) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes.L2::cache_hint"
      " [%0], [%1, {%2, %3, %4}], [%5], %6;" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(x), "r"(y), "r"(z), "r"(smem_u32(bar)),
      "l"(policy)
      : "memory");
}

__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// Streaming (evict-first) 16-byte output store.
__device__ __forceinline__ void st_cs_v4(void* p, uint4 v) {
  asm volatile("st.global.cs.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y),
               "r"(v.z), "r"(v.w)
               : "memory");
}

// ---------------------------------------------------------------------------
// Lane-group vectors: a lane owns G groups of E consecutive elements of a
// TW-wide tile row; group g covers columns g*32*E + lane*E + [0, E).

template <int P>
struct Vec {
  using C = Cfg<P>;
  typename C::TB v[C::G][C::E];
};

template <int P>
__device__ __forceinline__ int col_of(int g, int lane) {
  return g * 32 * Cfg<P>::E + lane * Cfg<P>::E;
}

template <typename T, int E>
__device__ __forceinline__ uint4 pack16(const T (&v)[E]) {
  static_assert(sizeof(T) * E == 16, "16-byte groups");
  uint4 r;
  memcpy(&r, v, 16);
  return r;
}

template <typename T, int E>
__device__ __forceinline__ void unpack16(uint4 r, T (&v)[E]) {
  memcpy(v, &r, 16);
}

// ---------------------------------------------------------------------------
// a2 + a3 + a5: scan one tile row (horizontal) and accumulate it into the
// running column sums `acc` (vertical).  `row` points at the smem tile row.

__device__ __forceinline__ void row_step(const uint8_t* row, int lane, uint32_t& rowcarry,
                                         uint32_t (&acc)[2][4]) {
  // a1/a2: two 4-byte groups per lane; group totals via byte dot-products.
  const uint32_t w0 = *reinterpret_cast<const uint32_t*>(row + 4 * lane);
  const uint32_t w1 = *reinterpret_cast<const uint32_t*>(row + 128 + 4 * lane);
  const uint32_t t0 = __dp4a(w0, 0x01010101u, 0u);
  const uint32_t t1 = __dp4a(w1, 0x01010101u, 0u);
  // a3: Kogge-Stone over lanes on packed 16-bit halves (each half <= 32640).
  const uint32_t own = t0 | (t1 << 16);
  uint32_t inc = own;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const uint32_t o = __shfl_up_sync(kFull, inc, d);
    if (lane >= d) inc += o;
  }
  const uint32_t tot = __shfl_sync(kFull, inc, 31);
  const uint32_t ex = inc - own;
  const uint32_t tot0 = tot & 0xFFFFu;
  const uint32_t base0 = rowcarry + (ex & 0xFFFFu);
  const uint32_t base1 = rowcarry + tot0 + (ex >> 16);
  rowcarry += tot0 + (tot >> 16);
  // a2 + a5: in-group prefix (byte masks) + carry, accumulated down the column.
  acc[0][0] += __dp4a(w0, 0x00000001u, base0);
  acc[0][1] += __dp4a(w0, 0x00000101u, base0);
  acc[0][2] += __dp4a(w0, 0x00010101u, base0);
  acc[0][3] += __dp4a(w0, 0x01010101u, base0);
  acc[1][0] += __dp4a(w1, 0x00000001u, base1);
  acc[1][1] += __dp4a(w1, 0x00000101u, base1);
  acc[1][2] += __dp4a(w1, 0x00010101u, base1);
  acc[1][3] += __dp4a(w1, 0x01010101u, base1);
}

__device__ __forceinline__ void row_step(const float* row, int lane, float& rowcarry,
                                         float (&acc)[1][4]) {
  const float4 a = *reinterpret_cast<const float4*>(row + 4 * lane);
  const float p0 = a.x, p1 = p0 + a.y, p2 = p1 + a.z, p3 = p2 + a.w;  // Alg. 2
  float inc = p3;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {  // Alg. 3
    const float o = __shfl_up_sync(kFull, inc, d);
    if (lane >= d) inc += o;
  }
  const float tot = __shfl_sync(kFull, inc, 31);
  float ex = __shfl_up_sync(kFull, inc, 1);
  if (lane == 0) ex = 0.0f;
  const float base = rowcarry + ex;
  rowcarry += tot;
  acc[0][0] += base + p0;
  acc[0][1] += base + p1;
  acc[0][2] += base + p2;
  acc[0][3] += base + p3;
}

__device__ __forceinline__ void row_step(const double* row, int lane, double& rowcarry,
                                         double (&acc)[1][2]) {
  const double2 a = *reinterpret_cast<const double2*>(row + 2 * lane);
  const double p0 = a.x, p1 = p0 + a.y;
  double inc = p1;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const double o = __shfl_up_sync(kFull, inc, d);
    if (lane >= d) inc += o;
  }
  const double tot = __shfl_sync(kFull, inc, 31);
  double ex = __shfl_up_sync(kFull, inc, 1);
  if (lane == 0) ex = 0.0;
  const double base = rowcarry + ex;
  rowcarry += tot;
  acc[0][0] += base + p0;
  acc[0][1] += base + p1;
}

// Carry payloads are epoch-TAGGED 64-bit words: (epoch << 32) | 32 value bits
// (an fp64 value takes two words, low then high half).  A 64-bit store is
// single-copy atomic, so a reader that sees the current epoch in a word also
// sees that word's value: publication needs no memory fence, and the
// per-tile status word is only a hint telling readers which vector to read.
// A lane's group of E elements is always 4 words (32 bytes).
template <int P>
struct Tag;
template <>
struct Tag<P8U32S> {
  static __device__ __forceinline__ void enc(const uint32_t (&v)[4], uint32_t t, uint64_t (&w)[4]) {
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = ((uint64_t)t << 32) | v[e];
  }
  static __device__ __forceinline__ void dec(const uint64_t (&w)[4], uint32_t (&v)[4]) {
#pragma unroll
    for (int e = 0; e < 4; ++e) v[e] = (uint32_t)w[e];
  }
};
template <>
struct Tag<P32F32F> {
  static __device__ __forceinline__ void enc(const float (&v)[4], uint32_t t, uint64_t (&w)[4]) {
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = ((uint64_t)t << 32) | __float_as_uint(v[e]);
  }
  static __device__ __forceinline__ void dec(const uint64_t (&w)[4], float (&v)[4]) {
#pragma unroll
    for (int e = 0; e < 4; ++e) v[e] = __uint_as_float((uint32_t)w[e]);
  }
};
template <>
struct Tag<P64F64F> {
  static __device__ __forceinline__ void enc(const double (&v)[2], uint32_t t, uint64_t (&w)[4]) {
#pragma unroll
    for (int e = 0; e < 2; ++e) {
      const uint64_t b = (uint64_t)__double_as_longlong(v[e]);
      w[2 * e] = ((uint64_t)t << 32) | (b & 0xffffffffull);
      w[2 * e + 1] = ((uint64_t)t << 32) | (b >> 32);
    }
  }
  static __device__ __forceinline__ void dec(const uint64_t (&w)[4], double (&v)[2]) {
#pragma unroll
    for (int e = 0; e < 2; ++e)
      v[e] = __longlong_as_double((long long)((w[2 * e] & 0xffffffffull) | (w[2 * e + 1] << 32)));
  }
};

__device__ __forceinline__ void st_relaxed_v2_u64(uint64_t* p, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.gpu.global.v2.u64 [%0], {%1, %2};" ::"l"(p), "l"(a), "l"(b) : "memory");
}

__device__ __forceinline__ void ld_relaxed_v2_u64(const uint64_t* p, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(p) : "memory");
}

__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Words of one payload vector: TW elements * (4 / E) words per element.
template <int P>
constexpr int kVecWords = Cfg<P>::TW * 4 / Cfg<P>::E;

template <int P>
__device__ __forceinline__ uint64_t* payload_row(const KParams& p, int64_t band, int32_t chunk,
                                                 int kind) {
  return reinterpret_cast<uint64_t*>(p.payload) +
         (((band * p.nchunks + chunk) * 2 + kind) * (int64_t)kVecWords<P>);
}

template <int P>
__device__ __forceinline__ void publish(const KParams& p, int64_t band, int32_t chunk, int kind,
                                        const typename Cfg<P>::TB (&v)[Cfg<P>::G][Cfg<P>::E],
                                        int lane) {
  using C = Cfg<P>;
  uint64_t* row = payload_row<P>(p, band, chunk, kind);
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    uint64_t w[4];
    Tag<P>::enc(v[g], p.epoch, w);
    uint64_t* dst = row + (g * 32 + lane) * 4;
    st_relaxed_v2_u64(dst, w[0], w[1]);
    st_relaxed_v2_u64(dst + 2, w[2], w[3]);
  }
  __syncwarp();
  if (lane == 0)  // hint only: readers validate every payload word's tag
    st_relaxed_u32(p.flags + band * p.nchunks + chunk,
                   (p.epoch << 2) | (kind == 0 ? kStAgg : kStIncl));
}

// Sum published vectors d = 0..dmax of the window (band j - d; kind AGG for
// d < kk, INCL for d == kk) into acc.  Loads of a batch of kBatch vectors are
// issued together (one L2 round trip per batch); a batch is re-read until
// every word carries this launch's epoch.
template <int P>
constexpr int kBatch = Cfg<P>::G == 1 ? 4 : 2;

template <int P>
__device__ __forceinline__ void read_window(const KParams& p, int64_t j, int32_t chunk, int kk,
                                            int dmax,
                                            typename Cfg<P>::TB (&acc)[Cfg<P>::G][Cfg<P>::E],
                                            int lane) {
  using C = Cfg<P>;
  constexpr int B = kBatch<P>;
  for (int d0 = 0; d0 <= dmax; d0 += B) {
    uint64_t w[B][C::G][4];
    for (;;) {
      bool ok = true;
#pragma unroll
      for (int b = 0; b < B; ++b) {
        const int d = d0 + b;
        if (d <= dmax) {
          const uint64_t* row = payload_row<P>(p, j - d, chunk, d == kk ? 1 : 0);
#pragma unroll
          for (int g = 0; g < C::G; ++g) {
            const uint64_t* src = row + (g * 32 + lane) * 4;
            ld_relaxed_v2_u64(src, w[b][g][0], w[b][g][1]);
            ld_relaxed_v2_u64(src + 2, w[b][g][2], w[b][g][3]);
          }
        }
      }
#pragma unroll
      for (int b = 0; b < B; ++b)
        if (d0 + b <= dmax)
#pragma unroll
          for (int g = 0; g < C::G; ++g)
#pragma unroll
            for (int e = 0; e < 4; ++e) ok &= (uint32_t)(w[b][g][e] >> 32) == p.epoch;
      if (__all_sync(kFull, ok)) break;
      __nanosleep(20);
    }
#pragma unroll
    for (int b = 0; b < B; ++b)
      if (d0 + b <= dmax)
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
          typename C::TB t[C::E];
          Tag<P>::dec(w[b][g], t);
#pragma unroll
          for (int e = 0; e < C::E; ++e) acc[g][e] += t[e];
        }
  }
}

// Decoupled look-back up the tile column: V = sum of predecessors' aggregates
// down to (and including) the nearest inclusive prefix.  32 predecessors are
// probed per round, one status word per lane.
template <int P>
__device__ __forceinline__ void lookback(Smem<P>& sm, const KParams& p, int64_t band, int64_t first,
                                         int32_t chunk, typename Cfg<P>::TB (&V)[Cfg<P>::G][Cfg<P>::E],
                                         int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) V[g][e] = TB(0);
  int64_t j = band - 1;
  for (;;) {
    const int64_t jj = j - lane;
    uint32_t st = kStIncl;  // lanes past the image's first band: never reached
    if (jj >= first) {
      const uint32_t f = ld_relaxed_u32(p.flags + jj * p.nchunks + chunk);
      st = ((f >> 2) == p.epoch) ? (f & 3u) : 0u;
    }
    const uint32_t inclm = __ballot_sync(kFull, st == kStIncl);
    const uint32_t nonem = __ballot_sync(kFull, st == 0u);
    const int kk = inclm ? (__ffs(inclm) - 1) : 32;
    const uint32_t need = (kk >= 31) ? kFull : ((2u << kk) - 1u);
    if (nonem & need) {
      SAT_PADD(sm, kPfLbRetries, 1);
      __nanosleep(20);
      continue;
    }
    SAT_PADD(sm, kPfLbDepth, (kk < 32 ? kk : 31) + 1);
    const int dmax = kk < 32 ? kk : 31;
    read_window<P>(p, j, chunk, kk, dmax, V, lane);
    if (kk < 32) break;
    j -= 32;
  }
}

template <int P>
__device__ __forceinline__ void lookback_warp(Smem<P>& sm, const KParams& p, int lbw, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int NT = kNTot<P>;
  for (uint32_t q = lbw;; q += kNLB) {
    const int t = q % NT;
    SAT_PT(t0);
    mbar_wait(&sm.tot_full[t], (q / NT) & 1);
    SAT_PT(t1);
    SAT_PADD(sm, kPfLbWaitTot, t1 - t0);
    const int64_t band = sm.tot_band[t];
    const int32_t chunk = sm.tot_chunk[t];
    if (band < 0) break;
    SAT_PADD(sm, kPfLbChunks, 1);
    const int64_t n = sm.tot_img[t];
    const int64_t k = sm.tot_k[t];
    const bool has_succ = k + 1 < p.bands_per_image;
    TB V[C::G][C::E];
    if (k == 0) {
      // Image's top band: the predecessor is the (optional) carry-in row.
#pragma unroll
      for (int g = 0; g < C::G; ++g)
#pragma unroll
        for (int e = 0; e < C::E; ++e) {
          const int64_t x = (int64_t)chunk * C::TW + col_of<P>(g, lane) + e;
          V[g][e] = (p.carry_in != nullptr && x < p.W)
                        ? reinterpret_cast<const TB*>(p.carry_in)[x]
                        : TB(0);
        }
    } else {
      if (has_succ) {
        TB agg[C::G][C::E];
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
#pragma unroll
          for (int e = 0; e < C::E; ++e) agg[g][e] = TB(0);
#pragma unroll
          for (int w = 0; w < kNCW; ++w) {
            TB tt[C::E];
            unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.tot[t][w][col_of<P>(g, lane)]),
                               tt);
#pragma unroll
            for (int e = 0; e < C::E; ++e) agg[g][e] += tt[e];
          }
        }
        publish<P>(p, band, chunk, 0, agg, lane);
      }
      SAT_PT(t2);
      SAT_PADD(sm, kPfLbPublishAgg, t2 - t1);
      lookback<P>(sm, p, band, n * p.bands_per_image, chunk, V, lane);
      SAT_PT(t3);
      SAT_PADD(sm, kPfLbLookback, t3 - t2);
    }
    SAT_PT(t4);
    // Fix-up offsets, in place: tot[w] <- V + sum_{w' < w} tot[w'] (Fig. 3c step #2).
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
#pragma unroll
      for (int w = 0; w < kNCW; ++w) {
        uint4* cell = reinterpret_cast<uint4*>(&sm.tot[t][w][col_of<P>(g, lane)]);
        TB tt[C::E];
        unpack16<TB, C::E>(*cell, tt);
        *cell = pack16<TB, C::E>(V[g]);
#pragma unroll
        for (int e = 0; e < C::E; ++e) V[g][e] += tt[e];
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.carry_full[t]);
    // V is now the inclusive prefix S(r1 - 1, .) of this tile column.
    if (has_succ) publish<P>(p, band, chunk, 1, V, lane);
    SAT_PT(t5);
    SAT_PADD(sm, kPfLbRest, t5 - t4);
  }
}

// ---------------------------------------------------------------------------
// Compute warps

// Pass A of chunk q (stage s): row + column scans of this warp's RW rows; the
// column totals go to tot[q % NT][warp]; the row carries entering the tile are
// saved for pass B.  Returns false at the end-of-work sentinel.
template <int P>
__device__ __forceinline__ bool pass_a(Smem<P>& sm, uint32_t q, int s, uint32_t ph,
                                       typename Cfg<P>::TB (&rowcarry)[Cfg<P>::TH / kNCW],
                                       int warp, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  SAT_PT(t0);
  mbar_wait(&sm.full[s], ph);
  SAT_PT(t1);
  if (warp == 0) SAT_PADD(sm, kPfComputeWaitFull, t1 - t0);
  const int64_t band = sm.stage_band[s];
  if (band < 0) return false;
  const int32_t chunk = sm.stage_chunk[s];
  if (chunk == 0) {
#pragma unroll
    for (int i = 0; i < RW; ++i) rowcarry[i] = TB(0);
  }
  if (lane < RW) {
    TB rc = rowcarry[0];
#pragma unroll
    for (int i = 1; i < RW; ++i)
      if (lane == i) rc = rowcarry[i];
    sm.rc_in[s][warp * RW + lane] = rc;
  }
  const typename C::TA* tile = &sm.in[s][warp * RW][0];
  TB acc[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) acc[g][e] = TB(0);
#pragma unroll
  for (int i = 0; i < RW; ++i) row_step(tile + i * C::TW, lane, rowcarry[i], acc);
  // a4: this warp's column totals for the block partial-sum scan.
  const int t = q % kNTot<P>;
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    *reinterpret_cast<uint4*>(&sm.tot[t][warp][col_of<P>(g, lane)]) = pack16<TB, C::E>(acc[g]);
  if (warp == 0 && lane == 0) {
    sm.tot_band[t] = band;
    sm.tot_img[t] = sm.stage_img[s];
    sm.tot_k[t] = sm.stage_k[s];
    sm.tot_chunk[t] = chunk;
    sm.passA_done = q + 1;
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.tot_full[t]);
  SAT_PT(t2);
  if (warp == 0) SAT_PADD(sm, kPfComputeLocal, t2 - t1);
  return true;
}

// Pass B of chunk q (stage s): wait for the offsets, re-run the scans from the
// resident tile, add the offsets, store; release the stage.
template <int P, bool kVecOut>
__device__ __forceinline__ void pass_b(Smem<P>& sm, const KParams& p, uint32_t q, int s, int warp,
                                       int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  const int t = q % kNTot<P>;
  SAT_PT(t0);
  mbar_wait(&sm.carry_full[t], (q / kNTot<P>) & 1);
  SAT_PT(t1);
  if (warp == 0) SAT_PADD(sm, kPfComputeWaitCarry, t1 - t0);
  TB acc[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.tot[t][warp][col_of<P>(g, lane)]),
                       acc[g]);
  const int64_t n = sm.stage_img[s];
  const int64_t k = sm.stage_k[s];
  const int32_t chunk = sm.stage_chunk[s];
  char* obase = p.out + n * p.out_img_stride;
  const int64_t x0 = (int64_t)chunk * C::TW;
  const typename C::TA* tile = &sm.in[s][warp * RW][0];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    TB rc = sm.rc_in[s][warp * RW + i];
    row_step(tile + i * C::TW, lane, rc, acc);  // acc = offset + S'(row i)
    const int64_t y = k * C::TH + warp * RW + i;
    if (y < p.H) {
      TB* orow = reinterpret_cast<TB*>(obase + y * p.out_pitch);
#pragma unroll
      for (int g = 0; g < C::G; ++g) {
        const int64_t x = x0 + col_of<P>(g, lane);
        if (kVecOut && x + C::E <= p.W) {
          st_cs_v4(orow + x, pack16<TB, C::E>(acc[g]));
        } else {
#pragma unroll
          for (int e = 0; e < C::E; ++e)
            if (x + e < p.W) orow[x + e] = acc[g][e];
        }
      }
    }
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.empty[s]);
  SAT_PT(t2);
  if (warp == 0) SAT_PADD(sm, kPfComputeFixup, t2 - t1);
}

template <int P, bool kVecOut>
__device__ __forceinline__ void compute_warp(Smem<P>& sm, const KParams& p, int warp, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  TB rowcarry[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) rowcarry[i] = TB(0);
  uint32_t qa = 0, qb = 0;
  bool ended = false;
  for (;;) {
    if (!ended) {
      if (pass_a<P>(sm, qa, qa % C::NSTAGE, (qa / C::NSTAGE) & 1, rowcarry, warp, lane))
        ++qa;
      else
        ended = true;
    }
    if (qb < qa && (ended || qa - qb > (uint32_t)C::LOOK)) {
      pass_b<P, kVecOut>(sm, p, qb, qb % C::NSTAGE, warp, lane);
      ++qb;
    } else if (ended) {
      break;
    }
  }
  // One end-of-work sentinel per look-back warp (slots are free: all pass B done).
  for (int i = 0; i < kNLB; ++i) {
    const uint32_t q = qa + i;
    const int t = q % kNTot<P>;
    if (warp == 0 && lane == 0) sm.tot_band[t] = -1;
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.tot_full[t]);
    // the next sentinel reuses a slot only after its look-back warp left
  }
}

// ---------------------------------------------------------------------------
// Producer warp

template <int P, bool kTMA>
__device__ __forceinline__ void producer_warp(Smem<P>& sm, const KParams& p, const CUtensorMap* map,
                                              int lane) {
  using C = Cfg<P>;
  using TA = typename C::TA;
  constexpr uint32_t kTileBytes = C::TH * C::TW * sizeof(TA);
  constexpr uint32_t kTicketLead = 2;  // chunks of the current band still ahead of pass A
  uint32_t q = 0;
  uint64_t pol = 0;
  if (kTMA) pol = policy_evict_first();
  for (;;) {
    // Draw the next band only when pass A is within kTicketLead chunks of the
    // end of what was issued, so a drawn band is never queued behind a whole
    // band (its successors would stall on it).
    SAT_PT(t0);
    while (q > kTicketLead && sm.passA_done + kTicketLead < q) __nanosleep(64);
    SAT_PT(t1);
    if (lane == 0) SAT_PADD(sm, kPfProdWaitTicket, t1 - t0);
    int64_t t = 0;
    if (lane == 0) t = (int64_t)(atomicAdd(p.counter, 1ull) - p.ticket_base);
    t = __shfl_sync(kFull, t, 0);
    const bool done = t >= p.total_bands;
    const int64_t n = done ? 0 : t / p.bands_per_image;
    const int64_t k = done ? 0 : t - n * p.bands_per_image;
    const int32_t nch = done ? 1 : p.nchunks;
    for (int32_t c = 0; c < nch; ++c, ++q) {
      const int s = q % C::NSTAGE;
      mbar_wait(&sm.empty[s], ((q / C::NSTAGE) & 1) ^ 1u);
      if (done) {
        if (lane == 0) {
          sm.stage_band[s] = -1;
          sm.stage_chunk[s] = 0;
          mbar_arrive(&sm.full[s]);
        }
      } else if (kTMA) {
        if (lane == 0) {
          sm.stage_band[s] = t;
          sm.stage_img[s] = (int32_t)n;
          sm.stage_k[s] = (int32_t)k;
          sm.stage_chunk[s] = c;
          mbar_arrive_expect_tx(&sm.full[s], kTileBytes);
          tma_load_3d(&sm.in[s][0][0], map, &sm.full[s], c * C::TW, (int32_t)(k * C::TH),
                      (int32_t)n, pol);
        }
      } else {
        // Generic path: plain loads, zero fill outside the image.
        const char* ibase = p.in + n * p.in_img_stride;
        for (int r = 0; r < C::TH; ++r) {
          const int64_t y = k * C::TH + r;
          for (int x = lane; x < C::TW; x += 32) {
            const int64_t xx = (int64_t)c * C::TW + x;
            TA v = TA(0);
            if (y < p.H && xx < p.W) v = reinterpret_cast<const TA*>(ibase + y * p.in_pitch)[xx];
            sm.in[s][r][x] = v;
          }
        }
        __syncwarp();
        if (lane == 0) {
          sm.stage_band[s] = t;
          sm.stage_img[s] = (int32_t)n;
          sm.stage_k[s] = (int32_t)k;
          sm.stage_chunk[s] = c;
          mbar_arrive(&sm.full[s]);
        }
      }
      __syncwarp();
    }
    if (done) break;
  }
}

// ---------------------------------------------------------------------------

template <int P, bool kTMA, bool kVecOut>
__global__ void __launch_bounds__(kThreads, 2)
    sat_tile_kernel(const __grid_constant__ CUtensorMap map, const KParams p) {
  using C = Cfg<P>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  Smem<P>& sm = *reinterpret_cast<Smem<P>*>(smem_raw);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::NSTAGE; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], kNCW);
    }
    for (int t = 0; t < kNTot<P>; ++t) {
      mbar_init(&sm.tot_full[t], kNCW);
      mbar_init(&sm.carry_full[t], 1);
    }
    sm.passA_done = 0;
#ifdef SAT_PROFILE
    for (int i = 0; i < 16; ++i) sm.prof[i] = 0;
#endif
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (kTMA)
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map)) : "memory");
  }
  __syncthreads();

  if (warp == kProducerWarp) {
    producer_warp<P, kTMA>(sm, p, &map, lane);
  } else if (warp >= kFirstLbWarp) {
    lookback_warp<P>(sm, p, warp - kFirstLbWarp, lane);
  } else {
    compute_warp<P, kVecOut>(sm, p, warp, lane);
  }
#ifdef SAT_PROFILE
  __syncthreads();
  if (threadIdx.x < 16) atomicAdd(&g_sat_prof[threadIdx.x], sm.prof[threadIdx.x]);
#endif
}

}  // namespace sat
