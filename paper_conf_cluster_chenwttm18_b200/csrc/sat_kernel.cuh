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
//   a4  the 8 compute warps' column totals are combined in shared memory by
//       the look-back warp (block partial-sum scan, Fig. 3c).
//
// Warp roles (one CTA = 8 compute warps + 1 producer warp + 1 look-back warp):
//   producer : draws band tickets (atomic counter => forward progress) and
//              streams the band's tiles into an NSTAGE-deep shared-memory ring
//              with TMA (cp.async.bulk.tensor.3d, mbarrier complete_tx), or
//              with plain loads on the generic (unaligned) path;
//   compute  : local pass of chunk c, then the fix-up + store of chunk c-1
//              (so the look-back of chunk c-1 overlaps the local pass of c);
//   look-back: per chunk, publishes the aggregate, looks back up the tile
//              column (32 predecessors per probe), publishes the inclusive
//              prefix and writes per-warp fix-up offsets.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace sat {

enum Pair : int { P8U32S = 0, P32F32F = 1, P64F64F = 2 };

constexpr int kNCW = 8;                     // compute warps
constexpr int kThreads = (kNCW + 2) * 32;   // + producer warp + look-back warp
constexpr int kProducerWarp = kNCW;
constexpr int kLookbackWarp = kNCW + 1;
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
  static constexpr int NSTAGE = 6;
};
template <>
struct Cfg<P32F32F> {
  using TA = float;
  using TB = float;
  static constexpr int E = 4;
  static constexpr int G = 1;
  static constexpr int TW = 128;
  static constexpr int TH = 32;
  static constexpr int NSTAGE = 4;
};
template <>
struct Cfg<P64F64F> {
  using TA = double;
  using TB = double;
  static constexpr int E = 2;
  static constexpr int G = 1;
  static constexpr int TW = 64;
  static constexpr int TH = 32;
  static constexpr int NSTAGE = 4;
};

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
  uint32_t* flags;                       // [total_bands][nchunks] status words
  void* payload;                         // [total_bands][nchunks][2][TW] carries
  const void* carry_in;                  // optional S(r0-1, .) row (W elems of TB) for band 0
};

template <int P>
struct __align__(128) Smem {
  using C = Cfg<P>;
  typename C::TA in[C::NSTAGE][C::TH][C::TW];  // TMA destination ring
  typename C::TB tot[2][kNCW][C::TW];          // per-warp column totals -> fix-up offsets
  uint64_t full[C::NSTAGE];
  uint64_t empty[C::NSTAGE];
  uint64_t tot_full[2];
  uint64_t carry_full[2];
  int64_t stage_band[C::NSTAGE];
  int32_t stage_chunk[C::NSTAGE];
  int64_t tot_band[2];
  int32_t tot_chunk[2];
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
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(addr),
      "r"(parity)
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

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

// 16-byte coherent (L1-bypassing, gpu-scope relaxed) payload load.
__device__ __forceinline__ uint4 ld_relaxed_v4(const void* p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}

__device__ __forceinline__ void st_v4(void* p, uint4 v) {
  asm volatile("st.global.v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z),
               "r"(v.w)
               : "memory");
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

// ---------------------------------------------------------------------------
// Compute-warp state and steps

template <int P>
struct ComputeState {
  using C = Cfg<P>;
  static constexpr int RW = C::TH / kNCW;
  int s;          // input ring stage
  uint32_t ph;    // input ring phase
  uint32_t q;     // chunks processed by this CTA (tot/carry double-buffer index)
  int64_t prev_band;
  int32_t prev_chunk;
  bool has_prev;
  typename C::TB rowcarry[RW];
};

template <int P, bool kVecOut>
__device__ __forceinline__ void fixup_store(Smem<P>& sm, const KParams& p,
                                            const typename Cfg<P>::TB (&S)[Cfg<P>::TH / kNCW]
                                                                          [Cfg<P>::G][Cfg<P>::E],
                                            int64_t band, int32_t chunk, uint32_t q, int warp,
                                            int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  const int b = q & 1;
  mbar_wait(&sm.carry_full[b], (q >> 1) & 1);
  TB off[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.tot[b][warp][col_of<P>(g, lane)]),
                       off[g]);
  const int64_t n = band / p.bands_per_image;
  const int64_t k = band - n * p.bands_per_image;
  char* obase = p.out + n * p.out_img_stride;
  const int64_t x0 = (int64_t)chunk * C::TW;
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const int64_t y = k * C::TH + warp * RW + i;
    if (y >= p.H) break;
    TB* orow = reinterpret_cast<TB*>(obase + y * p.out_pitch);
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      const int64_t x = x0 + col_of<P>(g, lane);
      TB v[C::E];
#pragma unroll
      for (int e = 0; e < C::E; ++e) v[e] = S[i][g][e] + off[g][e];
      if (kVecOut && x + C::E <= p.W) {
        st_cs_v4(orow + x, pack16<TB, C::E>(v));
      } else {
#pragma unroll
        for (int e = 0; e < C::E; ++e)
          if (x + e < p.W) orow[x + e] = v[e];
      }
    }
  }
}

// One chunk of the compute warps: local pass into `cur`, then fix-up of the
// previous chunk held in `prev`.  Returns false at the end-of-work sentinel.
template <int P, bool kVecOut>
__device__ __forceinline__ bool compute_step(
    Smem<P>& sm, const KParams& p, ComputeState<P>& st,
    typename Cfg<P>::TB (&cur)[Cfg<P>::TH / kNCW][Cfg<P>::G][Cfg<P>::E],
    const typename Cfg<P>::TB (&prev)[Cfg<P>::TH / kNCW][Cfg<P>::G][Cfg<P>::E], int warp,
    int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  mbar_wait(&sm.full[st.s], st.ph);
  const int64_t band = sm.stage_band[st.s];
  const int32_t chunk = sm.stage_chunk[st.s];
  const int b = st.q & 1;
  if (band < 0) {
    if (st.has_prev)
      fixup_store<P, kVecOut>(sm, p, prev, st.prev_band, st.prev_chunk, st.q - 1, warp, lane);
    if (warp == 0 && lane == 0) sm.tot_band[b] = -1;
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.tot_full[b]);
    return false;
  }
  if (chunk == 0) {
#pragma unroll
    for (int i = 0; i < RW; ++i) st.rowcarry[i] = TB(0);
  }
  const typename C::TA* tile = &sm.in[st.s][warp * RW][0];
  TB acc[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) acc[g][e] = TB(0);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    row_step(tile + i * C::TW, lane, st.rowcarry[i], acc);
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) cur[i][g][e] = acc[g][e];
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.empty[st.s]);
  if (++st.s == C::NSTAGE) {
    st.s = 0;
    st.ph ^= 1u;
  }
  // a4: this warp's column totals for the block partial-sum scan.
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    *reinterpret_cast<uint4*>(&sm.tot[b][warp][col_of<P>(g, lane)]) =
        pack16<TB, C::E>(acc[g]);
  if (warp == 0 && lane == 0) {
    sm.tot_band[b] = band;
    sm.tot_chunk[b] = chunk;
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.tot_full[b]);
  if (st.has_prev)
    fixup_store<P, kVecOut>(sm, p, prev, st.prev_band, st.prev_chunk, st.q - 1, warp, lane);
  st.has_prev = true;
  st.prev_band = band;
  st.prev_chunk = chunk;
  st.q++;
  return true;
}

// ---------------------------------------------------------------------------
// Look-back warp

template <int P>
__device__ __forceinline__ typename Cfg<P>::TB* payload_row(const KParams& p, int64_t band,
                                                            int32_t chunk, int kind) {
  using C = Cfg<P>;
  return reinterpret_cast<typename C::TB*>(p.payload) +
         (((band * p.nchunks + chunk) * 2 + kind) * C::TW);
}

template <int P>
__device__ __forceinline__ void publish(const KParams& p, int64_t band, int32_t chunk, int kind,
                                        const typename Cfg<P>::TB (&v)[Cfg<P>::G][Cfg<P>::E],
                                        int lane) {
  using C = Cfg<P>;
  typename C::TB* row = payload_row<P>(p, band, chunk, kind);
#pragma unroll
  for (int g = 0; g < C::G; ++g) st_v4(row + col_of<P>(g, lane), pack16<typename C::TB, C::E>(v[g]));
  __threadfence();  // each lane orders its payload stores (gpu scope) ...
  __syncwarp();     // ... before lane 0 raises the status word
  if (lane == 0)
    st_relaxed_u32(p.flags + band * p.nchunks + chunk,
                   (p.epoch << 2) | (kind == 0 ? kStAgg : kStIncl));
}

// Decoupled look-back up the tile column: V = sum of predecessors' aggregates
// down to (and including) the nearest inclusive prefix.  32 predecessors are
// probed per round, one per lane.
template <int P>
__device__ __forceinline__ void lookback(const KParams& p, int64_t band, int64_t first,
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
      const uint32_t f = ld_acquire_u32(p.flags + jj * p.nchunks + chunk);
      st = ((f >> 2) == p.epoch) ? (f & 3u) : 0u;
    }
    const uint32_t inclm = __ballot_sync(kFull, st == kStIncl);
    const uint32_t nonem = __ballot_sync(kFull, st == 0u);
    const int kk = inclm ? (__ffs(inclm) - 1) : 32;
    const uint32_t need = (kk >= 31) ? kFull : ((2u << kk) - 1u);
    if (nonem & need) {
      __nanosleep(32);
      continue;
    }
    __syncwarp();
    const int dmax = kk < 32 ? kk : 31;
    for (int d = 0; d <= dmax; ++d) {
      const int kind = (d == kk) ? 1 : 0;
      const TB* row = payload_row<P>(p, j - d, chunk, kind);
#pragma unroll
      for (int g = 0; g < C::G; ++g) {
        TB t[C::E];
        unpack16<TB, C::E>(ld_relaxed_v4(row + col_of<P>(g, lane)), t);
#pragma unroll
        for (int e = 0; e < C::E; ++e) V[g][e] += t[e];
      }
    }
    if (kk < 32) break;
    j -= 32;
  }
}

template <int P>
__device__ __forceinline__ void lookback_warp(Smem<P>& sm, const KParams& p, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  for (uint32_t q = 0;; ++q) {
    const int b = q & 1;
    mbar_wait(&sm.tot_full[b], (q >> 1) & 1);
    const int64_t band = sm.tot_band[b];
    const int32_t chunk = sm.tot_chunk[b];
    if (band < 0) break;
    const int64_t n = band / p.bands_per_image;
    const int64_t k = band - n * p.bands_per_image;
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
            TB t[C::E];
            unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.tot[b][w][col_of<P>(g, lane)]),
                               t);
#pragma unroll
            for (int e = 0; e < C::E; ++e) agg[g][e] += t[e];
          }
        }
        publish<P>(p, band, chunk, 0, agg, lane);
      }
      lookback<P>(p, band, n * p.bands_per_image, chunk, V, lane);
    }
    // Fix-up offsets, in place: tot[w] <- V + sum_{w' < w} tot[w'] (Fig. 3c step #2).
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
#pragma unroll
      for (int w = 0; w < kNCW; ++w) {
        uint4* cell = reinterpret_cast<uint4*>(&sm.tot[b][w][col_of<P>(g, lane)]);
        TB t[C::E];
        unpack16<TB, C::E>(*cell, t);
        *cell = pack16<TB, C::E>(V[g]);
#pragma unroll
        for (int e = 0; e < C::E; ++e) V[g][e] += t[e];
      }
    }
    // V is now the inclusive prefix S(r1 - 1, .) of this tile column.
    if (has_succ) publish<P>(p, band, chunk, 1, V, lane);
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.carry_full[b]);
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
  int s = 0;
  uint32_t ph = 0;
  uint64_t pol = 0;
  if (kTMA) pol = policy_evict_first();
  for (;;) {
    int64_t t = 0;
    if (lane == 0) t = (int64_t)(atomicAdd(p.counter, 1ull) - p.ticket_base);
    t = __shfl_sync(kFull, t, 0);
    const bool done = t >= p.total_bands;
    const int64_t n = done ? 0 : t / p.bands_per_image;
    const int64_t k = done ? 0 : t - n * p.bands_per_image;
    const int32_t nch = done ? 1 : p.nchunks;
    for (int32_t c = 0; c < nch; ++c) {
      mbar_wait(&sm.empty[s], ph ^ 1u);
      if (done) {
        if (lane == 0) {
          sm.stage_band[s] = -1;
          sm.stage_chunk[s] = 0;
          mbar_arrive(&sm.full[s]);
        }
      } else if (kTMA) {
        if (lane == 0) {
          sm.stage_band[s] = t;
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
          sm.stage_chunk[s] = c;
          mbar_arrive(&sm.full[s]);
        }
      }
      __syncwarp();
      if (++s == C::NSTAGE) {
        s = 0;
        ph ^= 1u;
      }
    }
    if (done) break;
  }
}

// ---------------------------------------------------------------------------

template <int P, bool kTMA, bool kVecOut>
__global__ void __launch_bounds__(kThreads, 2)
    sat_tile_kernel(const __grid_constant__ CUtensorMap map, const KParams p) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  Smem<P>& sm = *reinterpret_cast<Smem<P>*>(smem_raw);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < C::NSTAGE; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], kNCW);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&sm.tot_full[b], kNCW);
      mbar_init(&sm.carry_full[b], 1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (kTMA)
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map)) : "memory");
  }
  __syncthreads();

  if (warp == kProducerWarp) {
    producer_warp<P, kTMA>(sm, p, &map, lane);
  } else if (warp == kLookbackWarp) {
    lookback_warp<P>(sm, p, lane);
  } else {
    ComputeState<P> st;
    st.s = 0;
    st.ph = 0;
    st.q = 0;
    st.prev_band = -1;
    st.prev_chunk = 0;
    st.has_prev = false;
#pragma unroll
    for (int i = 0; i < RW; ++i) st.rowcarry[i] = TB(0);
    TB sa[RW][C::G][C::E], sb[RW][C::G][C::E];
    for (;;) {
      if (!compute_step<P, kVecOut>(sm, p, st, sa, sb, warp, lane)) break;
      if (!compute_step<P, kVecOut>(sm, p, st, sb, sa, warp, lane)) break;
    }
  }
}

}  // namespace sat
