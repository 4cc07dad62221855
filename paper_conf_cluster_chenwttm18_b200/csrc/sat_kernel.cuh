// sat_kernel.cuh -- single-pass summed-area-table kernel for sm_100a.
//
// What it computes: the inclusive SAT S(i,j) = sum_{y<=i, x<=j} A(y,x)
// (Eq. 1) of pitched row-major images, in one HBM pass, for
// the pairs 8u->32s, 32f->32f, 64f->64f (BASELINE north star), 8u->32f and
// 32s->32s (Cfg<P>; P + kShort = the same pair with 16-row bands).  The same
// kernel also stores the exclusive layout (Eq. 2, template flag kEx: shifted
// 16-byte stores) and chains bands through per-chunk carry vectors
// (KParams::chain_in / chain_out; the single-pass multi-GPU building block).
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
// The vertical carry V_up is the only cross-CTA quantity.  CL consecutive
// bands form a thread-block CLUSTER (one CTA per band): their column totals
// are combined through distributed shared memory (st.async + remote mbarrier
// complete_tx) by the cluster's leader CTA, which alone takes part in a
// decoupled look-back up the tile column across clusters: it publishes the
// cluster's vertical aggregate, sums predecessors' aggregates down to the
// nearest inclusive prefix, publishes the cluster's inclusive prefix and sends
// every band its V_up.  The chain of concurrently active look-back
// participants is CL times shorter than with one band per participant, and
// the global carry traffic CL times smaller.
//
// Inside a tile (Alg. 2 and Alg. 3; PAPER.md:191 block
// partial-sum scan):
//   a2  each lane serially scans its E consecutive elements (Alg. 2);
//   a3  a Kogge-Stone shfl.up scan over the 32 lanes combines the per-lane
//       totals (Alg. 3, condition read as lane >= d, reading R10);
//   a5  each compute warp owns RW consecutive rows and keeps a per-thread
//       running column sum (serial scan down the rows, Alg. 2);
//   a4  the compute warps' column totals are combined in shared memory by
//       the look-back warps (block partial-sum scan, Fig. 3c);
//       the same scan over the cluster's CTAs runs in the leader.
//
// Warp roles (one CTA = NCW compute warps + producer + aggregate + offset +
// kNLW leader warps):
//   producer : the leader's producer draws cluster tickets (atomic counter =>
//              forward progress), late enough that a drawn band is active, and
//              hands them to the cluster's other producers through DSMEM; each
//              producer streams its band's tiles into an NSTAGE-deep smem ring
//              with TMA (cp.async.bulk.tensor.3d + mbarrier complete_tx), or
//              with plain loads on the generic (unaligned) path;
//   aggregate: as soon as a tile lands, computes the band's vertical aggregate
//              for that chunk straight from the input -- the column totals of
//              R over the band's rows = (band input left of the chunk) + the
//              prefix over x of the tile's column sums -- and sends it to the
//              chunk's leader CTA.  Aggregates thus leave NSTAGE + LOOK + 1
//              chunks ahead of the stores that need the carries, so the
//              cross-cluster look-back mostly finds published predecessors;
//   compute  : pass A of chunk q (row + column scans -> TMEM S' and the warp's
//              column totals, row carries advanced), and, LOOK chunks later,
//              pass B of chunk q: S' back from TMEM plus the fix-up offset,
//              stored straight to HBM;
//   offset   : the block partial-sum scan over the compute warps' column totals
//               -> per-warp fix-up offsets;
//   leader   : for the chunks this CTA leads (q = rank mod CL): segmented scan
//              of the cluster's aggregates, global look-back, publication of
//              the cluster's inclusive prefix, V_up to every band of the cluster.
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <type_traits>

namespace sat {

// P8USQ: 8u -> (S, S of squares), both u32 mod 2^32, interleaved per pixel
// (Viola-Jones variance normalisation); P8UHIST4: 8u -> 4 bins of an integral
// histogram (counts u32), interleaved per pixel.  Both are SATs of a per-pixel
// vector f(a) (Eq. 1 applied channel by channel) on the same single pass.
enum Pair : int { P8U32S = 0, P32F32F = 1, P64F64F = 2, P8U32F = 3, P32S32S = 4, P8USQ = 5,
                  P8UHIST4 = 6 };
// Short-band variants (P + kShort): the same pair with 16-row bands (2 rows per
// compute warp), chosen for short, wide images whose 32-row bands would leave
// most of the machine idle (H / 4 compute warps in total otherwise).
constexpr int kShort = 8;
template <int P>
constexpr int kBase = P % kShort;
template <int P>
struct Cfg;

#ifndef SAT_NLW
#define SAT_NLW 1
#endif
constexpr int kNLWDefault = SAT_NLW;             // leader (look-back) warps unless Cfg says
constexpr uint32_t kFull = 0xffffffffu;

// Carry word tag (high 32 bits): (epoch << 2) | st,  st: 1 aggregate, 2 inclusive.
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
#ifndef SAT_LOOK8
#define SAT_LOOK8 3
#endif
  static constexpr int LOOK = SAT_LOOK8;  // pass B runs LOOK chunks behind pass A
#ifndef SAT_NCW8
#define SAT_NCW8 8
#endif
  static constexpr int NCW = SAT_NCW8;   // compute warps
#ifndef SAT_TH8
#define SAT_TH8 32
#endif
  static constexpr int TH = SAT_TH8;     // band height (TH / NCW rows per compute warp)
#ifndef SAT_NST8
#define SAT_NST8 5
#endif
  static constexpr int NSTAGE = SAT_NST8;  // TMA prefetch depth (stages free after pass A)
#ifndef SAT_MINB8
#define SAT_MINB8 2
#endif
  static constexpr int MINB = SAT_MINB8;   // resident CTAs per SM
#ifndef SAT_NLW8
#define SAT_NLW8 SAT_NLW
#endif
  static constexpr int NLW = SAT_NLW8;     // leader (look-back) warps
};
template <>
struct Cfg<P32F32F> {
  using TA = float;
  using TB = float;
  static constexpr int E = 4;
  static constexpr int G = 1;
  static constexpr int TW = 128;
  static constexpr int TH = 32;
#ifndef SAT_LOOK32
#define SAT_LOOK32 7
#endif
  static constexpr int LOOK = SAT_LOOK32;
  static constexpr int NCW = 8;
#ifndef SAT_NST32
#define SAT_NST32 3
#endif
  static constexpr int NSTAGE = SAT_NST32;
};
template <>
struct Cfg<P64F64F> {
  using TA = double;
  using TB = double;
  static constexpr int E = 2;
  static constexpr int G = 1;
  static constexpr int TW = 64;
  static constexpr int TH = 32;
#ifndef SAT_LOOK64
#define SAT_LOOK64 4
#endif
  static constexpr int LOOK = SAT_LOOK64;
  static constexpr int NCW = 8;
#ifndef SAT_NST64
#define SAT_NST64 4
#endif
  static constexpr int NSTAGE = SAT_NST64;
};
// 8u -> 32f (NPP's nppiIntegral_8u32f): the 8u->32s geometry (256-column
// tiles, two 4-byte lane groups), fp32 values and scans.
template <>
struct Cfg<P8U32F> : Cfg<P8U32S> {
  using TB = float;
};
// 32s -> 32s: the 32f geometry with wrap-around u32 integer scans (R2).
template <>
struct Cfg<P32S32S> : Cfg<P32F32F> {
  using TA = uint32_t;
  using TB = uint32_t;
};

// K-channel u32 element (wrap-around adds per channel, exact mod 2^32).
template <int K>
struct ChanVec {
  uint32_t c[K];
  __device__ __forceinline__ ChanVec() {}
  __device__ __forceinline__ ChanVec(int z) {
#pragma unroll
    for (int k = 0; k < K; ++k) c[k] = (uint32_t)z;
  }
  __device__ __forceinline__ ChanVec& operator+=(const ChanVec& o) {
#pragma unroll
    for (int k = 0; k < K; ++k) c[k] += o.c[k];
    return *this;
  }
  __device__ __forceinline__ ChanVec operator+(const ChanVec& o) const {
    ChanVec r = *this;
    r += o;
    return r;
  }
};
template <int K>
__device__ __forceinline__ ChanVec<K> shfl_up(const ChanVec<K>& v, int d) {
  ChanVec<K> r;
#pragma unroll
  for (int k = 0; k < K; ++k) r.c[k] = __shfl_up_sync(0xffffffffu, v.c[k], d);
  return r;
}
template <int K>
__device__ __forceinline__ ChanVec<K> shfl_idx(const ChanVec<K>& v, int l) {
  ChanVec<K> r;
#pragma unroll
  for (int k = 0; k < K; ++k) r.c[k] = __shfl_sync(0xffffffffu, v.c[k], l);
  return r;
}
// 8u -> (a, a^2): 128-column tiles, a lane owns two groups of 2 pixels (16 B out each).
template <>
struct Cfg<P8USQ> {
  using TA = uint8_t;
  using TB = ChanVec<2>;
  static constexpr int K = 2;
  static constexpr int E = 2;
  static constexpr int G = 2;
  static constexpr int TW = 32 * E * G;  // 128
  static constexpr int LOOK = 3;
  static constexpr int NCW = 8;
  static constexpr int TH = 32;
  static constexpr int NSTAGE = 4;
};
// 8u -> 4 histogram bins: 64-column tiles, a lane owns two groups of 1 pixel.
template <>
struct Cfg<P8UHIST4> {
  using TA = uint8_t;
  using TB = ChanVec<4>;
  static constexpr int K = 4;
  static constexpr int E = 1;
  static constexpr int G = 2;
  static constexpr int TW = 32 * E * G;  // 64
  static constexpr int LOOK = 3;
  static constexpr int NCW = 8;
  static constexpr int TH = 32;
  static constexpr int NSTAGE = 4;
};
template <int P>
constexpr bool kChan = kBase<P> == P8USQ || kBase<P> == P8UHIST4;

// Optional per-configuration members: MINB (resident CTAs per SM; default 2,
// or 1 with more than 8 compute warps) and NLW (leader warps).
template <int P, class = void>
struct MinBlocksOf {
  static constexpr int v = Cfg<P>::NCW > 8 ? 1 : 2;
};
template <int P>
struct MinBlocksOf<P, std::void_t<decltype(Cfg<P>::MINB)>> {
  static constexpr int v = Cfg<P>::MINB;
};
template <int P, class = void>
struct NlwOf {
  static constexpr int v = kNLWDefault;
};
template <int P>
struct NlwOf<P, std::void_t<decltype(Cfg<P>::NLW)>> {
  static constexpr int v = Cfg<P>::NLW;
};
template <int P>
constexpr int kNLW = NlwOf<P>::v;

template <int P>
struct CfgShort : Cfg<P> {
  static constexpr int TH = Cfg<P>::TH / 2;
};
template <>
struct Cfg<P8U32S + kShort> : CfgShort<P8U32S> {};
template <>
struct Cfg<P32F32F + kShort> : CfgShort<P32F32F> {};
template <>
struct Cfg<P64F64F + kShort> : CfgShort<P64F64F> {};
template <>
struct Cfg<P8U32F + kShort> : CfgShort<P8U32F> {};
template <>
struct Cfg<P32S32S + kShort> : CfgShort<P32S32S> {};

// Deep-ring variants (P + kDeep): the pair's geometry with one CTA per SM, a
// deeper TMA ring and twice the TMEM slots, for launches of at most one band
// per SM (wide, short images: 4096 x 65536).  Two CTAs per SM would leave
// half the slots empty there, and one CTA's bytes in flight (NSTAGE tiles)
// bound its bandwidth: 64f 4096 x 65536 needs ~41 GB/s per band at 0.8 of
// the copy peak against ~32 GB/s from three 16 KB stages.
constexpr int kDeep = 16;
template <int P>
constexpr bool kIsShort = P >= kShort && P < kDeep;
template <int P>
constexpr bool kIsDeep = P >= kDeep;
template <int P, int NST>
struct CfgDeep : Cfg<P> {
  static constexpr int MINB = 1;
  static constexpr int NSTAGE = NST;
  static constexpr int LOOK = 2 * Cfg<P>::LOOK + 1;  // 512 TMEM columns instead of 256
};
template <>
struct Cfg<P8U32S + kDeep> : CfgDeep<P8U32S, 10> {};
template <>
struct Cfg<P32F32F + kDeep> : CfgDeep<P32F32F, 6> {};
template <>
struct Cfg<P64F64F + kDeep> : CfgDeep<P64F64F, 8> {};
template <>
struct Cfg<P8U32F + kDeep> : CfgDeep<P8U32F, 10> {};
template <>
struct Cfg<P32S32S + kDeep> : CfgDeep<P32S32S, 6> {};


// Warp roles: NCW compute warps, the producer, the aggregate warp, the offset
// warp, then kNLW leader warps.
template <int P>
constexpr int kNCW = Cfg<P>::NCW;
template <int P>
constexpr int kProducerWarp = kNCW<P>;
template <int P>
constexpr int kAggWarp = kNCW<P> + 1;
template <int P>
constexpr int kOffWarp = kNCW<P> + 2;
template <int P>
constexpr int kFirstLwWarp = kNCW<P> + 3;
template <int P>
constexpr int kThreads = (kFirstLwWarp<P> + kNLW<P>) * 32;

// Words of one carry payload vector: TW elements * (4 / E) 64-bit words per element.
template <int P>
constexpr int kVecWords = Cfg<P>::TW * 4 / Cfg<P>::E;
// Payload vectors one look-back round lands in shared memory (kLandWords * 8 B
// per look-back warp).
#ifndef SAT_LB_LDG
#define SAT_LB_LDG 0  // look-back reads: 0 bulk copies into shared memory, 1 per-lane loads
#endif
#ifndef SAT_LAND_WORDS
#define SAT_LAND_WORDS 256
#endif
// Counted reduction tree (integer pairs, SAT_FEN=1): the cross-cluster carry
// is a Fenwick (binary indexed) tree per image over the clusters' column
// contributions, built with element-wise atomic bulk reductions (TMA) the
// moment a cluster's aggregates are gathered; a reader sums the <= log2(D)
// tree nodes of its prefix in one round -- no chain of inclusive prefixes,
// so the carry latency does not grow with the depth of the tile column.
// Each node word is 64 bits: value (bits 0-31, mod 2^32), the carries out of
// it (bits 32-47) and the number of contributions (bits 48-63), so a word
// whose count matches the node's writer count holds the complete sum.
// Exact (wrap-around integer adds commute), hence integer pairs only; the
// float pairs keep the look-back (fixed summation order).
// SAT_FEN: 1 compiles the tree into the integer-pair kernels next to the
// look-back; KParams::tree selects it per launch (the runtime's shape rule).
#ifndef SAT_FEN
#define SAT_FEN 1
#endif
template <int P>
constexpr bool kFen = SAT_FEN != 0 && (kBase<P> == P8U32S || kBase<P> == P32S32S ||
                                       kBase<P> == P8USQ || kBase<P> == P8UHIST4);
constexpr uint64_t kFenOne = 1ull << 48;  // one contribution, in a node word's count field
#ifndef SAT_FEN_LAND
#define SAT_FEN_LAND 6
#endif
template <int P>
constexpr int kLandVecs = kFen<P> ? (SAT_FEN_LAND)
                        : (SAT_LAND_WORDS) / kVecWords<P> > 2 ? (SAT_LAND_WORDS) / kVecWords<P> : 2;

// Chunk slots between pass A and pass B (TMEM S', column totals, metadata).
template <int P>
constexpr int kNTot = Cfg<P>::LOOK + 1;
// V_up ring: the aggregate warp (which arms a slot) runs at most NSTAGE + kNTot
// chunks ahead of pass B (which drains it): a stage is refilled only after
// every compute warp's pass A of it, which follows that warp's pass B of the
// chunk kNTot earlier.
template <int P>
constexpr int kNV = Cfg<P>::NSTAGE + kNTot<P>;

// Tensor memory (TMEM) holds pass A's column-scanned rows S' until pass B:
// per warp and chunk slot, RW rows x G x E values of 32-bit words (fp64: 2 words).
template <int P>
constexpr int kTmemColsPerWarp =
    (Cfg<P>::TH / kNCW<P>) * Cfg<P>::G * Cfg<P>::E * (int)(sizeof(typename Cfg<P>::TB) / 4);
template <int P>
constexpr int kMinBlocks = MinBlocksOf<P>::v;  // resident CTAs per SM
// TMEM columns per CTA: the SM's 512 columns shared by its resident CTAs.
template <int P>
constexpr int kTmemCols = 512 / kMinBlocks<P>;
template <int P>
constexpr int kTmemColsPerSlot = kTmemColsPerWarp<P> * (kNCW<P> / 4);  // NCW/4 warps per subpartition
static_assert(kTmemColsPerSlot<P8U32S> * kNTot<P8U32S> <= kTmemCols<P8U32S>, "TMEM budget (8u)");
static_assert(kTmemColsPerSlot<P32F32F> * kNTot<P32F32F> <= kTmemCols<P32F32F>, "TMEM budget (32f)");
static_assert(kTmemColsPerSlot<P64F64F> * kNTot<P64F64F> <= kTmemCols<P64F64F>, "TMEM budget (64f)");
static_assert(kTmemColsPerSlot<P8U32F> * kNTot<P8U32F> <= kTmemCols<P8U32F>, "TMEM budget (8u32f)");
static_assert(kTmemColsPerSlot<P32S32S> * kNTot<P32S32S> <= kTmemCols<P32S32S>, "TMEM budget (32s)");
static_assert(kTmemColsPerSlot<P8USQ> * kNTot<P8USQ> <= kTmemCols<P8USQ>, "TMEM budget (8u sq)");
static_assert(kTmemColsPerSlot<P8UHIST4> * kNTot<P8UHIST4> <= kTmemCols<P8UHIST4>, "TMEM budget (hist)");

struct KParams {
  const char* in;       // generic-path input base (TMA path uses the tensor map)
  char* out;
  int64_t H, W;
  int64_t in_pitch, out_pitch;           // bytes
  int64_t in_img_stride, out_img_stride; // bytes
  int64_t bands_per_image;               // ceil(H / TH)
  int64_t total_bands;                   // batch * bands_per_image
  int64_t total_tickets;                 // ceil(total_bands / CL) cluster tickets
  int32_t nchunks;                       // ceil(W / TW)
  uint32_t epoch;                        // status-word epoch of this launch
  uint64_t ticket_base;                  // counter value at launch
  unsigned long long* counter;           // ticket counter (workspace)
  void* payload;                         // [tickets][nchunks][kVecWords] status-tagged carries
                                         // (kFen pairs: the counted reduction tree's nodes)
  uint32_t* tree_rd;                     // kFen: [tickets][nchunks] node read counters
  int32_t tree;                          // kFen pairs: 1 carries by the tree, 0 by the look-back
  uint32_t ticket_lead;                  // draw the next ticket when pass A is this many
                                         // chunks from the end of the issued tiles
  const void* carry_in;                  // optional S(r0-1, .) row (W elems of TB) for image starts
  // Exclusive layout (kernels instantiated with kEx): S(y, x) is stored at
  // output row y (out already points at row 1 of the exclusive array) and
  // column x + 1; column 0 holds nval; columns >= out_cols are not written.
  int64_t out_cols;
  uint64_t nval_bits;                    // nVal, a TB value's bits (added to every element)
  // Chained bands: the carry row S(r0-1, .) arrives per
  // chunk as an epoch-tagged vector (payload layout) written by the kernel of
  // the band above -- possibly on another GPU through peer memory -- and this
  // band's bottom row S(r1-1, .) is published the same way for the band below.
  // Flow control (double-buffered slots): the band below acknowledges each
  // consumed chunk by writing the epoch into the upper band's ack word; a band
  // overwrites a slot (epoch e, slot e & 1) only after the band below has
  // acknowledged epoch e - 2 of that chunk.  No host or NCCL barrier per call.
  const uint64_t* chain_in;              // this call's receive slot [nchunks][kVecWords] or NULL
  uint64_t* chain_out;                   // the band below's receive slot or NULL
  uint32_t* chain_ack_out;               // the band above's ack words [nchunks] (with chain_in)
  const uint32_t* chain_ack_in;          // this band's ack words (with chain_out)
  uint32_t chain_epoch;                  // >= 1; tag = (chain_epoch << 2) | kStIncl
  // Bounded waits: a cross-CTA / cross-GPU carry wait that exceeds spin_ns
  // sets bit 0 of *err, takes zeros and lets the launch finish (the host
  // reports SAT_ERR_TIMEOUT) instead of hanging the GPU.
  uint32_t* err;
  uint64_t spin_ns;
  // Integral histogram (P8UHIST4): bin of every byte value; this launch
  // counts bins [bin0, bin0 + 4).
  uint8_t bin_of[256];
  int32_t bin0;
};

// Optional phase profiling (debug builds with -DSAT_PROFILE): per-CTA shared
// counters summed into g_sat_prof at exit.
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
// Optional timeline (debug builds with -DSAT_TIMELINE): globaltimer at every
// pass B of the first band each CTA processes, plus that band's index.
#ifdef SAT_TIMELINE
constexpr int kTlChunks = 256;
__device__ unsigned long long g_sat_tl[1024][2 + kTlChunks];
__device__ unsigned long long g_sat_tl_agg[1024][kTlChunks];  // aggregate sent (first band)
__device__ unsigned long long g_sat_tl_v[1024][kTlChunks];    // V_up landed (first band)
__device__ unsigned long long g_sat_tl_ls[1024][kTlChunks];   // leader: gather complete (led chunks)
__device__ unsigned long long g_sat_tl_lt[1024][kTlChunks];   // leader: prefix known
__device__ unsigned long long g_sat_tl_ld[1024][kTlChunks];   // leader: V_up sent
__device__ unsigned int g_sat_tl_rounds[1024][kTlChunks][2];  // leader: look-back rounds, retries
constexpr int kTlBands = 16384;
__device__ unsigned long long g_sat_band_t[kTlBands][2];        // every band: first / last pass B
__device__ __forceinline__ uint64_t tl_now() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#endif
enum ProfSlot {
  kPfComputeWaitFull = 0,   // warp 0: waiting for TMA data
  kPfComputeWaitCarry = 1,  // warp 0: waiting for the look-back result
  kPfComputeLocal = 2,      // warp 0: pass A
  kPfComputeFixup = 3,      // warp 0: pass B (after the wait)
  kPfLbWaitTot = 4,         // look-back warps: waiting for the column totals
  kPfLbCluster = 5,         // leader: waiting for the cluster's band aggregates
  kPfLbLookback = 6,        // leader: global probe + payload reads
  kPfLbDepth = 7,           // vectors summed
  kPfLbRetries = 8,         // probe rounds that found a missing predecessor
  kPfLbChunks = 9,          // chunks handled (all look-back warps)
  kPfLbWaitV = 10,          // all: waiting for V_up from the leader
  kPfProdWaitTicket = 11,   // producer: holding the next ticket back
  kPfLeaderChunks = 12,     // chunks handled by leaders
  kPfLbRoundTime = 13,      // leader: issue -> landed time of look-back rounds
  kPfLbRounds = 14,         // leader: look-back rounds issued
  kPfLbIssue = 15,          // leader: fence + bulk-copy issue time
};

// Chunk q of a cluster is led by CTA q % CL (rotating leadership spreads the
// global look-backs over all the cluster's leader warps).  A leader's gather
// slot is reused CL * kNLead chunks later.  A band's aggregate warp reaches
// chunk q only after the band's pass B of chunk q - NSTAGE - kNTot, i.e. after
// that chunk's leader has read the band's earlier aggregate, so CL * kNLead >=
// NSTAGE + kNTot keeps a slot from being overwritten while its leader reads it.
// The end-of-work sentinels go up to CL * kNLW - 1 chunks further (the next
// chunk each leader warp would lead), hence the extra CL * kNLW - 1.
template <int P, int CL>
constexpr int kNLeadRaw = (Cfg<P>::NSTAGE + kNTot<P> + CL * kNLW<P> - 1 + CL - 1) / CL;
template <int P, int CL>
constexpr int kNLead = kNLeadRaw<P, CL> > kNLW<P> ? kNLeadRaw<P, CL> : kNLW<P>;

template <int P, int CL>
struct __align__(128) Smem {
  using C = Cfg<P>;
  typename C::TA in[C::NSTAGE][C::TH][C::TW];   // TMA destination ring
  alignas(128) typename C::TB tot[kNTot<P>][kNCW<P>][C::TW];    // per-warp column totals -> fix-up offsets
  alignas(128) typename C::TB lead_in[kNLead<P, CL>][CL][C::TW];  // chunk leader: the bands' aggregates
  alignas(128) typename C::TB vin[kNV<P>][C::TW];            // V_up of this band (from the leader)
  int32_t meta[kNCW<P>][kNTot<P>][4];              // per warp: (band lo, img, k, chunk) of each slot
  uint32_t tmem_base;                           // TMEM address from tcgen05.alloc
  alignas(128) uint64_t land[kNLW<P>][kLandVecs<P>][kVecWords<P>];  // look-back landing (bulk copies)
  alignas(128) uint64_t fstage[kNLW<P>][kFen<P> ? kVecWords<P> : 2];  // tree: staged contribution
  uint64_t full[C::NSTAGE];
  uint64_t empty[C::NSTAGE];
  uint64_t tot_full[kNTot<P>];
  uint64_t carry_full[kNTot<P>];
  uint64_t lead_full[kNLead<P, CL>];            // CL aggregates landed in lead_in (+ leader's arrive)
  int64_t lead_band[kNLead<P, CL>];             // leader: its own band of the slot's chunk (-1: end)
  int32_t lead_chunk[kNLead<P, CL>];
  uint64_t vin_full[kNV<P>];                    // tx: V_up landed in vin
  uint64_t land_full[kNLW<P>];                     // tx: a look-back round landed
  uint64_t tk_full;                             // tx: ticket landed in tk_slot
  uint64_t tk_empty;                            // leader: peers consumed the ticket
  int64_t tk_slot;
  int64_t stage_band[C::NSTAGE];   // global band index, -1 = end of work
  int32_t stage_img[C::NSTAGE];    // image index n (-1: padding band of a partial cluster)
  int32_t stage_k[C::NSTAGE];      // band index within the image
  int32_t stage_chunk[C::NSTAGE];
  int64_t tot_band[kNTot<P>];
  int32_t tot_img[kNTot<P>];
  int32_t tot_k[kNTot<P>];
  int32_t tot_chunk[kNTot<P>];
  volatile uint32_t passA_done;                 // chunks through pass A (ticket pacing)
  uint8_t bin_of[256];                          // P8UHIST4: byte -> bin (from KParams, in smem:
                                                // divergent constant-bank reads serialise)
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

// Long waits (a warp that typically waits microseconds): non-blocking
// test_wait polls with an exponential __nanosleep back-off.  The hardware
// try_wait suspend loop wakes on every mbarrier event of the CTA and re-polls,
// which burnt ~20% of the 8u kernel's issue slots in spin iterations (ncu).
#ifndef SAT_BO_MAX
#define SAT_BO_MAX 256
#endif
__device__ __forceinline__ bool mbar_test(uint32_t addr, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n\t}"
      : "=r"(ok)
      : "r"(addr), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
  const uint32_t addr = smem_u32(bar);
  if (mbar_test(addr, parity)) return;
  uint32_t ns = 32;
  for (;;) {
    __nanosleep(ns);
    if (mbar_test(addr, parity)) return;
    if (ns < (SAT_BO_MAX)) ns <<= 1;
  }
}
#ifndef SAT_BO_CARRY
#define SAT_BO_CARRY 1
#endif

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


// Streaming (evict-first) 16-byte output store.
#ifndef SAT_ST_HINT
#define SAT_ST_HINT ".cs"
#endif
__device__ __forceinline__ void st_cs_v4(void* p, uint4 v) {
  asm volatile("st.global" SAT_ST_HINT ".v4.u32 [%0], {%1, %2, %3, %4};" ::"l"(p), "r"(v.x), "r"(v.y),
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
// Cluster / distributed-shared-memory helpers

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}

// Address of the same shared variable in CTA `rank` of this cluster.
__device__ __forceinline__ uint32_t mapa(const void* local, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(smem_u32(local)), "r"(rank));
  return r;
}

// 16-byte store into a (possibly remote) CTA's smem, completing 16 tx-bytes on
// that CTA's mbarrier.
__device__ __forceinline__ void st_async16(uint32_t raddr, uint4 v, uint32_t rbar) {
  asm volatile(
      "st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(
          raddr),
      "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w), "r"(rbar)
      : "memory");
}

// Expect `bytes` of tx on a local mbarrier without arriving.
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.expect_tx.relaxed.cta.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}

// 16-byte hand-off into CTA `dst` of the cluster.  Remote: st.async with tx on
// its mbarrier.  Self (st.async needs a remote CTA -- a cluster of 1 has
// none): plain shared store; the caller then arrives (release) on the barrier,
// which was armed for the remote bytes only.
__device__ __forceinline__ void send16(void* local_dst, uint64_t* local_bar, uint32_t dst,
                                       uint32_t self, uint4 v) {
  if (dst == self)
    *reinterpret_cast<uint4*>(local_dst) = v;
  else
    st_async16(mapa(local_dst, dst), v, mapa(local_bar, dst));
}

__device__ __forceinline__ void st_async8(uint32_t raddr, uint64_t v, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(raddr),
               "l"(v), "r"(rbar)
               : "memory");
}

__device__ __forceinline__ void mbar_arrive_remote(uint32_t rbar) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(rbar) : "memory");
}

// Waits for data that peers deliver into this CTA's shared memory with
// st.async + complete_tx (aggregates, V_up).  The cluster-scope acquire
// compiles to an L1 invalidation (CCTL.IVALL) per wait (5% of the 8u kernel's
// stall samples, ncu r02b); SAT_ACQ_CTA=1 waits with a CTA-scope acquire
// instead (the phase cannot complete before the bytes have landed here), which
// measured within same-box noise (16384^2 -1.4%), so the formally matching
// cluster scope stays the default.
#ifndef SAT_ACQ_CTA
#define SAT_ACQ_CTA 0
#endif
__device__ __forceinline__ void mbar_wait_peer_data(uint64_t* bar, uint32_t parity);
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t parity) {
  uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAITC_%=:\n\t"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 p, [%0], %1, %2;\n\t"
      "@!p bra WAITC_%=;\n\t}" ::"r"(addr),
      "r"(parity), "r"(0x100000u)
      : "memory");
}
__device__ __forceinline__ void mbar_wait_peer_data(uint64_t* bar, uint32_t parity) {
#if SAT_ACQ_CTA
  mbar_wait(bar, parity);
#else
  mbar_wait_cluster(bar, parity);
#endif
}

__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}

// ---------------------------------------------------------------------------
// Tensor-memory (TMEM) helpers: 32x32b shape = thread i of the warp <-> TMEM
// lane (subpartition base + i), .xN = N consecutive 32-bit columns.

__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
      "%11, %12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, "
      "%29, %30, %31, %32};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
      "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15]),
      "r"(v[16]), "r"(v[17]), "r"(v[18]), "r"(v[19]), "r"(v[20]), "r"(v[21]), "r"(v[22]),
      "r"(v[23]), "r"(v[24]), "r"(v[25]), "r"(v[26]), "r"(v[27]), "r"(v[28]), "r"(v[29]),
      "r"(v[30]), "r"(v[31])
      : "memory");
}
__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8, %9, %10, "
      "%11, %12, %13, %14, %15, %16};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]),
      "r"(v[8]), "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&v)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
      "%12, %13, %14, %15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, "
      "%30, %31}, [%32];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
        "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]),
        "=r"(v[20]), "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]),
        "=r"(v[26]), "=r"(v[27]), "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void tmem_st(uint32_t taddr, const uint32_t (&v)[8]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1, %2, %3, %4, %5, %6, %7, %8};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
      : "memory");
}
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&v)[8]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void tmem_ld(uint32_t taddr, uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, "
      "%12, %13, %14, %15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
        "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
        "=r"(v[14]), "=r"(v[15])
      : "r"(taddr)
      : "memory");
}
__device__ __forceinline__ void tmem_wait_st() {
  asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}

// Pack / unpack a lane's RW x G x E values as 32-bit words for TMEM.
__device__ __forceinline__ uint32_t w_lo(uint32_t v) { return v; }
__device__ __forceinline__ uint32_t w_lo(float v) { return __float_as_uint(v); }
template <typename T>
struct IsChan : std::false_type {};
template <int K>
struct IsChan<ChanVec<K>> : std::true_type {};
template <typename TB, int N>
__device__ __forceinline__ void put_words(uint32_t (&w)[N], int idx, TB v) {
  if constexpr (IsChan<TB>::value) {
#pragma unroll
    for (int k = 0; k < (int)(sizeof(TB) / 4); ++k) w[idx * (int)(sizeof(TB) / 4) + k] = v.c[k];
  } else if constexpr (sizeof(TB) == 8) {
    const uint64_t b = (uint64_t)__double_as_longlong(v);
    w[2 * idx] = (uint32_t)b;
    w[2 * idx + 1] = (uint32_t)(b >> 32);
  } else {
    w[idx] = w_lo(v);
  }
}
template <typename TB, int N>
__device__ __forceinline__ TB get_words(const uint32_t (&w)[N], int idx) {
  if constexpr (IsChan<TB>::value) {
    TB v;
#pragma unroll
    for (int k = 0; k < (int)(sizeof(TB) / 4); ++k) v.c[k] = w[idx * (int)(sizeof(TB) / 4) + k];
    return v;
  } else if constexpr (sizeof(TB) == 8) {
    return __longlong_as_double((long long)(((uint64_t)w[2 * idx + 1] << 32) | w[2 * idx]));
  } else if constexpr (sizeof(TB) == 4 && TB(0.5) != TB(0)) {
    return __uint_as_float(w[idx]);
  } else {
    return (TB)w[idx];
  }
}

// One Kogge-Stone step in place, v += v(lane - d) for lane >= d (Alg. 3,
// reading R10): shfl.up's in-range predicate guards the add -- two
// instructions per step (the C++ form compiled to shuffle + predicated add +
// move).  Same operation and order, so results are unchanged.
__device__ __forceinline__ void ks_step(uint32_t& v, int d) {
  asm("{\n\t.reg .pred p;\n\t.reg .b32 t;\n\t"
      "shfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t"
      "@p add.u32 %0, %0, t;\n\t}"
      : "+r"(v)
      : "r"(d));
}
__device__ __forceinline__ void ks_step(float& v, int d) {
  asm("{\n\t.reg .pred p;\n\t.reg .f32 t;\n\t"
      "shfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t"
      "@p add.rn.f32 %0, %0, t;\n\t}"
      : "+f"(v)
      : "r"(d));
}

// ---------------------------------------------------------------------------
// a2 + a3: scan the RW rows a warp owns, all rows advancing through the
// Kogge-Stone stages together (RW-way ILP on the shuffle latency).  Produces
// R[i] = rowcarry_i + (in-row prefix), the row-prefixed values of row i for
// this lane's columns, and advances the row carries.  `tile` points at the
// warp's first smem row; rows are TW elements apart.

template <int RW>
__device__ __forceinline__ void rows_scan(const uint8_t* tile, int lane, uint32_t (&rowcarry)[RW],
                                          uint32_t (&R)[RW][2][4]) {
  constexpr int TW = 256;
  uint32_t w0[RW], w1[RW], own[RW], inc[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    w0[i] = *reinterpret_cast<const uint32_t*>(tile + i * TW + 4 * lane);
    w1[i] = *reinterpret_cast<const uint32_t*>(tile + i * TW + 128 + 4 * lane);
  }
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    // a2: group totals by byte dot-products; two groups packed as 16-bit
    // halves (each prefix <= 32640, no carry between halves).
    own[i] = __dp4a(w0[i], 0x01010101u, 0u) | (__dp4a(w1[i], 0x01010101u, 0u) << 16);
    inc[i] = own[i];
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)  // a3: Alg. 3, lane >= d (reading R10)
#pragma unroll
    for (int i = 0; i < RW; ++i) ks_step(inc[i], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const uint32_t tot = __shfl_sync(kFull, inc[i], 31);
    const uint32_t ex = inc[i] - own[i];
    const uint32_t tot0 = tot & 0xFFFFu;
    const uint32_t base0 = rowcarry[i] + (ex & 0xFFFFu);
    const uint32_t base1 = rowcarry[i] + tot0 + (ex >> 16);
    rowcarry[i] += tot0 + (tot >> 16);
    // in-group prefixes + carry: dp4a with byte masks (Alg. 2 on 4 elements)
    R[i][0][0] = __dp4a(w0[i], 0x00000001u, base0);
    R[i][0][1] = __dp4a(w0[i], 0x00000101u, base0);
    R[i][0][2] = __dp4a(w0[i], 0x00010101u, base0);
    R[i][0][3] = __dp4a(w0[i], 0x01010101u, base0);
    R[i][1][0] = __dp4a(w1[i], 0x00000001u, base1);
    R[i][1][1] = __dp4a(w1[i], 0x00000101u, base1);
    R[i][1][2] = __dp4a(w1[i], 0x00010101u, base1);
    R[i][1][3] = __dp4a(w1[i], 0x01010101u, base1);
  }
}

template <int RW>
__device__ __forceinline__ void rows_scan(const float* tile, int lane, float (&rowcarry)[RW],
                                          float (&R)[RW][1][4]) {
  constexpr int TW = 128;
  float p[RW][4], inc[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const float4 a = *reinterpret_cast<const float4*>(tile + i * TW + 4 * lane);
    p[i][0] = a.x;  // Alg. 2
    p[i][1] = p[i][0] + a.y;
    p[i][2] = p[i][1] + a.z;
    p[i][3] = p[i][2] + a.w;
    inc[i] = p[i][3];
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)  // Alg. 3
#pragma unroll
    for (int i = 0; i < RW; ++i) ks_step(inc[i], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const float tot = __shfl_sync(kFull, inc[i], 31);
    float ex = __shfl_up_sync(kFull, inc[i], 1);
    if (lane == 0) ex = 0.0f;
    const float base = rowcarry[i] + ex;
    rowcarry[i] += tot;
#pragma unroll
    for (int e = 0; e < 4; ++e) R[i][0][e] = base + p[i][e];
  }
}

// 8u -> 32f, 256-column tiles: each lane widens two 4-byte groups (columns
// 4l.. and 128+4l..) to fp32, prefix within the group (Alg. 2), and scans the
// two group totals across the warp (Alg. 3, one Kogge-Stone per group).
template <int RW>
__device__ __forceinline__ void rows_scan(const uint8_t* tile, int lane, float (&rowcarry)[RW],
                                          float (&R)[RW][2][4]) {
  // The in-chunk prefixes of bytes are integers <= 65280: scan them exactly
  // as the 8u->32s path does (dp4a group sums packed in 16-bit halves, one
  // predicated-shuffle Kogge-Stone per row, dp4a in-group prefixes), then
  // one rounding each: R = rowcarry + float(prefix), rowcarry += float(total).
  constexpr int TW = 256;
  uint32_t w0[RW], w1[RW], own[RW], inc[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    w0[i] = *reinterpret_cast<const uint32_t*>(tile + i * TW + 4 * lane);
    w1[i] = *reinterpret_cast<const uint32_t*>(tile + i * TW + 128 + 4 * lane);
    own[i] = __dp4a(w0[i], 0x01010101u, 0u) | (__dp4a(w1[i], 0x01010101u, 0u) << 16);
    inc[i] = own[i];
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)  // Alg. 3, lane >= d (reading R10)
#pragma unroll
    for (int i = 0; i < RW; ++i) ks_step(inc[i], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const uint32_t tot = __shfl_sync(kFull, inc[i], 31);
    const uint32_t ex = inc[i] - own[i];
    const uint32_t tot0 = tot & 0xFFFFu;
    const uint32_t base0 = ex & 0xFFFFu;
    const uint32_t base1 = tot0 + (ex >> 16);
    const float rc = rowcarry[i];
    rowcarry[i] = rc + (float)(tot0 + (tot >> 16));
    R[i][0][0] = rc + (float)__dp4a(w0[i], 0x00000001u, base0);
    R[i][0][1] = rc + (float)__dp4a(w0[i], 0x00000101u, base0);
    R[i][0][2] = rc + (float)__dp4a(w0[i], 0x00010101u, base0);
    R[i][0][3] = rc + (float)__dp4a(w0[i], 0x01010101u, base0);
    R[i][1][0] = rc + (float)__dp4a(w1[i], 0x00000001u, base1);
    R[i][1][1] = rc + (float)__dp4a(w1[i], 0x00000101u, base1);
    R[i][1][2] = rc + (float)__dp4a(w1[i], 0x00010101u, base1);
    R[i][1][3] = rc + (float)__dp4a(w1[i], 0x01010101u, base1);
  }
}

// 32s -> 32s: as the 32f scan, in wrap-around uint32 arithmetic (exact mod 2^32).
template <int RW>
__device__ __forceinline__ void rows_scan(const uint32_t* tile, int lane, uint32_t (&rowcarry)[RW],
                                          uint32_t (&R)[RW][1][4]) {
  constexpr int TW = 128;
  uint32_t p[RW][4], inc[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const uint4 a = *reinterpret_cast<const uint4*>(tile + i * TW + 4 * lane);
    p[i][0] = a.x;  // Alg. 2
    p[i][1] = p[i][0] + a.y;
    p[i][2] = p[i][1] + a.z;
    p[i][3] = p[i][2] + a.w;
    inc[i] = p[i][3];
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)  // a3: Alg. 3, lane >= d (reading R10)
#pragma unroll
    for (int i = 0; i < RW; ++i) ks_step(inc[i], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const uint32_t tot = __shfl_sync(kFull, inc[i], 31);
    const uint32_t base = rowcarry[i] + (inc[i] - p[i][3]);
    rowcarry[i] += tot;
#pragma unroll
    for (int e = 0; e < 4; ++e) R[i][0][e] = base + p[i][e];
  }
}

template <int RW>
__device__ __forceinline__ void rows_scan(const double* tile, int lane, double (&rowcarry)[RW],
                                          double (&R)[RW][1][2]) {
  constexpr int TW = 64;
  double p[RW][2], inc[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const double2 a = *reinterpret_cast<const double2*>(tile + i * TW + 2 * lane);
    p[i][0] = a.x;
    p[i][1] = a.x + a.y;
    inc[i] = p[i][1];
  }
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    double o[RW];
#pragma unroll
    for (int i = 0; i < RW; ++i) o[i] = __shfl_up_sync(kFull, inc[i], d);
#pragma unroll
    for (int i = 0; i < RW; ++i)
      if (lane >= d) inc[i] += o[i];
  }
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const double tot = __shfl_sync(kFull, inc[i], 31);
    double ex = __shfl_up_sync(kFull, inc[i], 1);
    if (lane == 0) ex = 0.0;
    const double base = rowcarry[i] + ex;
    rowcarry[i] += tot;
    R[i][0][0] = base + p[i][0];
    R[i][0][1] = base + p[i][1];
  }
}

// Multi-channel pairs: a per-pixel vector f(a) whose channel-wise SAT is the
// output (Eq. 1 per channel).  P8USQ: f(a) = (a, a^2) -- the SAT and the SAT
// of squares of Viola-Jones variance normalisation ([2]);
// P8UHIST4: f(a) = the indicator vector of bins [bin0, bin0 + 4) -- the
// integral histogram ([34], [38]).
template <int P>
struct Xf;
template <>
struct Xf<P8USQ> {
  static __device__ __forceinline__ ChanVec<2> f(uint32_t a, const KParams&) {
    ChanVec<2> r;
    r.c[0] = a;
    r.c[1] = a * a;
    return r;
  }
};
template <>
struct Xf<P8UHIST4> {
  static __device__ __forceinline__ ChanVec<4> f(uint32_t a, const KParams& p) {
    const int b = (int)p.bin_of[a] - p.bin0;
    ChanVec<4> r;
#pragma unroll
    for (int k = 0; k < 4; ++k) r.c[k] = b == k ? 1u : 0u;
    return r;
  }
};

// The lane's E consecutive bytes of group g of a tile row.
template <int E>
__device__ __forceinline__ uint32_t lane_bytes(const uint8_t* row, int col) {
  if constexpr (E == 2) return *reinterpret_cast<const uint16_t*>(row + col);
  else return row[col];
}

// a2 + a3 for the multi-channel pairs: per-lane serial prefix of the E pixels
// of each group (Alg. 2), Kogge-Stone over the lanes (Alg. 3, lane >= d).
template <int P, int RW>
__device__ __forceinline__ void rows_scan_xf(const uint8_t* tile, int lane, const KParams& p,
                                             typename Cfg<P>::TB (&rowcarry)[RW],
                                             typename Cfg<P>::TB (&R)[RW][Cfg<P>::G][Cfg<P>::E]);

// Integral histogram: a pixel's 4 bin indicators packed as 8-bit lanes of one
// word (a tile row's prefix counts are <= 64), so the lane scan is ONE
// Kogge-Stone on u32 words; unpacked onto the u32 row carries at the end.
__device__ __forceinline__ uint32_t hist_pack(uint32_t a, const uint8_t* bin_of, int bin0) {
  const int b = (int)bin_of[a] - bin0;
  return (b >= 0 && b < 4) ? 1u << (8 * b) : 0u;
}

template <int RW>
__device__ __forceinline__ void rows_scan_hist4(const uint8_t* tile, int lane, const uint8_t* lut,
                                                int bin0, ChanVec<4> (&rowcarry)[RW],
                                                ChanVec<4> (&R)[RW][2][1]) {
  constexpr int TW = Cfg<P8UHIST4>::TW;  // 64: lane owns columns l and 32 + l
  uint32_t own[RW][2], inc[RW][2];
#pragma unroll
  for (int i = 0; i < RW; ++i)
#pragma unroll
    for (int g = 0; g < 2; ++g) inc[i][g] = own[i][g] = hist_pack(tile[i * TW + g * 32 + lane], lut, bin0);
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < 2; ++g) ks_step(inc[i][g], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    const uint32_t t0 = __shfl_sync(kFull, inc[i][0], 31), t1 = __shfl_sync(kFull, inc[i][1], 31);
    const uint32_t p0 = inc[i][0], p1 = t0 + inc[i][1];  // inclusive prefixes, packed (<= 64 each)
    const uint32_t tt = t0 + t1;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      R[i][0][0].c[k] = rowcarry[i].c[k] + ((p0 >> (8 * k)) & 0xffu);
      R[i][1][0].c[k] = rowcarry[i].c[k] + ((p1 >> (8 * k)) & 0xffu);
      rowcarry[i].c[k] += (tt >> (8 * k)) & 0xffu;
    }
  }
}

template <int P, int RW>
__device__ __forceinline__ void rows_scan_chan(const uint8_t* tile, int lane, const KParams& p,
                                               const uint8_t* lut,
                                               typename Cfg<P>::TB (&rowcarry)[RW],
                                               typename Cfg<P>::TB (&R)[RW][Cfg<P>::G][Cfg<P>::E]) {
  if constexpr (P == P8UHIST4) {
    rows_scan_hist4<RW>(tile, lane, lut, p.bin0, rowcarry, R);
  } else {
    rows_scan_xf<P, RW>(tile, lane, p, rowcarry, R);
  }
}

template <int P, int RW>
__device__ __forceinline__ void rows_scan_xf(const uint8_t* tile, int lane, const KParams& p,
                                             typename Cfg<P>::TB (&rowcarry)[RW],
                                             typename Cfg<P>::TB (&R)[RW][Cfg<P>::G][Cfg<P>::E]) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  TB inc[RW][C::G];  // R first holds the in-lane prefixes, then gets the bases added
#pragma unroll
  for (int i = 0; i < RW; ++i)
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      const uint32_t b = lane_bytes<C::E>(tile + i * C::TW, g * 32 * C::E + lane * C::E);
#pragma unroll
      for (int e = 0; e < C::E; ++e) {
        const TB v = Xf<P>::f((b >> (8 * e)) & 0xffu, p);
        R[i][g][e] = e == 0 ? v : R[i][g][e - 1] + v;
      }
      inc[i][g] = R[i][g][C::E - 1];
    }
  // a3 per channel with predicated-shuffle steps; the exclusive prefix is
  // inc - own (wrap-around u32, exact) instead of a further shuffle
#pragma unroll
  for (int d = 1; d < 32; d <<= 1)
#pragma unroll
    for (int i = 0; i < RW; ++i)
#pragma unroll
      for (int g = 0; g < C::G; ++g)
#pragma unroll
        for (int k = 0; k < C::K; ++k) ks_step(inc[i][g].c[k], d);
#pragma unroll
  for (int i = 0; i < RW; ++i) {
    TB base = rowcarry[i];
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      const TB tot = shfl_idx(inc[i][g], 31);
      TB ex;
#pragma unroll
      for (int k = 0; k < C::K; ++k) ex.c[k] = inc[i][g].c[k] - R[i][g][C::E - 1].c[k];
      const TB bx = base + ex;
#pragma unroll
      for (int e = 0; e < C::E; ++e) R[i][g][e] = bx + R[i][g][e];
      base += tot;
    }
    rowcarry[i] = base;
  }
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
struct Tag<P8U32F> : Tag<P32F32F> {};
template <>
struct Tag<P32S32S> : Tag<P8U32S> {};
// K-channel elements: a 16-byte group is 4 u32 words whatever K is.
template <int K, int E>
struct TagChan {
  static __device__ __forceinline__ void enc(const ChanVec<K> (&v)[E], uint32_t t, uint64_t (&w)[4]) {
    uint32_t u[4];
    memcpy(u, v, 16);
#pragma unroll
    for (int e = 0; e < 4; ++e) w[e] = ((uint64_t)t << 32) | u[e];
  }
  static __device__ __forceinline__ void dec(const uint64_t (&w)[4], ChanVec<K> (&v)[E]) {
    uint32_t u[4];
#pragma unroll
    for (int e = 0; e < 4; ++e) u[e] = (uint32_t)w[e];
    memcpy(v, u, 16);
  }
};
template <>
struct Tag<P8USQ> : TagChan<2, 2> {};
template <>
struct Tag<P8UHIST4> : TagChan<4, 1> {};
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



template <int P>
__device__ __forceinline__ uint64_t* payload_row(const KParams& p, int64_t T, int32_t chunk) {
  return reinterpret_cast<uint64_t*>(p.payload) + ((T * p.nchunks + chunk) * (int64_t)kVecWords<P>);
}

__device__ __forceinline__ uint64_t gclock() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// A bounded wait ran out: flag it (the host turns it into SAT_ERR_TIMEOUT).
__device__ __forceinline__ void flag_timeout(const KParams& p) {
  if (p.err) atomicOr(p.err, 1u);
}

// Status-tagged words: high 32 bits = (epoch << 2) | st, st = kStAgg or kStIncl.
// One vector per (cluster ticket, chunk): written first as the aggregate, then
// overwritten in place by the inclusive prefix.  A reader classifies a vector
// by its words' tags (all AGG, all INCL, or not ready / mixed -> re-read).
// Debug builds (-DSAT_DEBUG_DELAY) sleep a pseudo-random 0..~4 us before every
// carry publication, look-back round and DSMEM hand-off, so tests exercise
// late predecessors, mixed aggregate/inclusive windows and retries.
#ifdef SAT_DEBUG_DELAY
__device__ __forceinline__ void debug_delay(uint32_t salt) {
  uint32_t x = (uint32_t)clock64() ^ (salt * 0x9E3779B9u) ^ (blockIdx.x * 0x85EBCA6Bu);
  x ^= x >> 16;
  x *= 0x7FEB352Du;
  x ^= x >> 15;
  if ((x & 3u) == 0) __nanosleep((x >> 4) & 4095u);
}
#define SAT_DELAY(salt) debug_delay(salt)
#else
#define SAT_DELAY(salt)
#endif

template <int P>
__device__ __forceinline__ void publish(const KParams& p, uint64_t* row, uint32_t st,
                                        const typename Cfg<P>::TB (&v)[Cfg<P>::G][Cfg<P>::E],
                                        int lane) {
  using C = Cfg<P>;
  SAT_DELAY(st + 17u * (uint32_t)(uintptr_t)row);
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    uint64_t w[4];
    Tag<kBase<P>>::enc(v[g], (p.epoch << 2) | st, w);
    uint64_t* dst = row + (g * 32 + lane) * 4;
    st_relaxed_v2_u64(dst, w[0], w[1]);
    st_relaxed_v2_u64(dst + 2, w[2], w[3]);
  }
}

// One bulk (TMA) copy global -> shared, completing `bytes` tx on a local mbarrier.
// Bulk copies run on the TMA engine, not in the SM's LSU queue behind the
// compute warps' output stores.
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

// Decoupled look-back up the tile column over cluster tickets:
// V = sum of the predecessors' aggregates down to (and including) the nearest
// inclusive prefix.  Each round lands up to kLandVecs predecessor vectors in shared
// memory with bulk copies (one per vector, on the TMA engine): one L2 round
// trip per round, no separate status probe.  Vectors are classified by warp
// votes on the word tags (each lane checks its own words).
template <int P, class SM>
__device__ __forceinline__ void lookback(SM& sm, uint64_t (&land)[kLandVecs<P>][kVecWords<P>],
                                         uint64_t* land_bar, uint32_t& land_ph, const KParams& p,
                                         int64_t T, int64_t first, int32_t chunk,
                                         typename Cfg<P>::TB (&V)[Cfg<P>::G][Cfg<P>::E],
                                         int lane) {
  constexpr uint32_t kVecBytes = kVecWords<P> * 8;
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int B = kLandVecs<P>;
  const uint32_t tag_agg = (p.epoch << 2) | kStAgg, tag_incl = (p.epoch << 2) | kStIncl;
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) V[g][e] = TB(0);
  int64_t j = T - 1;
  uint64_t t_start = 0;
#if SAT_LB_LDG
  uint64_t wl[B][C::G][4];
#define LBW(b, g, e) wl[b][g][e]
#else
#define LBW(b, g, e) land[b][((g) * 32 + lane) * 4 + (e)]
#endif
  for (;;) {
    const int nb = (j - first + 1) < B ? (int)(j - first + 1) : B;
    int kk = nb;  // index of the inclusive vector in this round (nb: none)
    for (;;) {
      __syncwarp();  // every lane is done reading the previous round's landing zone
      SAT_DELAY(31u + (uint32_t)j);
      SAT_PT(i0);
#if SAT_LB_LDG
      // every lane loads its own words of the round's vectors straight into
      // registers (relaxed 16-byte loads: each 8-byte word single-copy atomic)
#pragma unroll
      for (int b = 0; b < B; ++b)
        if (b < nb)
#pragma unroll
          for (int g = 0; g < C::G; ++g) {
            const uint64_t* src = payload_row<P>(p, j - b, chunk) + (g * 32 + lane) * 4;
            ld_relaxed_v2_u64(src, wl[b][g][0], wl[b][g][1]);
            ld_relaxed_v2_u64(src + 2, wl[b][g][2], wl[b][g][3]);
          }
      SAT_PT(r0);
      SAT_PT(r1);
#else
      // lane b fetches vector b (parallel issue); lane 0 arms the barrier.  The
      // previous round's generic reads of the landing zone were consumed before
      // the __syncwarp above, so the async-proxy overwrite cannot overtake them.
      if (lane == 0) mbar_arrive_expect_tx(land_bar, nb * kVecBytes);
      if (lane < nb) bulk_g2s(&land[lane][0], payload_row<P>(p, j - lane, chunk), kVecBytes, land_bar);
      SAT_PT(r0);
      SAT_PADD(sm, kPfLbIssue, r0 - i0);
      mbar_wait(land_bar, land_ph);
      SAT_PT(r1);
      land_ph ^= 1u;
#endif
      SAT_PADD(sm, kPfLbRoundTime, r1 - r0);
      SAT_PADD(sm, kPfLbRounds, 1);
      bool ready = true;
      kk = nb;
      for (int b = 0; b < nb; ++b) {
        bool all_incl = true, all_agg = true;
#pragma unroll
        for (int g = 0; g < C::G; ++g)
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const uint32_t tg = (uint32_t)(LBW(b, g, e) >> 32);
            all_incl &= tg == tag_incl;
            all_agg &= tg == tag_agg;
          }
        if (__all_sync(kFull, all_incl)) {
          kk = b;
          break;
        }
        if (!__all_sync(kFull, all_agg)) {
          ready = false;  // predecessor not published yet (or mid-overwrite)
          break;
        }
      }
#ifdef SAT_TIMELINE
      if (lane == 0 && blockIdx.x < 1024 && chunk < kTlChunks) {
        g_sat_tl_rounds[blockIdx.x][chunk][0]++;
        if (!ready) g_sat_tl_rounds[blockIdx.x][chunk][1]++;
      }
#endif
      if (ready) break;
      SAT_PADD(sm, kPfLbRetries, 1);
      if (t_start == 0) t_start = gclock();
      if (gclock() - t_start > p.spin_ns) {  // bounded wait: flag, go on with what is summed
        if (lane == 0) flag_timeout(p);
        return;
      }
#ifndef SAT_LB_SLEEP
#define SAT_LB_SLEEP 32
#endif
      if (SAT_LB_SLEEP > 0) __nanosleep(SAT_LB_SLEEP);
    }
    const int nsum = kk < nb ? kk + 1 : nb;
    SAT_PADD(sm, kPfLbDepth, nsum);
    for (int b = 0; b < nsum; ++b)
#pragma unroll
      for (int g = 0; g < C::G; ++g) {
        uint64_t w[4];
#pragma unroll
        for (int e = 0; e < 4; ++e) w[e] = LBW(b, g, e);
        TB t[C::E];
        Tag<kBase<P>>::dec(w, t);
#pragma unroll
        for (int e = 0; e < C::E; ++e) V[g][e] += t[e];
      }
    if (kk < nb) break;
    j -= nb;
  }
#undef LBW
}

// ---------------------------------------------------------------------------
// Counted reduction tree (kFen pairs).  Image n is covered by the cluster
// tickets T0(n) .. T1(n) (D(n) = T1 - T0 + 1 of them); cluster T0 + u
// (u <= D - 2) contributes c_u = the column totals of its bands in image n
// (its tail segment, plus the image's carry-in row where the segment starts
// the image).  The carry of cluster T0 + t is the exclusive prefix
// sum_{u < t} c_u = sum of the Fenwick nodes t, t - lowbit(t), ... (> 0);
// node i (1 <= i <= D - 1) sums c_u for u in [i - lowbit(i), i), so it is complete
// when its words count lowbit(i) contributions.  Node i of image n, chunk q
// lives in the payload at vector (T0(n) + i - 1, q); its readers are the
// clusters t in [i, min(i + lowbit(i), D)), and the last of them (read
// counter) zeroes it again, so every launch finds the tree zeroed.
template <int CL>
__device__ __forceinline__ int64_t img_first_ticket(const KParams& p, int64_t n) {
  return (n * p.bands_per_image) / CL;
}
template <int CL>
__device__ __forceinline__ int64_t img_tickets(const KParams& p, int64_t n) {
  return ((n + 1) * p.bands_per_image - 1) / CL - (n * p.bands_per_image) / CL + 1;
}
__device__ __forceinline__ int64_t lowbit(int64_t i) { return i & -i; }

__device__ __forceinline__ void bulk_red_add_u64(void* gdst, const void* ssrc, uint32_t bytes) {
  asm volatile("cp.reduce.async.bulk.global.shared::cta.bulk_group.add.u64 [%0], [%1], %2;" ::"l"(gdst),
               "r"(smem_u32(ssrc)), "r"(bytes)
               : "memory");
}

// Add cluster t's contribution c (image n with D clusters, chunk q) to the
// nodes t + 1, then i + lowbit(i), ... (< D): one bulk reduction per node,
// issued by lane k for the k-th node, from a staged copy in shared memory.
template <int P, int CL, class SM>
__device__ __forceinline__ void tree_update(SM& sm, const KParams& p, int lbw, int64_t n, int64_t t,
                                            int64_t D, int32_t chunk,
                                            const typename Cfg<P>::TB (&c)[Cfg<P>::G][Cfg<P>::E],
                                            int lane) {
  using C = Cfg<P>;
  constexpr uint32_t kVecBytes = kVecWords<P> * 8;
  uint64_t* st = sm.fstage[lbw];
  SAT_DELAY(101u + (uint32_t)t);
  // the previous update's reductions have read the staged vector
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  __syncwarp();
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    const uint4 u = pack16<typename C::TB, C::E>(c[g]);
    uint64_t* d = st + (g * 32 + lane) * 4;
    d[0] = kFenOne | u.x;
    d[1] = kFenOne | u.y;
    d[2] = kFenOne | u.z;
    d[3] = kFenOne | u.w;
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic writes -> async proxy
  __syncwarp();
  const int64_t base = img_first_ticket<CL>(p, n) - 1;
  int k = 0;
  for (int64_t i = t + 1; i <= D - 1; i += lowbit(i), ++k) {
    if (k == lane) {
      bulk_red_add_u64(payload_row<P>(p, base + i, chunk), st, kVecBytes);
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    }
  }
}

// Read counters of the nodes a query summed: every reader adds one; the last
// reader zeroes the node and its counter.  The counter adds are issued in
// tree_query; tree_release (called after the V_up hand-offs) consumes their
// results, so their round trip is off the critical path.
struct TreeRel {
  uint32_t old;    // this lane's counter value before its add (lane < nodes)
  int64_t node;    // this lane's node (payload vector index), -1: none
  uint32_t readers;
};

template <int P>
__device__ __forceinline__ void tree_release(const KParams& p, int32_t chunk, const TreeRel& r,
                                             int lane) {
  using C = Cfg<P>;
  const bool last = r.node >= 0 && r.old + 1 == r.readers;
  uint32_t m = __ballot_sync(kFull, last);
  while (m) {
    const int k = __ffs(m) - 1;
    m &= m - 1;
    const int64_t node = __shfl_sync(kFull, r.node, k);
    uint64_t* row = payload_row<P>(p, node, chunk);
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      uint64_t* d = row + (g * 32 + lane) * 4;
      st_relaxed_v2_u64(d, 0ull, 0ull);
      st_relaxed_v2_u64(d + 2, 0ull, 0ull);
    }
    if (lane == k) p.tree_rd[node * p.nchunks + chunk] = 0u;
  }
}

// V = sum of the nodes t, t - lowbit(t), ... of image n's tree (chunk q), each
// once it is complete.  Rounds land up to kLandVecs nodes (bulk copies);
// incomplete nodes are re-read.  Returns the last round's read-counter state.
template <int P, int CL, class SM>
__device__ __forceinline__ TreeRel tree_query(SM& sm, uint64_t (&land)[kLandVecs<P>][kVecWords<P>],
                                              uint64_t* land_bar, uint32_t& land_ph,
                                              const KParams& p, int64_t n, int64_t t, int64_t D,
                                              int32_t chunk,
                                              typename Cfg<P>::TB (&V)[Cfg<P>::G][Cfg<P>::E],
                                              int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr uint32_t kVecBytes = kVecWords<P> * 8;
  constexpr int B = kLandVecs<P>;
  uint32_t acc[C::G][4];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < 4; ++e) acc[g][e] = 0u;
  const int64_t base = img_first_ticket<CL>(p, n) - 1;
  TreeRel rel{0u, -1, 0u};
  int64_t i = t;
  while (i > 0) {
    // this round's nodes: lane k < nn owns node k of the round
    int nn = 0;
    int64_t mine = -1, ii = i;
    for (; nn < B && ii > 0; ++nn, ii -= lowbit(ii))
      if (nn == lane) mine = ii;
    uint32_t pending = (1u << nn) - 1u;
    uint64_t t_start = 0;
    while (pending) {
      __syncwarp();  // every lane is done reading the previous round's landing zone
      SAT_DELAY(131u + (uint32_t)i);
#if SAT_LB_LDG
      // debug variant: per-lane relaxed loads of every pending node, one at a time
      for (int k = 0; k < nn; ++k) {
        if (!(pending >> k & 1u)) continue;
        const int64_t nk = __shfl_sync(kFull, mine, k);
        const uint64_t* src = payload_row<P>(p, base + nk, chunk);
        uint64_t w[C::G][4];
        bool ok = true;
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
          ld_relaxed_v2_u64(src + (g * 32 + lane) * 4, w[g][0], w[g][1]);
          ld_relaxed_v2_u64(src + (g * 32 + lane) * 4 + 2, w[g][2], w[g][3]);
#pragma unroll
          for (int e = 0; e < 4; ++e) ok &= (w[g][e] >> 48) == (uint64_t)lowbit(nk);
        }
        if (__all_sync(kFull, ok)) {
#pragma unroll
          for (int g = 0; g < C::G; ++g)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[g][e] += (uint32_t)w[g][e];
          pending &= ~(1u << k);
        }
      }
#else
      if (lane == 0) mbar_arrive_expect_tx(land_bar, __popc(pending) * kVecBytes);
      if (mine > 0 && (pending >> lane & 1u))
        bulk_g2s(&land[lane][0], payload_row<P>(p, base + mine, chunk), kVecBytes, land_bar);
      mbar_wait(land_bar, land_ph);
      land_ph ^= 1u;
      for (int k = 0; k < nn; ++k) {
        if (!(pending >> k & 1u)) continue;
        const uint64_t want = (uint64_t)lowbit(__shfl_sync(kFull, mine, k));
        bool ok = true;
#pragma unroll
        for (int g = 0; g < C::G; ++g)
#pragma unroll
          for (int e = 0; e < 4; ++e) ok &= (land[k][(g * 32 + lane) * 4 + e] >> 48) == want;
        if (__all_sync(kFull, ok)) {
#pragma unroll
          for (int g = 0; g < C::G; ++g)
#pragma unroll
            for (int e = 0; e < 4; ++e) acc[g][e] += (uint32_t)land[k][(g * 32 + lane) * 4 + e];
          pending &= ~(1u << k);
        }
      }
#endif
      if (pending) {
        if (t_start == 0) t_start = gclock();
        if (gclock() - t_start > p.spin_ns) {  // bounded wait: flag, go on with what is summed
          if (lane == 0) flag_timeout(p);
          pending = 0;
          mine = -1;  // a node left incomplete is not released (the host clears the tree)
        } else {
          __nanosleep(32);
        }
      }
    }
    // the previous round's counters (more than B nodes: long images only)
    tree_release<P>(p, chunk, rel, lane);
    rel.node = mine > 0 ? base + mine : -1;
    rel.readers = mine > 0 ? (uint32_t)min(lowbit(mine), D - mine) : 0u;
    rel.old = mine > 0 ? atomicAdd(&p.tree_rd[rel.node * p.nchunks + chunk], 1u) : 0u;
    i = ii;
  }
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    uint4 u = make_uint4(acc[g][0], acc[g][1], acc[g][2], acc[g][3]);
    unpack16<TB, C::E>(u, V[g]);
  }
  return rel;
}

// Chained-band carry vectors: system-scope relaxed 64-bit accesses (peer GPU
// memory over NVLink keeps aligned 8-byte stores single-copy atomic, so a word
// with the expected tag also holds its value).
__device__ __forceinline__ void st_sys_v2_u64(uint64_t* q, uint64_t a, uint64_t b) {
  asm volatile("st.relaxed.sys.global.v2.u64 [%0], {%1, %2};" ::"l"(q), "l"(a), "l"(b) : "memory");
}
__device__ __forceinline__ void ld_sys_v2_u64(const uint64_t* q, uint64_t& a, uint64_t& b) {
  asm volatile("ld.relaxed.sys.global.v2.u64 {%0, %1}, [%2];" : "=l"(a), "=l"(b) : "l"(q) : "memory");
}

template <int P>
__device__ __forceinline__ void chain_publish(const KParams& p, int32_t chunk,
                                              const typename Cfg<P>::TB (&v)[Cfg<P>::G][Cfg<P>::E],
                                              int lane) {
  using C = Cfg<P>;
  uint64_t* row = p.chain_out + (int64_t)chunk * kVecWords<P>;
  // The slot was last used by epoch e - 2: wait until the band below consumed it.
  if (p.chain_ack_in != nullptr && p.chain_epoch > 2) {
    const uint32_t need = p.chain_epoch - 2;
    const uint64_t t_start = gclock();
    for (;;) {
      uint32_t a = 0;
      if (lane == 0)
        asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(a) : "l"(p.chain_ack_in + chunk) : "memory");
      a = __shfl_sync(kFull, a, 0);
      if ((int32_t)(a - need) >= 0) break;
      if (gclock() - t_start > p.spin_ns) {
        if (lane == 0) flag_timeout(p);
        break;
      }
      __nanosleep(64);
    }
  }
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    uint64_t w[4];
    Tag<kBase<P>>::enc(v[g], (p.chain_epoch << 2) | kStIncl, w);
    uint64_t* dst = row + (g * 32 + lane) * 4;
    st_sys_v2_u64(dst, w[0], w[1]);
    st_sys_v2_u64(dst + 2, w[2], w[3]);
  }
}

template <int P>
__device__ __forceinline__ void chain_wait(const KParams& p, int32_t chunk,
                                           typename Cfg<P>::TB (&V)[Cfg<P>::G][Cfg<P>::E], int lane) {
  using C = Cfg<P>;
  const uint64_t* row = p.chain_in + (int64_t)chunk * kVecWords<P>;
  const uint32_t want = (p.chain_epoch << 2) | kStIncl;
  const uint64_t t_start = gclock();
  for (;;) {
    bool ok = true;
    uint64_t w[C::G][4];
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      const uint64_t* src = row + (g * 32 + lane) * 4;
      ld_sys_v2_u64(src, w[g][0], w[g][1]);
      ld_sys_v2_u64(src + 2, w[g][2], w[g][3]);
#pragma unroll
      for (int e = 0; e < 4; ++e) ok &= (uint32_t)(w[g][e] >> 32) == want;
    }
    if (__all_sync(kFull, ok)) {
#pragma unroll
      for (int g = 0; g < C::G; ++g) Tag<kBase<P>>::dec(w[g], V[g]);
      // every lane holds its words: release the slot to the band above
      if (lane == 0 && p.chain_ack_out != nullptr)
        asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(p.chain_ack_out + chunk),
                     "r"(p.chain_epoch)
                     : "memory");
      return;
    }
    if (gclock() - t_start > p.spin_ns) {  // the band above never published: zeros, flag
      if (lane == 0) flag_timeout(p);
#pragma unroll
      for (int g = 0; g < C::G; ++g)
#pragma unroll
        for (int e = 0; e < C::E; ++e) V[g][e] = typename C::TB(0);
      return;
    }
    __nanosleep(64);
  }
}

template <int P>
__device__ __forceinline__ void load_carry_in(const KParams& p, int32_t chunk,
                                              typename Cfg<P>::TB (&V)[Cfg<P>::G][Cfg<P>::E],
                                              int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) {
      const int64_t x = (int64_t)chunk * C::TW + col_of<P>(g, lane) + e;
      V[g][e] = (p.carry_in != nullptr && x < p.W) ? reinterpret_cast<const TB*>(p.carry_in)[x]
                                                   : TB(0);
    }
}

// Leader CTA, chunk q (V_up slot v, gather slot ls, whose CL band aggregates
// have landed): publish / look back for the cluster, publish its inclusive
// prefix, and send every band of the cluster its V_up (segmented at image
// starts inside the cluster).
template <int P, int CL>
__device__ __forceinline__ void leader_chunk(Smem<P, CL>& sm, const KParams& p, int lbw,
                                             uint32_t& land_ph, int v, int ls, int64_t g0,
                                             int32_t chunk, uint32_t qdbg, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  const int32_t n0 = (int32_t)(g0 / p.bands_per_image);
  const int32_t k0 = (int32_t)(g0 - (int64_t)n0 * p.bands_per_image);
  SAT_PADD(sm, kPfLeaderChunks, 1);
  const int64_t T = g0 / CL;
  const int64_t bpi = p.bands_per_image;
  // Pass 1: the tail segment (bands of the cluster's last image) and its sum.
  TB tail[C::G][C::E];
  bool tail_self = (k0 == 0);
  int64_t tail_last_k = k0;
  {
    int64_t k = k0;
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) tail[g][e] = TB(0);
    for (int r = 0; r < CL; ++r) {
      if (g0 + r >= p.total_bands) break;
      if (r > 0 && k == 0) {
        tail_self = true;
#pragma unroll
        for (int g = 0; g < C::G; ++g)
#pragma unroll
          for (int e = 0; e < C::E; ++e) tail[g][e] = TB(0);
      }
#pragma unroll
      for (int g = 0; g < C::G; ++g) {
        TB a[C::E];
        unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.lead_in[ls][r][col_of<P>(g, lane)]), a);
#pragma unroll
        for (int e = 0; e < C::E; ++e) tail[g][e] += a[e];
      }
      tail_last_k = k;
      if (++k == bpi) k = 0;
    }
  }
  const bool has_succ = tail_last_k + 1 < bpi;
  const bool head_self = (k0 == 0);
  TB carry0[C::G][C::E];
  if (p.chain_in != nullptr && (head_self || tail_self))
    chain_wait<P>(p, chunk, carry0, lane);  // the band above publishes it chunk by chunk
  else
    load_carry_in<P>(p, chunk, carry0, lane);
  // The cluster's contribution to its tail image goes out first -- the clusters
  // below need it -- then, as a reader of its head image, the look-back.
  TB contrib[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) contrib[g][e] = tail_self ? carry0[g][e] + tail[g][e] : tail[g][e];
  TB Vcl[C::G][C::E];
  TreeRel rel{0u, -1, 0u};
  if (kFen<P> && p.tree) {
    // Counted reduction tree: contribute to the tail image's tree, then (as a
    // reader of the head image) sum this cluster's prefix nodes.
    if (has_succ) {
      const int64_t g_last = (g0 + CL < p.total_bands ? g0 + CL : p.total_bands) - 1;
      const int64_t nt = g_last / bpi;
      tree_update<P, CL>(sm, p, lbw, nt, T - img_first_ticket<CL>(p, nt), img_tickets<CL>(p, nt),
                         chunk, contrib, lane);
    }
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) Vcl[g][e] = TB(0);
    if (!head_self) {
      SAT_PT(t2);
      rel = tree_query<P, CL>(sm, sm.land[lbw], &sm.land_full[lbw], land_ph, p, n0,
                              T - img_first_ticket<CL>(p, n0), img_tickets<CL>(p, n0), chunk, Vcl,
                              lane);
      SAT_PT(t3);
      SAT_PADD(sm, kPfLbLookback, t3 - t2);
    }
  } else {
  // aggregate, or -- when the tail segment starts its image -- already inclusive
  if (has_succ)
    publish<P>(p, payload_row<P>(p, T, chunk), tail_self ? kStIncl : kStAgg, contrib, lane);
#ifdef SAT_DEBUG_NO_LOOKBACK  // timing experiments only: wrong results, no cross-cluster wait
#pragma unroll
  for (int g = 0; g < C::G; ++g)
#pragma unroll
    for (int e = 0; e < C::E; ++e) Vcl[g][e] = TB(0);
  if (false) {
#else
  if (!head_self) {
#endif
    SAT_PT(t2);
    const int64_t T0 = ((int64_t)n0 * bpi) / CL;  // first cluster of the head image
    lookback<P>(sm, sm.land[lbw], &sm.land_full[lbw], land_ph, p, T, T0, chunk, Vcl, lane);
    if (has_succ && !tail_self) {  // the cluster's inclusive prefix (overwrites its aggregate)
      TB incl[C::G][C::E];
#pragma unroll
      for (int g = 0; g < C::G; ++g)
#pragma unroll
        for (int e = 0; e < C::E; ++e) incl[g][e] = Vcl[g][e] + tail[g][e];
      publish<P>(p, payload_row<P>(p, T, chunk), kStIncl, incl, lane);
    }
    SAT_PT(t3);
    SAT_PADD(sm, kPfLbLookback, t3 - t2);
  }
  }
#ifdef SAT_TIMELINE
  if (lane == 0 && blockIdx.x < 1024 && qdbg < kTlChunks) g_sat_tl_lt[blockIdx.x][qdbg] = tl_now();
#endif
  // Pass 2: V_up of every band of the cluster (padding CTAs get zeros).
  {
    const uint32_t self = CL > 1 ? cluster_rank() : 0u;
    TB run[C::G][C::E];
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) run[g][e] = head_self ? carry0[g][e] : Vcl[g][e];
    int64_t k = k0;
    for (int r = 0; r < CL; ++r) {
      const bool valid = g0 + r < p.total_bands;
      if (valid && r > 0 && k == 0) {
#pragma unroll
        for (int g = 0; g < C::G; ++g)
#pragma unroll
          for (int e = 0; e < C::E; ++e) run[g][e] = carry0[g][e];
      }
#pragma unroll
      for (int g = 0; g < C::G; ++g) {
        TB vv[C::E], a[C::E];
        // read this band's aggregate BEFORE sending it its V_up: once CTA r has
        // its V_up it may eventually overwrite lead_in[ls][r] for a later chunk
        unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.lead_in[ls][r][col_of<P>(g, lane)]),
                           a);
#pragma unroll
        for (int e = 0; e < C::E; ++e) {
          vv[e] = valid ? run[g][e] : TB(0);
          if (valid) run[g][e] += a[e];
        }
        send16(&sm.vin[v][col_of<P>(g, lane)], &sm.vin_full[v], (uint32_t)r, self, pack16<TB, C::E>(vv));
      }
      if ((uint32_t)r == self) {
        __syncwarp();
        if (lane == 0) mbar_arrive(&sm.vin_full[v]);
      }
      if (++k == bpi) k = 0;
    }
    // The image's bottom row S(r1-1, .) = the tail segment's inclusive value.
    if (!has_succ && p.chain_out != nullptr) chain_publish<P>(p, chunk, run, lane);
  }
  if (kFen<P> && p.tree) tree_release<P>(p, chunk, rel, lane);
}

template <typename TB>
__device__ __forceinline__ TB from_bits(uint64_t b) {
  TB v;
  memcpy(&v, &b, sizeof(TB));
  return v;
}

// Offset step (chunk q, its column totals and V_up landed): block partial-sum
// scan (Fig. 3c) over the compute warps' column totals, started
// from the band's V_up (and the exclusive layout's nVal) -> each compute
// warp's complete fix-up offset, in place.  One warp per CTA waits for V_up
// (cluster-scope acquire); the compute warps wait only for its local arrival.
template <int P, int CL, bool kEx>
__device__ __forceinline__ void offset_step(Smem<P, CL>& sm, const KParams& p, uint32_t q,
                                            int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  const int t = q % kNTot<P>;
  const int vs = q % kNV<P>;
#ifdef SAT_TIMELINE
  if (lane == 0 && blockIdx.x < 1024 && q < kTlChunks) g_sat_tl_v[blockIdx.x][q] = tl_now();
#endif
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    TB run[C::E];
    unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.vin[vs][col_of<P>(g, lane)]), run);
    if constexpr (kEx) {
#pragma unroll
      for (int e = 0; e < C::E; ++e) run[e] += from_bits<TB>(p.nval_bits);
    }
#pragma unroll
    for (int w = 0; w < kNCW<P>; ++w) {
      uint4* cell = reinterpret_cast<uint4*>(&sm.tot[t][w][col_of<P>(g, lane)]);
      TB tt[C::E];
      unpack16<TB, C::E>(*cell, tt);
      *cell = pack16<TB, C::E>(run);
#pragma unroll
      for (int e = 0; e < C::E; ++e) run[e] += tt[e];
    }
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.carry_full[t]);
}

// Leader warp lw: the chunks this CTA leads, q = rank + CL * j for
// j = lw (mod kNLW), each as soon as the cluster's aggregates have landed.
template <int P, int CL>
__device__ __forceinline__ void leader_warp(Smem<P, CL>& sm, const KParams& p, int lw,
                                            uint32_t rank, int lane) {
  uint32_t land_ph = 0;
  for (uint32_t j = lw;; j += kNLW<P>) {
    const int ls = j % kNLead<P, CL>;
    SAT_PT(t0);
    mbar_wait_peer_data(&sm.lead_full[ls], (j / kNLead<P, CL>) & 1);
    SAT_PT(t1);
    SAT_PADD(sm, kPfLbCluster, t1 - t0);
    const int64_t band = sm.lead_band[ls];
    if (band < 0) break;
    SAT_PADD(sm, kPfLbChunks, 1);
    const uint32_t q = rank + CL * j;
#ifdef SAT_TIMELINE
    if (lane == 0 && blockIdx.x < 1024 && q < kTlChunks) g_sat_tl_ls[blockIdx.x][q] = tl_now();
#endif
    leader_chunk<P, CL>(sm, p, lw, land_ph, (int)(q % kNV<P>), ls, band - rank, sm.lead_chunk[ls],
                        q, lane);
#ifdef SAT_TIMELINE
    if (lane == 0 && blockIdx.x < 1024 && q < kTlChunks) g_sat_tl_ld[blockIdx.x][q] = tl_now();
#endif
  }
  // the last node stores / tree reductions must have read their staging buffer
  // before the CTA exits
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  __syncwarp();
}

// Aggregate warp helpers: the band's vertical aggregate of a landed tile,
//   agg(x) = L + sum_{x0 <= x' <= x} colsum(x'),  colsum(x') = sum_{y in band} A(y, x'),
// L = the band's input left of the chunk (= sum_y rowcarry(y)); this equals
// sum_y R(y, x), the column total of the row-prefixed values (Sec. 5).
// 8u: column sums of bytes in packed 16-bit lanes (<= TH * 255 < 2^16), then
// the in-lane prefix and a Kogge-Stone scan of the lane totals (Alg. 2, 3).
template <int TH>
__device__ __forceinline__ void colsum8(const uint8_t* tile, int lane, uint32_t (&c)[2][4]) {
  uint32_t lo[2] = {0u, 0u}, hi[2] = {0u, 0u};
#pragma unroll 8
  for (int r = 0; r < TH; ++r) {
#pragma unroll
    for (int g = 0; g < 2; ++g) {
      const uint32_t w = *reinterpret_cast<const uint32_t*>(tile + r * 256 + g * 128 + 4 * lane);
      lo[g] += __byte_perm(w, 0u, 0x4240);  // bytes 0, 2 -> 16-bit lanes
      hi[g] += __byte_perm(w, 0u, 0x4341);  // bytes 1, 3
    }
  }
#pragma unroll
  for (int g = 0; g < 2; ++g) {
    c[g][0] = lo[g] & 0xFFFFu;
    c[g][1] = hi[g] & 0xFFFFu;
    c[g][2] = lo[g] >> 16;
    c[g][3] = hi[g] >> 16;
  }
}

template <typename T>
__device__ __forceinline__ T warp_incl(T v, int lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    if constexpr (std::is_same<T, uint32_t>::value || std::is_same<T, float>::value) {
      ks_step(v, d);
    } else {
      T o;
      if constexpr (IsChan<T>::value)
        o = shfl_up(v, d);
      else
        o = __shfl_up_sync(kFull, v, d);
      if (lane >= d) v += o;
    }
  }
  return v;
}

// Per-pair aggregate of one tile; `L` is the running band-left sum (reset at chunk 0).
template <int P>
struct Agg;
template <>
struct Agg<P8U32S> {
  using Acc = uint32_t;
  template <int TH>
  static __device__ __forceinline__ void run(const uint8_t* tile, int lane, Acc& L,
                                             uint32_t (&agg)[2][4]) {
    uint32_t c[2][4];
    colsum8<TH>(tile, lane, c);
    uint32_t pg[2][4], inc[2];
#pragma unroll
    for (int g = 0; g < 2; ++g) {
      pg[g][0] = c[g][0];
#pragma unroll
      for (int e = 1; e < 4; ++e) pg[g][e] = pg[g][e - 1] + c[g][e];
      inc[g] = warp_incl(pg[g][3], lane);
    }
    const uint32_t tot0 = __shfl_sync(kFull, inc[0], 31), tot1 = __shfl_sync(kFull, inc[1], 31);
    const uint32_t b0 = L + (inc[0] - pg[0][3]), b1 = L + tot0 + (inc[1] - pg[1][3]);
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      agg[0][e] = b0 + pg[0][e];
      agg[1][e] = b1 + pg[1][e];
    }
    L += tot0 + tot1;
  }
};
template <>
struct Agg<P8U32F> {
  using Acc = uint64_t;  // exact integer sums, rounded once to fp32
  template <int TH>
  static __device__ __forceinline__ void run(const uint8_t* tile, int lane, Acc& L,
                                             float (&agg)[2][4]) {
    uint32_t c[2][4];
    colsum8<TH>(tile, lane, c);
    uint32_t pg[2][4], inc[2];
#pragma unroll
    for (int g = 0; g < 2; ++g) {
      pg[g][0] = c[g][0];
#pragma unroll
      for (int e = 1; e < 4; ++e) pg[g][e] = pg[g][e - 1] + c[g][e];
      inc[g] = warp_incl(pg[g][3], lane);
    }
    const uint32_t tot0 = __shfl_sync(kFull, inc[0], 31), tot1 = __shfl_sync(kFull, inc[1], 31);
    const uint32_t b0 = inc[0] - pg[0][3], b1 = tot0 + (inc[1] - pg[1][3]);
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      agg[0][e] = (float)(L + (uint64_t)(b0 + pg[0][e]));
      agg[1][e] = (float)(L + (uint64_t)(b1 + pg[1][e]));
    }
    L += (uint64_t)tot0 + tot1;
  }
};
template <typename T>
struct AggWide {  // 4-byte elements, 128-column tiles: lane owns columns 4l .. 4l+3
  using Acc = T;
  template <int TH>
  static __device__ __forceinline__ void run(const T* tile, int lane, Acc& L, T (&agg)[1][4]) {
    T c[4] = {T(0), T(0), T(0), T(0)};
#pragma unroll 8
    for (int r = 0; r < TH; ++r) {
      const uint4 w = *reinterpret_cast<const uint4*>(tile + r * 128 + 4 * lane);
      T a[4];
      unpack16<T, 4>(w, a);
#pragma unroll
      for (int e = 0; e < 4; ++e) c[e] += a[e];
    }
    T pg[4];
    pg[0] = c[0];
#pragma unroll
    for (int e = 1; e < 4; ++e) pg[e] = pg[e - 1] + c[e];
    const T inc = warp_incl(pg[3], lane);
    const T tot = __shfl_sync(kFull, inc, 31);
    T ex = __shfl_up_sync(kFull, inc, 1);
    if (lane == 0) ex = T(0);
    const T b = L + ex;
#pragma unroll
    for (int e = 0; e < 4; ++e) agg[0][e] = b + pg[e];
    L += tot;
  }
};
template <>
struct Agg<P32F32F> : AggWide<float> {};
template <>
struct Agg<P32S32S> : AggWide<uint32_t> {};
template <>
struct Agg<P64F64F> {
  using Acc = double;
  template <int TH>
  static __device__ __forceinline__ void run(const double* tile, int lane, Acc& L,
                                             double (&agg)[1][2]) {
    double c0 = 0.0, c1 = 0.0;
#pragma unroll 8
    for (int r = 0; r < TH; ++r) {
      const double2 a = *reinterpret_cast<const double2*>(tile + r * 64 + 2 * lane);
      c0 += a.x;
      c1 += a.y;
    }
    const double p1 = c0 + c1;
    const double inc = warp_incl(p1, lane);
    const double tot = __shfl_sync(kFull, inc, 31);
    double ex = __shfl_up_sync(kFull, inc, 1);
    if (lane == 0) ex = 0.0;
    const double b = L + ex;
    agg[0][0] = b + c0;
    agg[0][1] = b + p1;
    L += tot;
  }
};

template <int P>
struct AggChan {
  using TB = typename Cfg<P>::TB;
  using Acc = TB;
  template <int TH>
  static __device__ __forceinline__ void run(const uint8_t* tile, int lane, Acc& L,
                                             TB (&agg)[Cfg<P>::G][Cfg<P>::E], const KParams& p,
                                             const uint8_t* lut) {
    using C = Cfg<P>;
    TB c[C::G][C::E];
    if constexpr (P == P8UHIST4) {  // column counts <= TH < 256: packed 8-bit lanes
      static_assert(TH < 256, "packed histogram column counts");
      uint32_t pk[2] = {0u, 0u};
#pragma unroll 8
      for (int r = 0; r < TH; ++r)
#pragma unroll
        for (int g = 0; g < 2; ++g) pk[g] += hist_pack(tile[r * C::TW + g * 32 + lane], lut, p.bin0);
#pragma unroll
      for (int g = 0; g < 2; ++g)
#pragma unroll
        for (int k = 0; k < 4; ++k) c[g][0].c[k] = (pk[g] >> (8 * k)) & 0xffu;
    } else {
#pragma unroll
      for (int g = 0; g < C::G; ++g)
#pragma unroll
        for (int e = 0; e < C::E; ++e) c[g][e] = TB(0);
#pragma unroll 4
      for (int r = 0; r < TH; ++r)
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
          const uint32_t b = lane_bytes<C::E>(tile + r * C::TW, g * 32 * C::E + lane * C::E);
#pragma unroll
          for (int e = 0; e < C::E; ++e) c[g][e] += Xf<P>::f((b >> (8 * e)) & 0xffu, p);
        }
    }
    TB base = L;
#pragma unroll
    for (int g = 0; g < C::G; ++g) {
      TB pg[C::E];
#pragma unroll
      for (int e = 0; e < C::E; ++e) pg[e] = e == 0 ? c[g][0] : pg[e - 1] + c[g][e];
      const TB inc = warp_incl(pg[C::E - 1], lane);
      const TB tot = shfl_idx(inc, 31);
      TB ex = shfl_up(inc, 1);
      if (lane == 0) ex = TB(0);
#pragma unroll
      for (int e = 0; e < C::E; ++e) agg[g][e] = (base + ex) + pg[e];
      base += tot;
    }
    L = base;
  }
};
template <>
struct Agg<P8USQ> : AggChan<P8USQ> {};
template <>
struct Agg<P8UHIST4> : AggChan<P8UHIST4> {};

// Aggregate step (stage of chunk q landed): the band aggregate of the tile ->
// the chunk's leader.  Returns false at the end-of-work sentinel, after giving
// every leader warp of this CTA a sentinel in the gather slot of the next
// chunk it would lead (its peers send nothing there).
template <int P, int CL>
__device__ __forceinline__ bool aggregate_step(Smem<P, CL>& sm, const KParams& p, uint32_t rank,
                                               uint32_t q, typename Agg<kBase<P>>::Acc& L,
                                               int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  using A = Agg<kBase<P>>;
  constexpr uint32_t kVecBytes = C::TW * sizeof(TB);
  const int s = q % C::NSTAGE;
  const int64_t band = sm.stage_band[s];
  const uint32_t lead = q % CL;
  if (band < 0) {
    if (lane == 0) {
      const uint32_t jn = q <= rank ? 0u : (q - rank + CL - 1) / CL;
      for (int i = 0; i < kNLW<P>; ++i) {
        const uint32_t j = jn + (uint32_t)(((i - (int)(jn % kNLW<P>)) % kNLW<P> + kNLW<P>) % kNLW<P>);
        const int ls = j % kNLead<P, CL>;
        sm.lead_band[ls] = -1;
        mbar_arrive(&sm.lead_full[ls]);
      }
    }
    return false;
  }
  const int32_t chunk = sm.stage_chunk[s];
  TB agg[C::G][C::E];
  if (chunk == 0) L = typename A::Acc(0);
  if constexpr (kChan<P>)
    A::template run<C::TH>(&sm.in[s][0][0], lane, L, agg, p, sm.bin_of);
  else
    A::template run<C::TH>(&sm.in[s][0][0], lane, L, agg);
  if (sm.stage_img[s] < 0) {  // padding band of a partial cluster: stage not loaded
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) agg[g][e] = TB(0);
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.empty[s]);
  const int ls = (q / CL) % kNLead<P, CL>;
  // Arm the V_up receive before our aggregate can reach the leader.  The
  // leader's own hand-offs are shared stores + arrive (see send16), so it
  // arms only the bytes of its CL-1 peers.
  if (lane == 0) {
    if (rank != lead) {
      mbar_arrive_expect_tx(&sm.vin_full[q % kNV<P>], kVecBytes);
    } else {
      if (CL > 1) mbar_expect_tx(&sm.lead_full[ls], (CL - 1) * kVecBytes);
      sm.lead_band[ls] = band;
      sm.lead_chunk[ls] = chunk;
    }
  }
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    send16(&sm.lead_in[ls][rank][col_of<P>(g, lane)], &sm.lead_full[ls], lead, rank,
           pack16<TB, C::E>(agg[g]));
  if (lead == rank) {  // own contribution went by shared stores
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.lead_full[ls]);
  }
#ifdef SAT_TIMELINE
  if (lane == 0 && blockIdx.x < 1024 && q < kTlChunks) g_sat_tl_agg[blockIdx.x][q] = tl_now();
#endif
  return true;
}

// ---------------------------------------------------------------------------
// Compute warps

// TMEM address of warp `warp`'s S' rows for chunk slot t.
template <int P, int CL>
__device__ __forceinline__ uint32_t tmem_addr(const Smem<P, CL>& sm, int t, int warp) {
  return sm.tmem_base + ((uint32_t)(32 * (warp & 3)) << 16) +
         (uint32_t)(t * kTmemColsPerSlot<P> + (warp >> 2) * kTmemColsPerWarp<P>);
}

// Pass A of chunk q (stage s): row + column scans of this warp's RW rows
// (a2, a3, a5).  The column-scanned rows S' go to TMEM, the column totals to
// tot[q % NT][warp]; the input stage is released at once.  Returns false at
// the end-of-work sentinel.
template <int P, int CL>
__device__ __forceinline__ bool pass_a(Smem<P, CL>& sm, const KParams& p, uint32_t q, int s,
                                       uint32_t ph,
                                       typename Cfg<P>::TB (&rowcarry)[Cfg<P>::TH / kNCW<P>],
                                       int warp, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW<P>;
  constexpr int NW = kTmemColsPerWarp<P>;
  SAT_PT(t0);
  mbar_wait(&sm.full[s], ph);
  SAT_PT(t1);
  if (warp == 0) SAT_PADD(sm, kPfComputeWaitFull, t1 - t0);
  const int64_t band = sm.stage_band[s];
  if (band < 0) return false;
  const int32_t chunk = sm.stage_chunk[s];
  const int32_t img = sm.stage_img[s];
  const int32_t kk = sm.stage_k[s];
  if (chunk == 0) {
#pragma unroll
    for (int i = 0; i < RW; ++i) rowcarry[i] = TB(0);
  }
  const typename C::TA* tile = &sm.in[s][warp * RW][0];
  TB R[RW][C::G][C::E];
  if constexpr (kChan<P>)
    rows_scan_chan<kBase<P>, RW>(tile, lane, p, sm.bin_of, rowcarry, R);
  else
    rows_scan<RW>(tile, lane, rowcarry, R);
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.empty[s]);  // the tile is consumed: refill the stage
  // a5: running column sums S'(row i) down the warp's rows -> TMEM
  const int t = q % kNTot<P>;
  TB acc[C::G][C::E];
  uint32_t w[NW];
#pragma unroll
  for (int i = 0; i < RW; ++i)
#pragma unroll
    for (int g = 0; g < C::G; ++g)
#pragma unroll
      for (int e = 0; e < C::E; ++e) {
        acc[g][e] = i == 0 ? R[0][g][e] : acc[g][e] + R[i][g][e];
        put_words<TB>(w, (i * C::G + g) * C::E + e, acc[g][e]);
      }
  tmem_st(tmem_addr(sm, t, warp), w);
  tmem_wait_st();
  // a4: this warp's column totals for the block partial-sum scan.
#pragma unroll
  for (int g = 0; g < C::G; ++g)
    *reinterpret_cast<uint4*>(&sm.tot[t][warp][col_of<P>(g, lane)]) = pack16<TB, C::E>(acc[g]);
  if (lane == 0) {
    sm.meta[warp][t][1] = img;
    sm.meta[warp][t][2] = kk;
    sm.meta[warp][t][3] = chunk;
  }
  if (warp == 0 && lane == 0) {
    sm.tot_band[t] = band;
    sm.tot_img[t] = img;
    sm.tot_k[t] = kk;
    sm.tot_chunk[t] = chunk;
    sm.passA_done = q + 1;
  }
  __syncwarp();
  if (lane == 0) mbar_arrive(&sm.tot_full[t]);
  SAT_PT(t2);
  if (warp == 0) SAT_PADD(sm, kPfComputeLocal, t2 - t1);
  return true;
}

// Pass B of chunk q: wait for the fix-up offsets, load S' back from TMEM,
// add, store (a8).

// Exclusive-layout store of one tile row (Eq. 2; NPP layout):
// S(y, x) goes to output column o = x + 1.  The 16-B aligned output vector of
// lane l / group g starts at o0 = x0 + col_of(g, l) and holds S(x = o0 - 1 ..
// o0 + E - 2): the previous lane's last element, then this lane's first E - 1.
// Lane 0 takes its first element from group g - 1 (lane 31) or, for g = 0, from
// the previous chunk (`prevlast`, nVal at chunk 0 = output column 0).
template <int P, bool kVecOut>
__device__ __forceinline__ void store_row_exclusive(
    const KParams& p, char* orow, int64_t x0, bool last_chunk,
    const typename Cfg<P>::TB (&v)[Cfg<P>::G][Cfg<P>::E], typename Cfg<P>::TB& prevlast, int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  TB sh[C::G][C::E];
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    const TB up = __shfl_up_sync(kFull, v[g][C::E - 1], 1);
    const TB l31 = g > 0 ? __shfl_sync(kFull, v[g > 0 ? g - 1 : 0][C::E - 1], 31) : prevlast;
    sh[g][0] = lane == 0 ? l31 : up;
#pragma unroll
    for (int e = 1; e < C::E; ++e) sh[g][e] = v[g][e - 1];
  }
  const TB newlast = __shfl_sync(kFull, v[C::G - 1][C::E - 1], 31);
  TB* o = reinterpret_cast<TB*>(orow);
#pragma unroll
  for (int g = 0; g < C::G; ++g) {
    const int64_t o0 = x0 + col_of<P>(g, lane);
    if (kVecOut && o0 + C::E <= p.out_cols) {
      st_cs_v4(o + o0, pack16<TB, C::E>(sh[g]));
    } else {
#pragma unroll
      for (int e = 0; e < C::E; ++e)
        if (o0 + e < p.out_cols) o[o0 + e] = sh[g][e];
    }
  }
  // W a multiple of TW: the last column (o = W) lies past this chunk's vectors.
  if (last_chunk && lane == 31 && x0 + C::TW < p.out_cols) o[x0 + C::TW] = newlast;
  prevlast = newlast;
}

template <int P, int CL, bool kVecOut, bool kEx>
__device__ __forceinline__ void pass_b(Smem<P, CL>& sm, const KParams& p, uint32_t q, int warp,
                                       int lane, typename Cfg<P>::TB (&prevlast)[Cfg<P>::TH / kNCW<P>]) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW<P>;
  constexpr int NW = kTmemColsPerWarp<P>;
  const int t = q % kNTot<P>;
  const int32_t img = sm.meta[warp][t][1];  // written by this warp's pass A
  uint32_t w[NW];
  SAT_PT(t0);
  // byte pairs: back-off polling (same-box A/B -0.4..-3%); floats: try_wait
  if constexpr (SAT_BO_CARRY != 0 && (kBase<P> == P8U32S || kChan<P>))
    mbar_wait_sleep(&sm.carry_full[t], (q / kNTot<P>) & 1);
  else
    mbar_wait(&sm.carry_full[t], (q / kNTot<P>) & 1);
  SAT_PT(t1);
  if (warp == 0) SAT_PADD(sm, kPfComputeWaitCarry, t1 - t0);
  if (img >= 0) {
    tmem_ld(tmem_addr(sm, t, warp), w);
    TB off[C::G][C::E];  // V_up + the warps above + nVal (offset warp)
#pragma unroll
    for (int g = 0; g < C::G; ++g)
      unpack16<TB, C::E>(*reinterpret_cast<const uint4*>(&sm.tot[t][warp][col_of<P>(g, lane)]),
                         off[g]);
    const int64_t k = sm.meta[warp][t][2];
    const int32_t chunk = sm.meta[warp][t][3];
    const int64_t y0 = k * C::TH + warp * RW;
    const int64_t x0 = (int64_t)chunk * C::TW;
    char* orow = p.out + (int64_t)img * p.out_img_stride + y0 * p.out_pitch;
    tmem_wait_ld();
    if constexpr (kEx) {
      if (chunk == 0) {
#pragma unroll
        for (int i = 0; i < RW; ++i) prevlast[i] = from_bits<TB>(p.nval_bits);
      }
      const bool last_chunk = chunk == p.nchunks - 1;
#pragma unroll
      for (int i = 0; i < RW; ++i, orow += p.out_pitch) {
        if (y0 + i >= p.H) break;  // warp-uniform
        TB v[C::G][C::E];
#pragma unroll
        for (int g = 0; g < C::G; ++g)
#pragma unroll
          for (int e = 0; e < C::E; ++e)
            v[g][e] = off[g][e] + get_words<TB>(w, (i * C::G + g) * C::E + e);
        store_row_exclusive<P, kVecOut>(p, orow, x0, last_chunk, v, prevlast[i], lane);
      }
    } else if (kVecOut && y0 + RW <= p.H && x0 + C::TW <= p.W) {
      // interior tile rows: no edge predicates, row pointers by increment
#pragma unroll
      for (int i = 0; i < RW; ++i, orow += p.out_pitch) {
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
          TB v[C::E];
#pragma unroll
          for (int e = 0; e < C::E; ++e)
            v[e] = off[g][e] + get_words<TB>(w, (i * C::G + g) * C::E + e);
          st_cs_v4(reinterpret_cast<TB*>(orow) + x0 + col_of<P>(g, lane), pack16<TB, C::E>(v));
        }
      }
    } else {
#pragma unroll
      for (int i = 0; i < RW; ++i, orow += p.out_pitch) {
        if (y0 + i >= p.H) break;
#pragma unroll
        for (int g = 0; g < C::G; ++g) {
          TB v[C::E];
#pragma unroll
          for (int e = 0; e < C::E; ++e)
            v[e] = off[g][e] + get_words<TB>(w, (i * C::G + g) * C::E + e);
          const int64_t x = x0 + col_of<P>(g, lane);
          TB* o = reinterpret_cast<TB*>(orow);
          if (kVecOut && x + C::E <= p.W) {
            st_cs_v4(o + x, pack16<TB, C::E>(v));
          } else {
#pragma unroll
            for (int e = 0; e < C::E; ++e)
              if (x + e < p.W) o[x + e] = v[e];
          }
        }
      }
    }
  }
  SAT_PT(t2);
  if (warp == 0) SAT_PADD(sm, kPfComputeFixup, t2 - t1);
#ifdef SAT_TIMELINE
  if (warp == 0 && lane == 0 && img >= 0) {
    const int32_t ch = sm.meta[0][t][3];
    const int64_t gb = (int64_t)img * p.bands_per_image + sm.meta[0][t][2];
    if (gb < kTlBands) {
      if (ch == 0) g_sat_band_t[gb][0] = tl_now();
      if (ch == p.nchunks - 1) g_sat_band_t[gb][1] = tl_now();
    }
  }
  if (warp == 0 && lane == 0 && blockIdx.x < 1024 && img >= 0 && q < kTlChunks &&
      q < (uint32_t)p.nchunks) {
    if (q == 0) g_sat_tl[blockIdx.x][1] = (unsigned long long)sm.meta[0][t][2] +
                                          ((unsigned long long)img << 32);
    g_sat_tl[blockIdx.x][2 + q] = tl_now();
  }
#endif
}

template <int P, int CL, bool kVecOut, bool kEx>
__device__ __forceinline__ void compute_warp(Smem<P, CL>& sm, const KParams& p, int warp,
                                             int lane) {
  using C = Cfg<P>;
  using TB = typename C::TB;
  constexpr int RW = C::TH / kNCW<P>;
  TB prevlast[RW];  // exclusive layout: each row's last value of the previous chunk
  TB rowcarry[RW];
#pragma unroll
  for (int i = 0; i < RW; ++i) rowcarry[i] = TB(0);
  uint32_t qa = 0, qb = 0;
  bool ended = false;
  for (;;) {
    if (!ended) {
      if (pass_a<P, CL>(sm, p, qa, qa % C::NSTAGE, (qa / C::NSTAGE) & 1, rowcarry, warp, lane))
        ++qa;
      else
        ended = true;
    }
    if (qb < qa && (ended || qa - qb > (uint32_t)C::LOOK)) {
      pass_b<P, CL, kVecOut, kEx>(sm, p, qb, warp, lane, prevlast);
      ++qb;
    } else if (ended) {
      break;
    }
  }
  // End-of-work sentinel for the offset warp (the slot is free: all pass B done).
  {
    const int t = qa % kNTot<P>;
    if (warp == 0 && lane == 0) sm.tot_band[t] = -1;
    __syncwarp();
    if (lane == 0) mbar_arrive(&sm.tot_full[t]);
  }
}

// ---------------------------------------------------------------------------
// Producer warp

template <int P, int CL, bool kTMA>
__device__ __forceinline__ void producer_warp(Smem<P, CL>& sm, const KParams& p,
                                              const CUtensorMap* map, uint32_t rank, int lane) {
  using C = Cfg<P>;
  using TA = typename C::TA;
  constexpr uint32_t kTileBytes = C::TH * C::TW * sizeof(TA);
  const uint32_t kTicketLead = p.ticket_lead;  // chunks of the current band still ahead of pass A
  uint32_t q = 0, draws = 0;
  uint64_t pol = 0;
  if (kTMA) pol = policy_evict_first();
  for (;;) {
    int64_t T = 0;
    if (rank == 0) {
      // Draw the next cluster ticket only when pass A is within kTicketLead
      // chunks of the end of what was issued, so a drawn band is never queued
      // behind a whole band (its successors would stall on it).
      SAT_PT(t0);
      while (q > kTicketLead && sm.passA_done + kTicketLead < q) __nanosleep(64);
      SAT_PT(t1);
      if (lane == 0) SAT_PADD(sm, kPfProdWaitTicket, t1 - t0);
      if (lane == 0) {
        T = (int64_t)(atomicAdd(p.counter, 1ull) - p.ticket_base);
        if (CL > 1) {
          if (draws > 0) mbar_wait_cluster(&sm.tk_empty, (draws - 1) & 1);
          for (uint32_t r = 1; r < (uint32_t)CL; ++r)
            st_async8(mapa(&sm.tk_slot, r), (uint64_t)T, mapa(&sm.tk_full, r));
        }
      }
      T = __shfl_sync(kFull, T, 0);
    } else {
      if (lane == 0) {
        mbar_arrive_expect_tx(&sm.tk_full, 8);
        mbar_wait_cluster(&sm.tk_full, draws & 1);
        T = sm.tk_slot;
        mbar_arrive_remote(mapa(&sm.tk_empty, 0));
      }
      T = __shfl_sync(kFull, T, 0);
    }
    ++draws;
    const bool done = T < 0 || T >= p.total_tickets;  // T < 0: a counter out of step (never with plan-ordered launches)
    const int64_t g = T * CL + rank;
    const bool valid = !done && g < p.total_bands;
    const int64_t n = valid ? g / p.bands_per_image : 0;
    const int64_t k = valid ? g - n * p.bands_per_image : 0;
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
          sm.stage_band[s] = g;
          sm.stage_img[s] = valid ? (int32_t)n : -1;
          sm.stage_k[s] = (int32_t)k;
          sm.stage_chunk[s] = c;
          if (valid) {
            mbar_arrive_expect_tx(&sm.full[s], kTileBytes);
            tma_load_3d(&sm.in[s][0][0], map, &sm.full[s], c * C::TW, (int32_t)(k * C::TH),
                        (int32_t)n, pol);
          } else {
            mbar_arrive(&sm.full[s]);  // padding band: contents unused (nothing stored)
          }
        }
      } else {
        // Generic path: plain loads, zero fill outside the image.
        if (valid) {
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
        }
        __syncwarp();
        if (lane == 0) {
          sm.stage_band[s] = g;
          sm.stage_img[s] = valid ? (int32_t)n : -1;
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

template <int P, int CL, bool kTMA, bool kVecOut, bool kEx = false>
__global__ void __launch_bounds__(kThreads<P>, kMinBlocks<P>)
    sat_tile_kernel(const __grid_constant__ CUtensorMap map, const __grid_constant__ KParams p) {
  using C = Cfg<P>;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  Smem<P, CL>& sm = *reinterpret_cast<Smem<P, CL>*>(smem_raw);
  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const uint32_t rank = CL > 1 ? cluster_rank() : 0;

  if constexpr (kBase<P> == P8UHIST4) {
    for (int i = threadIdx.x; i < 256; i += blockDim.x) sm.bin_of[i] = p.bin_of[i];
  }
  if (threadIdx.x == 0) {
    for (int s = 0; s < C::NSTAGE; ++s) {
      mbar_init(&sm.full[s], 1);
      mbar_init(&sm.empty[s], kNCW<P> + 1);  // compute warps' pass A + the aggregate warp
    }
    for (int t = 0; t < kNTot<P>; ++t) {
      mbar_init(&sm.tot_full[t], kNCW<P>);
      mbar_init(&sm.carry_full[t], 1);
    }
    for (int v = 0; v < kNV<P>; ++v) mbar_init(&sm.vin_full[v], 1);
    for (int i = 0; i < kNLead<P, CL>; ++i) mbar_init(&sm.lead_full[i], 1);
    for (int i = 0; i < kNLW<P>; ++i) mbar_init(&sm.land_full[i], 1);
    mbar_init(&sm.tk_full, 1);
    mbar_init(&sm.tk_empty, CL > 1 ? CL - 1 : 1);
    sm.passA_done = 0;
#ifdef SAT_PROFILE
    for (int i = 0; i < 16; ++i) sm.prof[i] = 0;
#endif
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (kTMA)
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&map)) : "memory");
  }
  if (warp == 0) {  // TMEM for the S' rows (one warp allocates and later frees)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&sm.tmem_base)),
                 "r"(kTmemCols<P>)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  // Every CTA's barriers exist before any peer can signal them.
  if (CL > 1)
    cluster_sync_all();
  else
    __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");

#ifdef SAT_TIMELINE
  if (threadIdx.x == 0 && blockIdx.x < 1024) g_sat_tl[blockIdx.x][0] = tl_now();
#endif
  if (warp == kProducerWarp<P>) {
    producer_warp<P, CL, kTMA>(sm, p, &map, rank, lane);
  } else if (warp == kAggWarp<P>) {
    typename Agg<kBase<P>>::Acc L = typename Agg<kBase<P>>::Acc(0);
    for (uint32_t q = 0;; ++q) {
      mbar_wait(&sm.full[q % Cfg<P>::NSTAGE], (q / Cfg<P>::NSTAGE) & 1);
      if (!aggregate_step<P, CL>(sm, p, rank, q, L, lane)) break;
    }
  } else if (warp == kOffWarp<P>) {
    for (uint32_t q = 0;; ++q) {
      mbar_wait(&sm.tot_full[q % kNTot<P>], (q / kNTot<P>) & 1);
      if (sm.tot_band[q % kNTot<P>] < 0) break;
      mbar_wait_peer_data(&sm.vin_full[q % kNV<P>], (q / kNV<P>) & 1);
      offset_step<P, CL, kEx>(sm, p, q, lane);
    }
  } else if (warp >= kFirstLwWarp<P>) {
    leader_warp<P, CL>(sm, p, warp - kFirstLwWarp<P>, rank, lane);
  } else {
    compute_warp<P, CL, kVecOut, kEx>(sm, p, warp, lane);
  }
#ifdef SAT_PROFILE
  __syncthreads();
  if (threadIdx.x < 16) atomicAdd(&g_sat_prof[threadIdx.x], sm.prof[threadIdx.x]);
#endif
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  // No CTA may leave while a peer can still write into its shared memory.
  if (CL > 1)
    cluster_sync_all();
  else
    __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(sm.tmem_base),
                 "r"(kTmemCols<P>)
                 : "memory");
  }
}

}  // namespace sat
