// sat_runtime.cu -- libsat host runtime: plans, validation, tensor-map
// encoding, epoch/ticket workspace management, launches, the streamed host
// path.  C ABI declared in include/libsat.h.
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>

#include <algorithm>
#include <mutex>

#include "../../include/libsat.h"
#include "sat_internal.h"
#include "sat_kernel.cuh"

// The third cluster size besides 4 and 8: 5, the default for the 8u pairs
// (clusters of >= 3 CTAs reach 142 of the 148 SMs; 5-CTA clusters place 280
// CTAs and shorten the look-back chain 1.25x against 4: same-box A/B 16384^2
// -1.5%, 4096x65536 -4%, 1080p batch -1%; 3 and 6 measured too).
#ifndef SAT_CLX
#define SAT_CLX 5
#endif

namespace {

thread_local char g_last_error[512] = "";

}  // namespace

namespace sat {

sat_status fail(sat_status s, const char* fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_last_error, sizeof(g_last_error), fmt, ap);
  va_end(ap);
  return s;
}

sat_status cuda_fail(cudaError_t e, const char* what) {
  return fail(e == cudaErrorMemoryAllocation ? SAT_ERR_OUT_OF_MEMORY : SAT_ERR_CUDA, "%s: %s (%s)",
              what, cudaGetErrorName(e), cudaGetErrorString(e));
}

bool multi_channel(sat_pair p) { return p == SAT_8U_SQ || p == SAT_8U_HIST4; }
size_t in_size(sat_pair p) {
  return (p == SAT_8U_32S || p == SAT_8U_32F || multi_channel(p)) ? 1 : (p == SAT_64F_64F ? 8 : 4);
}
size_t out_size(sat_pair p) {
  return p == SAT_64F_64F || p == SAT_8U_SQ ? 8 : p == SAT_8U_HIST4 ? 16 : 4;
}
int tile_w(sat_pair p) {
  switch (p) {
    case SAT_8U_32S: return Cfg<P8U32S>::TW;
    case SAT_32F_32F: return Cfg<P32F32F>::TW;
    case SAT_64F_64F: return Cfg<P64F64F>::TW;
    case SAT_8U_32F: return Cfg<P8U32F>::TW;
    case SAT_32S_32S: return Cfg<P32S32S>::TW;
    case SAT_8U_SQ: return Cfg<P8USQ>::TW;
    case SAT_8U_HIST4: return Cfg<P8UHIST4>::TW;
  }
  return 1;
}
int tile_h(sat_pair p) {
  switch (p) {
    case SAT_8U_32S: return Cfg<P8U32S>::TH;
    case SAT_32F_32F: return Cfg<P32F32F>::TH;
    case SAT_64F_64F: return Cfg<P64F64F>::TH;
    case SAT_8U_32F: return Cfg<P8U32F>::TH;
    case SAT_32S_32S: return Cfg<P32S32S>::TH;
    case SAT_8U_SQ: return Cfg<P8USQ>::TH;
    case SAT_8U_HIST4: return Cfg<P8UHIST4>::TH;
  }
  return 1;
}

// ---------------------------------------------------------------------------
// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda).
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*,
                                  const cuuint64_t*, const cuuint64_t*, const cuuint32_t*,
                                  const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

static EncodeTiledFn get_encode() {
  static EncodeTiledFn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
            cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<EncodeTiledFn>(p);
  });
  return fn;
}

template <int P>
static sat_status launch_t(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w,
                           int64_t ip, int64_t op, int64_t iis, int64_t ois, int64_t batch,
                           const void* carry_in, cudaStream_t stream, const ExSpec* ex,
                           const ChainSpec* chain, const HistSpec* hist) {
  using C = Cfg<P>;
  const bool tma = ((uintptr_t)in % 16 == 0) && (ip % 16 == 0) && (batch == 1 || iis % 16 == 0) &&
                   pl->force_generic == 0;
  const bool vec = ((uintptr_t)out % 16 == 0) && (op % 16 == 0) && (batch == 1 || ois % 16 == 0);
  KParams kp;
  kp.in = static_cast<const char*>(in);
  kp.out = static_cast<char*>(out);
  kp.H = h;
  kp.W = w;
  kp.in_pitch = ip;
  kp.out_pitch = op;
  kp.in_img_stride = iis;
  kp.out_img_stride = ois;
  kp.bands_per_image = (h + C::TH - 1) / C::TH;
  kp.total_bands = kp.bands_per_image * batch;
  kp.nchunks = (int32_t)((w + C::TW - 1) / C::TW);
  kp.carry_in = carry_in;
  kp.out_cols = ex ? ex->out_cols : w;
  kp.nval_bits = ex ? ex->nval_bits : 0;
  kp.chain_in = chain ? static_cast<const uint64_t*>(chain->in) : nullptr;
  kp.chain_out = chain ? static_cast<uint64_t*>(chain->out) : nullptr;
  kp.chain_ack_out = chain ? chain->ack_out : nullptr;
  kp.chain_ack_in = chain ? chain->ack_in : nullptr;
  kp.chain_epoch = chain ? chain->epoch : 0;
  memset(kp.bin_of, 0, sizeof(kp.bin_of));
  kp.bin0 = 0;
  if (hist) {
    memcpy(kp.bin_of, hist->bin_of, sizeof(kp.bin_of));
    kp.bin0 = hist->bin0;
  }

  CUtensorMap map;
  memset(&map, 0, sizeof(map));
  if (tma) {
    EncodeTiledFn enc = get_encode();
    if (!enc) return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
    const CUtensorMapDataType dt = (kBase<P> == P8U32S || kBase<P> == P8U32F || kChan<P>)
                                       ? CU_TENSOR_MAP_DATA_TYPE_UINT8
                                   : kBase<P> == P32F32F ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32
                                   : kBase<P> == P32S32S ? CU_TENSOR_MAP_DATA_TYPE_UINT32
                                                  : CU_TENSOR_MAP_DATA_TYPE_FLOAT64;
    cuuint64_t dims[3] = {(cuuint64_t)w, (cuuint64_t)h, (cuuint64_t)batch};
    cuuint64_t strides[2] = {(cuuint64_t)ip, (cuuint64_t)(batch > 1 ? iis : ip * h)};
    cuuint32_t box[3] = {(cuuint32_t)C::TW, (cuuint32_t)C::TH, 1};
    cuuint32_t estr[3] = {1, 1, 1};
    CUresult r = enc(&map, dt, 3, const_cast<void*>(in), dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (r != CUDA_SUCCESS) return fail(SAT_ERR_CUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  }

  // Cluster size: 8 bands per cluster for the float pairs when there are enough
  // bands to fill the machine (shorter look-back chains pay off there); 4 for
  // 8u->32s and for short/wide images (measured).
  int CL = default_cluster(kBase<P>, kp.total_bands);
  if (pl->cluster > 0) CL = pl->cluster;
  if (ex && CL != 4 && CL != 8) CL = 4;  // exclusive kernels: clusters of 4 and 8
  if (P >= kShort) CL = 4;               // short-band / deep-ring kernels: clusters of 4 only
  kp.total_tickets = (kp.total_bands + CL - 1) / CL;
  // Look-back workspace: one tagged carry vector per (cluster ticket, chunk).
  {
    const size_t need = (size_t)kp.total_tickets * kp.nchunks * kVecWords<P> * 8;
    const size_t have = pl->payload_bytes;
    if (need > have)
      return fail(SAT_ERR_INVALID_ARGUMENT,
                  "problem needs %zu bytes of carry workspace (cluster %d), plan holds %zu", need, CL,
                  have);
  }
  kp.err = pl->err;
  kp.spin_ns = pl->spin_ns;

  // Epoch: status words from earlier launches carry older epochs.
  if (pl->epoch + 1 >= (1u << 30)) {
    // status words hold 30 epoch bits and payload words 32: clear both on wrap
    cudaError_t e =
        cudaMemsetAsync(pl->payload, 0, pl->ws_bytes - ((char*)pl->payload - (char*)pl->ws), stream);
    if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(workspace)");
    pl->epoch = 0;
  }
  kp.epoch = ++pl->epoch;
  kp.counter = pl->counter;
  kp.payload = pl->payload;
  kp.tree_rd = pl->tree_rd;
  kp.tree = 0;
  // Ticket pacing: a CTA draws its next band when pass A is kp.ticket_lead
  // chunks from the end of what it has issued.  Short bands (batches of small
  // frames) draw early, so the next band's tiles and carries are under way
  // while the current one drains (1080p batch -7..9%); long bands draw late
  // (a drawn band must not queue behind a whole band).
#ifndef SAT_TICKET_LEAD
#define SAT_TICKET_LEAD 0
#endif
  kp.ticket_lead = SAT_TICKET_LEAD > 0 ? SAT_TICKET_LEAD
                                       : (kp.nchunks <= 16 ? (uint32_t)C::NSTAGE : 2u);
  if constexpr (kFen<P>) {
    // Carry mechanism (integer pairs): the counted reduction tree where the
    // look-back chain is what paces the launch -- images of few bands
    // (batches: every band start waits for its carry) and launches of at
    // most one wave of bands; the look-back where bands run two waves and
    // more (measured).  SAT_TREE=0/1 forces it.
    const int64_t slots = (int64_t)pl->active_clusters[kBase<P>][cluster_index(CL)][3] * CL;
    const bool tree_shape = kp.bands_per_image <= 64 || kp.total_bands <= slots;
    kp.tree = pl->tree_mode >= 0 ? pl->tree_mode : (tree_shape ? 1 : 0);
    if (kp.tree && (size_t)kp.total_tickets * kp.nchunks > (size_t)pl->tickets_cap * pl->max_chunks)
      return fail(SAT_ERR_INVALID_ARGUMENT, "problem exceeds the plan's carry-tree counters");
    if (kp.tree && kp.bands_per_image / CL + 2 >= (1 << 16)) kp.tree = 0;  // count field: look-back
    // The tree needs zeroed nodes (every tree launch leaves them zeroed); the
    // look-back leaves tagged words in the same workspace: clear the part a
    // tree launch uses when the plan's previous carry launch looked back.
    if (kp.tree && pl->lookback_dirty) {
      const size_t vecs = (size_t)kp.total_tickets * kp.nchunks;
      cudaError_t e = cudaMemsetAsync(pl->payload, 0, vecs * kVecWords<P> * 8, stream);
      if (e == cudaSuccess) e = cudaMemsetAsync(pl->tree_rd, 0, vecs * 4, stream);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemsetAsync(carry tree)");
    }
    pl->lookback_dirty = !kp.tree;
  }
  kp.ticket_base = pl->ticket_base;

  const int mode = (tma ? 1 : 0) | (vec ? 2 : 0);
  const int ci = cluster_index(CL);
  // Persistent grid: every co-resident cluster slot, but no more clusters than tickets.
  int64_t clusters =
      std::max(kIsDeep<P> ? pl->active_deep[kBase<P>]
               : P >= kShort ? pl->active_short[kBase<P>]
                             : pl->active_clusters[kBase<P>][ci][mode], 1);
  if (pl->max_clusters > 0) clusters = std::min<int64_t>(clusters, pl->max_clusters);
  if (pl->force_clusters > 0) clusters = pl->force_clusters;
  clusters = std::min<int64_t>(clusters, kp.total_tickets);
  const int64_t grid = clusters * CL;

  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(kThreads<P>);
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)CL;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  size_t smem = 0;
  cudaError_t e = cudaSuccess;
#define SAT_LAUNCH_CL(CLV, EX)                                                              \
  {                                                                                         \
    smem = sizeof(Smem<P, CLV>);                                                            \
    cfg.dynamicSmemBytes = smem;                                                            \
    switch (mode) {                                                                         \
      case 0: e = cudaLaunchKernelEx(&cfg, sat_tile_kernel<P, CLV, false, false, EX>, map, kp); break; \
      case 1: e = cudaLaunchKernelEx(&cfg, sat_tile_kernel<P, CLV, true, false, EX>, map, kp); break;  \
      case 2: e = cudaLaunchKernelEx(&cfg, sat_tile_kernel<P, CLV, false, true, EX>, map, kp); break;  \
      default: e = cudaLaunchKernelEx(&cfg, sat_tile_kernel<P, CLV, true, true, EX>, map, kp); break;  \
    }                                                                                       \
  }
  if constexpr (P >= kShort) {  // selected only for TMA + vector-store launches
    smem = sizeof(Smem<P, 4>);
    cfg.dynamicSmemBytes = smem;
    e = cudaLaunchKernelEx(&cfg, sat_tile_kernel<P, 4, true, true, false>, map, kp);
  } else {
    if constexpr (!kChan<P>) {
      if (ex) {
        if (CL == 4) SAT_LAUNCH_CL(4, true) else SAT_LAUNCH_CL(8, true)
      }
    }
    if (!ex) {
      if (CL == SAT_CLX) SAT_LAUNCH_CL(SAT_CLX, false) else if (CL == 4) SAT_LAUNCH_CL(4, false) else SAT_LAUNCH_CL(8, false)
    }
  }
#undef SAT_LAUNCH_CL
  if (e != cudaSuccess) return cuda_fail(e, "sat_tile_kernel launch");
  e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_fail(e, "sat_tile_kernel launch");
#ifdef SAT_TIMELINE
  {
    static unsigned long long tl[1024][2 + kTlChunks], ta[1024][kTlChunks], tv[1024][kTlChunks],
        t1[1024][kTlChunks], t2[1024][kTlChunks], t3[1024][kTlChunks];
    cudaStreamSynchronize(stream);
    cudaMemcpyFromSymbol(tl, g_sat_tl, sizeof(tl));
    cudaMemcpyFromSymbol(ta, g_sat_tl_agg, sizeof(ta));
    cudaMemcpyFromSymbol(tv, g_sat_tl_v, sizeof(tv));
    cudaMemcpyFromSymbol(t1, g_sat_tl_ls, sizeof(t1));
    cudaMemcpyFromSymbol(t2, g_sat_tl_lt, sizeof(t2));
    cudaMemcpyFromSymbol(t3, g_sat_tl_ld, sizeof(t3));
    static unsigned int rr[1024][kTlChunks][2];
    cudaMemcpyFromSymbol(rr, g_sat_tl_rounds, sizeof(rr));
    static unsigned int rz[1024][kTlChunks][2];
    cudaMemcpyToSymbol(g_sat_tl_rounds, rz, sizeof(rz));
    static unsigned long long zero[1024][2 + kTlChunks];
    cudaMemcpyToSymbol(g_sat_tl, zero, sizeof(zero));
    cudaMemcpyToSymbol(g_sat_tl_agg, zero, sizeof(ta));
    cudaMemcpyToSymbol(g_sat_tl_v, zero, sizeof(tv));
    cudaMemcpyToSymbol(g_sat_tl_ls, zero, sizeof(ta));
    cudaMemcpyToSymbol(g_sat_tl_lt, zero, sizeof(ta));
    cudaMemcpyToSymbol(g_sat_tl_ld, zero, sizeof(ta));
    const char* path = getenv("SAT_TIMELINE_OUT");
    FILE* f = path ? fopen(path, "a") : nullptr;
    static unsigned long long bt[kTlBands][2];
    cudaMemcpyFromSymbol(bt, g_sat_band_t, sizeof(bt));
    static unsigned long long bz[kTlBands][2];
    cudaMemcpyToSymbol(g_sat_band_t, bz, sizeof(bz));
    if (f) {
      for (int64_t b = 0; b < kp.total_bands && b < kTlBands; ++b)
        fprintf(f, "band %lld %llu %llu\n", (long long)b, bt[b][0], bt[b][1]);
      fprintf(f, "launch pair=%d h=%lld w=%lld batch=%lld CL=%d grid=%lld nchunks=%d\n", P,
              (long long)h, (long long)w, (long long)batch, CL, (long long)grid, kp.nchunks);
      const int nc = std::min<int>(kp.nchunks, kTlChunks);
      for (int64_t b = 0; b < grid && b < 1024; ++b) {
        fprintf(f, "cta %lld %llu %llu", (long long)b, tl[b][0], tl[b][1]);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", tl[b][2 + c]);
        fprintf(f, "\nagg %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", ta[b][c]);
        fprintf(f, "\nvup %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", tv[b][c]);
        fprintf(f, "\nls %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", t1[b][c]);
        fprintf(f, "\nlt %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", t2[b][c]);
        fprintf(f, "\nld %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %llu", t3[b][c]);
        fprintf(f, "\nrounds %lld", (long long)b);
        for (int c = 0; c < nc; ++c) fprintf(f, " %u/%u", rr[b][c][0], rr[b][c][1]);
        fprintf(f, "\n");
      }
      fclose(f);
    }
  }
#endif
#ifdef SAT_PROFILE
  {
    unsigned long long prof[16];
    cudaStreamSynchronize(stream);
    cudaMemcpyFromSymbol(prof, g_sat_prof, sizeof(prof));
    unsigned long long zero[16] = {};
    cudaMemcpyToSymbol(g_sat_prof, zero, sizeof(zero));
    const double ch = prof[kPfLbChunks] ? (double)prof[kPfLbChunks] : 1.0;
    const double ctas = (double)grid;
    const double lc = prof[kPfLeaderChunks] ? (double)prof[kPfLeaderChunks] : 1.0;
    fprintf(stderr,
            "[libsat prof] pair=%d %lldx%lld CL=%d grid=%lld chunks=%.0f | per chunk (ns): compute "
            "wait_full %.0f wait_carry %.0f passA %.0f passB %.0f | lb wait_tot %.0f wait_V %.0f | "
            "leader (per leader chunk): wait_cluster %.0f lookback %.0f depth %.2f retries %.2f "
            "rounds %.2f round_ns %.0f issue_ns %.0f\n",
            P, (long long)h, (long long)w, CL, (long long)grid, ch, prof[0] / ch, prof[1] / ch,
            prof[2] / ch, prof[3] / ch, prof[4] / ch, prof[10] / ch, prof[5] / lc, prof[6] / lc,
            prof[7] / lc, prof[8] / lc, prof[14] / lc,
            prof[14] ? (double)prof[13] / (double)prof[14] : 0.0,
            prof[14] ? (double)prof[15] / (double)prof[14] : 0.0);
    (void)ctas;
  }
#endif
  // Every cluster draws exactly one failing ticket.
  pl->ticket_base += (uint64_t)kp.total_tickets + (uint64_t)clusters;
  pl->launches++;
  if (pl->log)
    fprintf(stderr,
            "[libsat] pair=%d %lldx%lld batch=%lld tma=%d vec=%d cluster=%d grid=%lld smem=%zu "
            "epoch=%u tree=%d\n",
            P, (long long)h, (long long)w, (long long)batch, (int)tma, (int)vec, CL, (long long)grid,
            smem, kp.epoch, (int)kp.tree);
  return SAT_OK;
}

static sat_status launch_dispatch(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w,
                                  int64_t ip, int64_t op, int64_t iis, int64_t ois, int64_t batch,
                                  const void* carry_in, cudaStream_t stream, const ExSpec* ex,
                                  const ChainSpec* chain, const HistSpec* hist);

sat_status launch(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w, int64_t ip,
                  int64_t op, int64_t iis, int64_t ois, int64_t batch, const void* carry_in,
                  cudaStream_t stream, const ExSpec* ex, const ChainSpec* chain,
                  const HistSpec* hist) {
  if (multi_channel(pl->pair) && (carry_in || ex || chain))
    return fail(SAT_ERR_UNSUPPORTED,
                "the multi-channel pairs support sat_compute / _batched only (no carry-in, "
                "exclusive layout or chained bands)");
  if (pl->pair == SAT_8U_HIST4 && !hist)
    return fail(SAT_ERR_INVALID_ARGUMENT, "SAT_8U_HIST4 needs bins: use sat_compute_hist4");
  // Tickets and epochs are handed out by the host per launch: a captured
  // launch replayed from a graph would reuse them, so capture is refused.
  cudaStreamCaptureStatus cs = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(stream, &cs) == cudaSuccess && cs != cudaStreamCaptureStatusNone)
    return fail(SAT_ERR_UNSUPPORTED,
                "stream capture (CUDA graphs) is not supported: libsat hands out look-back "
                "tickets and epochs per launch on the host");
  // Launches of one plan share its workspace: order a launch on a new stream
  // after the plan's previous launch.
  if (pl->has_last && pl->last_stream != stream) {
    cudaError_t e = cudaStreamWaitEvent(stream, pl->last_ev, 0);
    if (e != cudaSuccess) return cuda_fail(e, "cudaStreamWaitEvent(plan order)");
  }
  sat_status st =
      launch_dispatch(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
  if (st == SAT_OK) {
    cudaError_t e = cudaEventRecord(pl->last_ev, stream);
    if (e != cudaSuccess) return cuda_fail(e, "cudaEventRecord(plan order)");
    pl->last_stream = stream;
    pl->has_last = true;
  }
  return st;
}

static sat_status launch_dispatch(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w,
                                  int64_t ip, int64_t op, int64_t iis, int64_t ois, int64_t batch,
                                  const void* carry_in, cudaStream_t stream, const ExSpec* ex,
                                  const ChainSpec* chain, const HistSpec* hist) {
  // Short, wide images: 32-row bands give only H/4 compute warps in total
  // (2 CTAs of 8 warps per SM leave most SMs idle below ~140 bands); 16-row
  // bands (2 rows per warp) double the warps in flight.
  const int th = tile_h(pl->pair);
  const int64_t bands32 = (h + th - 1) / th * batch;
  const bool aligned = ((uintptr_t)in % 16 == 0) && (ip % 16 == 0) && (batch == 1 || iis % 16 == 0) &&
                       ((uintptr_t)out % 16 == 0) && (op % 16 == 0) && (batch == 1 || ois % 16 == 0);
  const int sh_env = pl->short_bands;
  const bool use_short = !ex && !multi_channel(pl->pair) && aligned && pl->force_generic == 0 &&
                         pl->cluster == 0 &&
                         (sh_env >= 0 ? sh_env == 1 : 2 * bands32 <= (int64_t)pl->num_sms);
  // Deep-ring variant: at most one band per SM (and more than the short-band
  // rule takes) -- one CTA per SM with a deeper TMA ring.  By shape for the
  // 4-byte pairs only (4096 x 65536 32f -11%; 64f unchanged, 8u +4%, same-box
  // A/B); SAT_DEEP=0/1 forces it for every pair.
  const int dp_env = pl->deep_ring;
  const bool deep_pair = pl->pair == SAT_32F_32F || pl->pair == SAT_32S_32S;
  const bool use_deep = !use_short && !ex && !multi_channel(pl->pair) && aligned &&
                        pl->force_generic == 0 && pl->cluster == 0 &&
                        (dp_env >= 0 ? dp_env == 1 : deep_pair && bands32 <= (int64_t)pl->num_sms);
  if (use_deep) {
    switch (pl->pair) {
      case SAT_8U_32S:
        return launch_t<P8U32S + kDeep>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_32F_32F:
        return launch_t<P32F32F + kDeep>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_64F_64F:
        return launch_t<P64F64F + kDeep>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_8U_32F:
        return launch_t<P8U32F + kDeep>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_32S_32S:
        return launch_t<P32S32S + kDeep>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      default:
        break;
    }
  }
  if (use_short) {
    switch (pl->pair) {
      case SAT_8U_32S:
        return launch_t<P8U32S + kShort>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_32F_32F:
        return launch_t<P32F32F + kShort>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_64F_64F:
        return launch_t<P64F64F + kShort>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_8U_32F:
        return launch_t<P8U32F + kShort>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      case SAT_32S_32S:
        return launch_t<P32S32S + kShort>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
      default:
        break;
    }
  }
  switch (pl->pair) {
    case SAT_8U_32S:
      return launch_t<P8U32S>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_32F_32F:
      return launch_t<P32F32F>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_64F_64F:
      return launch_t<P64F64F>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_8U_32F:
      return launch_t<P8U32F>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_32S_32S:
      return launch_t<P32S32S>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_8U_SQ:
      return launch_t<P8USQ>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
    case SAT_8U_HIST4:
      return launch_t<P8UHIST4>(pl, in, out, h, w, ip, op, iis, ois, batch, carry_in, stream, ex, chain, hist);
  }
  return fail(SAT_ERR_INVALID_ARGUMENT, "bad pair");
}

int cluster_index(int cl) { return cl == SAT_CLX ? 0 : cl == 4 ? 1 : 2; }

int default_cluster(int base_pair, int64_t bands) {
  if (base_pair == P8U32S || base_pair == P8U32F) return SAT_CLX;
  if (base_pair == P8USQ || base_pair == P8UHIST4) return 4;
  return bands >= 224 ? 8 : 4;
}

int getenv_int(const char* name, int dflt) {
  const char* v = getenv(name);
  return v && *v ? atoi(v) : dflt;
}

// Occupancy proxy: the occupancy calculator treats any tcgen05 (TMEM) kernel as
// one CTA per SM, while the hardware co-schedules as many as TMEM allows (each
// CTA allocates kTmemCols of the SM's 512 columns).  The proxy has the same
// block size, dynamic shared memory, cluster shape and register bound, so its
// answer is the real residency, which is then capped by TMEM.
template <int P, int CL>
__global__ void __launch_bounds__(kThreads<P>, kMinBlocks<P>) sat_occupancy_proxy(int* sink) {
  extern __shared__ unsigned char s[];
  if (sink) sink[threadIdx.x] = s[threadIdx.x];
}

template <int P, int CL>
static sat_status configure_cl(sat_plan_st* pl) {
  const size_t smem = sizeof(Smem<P, CL>);
  void (*fns[4])(CUtensorMap, KParams) = {
      sat_tile_kernel<P, CL, false, false>, sat_tile_kernel<P, CL, true, false>,
      sat_tile_kernel<P, CL, false, true>, sat_tile_kernel<P, CL, true, true>};
  cudaError_t e0 = cudaFuncSetAttribute(sat_occupancy_proxy<P, CL>,
                                        cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e0 != cudaSuccess) return cuda_fail(e0, "cudaFuncSetAttribute(proxy)");
  if constexpr ((CL == 4 || CL == 8) && !kChan<P>) {
    void (*fx[4])(CUtensorMap, KParams) = {
        sat_tile_kernel<P, CL, false, false, true>, sat_tile_kernel<P, CL, true, false, true>,
        sat_tile_kernel<P, CL, false, true, true>, sat_tile_kernel<P, CL, true, true, true>};
    for (int m = 0; m < 4; ++m) {
      cudaError_t e = cudaFuncSetAttribute(fx[m], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(exclusive)");
    }
  }
  for (int m = 0; m < 4; ++m) {
    cudaError_t e = cudaFuncSetAttribute(fns[m], cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute");
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(CL * 64);
    cfg.blockDim = dim3(kThreads<P>);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr;
    attr.id = cudaLaunchAttributeClusterDimension;
    attr.val.clusterDim.x = CL;
    attr.val.clusterDim.y = 1;
    attr.val.clusterDim.z = 1;
    cfg.attrs = &attr;
    cfg.numAttrs = 1;
    int n = 0;
    e = cudaOccupancyMaxActiveClusters(&n, sat_occupancy_proxy<P, CL>, &cfg);
    if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveClusters");
    const int tmem_cap = pl->num_sms * (512 / kTmemCols<P>) / CL;
    pl->active_clusters[P][cluster_index(CL)][m] = std::min(n, tmem_cap);
  }
  return SAT_OK;
}

template <int P>
static sat_status configure_short(sat_plan_st* pl) {
  constexpr int PS = P + kShort, CL = 4;
  const size_t smem = sizeof(Smem<PS, CL>);
  cudaError_t e = cudaFuncSetAttribute(sat_occupancy_proxy<PS, CL>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sat_tile_kernel<PS, CL, true, true, false>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(short)");
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CL * 64);
  cfg.blockDim = dim3(kThreads<PS>);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr;
  attr.id = cudaLaunchAttributeClusterDimension;
  attr.val.clusterDim.x = CL;
  attr.val.clusterDim.y = 1;
  attr.val.clusterDim.z = 1;
  cfg.attrs = &attr;
  cfg.numAttrs = 1;
  int n = 0;
  e = cudaOccupancyMaxActiveClusters(&n, sat_occupancy_proxy<PS, CL>, &cfg);
  if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveClusters(short)");
  pl->active_short[P] = std::min(n, pl->num_sms * (512 / kTmemCols<PS>) / CL);
  return SAT_OK;
}

template <int P>
static sat_status configure_deep(sat_plan_st* pl) {
  constexpr int PD = P + kDeep, CL = 4;
  const size_t smem = sizeof(Smem<PD, CL>);
  cudaError_t e = cudaFuncSetAttribute(sat_occupancy_proxy<PD, CL>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(sat_tile_kernel<PD, CL, true, true, false>,
                             cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return cuda_fail(e, "cudaFuncSetAttribute(deep)");
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(CL * 64);
  cfg.blockDim = dim3(kThreads<PD>);
  cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute attr;
  attr.id = cudaLaunchAttributeClusterDimension;
  attr.val.clusterDim.x = CL;
  attr.val.clusterDim.y = 1;
  attr.val.clusterDim.z = 1;
  cfg.attrs = &attr;
  cfg.numAttrs = 1;
  int n = 0;
  e = cudaOccupancyMaxActiveClusters(&n, sat_occupancy_proxy<PD, CL>, &cfg);
  if (e != cudaSuccess) return cuda_fail(e, "cudaOccupancyMaxActiveClusters(deep)");
  pl->active_deep[P] = std::min(n, pl->num_sms * (512 / kTmemCols<PD>) / CL);
  return SAT_OK;
}

template <int P>
static sat_status configure_t(sat_plan_st* pl) {
  sat_status st = configure_cl<P, SAT_CLX>(pl);
  if (st == SAT_OK) st = configure_cl<P, 4>(pl);
  if (st == SAT_OK) st = configure_cl<P, 8>(pl);
  if constexpr (!kChan<P>)
    if (st == SAT_OK) st = configure_short<P>(pl);
  if constexpr (!kChan<P>)
    if (st == SAT_OK) st = configure_deep<P>(pl);
  return st;
}

sat_status configure(sat_plan_st* pl) {
  switch (pl->pair) {
    case SAT_8U_32S:
      return configure_t<P8U32S>(pl);
    case SAT_32F_32F:
      return configure_t<P32F32F>(pl);
    case SAT_64F_64F:
      return configure_t<P64F64F>(pl);
    case SAT_8U_32F:
      return configure_t<P8U32F>(pl);
    case SAT_32S_32S:
      return configure_t<P32S32S>(pl);
    case SAT_8U_SQ:
      return configure_t<P8USQ>(pl);
    case SAT_8U_HIST4:
      return configure_t<P8UHIST4>(pl);
  }
  return fail(SAT_ERR_INVALID_ARGUMENT, "bad pair");
}

// ---------------------------------------------------------------------------
// Validation (synchronous; nothing is launched on failure)

static bool ranges_overlap(const void* a, size_t an, const void* b, size_t bn) {
  const uintptr_t a0 = (uintptr_t)a, a1 = a0 + an, b0 = (uintptr_t)b, b1 = b0 + bn;
  return a0 < b1 && b0 < a1;
}

sat_status validate(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w, int64_t ip,
                    int64_t op, int64_t iis, int64_t ois, int64_t batch, sat_pair pair,
                    bool* empty) {
  *empty = false;
  if (!pl) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (pair != pl->pair)
    return fail(SAT_ERR_INVALID_ARGUMENT, "pair %d does not match the plan's pair %d", (int)pair,
                (int)pl->pair);
  if (h < 0 || w < 0 || batch < 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "negative extent (h=%lld w=%lld batch=%lld)",
                (long long)h, (long long)w, (long long)batch);
  if (h == 0 || w == 0 || batch == 0) {
    *empty = true;
    return SAT_OK;
  }
  if (!in || !out) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL input or output pointer");
  if (h > pl->max_h || w > pl->max_w || batch > pl->max_batch)
    return fail(SAT_ERR_INVALID_ARGUMENT,
                "extent %lldx%lld batch %lld exceeds plan limits %lldx%lld batch %lld",
                (long long)h, (long long)w, (long long)batch, (long long)pl->max_h,
                (long long)pl->max_w, (long long)pl->max_batch);
  const int64_t sa = (int64_t)in_size(pair), sb = (int64_t)out_size(pair);
  if (ip < w * sa || ip % sa != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "input pitch %lld invalid for w=%lld (elem %lld B)",
                (long long)ip, (long long)w, (long long)sa);
  if (op < w * sb || op % sb != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "output pitch %lld invalid for w=%lld (elem %lld B)",
                (long long)op, (long long)w, (long long)sb);
  if ((uintptr_t)in % sa != 0 || (uintptr_t)out % sb != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "pointer not aligned to its element size");
  if (batch > 1) {
    if (iis < h * ip || iis % sa != 0)
      return fail(SAT_ERR_INVALID_ARGUMENT, "input image stride %lld invalid", (long long)iis);
    if (ois < h * op || ois % sb != 0)
      return fail(SAT_ERR_INVALID_ARGUMENT, "output image stride %lld invalid", (long long)ois);
  }
  // Overlap: only exact in-place for equal element sizes and layouts.
  const size_t in_bytes = (size_t)((batch - 1) * (batch > 1 ? iis : 0) + (h - 1) * ip + w * sa);
  const size_t out_bytes = (size_t)((batch - 1) * (batch > 1 ? ois : 0) + (h - 1) * op + w * sb);
  if (ranges_overlap(in, in_bytes, out, out_bytes)) {
    const bool inplace = in == out && sa == sb && ip == op && (batch == 1 || iis == ois);
    if (!inplace)
      return fail(SAT_ERR_UNSUPPORTED, "input and output overlap (only exact in-place for 32f/64f)");
  }
  return SAT_OK;
}

}  // namespace sat

using namespace sat;

// ===========================================================================
// C ABI

extern "C" {

int sat_version(void) { return 20000; }

const char* sat_status_string(sat_status s) {
  switch (s) {
    case SAT_OK:
      return "SAT_OK";
    case SAT_ERR_INVALID_ARGUMENT:
      return "SAT_ERR_INVALID_ARGUMENT";
    case SAT_ERR_UNSUPPORTED:
      return "SAT_ERR_UNSUPPORTED";
    case SAT_ERR_CUDA:
      return "SAT_ERR_CUDA";
    case SAT_ERR_NCCL:
      return "SAT_ERR_NCCL";
    case SAT_ERR_OUT_OF_MEMORY:
      return "SAT_ERR_OUT_OF_MEMORY";
    case SAT_ERR_TIMEOUT:
      return "SAT_ERR_TIMEOUT";
  }
  return "SAT_ERR_UNKNOWN";
}

const char* sat_last_error(void) { return g_last_error; }

sat_status sat_plan_create(sat_plan* plan, int device, sat_pair pair, int64_t max_h, int64_t max_w,
                           int64_t max_batch) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan out-pointer is NULL");
  *plan = nullptr;
  if (pair != SAT_8U_32S && pair != SAT_32F_32F && pair != SAT_64F_64F && pair != SAT_8U_32F &&
      pair != SAT_32S_32S && pair != SAT_8U_SQ && pair != SAT_8U_HIST4)
    return fail(SAT_ERR_INVALID_ARGUMENT, "unknown pair %d", (int)pair);
  if (max_h <= 0 || max_w <= 0 || max_batch <= 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "plan limits must be positive");
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceCount");
  if (device < 0 || device >= ndev) return fail(SAT_ERR_CUDA, "no CUDA device %d", device);
  cudaDeviceProp prop;
  e = cudaGetDeviceProperties(&prop, device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDeviceProperties");
  if (prop.major != 10 || prop.minor != 0)
    return fail(SAT_ERR_CUDA, "device %d is sm_%d%d; libsat is built for sm_100a only", device,
                prop.major, prop.minor);
  int prev = 0;
  cudaGetDevice(&prev);
  e = cudaSetDevice(device);
  if (e != cudaSuccess) return cuda_fail(e, "cudaSetDevice");

  sat_plan_st* pl = new sat_plan_st();
  pl->device = device;
  pl->pair = pair;
  pl->max_h = max_h;
  pl->max_w = max_w;
  pl->max_batch = max_batch;
  pl->num_sms = prop.multiProcessorCount;
  // Environment knobs: read once, here (never on the launch path).
  pl->force_generic = getenv_int("SAT_FORCE_GENERIC", 0);
  {
    const int c = getenv_int("SAT_CLUSTER", 0);
    pl->cluster = (c == SAT_CLX || c == 4 || c == 8) ? c : 0;
  }
  pl->short_bands = getenv_int("SAT_SHORT", -1);
  pl->deep_ring = getenv_int("SAT_DEEP", -1);
  pl->max_clusters = getenv_int("SAT_MAX_CLUSTERS", 0);
  pl->force_clusters = getenv_int("SAT_FORCE_CLUSTERS", 0);
  pl->log = getenv_int("SAT_LOG", 0);
  pl->tree_mode = getenv_int("SAT_TREE", -1);
  const int64_t TH = tile_h(pair), TW = tile_w(pair);
  const int64_t bands = max_batch * ((max_h + TH - 1) / TH);
  pl->max_chunks = (max_w + TW - 1) / TW;
  pl->max_tiles = bands * pl->max_chunks;
  // Look-back capacity: one tagged vector (TW elements, 8 bytes per 32 value
  // bits) per (cluster ticket, chunk).  Tickets per launch follow the cluster policy
  // (default_cluster, or the forced size); short-band launches (<= #SMs / 2
  // normal bands) have at most num_sms / 4 tickets.
  int64_t tickets;
  if (pl->cluster > 0) {
    // a forced size other than 4 / 8 still runs exclusive launches with clusters of 4
    const int64_t c = std::min(pl->cluster, 4);
    tickets = (bands + c - 1) / c;
  } else if (pair == SAT_32F_32F || pair == SAT_64F_64F || pair == SAT_32S_32S) {
    tickets = (std::min<int64_t>(bands, 223) + 3) / 4;  // clusters of 4 below 224 bands
    tickets = std::max<int64_t>(tickets, (bands + 7) / 8);
  } else {
    tickets = (bands + 3) / 4;  // byte pairs: clusters of 5, exclusive launches 4
  }
  // short-band launches (<= #SMs / 2 normal bands): 16-row bands in clusters of 4
  tickets = std::max<int64_t>(tickets, std::min<int64_t>((2 * bands + 3) / 4, (pl->num_sms + 3) / 4));
  pl->tickets_cap = tickets;
  const size_t payload_bytes = (size_t)tickets * pl->max_chunks * TW * (out_size(pair) / 4) * 8;
  // integer pairs: one read counter per tree node (= per payload vector)
  const size_t rd_bytes = (size_t)tickets * pl->max_chunks * 4;
  pl->payload_bytes = payload_bytes;
  pl->ws_bytes = 256 + payload_bytes + rd_bytes;
  sat_status st = configure(pl);
  if (st == SAT_OK) {
    e = cudaEventCreateWithFlags(&pl->last_ev, cudaEventDisableTiming);
    if (e != cudaSuccess) st = cuda_fail(e, "cudaEventCreate");
  }
  if (st == SAT_OK) {
    e = cudaMalloc(&pl->ws, pl->ws_bytes);
    if (e != cudaSuccess) st = cuda_fail(e, "cudaMalloc(workspace)");
  }
  if (st == SAT_OK) {
    e = cudaMemset(pl->ws, 0, pl->ws_bytes);
    if (e != cudaSuccess) st = cuda_fail(e, "cudaMemset(workspace)");
  }
  if (st != SAT_OK) {
    if (pl->ws) cudaFree(pl->ws);
    if (pl->last_ev) cudaEventDestroy(pl->last_ev);
    delete pl;
    cudaSetDevice(prev);
    return st;
  }
  pl->counter = reinterpret_cast<unsigned long long*>(pl->ws);
  pl->err = reinterpret_cast<uint32_t*>(static_cast<char*>(pl->ws) + 64);
  pl->payload = static_cast<char*>(pl->ws) + 256;
  pl->tree_rd = reinterpret_cast<uint32_t*>(static_cast<char*>(pl->ws) + 256 + payload_bytes);
  cudaSetDevice(prev);
  *plan = pl;
  return SAT_OK;
}

sat_status sat_plan_set_timeout(sat_plan plan, uint64_t ns) {
  if (!plan || ns == 0) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL plan or zero timeout");
  plan->spin_ns = ns;
  return SAT_OK;
}

sat_status sat_plan_set_carry(sat_plan plan, sat_carry mode) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (mode != SAT_CARRY_AUTO && mode != SAT_CARRY_LOOKBACK && mode != SAT_CARRY_TREE)
    return fail(SAT_ERR_INVALID_ARGUMENT, "unknown carry mode %d", (int)mode);
  const bool integer = plan->pair == SAT_8U_32S || plan->pair == SAT_32S_32S ||
                       plan->pair == SAT_8U_SQ || plan->pair == SAT_8U_HIST4;
  if (mode == SAT_CARRY_TREE && !integer)
    return fail(SAT_ERR_UNSUPPORTED, "the carry tree is for the integer pairs only");
  plan->tree_mode = mode == SAT_CARRY_AUTO ? -1 : mode == SAT_CARRY_TREE ? 1 : 0;
  return SAT_OK;
}

sat_status sat_plan_status(sat_plan plan, void* stream) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  uint32_t h = 0;
  cudaError_t e = cudaMemcpyAsync(&h, plan->err, 4, cudaMemcpyDeviceToHost, s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e == cudaSuccess && h != 0) e = cudaMemsetAsync(plan->err, 0, 4, s);
  // a timed-out launch may leave carry-tree nodes partly summed: clear the tree
  if (e == cudaSuccess && h != 0)
    e = cudaMemsetAsync(plan->payload, 0, plan->ws_bytes - ((char*)plan->payload - (char*)plan->ws), s);
  if (e == cudaSuccess) e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "sat_plan_status");
  if (h & 1u)
    return fail(SAT_ERR_TIMEOUT,
                "a carry wait exceeded the plan's timeout (a band / rank above never published); "
                "the affected output is wrong");
  return SAT_OK;
}

sat_status sat_plan_workspace_bytes(sat_plan plan, size_t* bytes) {
  if (!plan || !bytes) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL argument");
  *bytes = plan->ws_bytes;
  return SAT_OK;
}

sat_status sat_plan_destroy(sat_plan plan) {
  if (!plan) return SAT_OK;
  int prev = 0;
  cudaGetDevice(&prev);
  cudaSetDevice(plan->device);
  host_path_release(plan);
  if (plan->ws) cudaFree(plan->ws);
  if (plan->dist_scratch) cudaFree(plan->dist_scratch);
  if (plan->last_ev) cudaEventDestroy(plan->last_ev);
  cudaSetDevice(prev);
  delete plan;
  return SAT_OK;
}

sat_status sat_compute_batched(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                               int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                               int64_t in_image_stride_bytes, int64_t out_image_stride_bytes,
                               int64_t batch, sat_pair pair, void* stream) {
  bool empty = false;
  sat_status st = validate(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                           in_image_stride_bytes, out_image_stride_bytes, batch, pair, &empty);
  if (st != SAT_OK || empty) return st;
  DeviceGuard g(plan->device);
  return launch(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                batch > 1 ? in_image_stride_bytes : h * in_pitch_bytes,
                batch > 1 ? out_image_stride_bytes : h * out_pitch_bytes, batch, nullptr,
                static_cast<cudaStream_t>(stream));
}

}  // extern "C"

namespace {
// rows x cols block of one value (the exclusive layout's nVal border)
template <typename T>
__global__ void fill2d_kernel(char* out, int64_t rows, int64_t cols, int64_t pitch, T v) {
  const int64_t n = rows * cols;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n;
       i += (int64_t)gridDim.x * blockDim.x)
    reinterpret_cast<T*>(out + (i / cols) * pitch)[i % cols] = v;
}

sat_status fill2d(sat_pair pair, void* out, int64_t rows, int64_t cols, int64_t pitch,
                  uint64_t bits, cudaStream_t s) {
  if (rows <= 0 || cols <= 0) return SAT_OK;
  const int64_t n = rows * cols;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 4096);
  if (pair == SAT_64F_64F) {
    double v;
    memcpy(&v, &bits, 8);
    fill2d_kernel<double><<<grid, 256, 0, s>>>((char*)out, rows, cols, pitch, v);
  } else {
    uint32_t v = (uint32_t)bits;
    fill2d_kernel<uint32_t><<<grid, 256, 0, s>>>((char*)out, rows, cols, pitch, v);
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? SAT_OK : cuda_fail(e, "fill2d_kernel launch");
}
}  // namespace

extern "C" {

sat_status sat_compute_exclusive(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                                 int64_t in_pitch_bytes, int64_t out_pitch_bytes, int full,
                                 const void* nval, sat_pair pair, void* stream) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (pair != plan->pair)
    return fail(SAT_ERR_INVALID_ARGUMENT, "pair %d does not match the plan's pair %d", (int)pair,
                (int)plan->pair);
  if (h < 0 || w < 0) return fail(SAT_ERR_INVALID_ARGUMENT, "negative extent");
  if (full != 0 && full != 1) return fail(SAT_ERR_INVALID_ARGUMENT, "full must be 0 or 1");
  const int64_t sa = (int64_t)in_size(pair), sb = (int64_t)out_size(pair);
  const int64_t out_rows = full ? h + 1 : h, out_cols = full ? w + 1 : w;
  if (out_rows == 0 || out_cols == 0) return SAT_OK;
  if (!out) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL output pointer");
  if (out_pitch_bytes < out_cols * sb || out_pitch_bytes % sb != 0 || (uintptr_t)out % sb != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "output pitch %lld / alignment invalid for %lld columns",
                (long long)out_pitch_bytes, (long long)out_cols);
  uint64_t bits = 0;
  if (nval) memcpy(&bits, nval, (size_t)sb);
  const int64_t hk = full ? h : h - 1;  // input rows whose SAT lands in the output
  if (hk > 0 && w > 0) {
    if (!in) return fail(SAT_ERR_INVALID_ARGUMENT, "NULL input pointer");
    const size_t in_bytes = (size_t)((h - 1) * in_pitch_bytes + w * sa);
    const size_t out_bytes = (size_t)((out_rows - 1) * out_pitch_bytes + out_cols * sb);
    if (ranges_overlap(in, in_bytes, out, out_bytes))
      return fail(SAT_ERR_UNSUPPORTED, "input and output overlap (exclusive layout is never in place)");
  }
  DeviceGuard g(plan->device);
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  if (hk <= 0 || w == 0) {  // border only: every element is nVal
    return fill2d(pair, out, out_rows, out_cols, out_pitch_bytes, bits, s);
  }
  bool empty = false;
  char* out1 = static_cast<char*>(out) + out_pitch_bytes;
  sat_status st = validate(plan, in, out1, hk, w, in_pitch_bytes, out_pitch_bytes,
                           hk * in_pitch_bytes, hk * out_pitch_bytes, 1, pair, &empty);
  if (st != SAT_OK || empty) return st;
  st = fill2d(pair, out, 1, out_cols, out_pitch_bytes, bits, s);  // row 0
  if (st != SAT_OK) return st;
  const ExSpec ex{out_cols, bits};
  return launch(plan, in, out1, hk, w, in_pitch_bytes, out_pitch_bytes, hk * in_pitch_bytes,
                hk * out_pitch_bytes, 1, nullptr, s, &ex);
}

sat_status sat_compute_hist4(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                             int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                             int64_t in_image_stride_bytes, int64_t out_image_stride_bytes,
                             int64_t batch, const uint8_t* bin_of, int bin0, void* stream) {
  if (!plan) return fail(SAT_ERR_INVALID_ARGUMENT, "plan is NULL");
  if (plan->pair != SAT_8U_HIST4)
    return fail(SAT_ERR_INVALID_ARGUMENT, "sat_compute_hist4 needs a SAT_8U_HIST4 plan");
  if (!bin_of) return fail(SAT_ERR_INVALID_ARGUMENT, "bin table is NULL");
  bool empty = false;
  sat_status st = validate(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                           in_image_stride_bytes, out_image_stride_bytes, batch, SAT_8U_HIST4, &empty);
  if (st != SAT_OK || empty) return st;
  DeviceGuard g(plan->device);
  const HistSpec hs{bin_of, bin0};
  return launch(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                batch > 1 ? in_image_stride_bytes : h * in_pitch_bytes,
                batch > 1 ? out_image_stride_bytes : h * out_pitch_bytes, batch, nullptr,
                static_cast<cudaStream_t>(stream), nullptr, nullptr, &hs);
}

sat_status sat_compute(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                       int64_t in_pitch_bytes, int64_t out_pitch_bytes, sat_pair pair,
                       void* stream) {
  return sat_compute_batched(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                             h * in_pitch_bytes, h * out_pitch_bytes, 1, pair, stream);
}

sat_status sat_compute_band(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                            int64_t in_pitch_bytes, int64_t out_pitch_bytes, const void* carry_in,
                            sat_pair pair, void* stream) {
  bool empty = false;
  sat_status st = validate(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes,
                           h * in_pitch_bytes, h * out_pitch_bytes, 1, pair, &empty);
  if (st != SAT_OK || empty) return st;
  if (carry_in && (uintptr_t)carry_in % out_size(pair) != 0)
    return fail(SAT_ERR_INVALID_ARGUMENT, "carry_in not aligned to its element size");
  DeviceGuard g(plan->device);
  return launch(plan, in, out, h, w, in_pitch_bytes, out_pitch_bytes, h * in_pitch_bytes,
                h * out_pitch_bytes, 1, carry_in, static_cast<cudaStream_t>(stream));
}

}  // extern "C"
