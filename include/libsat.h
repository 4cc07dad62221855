/* libsat.h -- C ABI of the B200-native summed-area-table library.
 *
 * Operation (Sec. III-A, Eq. 1; index reading R1 in DESIGN.md):
 * the 2D inclusive summed-area table (integral image)
 *
 *     S(i, j) = sum_{y <= i} sum_{x <= j} A(y, x),   0 <= i < h, 0 <= j < w,
 *
 * of a row-major pitched image A (h rows of w elements), for the paper's type
 * pairs T_A -> T_B (Sec. III-D):
 *     SAT_8U_32S  : uint8  -> int32, exact, two's-complement wrap mod 2^32 (R2)
 *     SAT_32F_32F : float  -> float  (accumulated in fp32; tolerance 1e-4 rel.)
 *     SAT_64F_64F : double -> double (accumulated in fp64; tolerance 1e-12 rel.)
 *     SAT_8U_32F  : uint8  -> float  (accumulated in fp32; tolerance 1e-4 rel.)
 *     SAT_32S_32S : int32  -> int32, exact, two's-complement wrap mod 2^32
 * (8u->32u is SAT_8U_32S's output read as uint32: the same bits mod 2^32.)
 * Output has the same h x w shape as the input (inclusive form).
 *
 * Conventions (all entry points):
 *  - Every call returns sat_status; no C++ exception crosses the ABI.  On a
 *    non-OK status, sat_last_error() returns a thread-local detail string.
 *  - Pointers `in`, `out`, `carry_in`, `in_band`, `out_band` are DEVICE
 *    pointers on the plan's device (except sat_compute_host, which takes HOST
 *    pointers).  The caller owns them; they must stay valid until the work
 *    queued on `stream` completes.
 *  - Pitches and strides are in BYTES, separately for input and output
 *    (NPP nSrcStep/nDstStep style, reading R8).  Any pitch that is a multiple
 *    of the element size and >= w * sizeof(T) is accepted; 16-byte aligned
 *    base/pitch/stride select the TMA-fed fast path, others a generic path.
 *  - Compute calls are asynchronous and stream-ordered: they validate
 *    synchronously, enqueue on `stream` (a cudaStream_t passed as void*;
 *    NULL = legacy default stream) and return without synchronising the host.
 *    Asynchronous device faults surface at the caller's next synchronisation.
 *  - A plan owns a workspace (look-back carry vectors, a ticket counter, an
 *    error word).  Launches of one plan are ordered: a launch on a stream
 *    other than the plan's previous one first waits (cudaStreamWaitEvent) for
 *    that launch, so two streams sharing a plan serialise instead of racing on
 *    the workspace.  Workspace is never re-zeroed per call: carry words carry a
 *    per-call epoch, and the carry tree's nodes are zeroed again by their last
 *    reader (after a timed-out launch sat_plan_status clears them).  Stream capture (CUDA graphs) of a compute call returns
 *    SAT_ERR_UNSUPPORTED (tickets and epochs are handed out per launch by the
 *    host).
 *  - Cross-CTA and cross-GPU carry waits are bounded (sat_plan_set_timeout,
 *    default 2 s): a wait that runs out (e.g. the band above in a chain never
 *    ran) lets the kernel finish with wrong values and records the event;
 *    sat_plan_status() then returns SAT_ERR_TIMEOUT.
 *  - h == 0 or w == 0 (or batch == 0) is SAT_OK and a no-op.
 *  - In-place (in == out, equal pitches/strides) is allowed for 32f/64f.
 *    Any other overlap of input and output ranges is SAT_ERR_UNSUPPORTED.
 *  - Validation failures return SAT_ERR_INVALID_ARGUMENT and launch nothing:
 *    NULL pointer with non-empty extent, negative h/w/batch, pitch smaller
 *    than w * sizeof(T) or not a multiple of sizeof(T), image stride smaller
 *    than h * pitch or not a multiple of sizeof(T), dims above the plan
 *    limits, `pair` different from the plan's pair.
 */
#ifndef LIBSAT_H
#define LIBSAT_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  SAT_OK = 0,
  SAT_ERR_INVALID_ARGUMENT = 1,
  SAT_ERR_UNSUPPORTED = 2,
  SAT_ERR_CUDA = 3,
  SAT_ERR_NCCL = 4,
  SAT_ERR_OUT_OF_MEMORY = 5,
  SAT_ERR_TIMEOUT = 6
} sat_status;

/* Type pairs T_A -> T_B.  SAT_8U_32F is NPP's second pair
 * (nppiIntegral_8u32f): uint8 input, float output accumulated in
 * fp32 (tolerance 1e-4 relative to the exact sum, as for 32f). */
/* Multi-channel pairs (SAT consumers that motivate the primitive):
 *   SAT_8U_SQ    : uint8 -> 2 x uint32 per pixel, interleaved (S, Q): S = the SAT
 *                  of A and Q = the SAT of A^2 (Viola-Jones variance
 *                  normalisation [2]), both exact mod 2^32 (reading R2), from ONE
 *                  read of A in ONE pass (1 + 8 bytes per pixel).  A rectangle sum
 *                  by four corners is exact when its true value is below
 *                  2^32: every window of A, and windows of A^2 up to 66051 pixels.
 *   SAT_8U_HIST4 : uint8 -> 4 x uint32 per pixel, interleaved: the integral
 *                  histogram ([34], [38]) of bins [bin0, bin0 + 4) for a byte-to-
 *                  bin table (sat_compute_hist4), counts exact mod 2^32.
 * Output pitches / strides are in bytes of these 8- / 16-byte elements.  These
 * pairs support sat_compute / sat_compute_batched (and sat_compute_hist4) only. */
typedef enum {
  SAT_8U_32S = 0, SAT_32F_32F = 1, SAT_64F_64F = 2, SAT_8U_32F = 3, SAT_32S_32S = 4,
  SAT_8U_SQ = 5, SAT_8U_HIST4 = 6
} sat_pair;

typedef struct sat_plan_st* sat_plan;
typedef struct sat_comm_st* sat_comm;

/* Library version as major*10000 + minor*100 + patch. */
int sat_version(void);

/* Create a plan for `pair` on CUDA device `device`, sized for images up to
 * max_h x max_w and batches up to max_batch (all >= 1).  Allocates the
 * workspace on that device (see sat_plan_workspace_bytes).  *plan receives
 * the handle; on failure *plan is NULL.
 * Errors: INVALID_ARGUMENT (NULL plan, bad pair, non-positive limits),
 * CUDA (no such device / not sm_100), OUT_OF_MEMORY. */
sat_status sat_plan_create(sat_plan* plan, int device, sat_pair pair, int64_t max_h, int64_t max_w,
                           int64_t max_batch);

/* Bytes of device workspace owned by the plan. */
sat_status sat_plan_workspace_bytes(sat_plan plan, size_t* bytes);

/* Bound (ns, > 0) on every cross-CTA / cross-GPU carry wait of later launches
 * of `plan` (default 2e9).  Errors: INVALID_ARGUMENT (NULL plan, ns == 0). */
sat_status sat_plan_set_timeout(sat_plan plan, uint64_t ns);

/* Cross-cluster vertical carry of the integer pairs (8u->32s, 32s->32s,
 * 8u->(S,S^2), integral histogram) -- V_up(x) = S(r0-1, x) of a cluster's
 * first band, PAPER.md:258-260 (Sec. IV-C, the carries between blocks).
 *  SAT_CARRY_LOOKBACK  decoupled look-back over epoch-tagged aggregate /
 *                      inclusive vectors (the float pairs always use it);
 *  SAT_CARRY_TREE      counted reduction tree: each cluster adds its column
 *                      totals into the Fenwick nodes above it with TMA bulk
 *                      reductions, a reader sums <= log2(D) complete nodes
 *                      (exact: wrap-around integer adds commute);
 *  SAT_CARRY_AUTO      per launch by shape (default; the tree for images of
 *                      <= 64 bands and launches of <= one wave of bands).
 * The initial mode comes from the environment variable SAT_TREE (-1/0/1) read
 * at plan creation.  Applies to later launches of `plan`.
 * Errors: INVALID_ARGUMENT (NULL plan, unknown mode), UNSUPPORTED (TREE on a
 * float pair). */
typedef enum { SAT_CARRY_AUTO = 0, SAT_CARRY_LOOKBACK = 1, SAT_CARRY_TREE = 2 } sat_carry;
sat_status sat_plan_set_carry(sat_plan plan, sat_carry mode);

/* Synchronises `stream` and reports (then clears) the plan's device error
 * word: SAT_ERR_TIMEOUT if a bounded carry wait of an earlier launch ran out
 * (that launch's output is wrong), SAT_OK otherwise; CUDA on a device fault. */
sat_status sat_plan_status(sat_plan plan, void* stream);

/* Free the plan and its workspace (and host-path staging buffers).  The caller
 * must ensure no work using the plan is still pending.  NULL is a no-op. */
sat_status sat_plan_destroy(sat_plan plan);

/* SAT of one h x w image: out = S(in).  One kernel launch (single HBM pass:
 * each input byte read once, each output byte written once). */
sat_status sat_compute(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                       int64_t in_pitch_bytes, int64_t out_pitch_bytes, sat_pair pair, void* stream);

/* SAT of `batch` independent images; image n starts at in + n*in_image_stride_bytes
 * (resp. out + n*out_image_stride_bytes).  Carries never cross images. */
sat_status sat_compute_batched(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                               int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                               int64_t in_image_stride_bytes, int64_t out_image_stride_bytes,
                               int64_t batch, sat_pair pair, void* stream);

/* Integral histogram, four bins per call (SAT_8U_HIST4 plans; PAPER.md:22,
 * [34], [38]): out(y, x, k) = #{ (y', x') : y' <= y, x' <= x,
 * bin_of[A(y', x')] == bin0 + k } for k < 4, uint32, interleaved per pixel
 * (16 bytes).  bin_of: 256 entries, HOST memory (copied into the launch);
 * values outside [bin0, bin0 + 4) are not counted.  K bins = ceil(K / 4)
 * calls, each one pass (1 + 16 bytes per pixel).  Batches as
 * sat_compute_batched.  Errors as sat_compute_batched; INVALID_ARGUMENT for
 * a NULL table or a plan of another pair. */
sat_status sat_compute_hist4(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                             int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                             int64_t in_image_stride_bytes, int64_t out_image_stride_bytes,
                             int64_t batch, const uint8_t* bin_of, int bin0, void* stream);

/* SAT of a row band with a carry-in row: out(i, j) = carry_in[j] + S_band(i, j),
 * where carry_in (device, w elements of T_B, contiguous) is the SAT row just
 * above the band, S(r0 - 1, .).  carry_in == NULL means zeros (== sat_compute).
 * This is the building block of the streamed host path and of the row-banded
 * multi-GPU path. */
sat_status sat_compute_band(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                            int64_t in_pitch_bytes, int64_t out_pitch_bytes, const void* carry_in,
                            sat_pair pair, void* stream);

/* End-to-end SAT of a HOST image into a HOST output (pinned memory
 * recommended).  The image is streamed through the device in row bands:
 * host->device copy, sat_compute_band with the previous band's last output
 * row as carry-in, device->host copy, overlapped on internal streams.  All
 * work is ordered after prior work on `stream`, and `stream` is made to wait
 * for its completion; synchronise `stream` before reading `out`.
 * Device staging buffers are allocated lazily and owned by the plan. */
sat_status sat_compute_host(sat_plan plan, const void* in_host, void* out_host, int64_t h,
                            int64_t w, int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                            sat_pair pair, void* stream);

/* Exclusive SAT (Eq. 2) with NPP's offset nVal
 * (nppiIntegral: pDst(j,i) = nVal + sum_{l<j} sum_{k<i}
 * pSrc(l,k)):
 *   J(y, x) = nVal                                   if x == 0 or y == 0
 *   J(y, x) = nVal + sum_{j<y} sum_{i<x} A(j, i)     otherwise.
 * full = 1: the (h+1) x (w+1) layout of NPP / OpenCV (last row and column
 *           hold the totals) -- a drop-in nppiIntegral_8u32s_C1R replacement
 *           for 8u->32s (in-place forbidden: J is shifted by one row/column);
 * full = 0: Eq. 2 as printed, an h x w output (the full layout cropped).
 * `out` (device) has out_pitch_bytes >= (w + full) * sizeof(T_B); nval points
 * to ONE host value of T_B (int32 / float / double), NULL means 0.  The first
 * row is filled by a small kernel, every other element by the single-pass SAT
 * kernel, which stores S(y, x) at (y + 1, x + 1) with 16-byte aligned vector
 * stores when `out` and the pitch are 16-byte aligned.  Asynchronous on
 * `stream`; validation as sat_compute, plus SAT_ERR_UNSUPPORTED on any
 * overlap of input and output.  h == 0 or w == 0 fills the border (full) or
 * is a no-op (Eq. 2). */
sat_status sat_compute_exclusive(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                                 int64_t in_pitch_bytes, int64_t out_pitch_bytes, int full,
                                 const void* nval, sat_pair pair, void* stream);

/* ---------------------------------------------------------------------------
 * SAT consumers: O(1) rectangle sums from an
 * inclusive SAT by the four-corner identity (motivation
 * PAPER.md:18-24).  `sat` is a device SAT as written by sat_compute (T_B
 * elements, sat_pitch_bytes per row).  For 8u->32s the SAT holds the sums
 * mod 2^32 and so do the results: exact whenever the rectangle's true sum is
 * below 2^32, even where the SAT itself wrapped. */

/* n rectangle sums.  rects: device int32[n][4] = {y0, x0, y1, x1} (16-byte
 * aligned), the half-open rectangle [y0, y1) x [x0, x1) of the image;
 * coordinates are clamped to [0, h] / [0, w] and an empty rectangle sums to 0.
 * out: device T_B[n]; for the multi-channel SATs (SAT_8U_SQ, SAT_8U_HIST4)
 * uint32[n][K] (K = 2: sum of A, sum of A^2 -- a window's variance is
 * Q/n - (S/n)^2; K = 4: the window's 4 bin counts). */
sat_status sat_rect_sums(sat_plan plan, const void* sat, int64_t h, int64_t w,
                         int64_t sat_pitch_bytes, const void* rects, int64_t n, void* out,
                         sat_pair pair, void* stream);

/* Box filter (box sum): out(y, x) = sum of A over [y-ry, y+ry] x [x-rx, x+rx]
 * clipped to the image, for every pixel; out is h x w of T_B (device, must not
 * overlap the SAT).  ry, rx >= 0.  Single-channel SATs only. */
sat_status sat_box_filter(sat_plan plan, const void* sat, void* out, int64_t h, int64_t w,
                          int64_t sat_pitch_bytes, int64_t out_pitch_bytes, int64_t ry,
                          int64_t rx, sat_pair pair, void* stream);

/* ---------------------------------------------------------------------------
 * Multi-GPU (one process per GPU, NCCL over NVLink/NVSwitch).
 * NCCL is loaded at run time (dlopen "libnccl.so.2"; the copy torch already
 * loaded is reused).  Errors from NCCL map to SAT_ERR_NCCL.
 */

/* Rows [*r0, *r1) of rank `rank` when h rows are split over nranks bands in
 * rank order: the first h mod nranks ranks get one extra row (reading R14).
 * Host-only arithmetic (no device needed).  Errors: INVALID_ARGUMENT. */
sat_status sat_band_partition(int64_t h, int nranks, int rank, int64_t* r0, int64_t* r1);

/* Bytes of an NCCL unique id (NCCL_UNIQUE_ID_BYTES). */
#define SAT_COMM_ID_BYTES 128

/* Rank 0 creates the id (SAT_COMM_ID_BYTES bytes at id_out) and broadcasts it
 * out of band (e.g. torch.distributed.broadcast). */
sat_status sat_comm_unique_id(void* id_out);

/* Collective over nranks processes: create the communicator of `rank` on
 * CUDA device `device`. */
sat_status sat_comm_create(sat_comm* comm, const void* id, int nranks, int rank, int device);

sat_status sat_comm_destroy(sat_comm comm);

/* Row-banded SAT of one image of height sum_r band_h_r distributed over the
 * communicator's ranks in rank order: rank r holds rows [r0, r0 + band_h) in
 * in_band / out_band (device, pitched).  Each rank reduces its band's column
 * totals, the W-vectors are all-gathered over NCCL, the exclusive prefix over
 * lower ranks is scanned horizontally into the carry-in row S(r0 - 1, .), and
 * the band SAT is computed with that carry-in.  All
 * ranks must call it collectively with the same w and pair; band_h may differ
 * per rank (0 allowed).  Ordered on `stream`. */
sat_status sat_compute_dist(sat_plan plan, sat_comm comm, const void* in_band, void* out_band,
                            int64_t band_h, int64_t w, int64_t in_pitch_bytes,
                            int64_t out_pitch_bytes, sat_pair pair, void* stream);

/* ---------------------------------------------------------------------------
 * Chained row bands: the single-pass multi-GPU path (
 * the paper motivates horizontal scaling but stays on one node).
 * Instead of a column-sum pre-pass and an all-gather, the kernel of band r
 * publishes its bottom row S(r1-1, .) chunk by chunk (epoch-tagged 64-bit
 * words, the look-back payload format) straight into the LINK of band r+1 --
 * on another GPU through peer memory -- whose top clusters wait for each
 * chunk's vector as the carry-in of their first band (Eq. 1 split at row r0:
 * S(y, x) = S(r0-1, x) + SAT of rows [r0, y]).  Bands are read once and
 * written once (sizeof(T_A) + sizeof(T_B) bytes per pixel) and overlap chunk
 * by chunk.
 *
 * A link (owned by band r, sat_chain_bytes(pair, w) bytes, zero before first
 * use, 256-byte aligned) holds ack words [nchunks] -- written by band r+1 --
 * and two receive slots -- written by band r-1.  A call with epoch e uses
 * slot e & 1; the band above writes a chunk of slot e & 1 only after band r
 * has acknowledged epoch e - 2 of that chunk, so successive calls need no
 * host or NCCL barrier: flow control is on the device.  Epochs: one value per
 * chained SAT, the same on every band, 1, 2, 3, ... (< 2^30); restarting at 1
 * needs zeroed links.  Waits are bounded by the plan timeout (SAT_ERR_TIMEOUT
 * via sat_plan_status). */

/* Bytes of one chain link for rows of width w (0 for a bad pair / w <= 0). */
size_t sat_chain_bytes(sat_pair pair, int64_t w);

/* Allocate (cudaMalloc, so it can be exported over CUDA IPC) and zero one link
 * on `device`; sat_chain_link_destroy frees it. */
sat_status sat_chain_link_create(int device, sat_pair pair, int64_t w, void** link);
sat_status sat_chain_link_destroy(void* link);

/* Bytes of a CUDA IPC memory handle (CUDA_IPC_HANDLE_SIZE). */
#define SAT_IPC_HANDLE_BYTES 64

/* Export a link created by sat_chain_link_create to another process
 * (SAT_IPC_HANDLE_BYTES at handle_out; ship them over any transport, e.g. a
 * torch process group), and map a peer's link into this process on `device`
 * (peer access: NVLink between GPUs, or the same GPU).  Close with
 * sat_chain_close_peer. */
sat_status sat_chain_ipc_handle(const void* link, void* handle_out);
sat_status sat_chain_open_peer(int device, const void* handle, void** peer_link);
sat_status sat_chain_close_peer(void* peer_link);

/* One band of a chain.  link_self: this band's link (required when it has a
 * neighbour); link_above: the link of the band above (NULL for the top band)
 * -- the carry-in comes from link_self's slot, the acknowledgement goes to
 * link_above; link_below: the link of the band below (NULL for the bottom
 * band) -- the bottom row goes into its slot, after link_self's ack words
 * allow it.  Device or peer-mapped pointers.  The band above must run
 * earlier or concurrently (a band waits in its kernel for its carry-in).
 * h, w >= 1. */
sat_status sat_compute_band_chained(sat_plan plan, const void* in, void* out, int64_t h, int64_t w,
                                    int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                                    void* link_self, void* link_above, void* link_below,
                                    uint32_t epoch, sat_pair pair, void* stream);

/* Collective convenience over a sat_comm: rank r holds rows
 * [sum_{r'<r} band_h_r', +band_h) (every band >= 1 row).  Links are created
 * and their IPC handles all-gathered over NCCL once per width; every call is
 * then ONE kernel per rank (epochs counted by the comm, no collective). */
sat_status sat_compute_dist_chained(sat_plan plan, sat_comm comm, const void* in_band,
                                    void* out_band, int64_t band_h, int64_t w,
                                    int64_t in_pitch_bytes, int64_t out_pitch_bytes, sat_pair pair,
                                    void* stream);

/* Building blocks of sat_compute_dist (steps 1 and 3), exported so the carry
 * algebra can be exercised without NCCL (e.g. "virtual ranks" on one GPU).
 * Accumulator type: uint32 for SAT_8U_32S (exact mod 2^32), double
 * (compensated sums) for the float pairs; sat_dist_acc_bytes gives its size. */
size_t sat_dist_acc_bytes(sat_pair pair);

/* acc_out[x] = sum_{y < band_h} in_band(y, x) for x < w (device, w accumulators). */
sat_status sat_dist_colsum(sat_plan plan, const void* in_band, int64_t band_h, int64_t w,
                           int64_t in_pitch_bytes, void* acc_out, void* stream);

/* carry_out[x] = sum_{x' <= x} sum_{r < rank} gathered[r][x'] rounded once to
 * T_B, i.e. the row S(r0 - 1, .) above rank `rank`'s band.  gathered is
 * [nranks][w] accumulators (device), carry_out w elements of T_B (device). */
sat_status sat_dist_carry(sat_plan plan, const void* gathered, int nranks, int rank, int64_t w,
                          void* carry_out, void* stream);

/* ---------------------------------------------------------------------------
 * ABLATION, not the product path: the paper's fastest
 * method, Register-based BRLT-ScanRow run twice (Sec. IV-B;
 * Alg. 5), ported to sm_100a so the single-pass kernel's
 * saving can be measured on the same box.  Pass 1 writes the transposed row
 * prefixes of `in` into `tmp` (w x h, T_B, tmp_pitch_bytes per row of h
 * elements), pass 2 those of tmp into `out` (h x w): the inclusive SAT, for
 * SAT_8U_32S / SAT_32F_32F / SAT_64F_64F, at sizeof(T_A) + 3 sizeof(T_B)
 * bytes per pixel.  Device pointers; stream-ordered. */
sat_status sat_compute_brlt(sat_pair pair, const void* in, void* out, void* tmp, int64_t h,
                            int64_t w, int64_t in_pitch_bytes, int64_t out_pitch_bytes,
                            int64_t tmp_pitch_bytes, void* stream);

/* Static description of a status code. */
const char* sat_status_string(sat_status s);

/* Thread-local detail for the last non-OK status returned on this thread. */
const char* sat_last_error(void);

#ifdef __cplusplus
}
#endif

#endif /* LIBSAT_H */
