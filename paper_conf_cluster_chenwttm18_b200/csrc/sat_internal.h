// sat_internal.h -- private declarations shared by the libsat host runtime
// translation units (not part of the ABI).
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/libsat.h"

namespace sat {
struct HostPath;
}

struct sat_plan_st {
  int device = 0;
  sat_pair pair = SAT_8U_32S;
  int64_t max_h = 0, max_w = 0, max_batch = 0;
  int num_sms = 0;
  int active_clusters[7][3][4] = {};  // [pair][cluster 2/4/8][mode: bit0 TMA, bit1 vec out]
  int active_short[7] = {};           // [pair] short-band variant, clusters of 4, TMA + vec out
  int active_deep[7] = {};            // [pair] deep-ring variant (one CTA per SM), clusters of 4
  // Tuning / diagnosis knobs, read from the environment ONCE at plan creation
  // (SAT_FORCE_GENERIC, SAT_CLUSTER, SAT_SHORT, SAT_MAX_CLUSTERS,
  // SAT_FORCE_CLUSTERS, SAT_LOG); launches never consult the environment.
  int force_generic = 0;
  int cluster = 0;        // forced CTAs (bands) per cluster: 0 = by shape, else 2 / 4 / 8
  int short_bands = -1;   // -1 by shape, 0 / 1 forced
  int deep_ring = -1;     // SAT_DEEP: -1 by shape, 0 / 1 forced
  int max_clusters = 0, force_clusters = 0;
  int log = 0;
  int tree_mode = -1;     // SAT_TREE: integer-pair carries -1 by shape, 0 look-back, 1 tree
  int64_t max_tiles = 0;       // max_batch * bands * chunks of the plan limits (normal bands)
  int64_t tickets_cap = 0;     // cluster tickets the look-back payload holds at the plan's max width
  int64_t max_chunks = 0;
  void* ws = nullptr;
  size_t ws_bytes = 0;
  unsigned long long* counter = nullptr;  // ticket counter
  uint32_t* err = nullptr;                // device error word (bit 0: a bounded wait timed out)
  void* payload = nullptr;                // aggregate / inclusive carry vectors (integer
                                          // pairs: the counted reduction tree's nodes)
  size_t payload_bytes = 0;
  uint32_t* tree_rd = nullptr;            // tree node read counters [tickets][chunks]
  bool lookback_dirty = false;            // a look-back launch left tagged words in the payload
  uint64_t spin_ns = 2000000000ull;       // bounded-wait limit (sat_plan_set_timeout)
  uint32_t epoch = 0;
  uint64_t ticket_base = 0;
  uint64_t launches = 0;
  // Launch ordering across streams: the workspace is shared by every launch of
  // the plan, so a launch on a different stream first waits for the previous one.
  cudaEvent_t last_ev = nullptr;
  cudaStream_t last_stream = nullptr;
  bool has_last = false;
  // scratch of sat_dist_colsum / sat_dist_carry (lazily allocated, grown)
  void* dist_scratch = nullptr;
  size_t dist_scratch_bytes = 0;
  uint32_t dist_epoch = 0;  // tile-flag epoch of the one-kernel carry
  // streamed host path (lazily allocated)
  sat::HostPath* host = nullptr;
};

namespace sat {

sat_status fail(sat_status s, const char* fmt, ...);
sat_status cuda_fail(cudaError_t e, const char* what);
int getenv_int(const char* name, int dflt);
int cluster_index(int cl);
int default_cluster(int base_pair, int64_t bands);
size_t in_size(sat_pair p);
size_t out_size(sat_pair p);
int tile_w(sat_pair p);
int tile_h(sat_pair p);

sat_status validate(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w, int64_t ip,
                    int64_t op, int64_t iis, int64_t ois, int64_t batch, sat_pair pair,
                    bool* empty);
// Exclusive-layout output (sat_compute_exclusive): `out` points at output
// row 1; S(y, x) lands in column x + 1 (< out_cols); every value gets nVal.
struct ExSpec {
  int64_t out_cols;
  uint64_t nval_bits;
};
// Chained bands: per-chunk tagged carry vectors in (from the band above) and
// out (this band's bottom row, for the band below); see KParams.
struct ChainSpec {
  const void* in;        // this call's receive slot (band above publishes), or NULL
  void* out;             // the band below's receive slot, or NULL
  uint32_t* ack_out;     // the band above's ack words (written after reading `in`)
  const uint32_t* ack_in;  // this band's ack words (read before writing `out`)
  uint32_t epoch;
};
// Integral histogram (SAT_8U_HIST4): bin of every byte value, first bin of this launch.
struct HistSpec {
  const uint8_t* bin_of;  // 256 entries (host)
  int bin0;
};
sat_status launch(sat_plan_st* pl, const void* in, void* out, int64_t h, int64_t w, int64_t ip,
                  int64_t op, int64_t iis, int64_t ois, int64_t batch, const void* carry_in,
                  cudaStream_t stream, const ExSpec* ex = nullptr, const ChainSpec* chain = nullptr,
                  const HistSpec* hist = nullptr);
bool multi_channel(sat_pair p);
void host_path_release(sat_plan_st* pl);

struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
    else prev = -1;
  }
  ~DeviceGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

}  // namespace sat
