"""Per-rank work of the two row-banded multi-GPU schemes, measured on ONE GPU
with virtual ranks (development tool).

For P ranks over one H x W image, each rank's device work is timed alone with
CUDA events (the ranks of a real run execute it concurrently on P GPUs):

  colsum scheme (sat_compute_dist):  column sums of the band (reads the band),
                                     carry row from the gathered sums, band SAT
                                     with the carry fused  -> (2 sa + sb) B/px
  chained scheme (N1):               band SAT whose top clusters take the band
                                     above's bottom row from a chain buffer
                                     -> (sa + sb) B/px

The NCCL all-gather (P x W x 8 bytes, ~10-20 us over NVLink) and the chained
scheme's pipeline fill (band r starts chunk c once band r-1 published it) are
not in these numbers.  Prints one JSON object.

    python tools/dist_model.py [PAIR H W P...]    (default: 1 65536 65536 2 4 8)
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

IN_B = {0: 1, 1: 4, 2: 8}
OUT_B = {0: 4, 1: 4, 2: 8}


def ev_time(fn, reps=5):
    fn()
    torch.cuda.synchronize()
    best = float("inf")
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b))
    return best


def main():
    args = [int(v) for v in sys.argv[1:]]
    pair, H, W = (args[:3] if len(args) >= 3 else [1, 65536, 65536])
    Ps = args[3:] or [2, 4, 8]
    dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64}[pair]
    x = torch.empty((H, W), dtype=dt, device="cuda")
    satgen.fill_device(x, seed=1004)
    out = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    full_ms = ev_time(lambda: sat.sat(x, out=out))
    res = {"pair": pair, "H": H, "W": W, "single_gpu_ms": full_ms, "ranks": []}
    for P in Ps:
        spans = [sat.band_partition(H, P, r) for r in range(P)]
        gathered = torch.stack([sat.dist_colsum(x[a:b]) for a, b in spans])
        links = [sat.new_chain_buffer(pair, W) for _ in range(P)]
        for r in range(P - 1):  # fill the links once (epoch 1) so band r sees its carry
            a, b = spans[r]
            sat.sat_band_chained(x[a:b], links[r], links[r - 1] if r > 0 else None, links[r + 1], 1,
                                 out=out[a:b])
        colsum_ms, chained_ms = [], []
        for r, (a, b) in enumerate(spans):
            def colsum_rank():
                sat.dist_colsum(x[a:b])
                c = sat.dist_carry(gathered, r, pair)
                sat.sat_band(x[a:b], carry_in=c if r > 0 else None, out=out[a:b])

            def chained_rank():
                # the band below is NOT written (None): only band r's own device work
                sat.sat_band_chained(x[a:b], links[r], links[r - 1] if r > 0 else None, None, 1,
                                     out=out[a:b])

            colsum_ms.append(ev_time(colsum_rank))
            if r == P - 1:
                parts = {"colsum": ev_time(lambda: sat.dist_colsum(x[a:b])),
                         "carry": ev_time(lambda: sat.dist_carry(gathered, r, pair)),
                         "band_sat": ev_time(lambda: sat.sat_band(x[a:b], carry_in=gathered[0, :W].to(out.dtype) if False else None, out=out[a:b]))}
            chained_ms.append(ev_time(chained_rank))
        px = H * W
        res["ranks"].append({
            "P": P, "colsum_max_rank_ms": max(colsum_ms), "chained_max_rank_ms": max(chained_ms),
            "colsum_gpx_s_model": px / max(colsum_ms) / 1e6,
            "chained_gpx_s_model": px / max(chained_ms) / 1e6,
            "colsum_bytes_per_px": 2 * IN_B[pair] + OUT_B[pair],
            "chained_bytes_per_px": IN_B[pair] + OUT_B[pair], "last_rank_parts_ms": parts})
    print(json.dumps(res))


if __name__ == "__main__":
    main()
