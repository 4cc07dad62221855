"""Time sat_compute over a list of shapes (development tool, not the bench contract).

usage: python tools/shape_scan.py PAIR HxWxN [HxWxN ...]   (PAIR 0 = 8u32s, 1 = 32f, 2 = 64f)
Env knobs of libsat (SAT_CLUSTER, SAT_FORCE_CLUSTERS, SAT_LIBRARY, ...) apply.
"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

IN_B = {0: 1, 1: 4, 2: 8}
OUT_B = {0: 4, 1: 4, 2: 8}
PEAK = 6527.5

pair = int(sys.argv[1])
steps = int(os.environ.get("STEPS", "15"))
dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64}[pair]
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for spec in sys.argv[2:]:
    parts = [int(v) for v in spec.split("x")]
    H, W = parts[0], parts[1]
    N = parts[2] if len(parts) > 2 else 1
    shape = (N, H, W) if N > 1 else (H, W)
    x = torch.empty(shape, dtype=dt, device="cuda")
    satgen.fill_device(x, seed=1)
    y = torch.empty(shape, dtype=sat.out_dtype(pair), device="cuda")
    for _ in range(3):
        sat.sat(x, out=y)
    torch.cuda.synchronize()
    small = H * W * N * (IN_B[pair] + OUT_B[pair]) < 4 * (126 << 20)
    ts = []
    for _ in range(steps):
        if small:
            flush.add_(1)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        sat.sat(x, out=y)
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = statistics.median(ts)
    gbs = H * W * N * (IN_B[pair] + OUT_B[pair]) / ms / 1e6
    print(f"pair={pair} {N}x{H}x{W}: {ms:.4f} ms (min {min(ts):.4f})  {H*W*N/ms/1e6:7.1f} Gpx/s  "
          f"{gbs:6.0f} GB/s  {gbs/PEAK:.3f} of peak", flush=True)
    del x, y
    torch.cuda.empty_cache()
