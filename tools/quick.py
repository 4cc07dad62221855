"""Quick per-config timing used during development (not the bench contract)."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

CONFIGS = [(0, 16384, 16384, 1), (0, 8192, 8192, 1), (1, 16384, 16384, 1), (2, 16384, 16384, 1),
           (0, 1080, 1920, 1024), (1, 65536, 4096, 1), (0, 4096, 65536, 1)]
if os.environ.get("QUICK_CONFIGS"):  # e.g. "5:16384:16384:1,6:16384:16384:1"
    CONFIGS = [tuple(int(v) for v in c.split(":")) for c in os.environ["QUICK_CONFIGS"].split(",")]
IN_B = {0: 1, 1: 4, 2: 8, 3: 1, 4: 4, 5: 1, 6: 1}
OUT_B = {0: 4, 1: 4, 2: 8, 3: 4, 4: 4, 5: 8, 6: 16}
steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
for pair, H, W, N in CONFIGS:
    dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64, 3: torch.uint8, 4: torch.int32, 5: torch.uint8,
          6: torch.uint8}[pair]
    shape = (N, H, W) if N > 1 else (H, W)
    x = torch.empty(shape, dtype=dt, device="cuda")
    satgen.fill_device(x, seed=1)
    oshape = {5: (*shape, 2), 6: (1, *shape, 4)}.get(pair, shape)
    y = torch.empty(oshape, dtype=sat.out_dtype(pair), device="cuda")
    run = {5: lambda: sat.sat_sq(x, out=y), 6: lambda: sat.integral_histogram(x, bins=4, out=y),
           3: lambda: sat.sat(x, out=y, out_dtype=torch.float32)}.get(pair, lambda: sat.sat(x, out=y))
    for _ in range(2):
        run()
    torch.cuda.synchronize()
    ts = []
    for _ in range(steps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); run(); b.record(); torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    ms = statistics.median(ts)
    gbs = H * W * N * (IN_B[pair] + OUT_B[pair]) / ms / 1e6
    print(f"pair={pair} {N}x{H}x{W}: {ms:.4f} ms  {H*W*N/ms/1e6:.1f} Gpx/s  {gbs:.0f} GB/s  {gbs/6449.7:.3f} of peak", flush=True)
    del x, y
    torch.cuda.empty_cache()
