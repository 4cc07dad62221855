"""Run a single SAT config a few times (for ncu captures)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

pair, H, W, N, reps = (int(v) for v in sys.argv[1:6])
dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64, 3: torch.uint8, 4: torch.int32,
      5: torch.uint8, 6: torch.uint8}[pair]
shape = (N, H, W) if N > 1 else (H, W)
x = torch.empty(shape, dtype=dt, device="cuda")
if pair == 4:
    x.random_(-2**31, 2**31 - 1)
else:
    satgen.fill_device(x, seed=1)
oshape = {5: (*shape, 2), 6: (1, *shape, 4)}.get(pair, shape)
y = torch.empty(oshape, dtype=sat.out_dtype(pair), device="cuda")
run = {5: lambda: sat.sat_sq(x, out=y), 6: lambda: sat.integral_histogram(x, bins=4, out=y)}.get(
    pair, lambda: sat.sat(x, out=y))
for _ in range(reps):
    run()
torch.cuda.synchronize()
