"""Does the pitch (power-of-two row strides) change the kernel's HBM rate?
Times sat() at one shape with dense and padded input / output pitches
(development tool).  usage: python tools/pitch_probe.py [PAIR:H:W ...]"""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

IN_B = {0: 1, 1: 4, 2: 8}
DT = {0: torch.uint8, 1: torch.float32, 2: torch.float64}
cfgs = sys.argv[1:] or ["0:16384:16384", "0:8192:8192", "1:16384:16384"]
for c in cfgs:
    pair, H, W = (int(v) for v in c.split(":"))
    for pin, pout in [(0, 0), (0, 128), (0, 512), (128, 0), (128, 128), (512, 512)]:
        xb = torch.empty(H, W + pin, dtype=DT[pair], device="cuda")
        x = xb[:, :W]
        satgen.fill_device(xb, seed=1)
        yb = torch.empty(H, W + pout, dtype=sat.out_dtype(pair), device="cuda")
        y = yb[:, :W]
        for _ in range(3):
            sat.sat(x, out=y)
        torch.cuda.synchronize()
        ts = []
        for _ in range(20):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(); sat.sat(x, out=y); b.record(); torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        ms = statistics.median(ts)
        gbs = H * W * (IN_B[pair] + 4 * (2 if pair == 2 else 1)) / ms / 1e6
        print(f"pair={pair} {H}x{W} pad_in={pin:4d} pad_out={pout:4d}: {ms:.4f} ms {gbs:7.0f} GB/s "
              f"{gbs / 6543.7:.3f} of peak", flush=True)
        del x, xb, y, yb
        torch.cuda.empty_cache()
