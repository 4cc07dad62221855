"""Same-box ablation: single-pass sat_compute vs the paper's
BRLT-ScanRow x 2 (two passes, transposed intermediate) at 16384^2 for 8u / 32f
/ 64f.  CUDA events, median of N runs; algorithmic bytes per pixel: single
pass sizeof(T_A)+sizeof(T_B), BRLT sizeof(T_A)+3 sizeof(T_B).  Prints one JSON
line per pair (development tool; results go to profiles/)."""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

N = int(os.environ.get("STEPS", "10"))
H = W = int(os.environ.get("SIZE", "16384"))
PEAK = 6543.7
for pair, dt, sa, sb in [(0, torch.uint8, 1, 4), (1, torch.float32, 4, 4), (2, torch.float64, 8, 8)]:
    x = torch.empty((H, W), dtype=dt, device="cuda")
    satgen.fill_device(x, seed=1001)
    y = torch.empty((H, W), dtype=sat.out_dtype(pair), device="cuda")
    tmp = torch.empty((W, H), dtype=sat.out_dtype(pair), device="cuda")

    def t(fn):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(N):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            fn()
            b.record()
            torch.cuda.synchronize()
            ts.append(a.elapsed_time(b))
        return statistics.median(ts)

    ms1 = t(lambda: sat.sat(x, out=y))
    ms2 = t(lambda: sat.sat_brlt(x, out=y, tmp=tmp))
    px = H * W
    print(json.dumps({"pair": sat.__dict__.get("PAIR_NAMES", {}).get(pair, pair), "H": H, "W": W,
                      "single_pass_ms": round(ms1, 4), "brlt_x2_ms": round(ms2, 4),
                      "speedup": round(ms2 / ms1, 2),
                      "single_pass_B_per_px": sa + sb, "brlt_B_per_px": sa + 3 * sb,
                      "single_pass_gbs": round(px * (sa + sb) / ms1 / 1e6, 1),
                      "brlt_gbs": round(px * (sa + 3 * sb) / ms2 / 1e6, 1),
                      "brlt_frac_of_peak": round(px * (sa + 3 * sb) / ms2 / 1e6 / PEAK, 3)}),
          flush=True)
    del x, y, tmp
    torch.cuda.empty_cache()
