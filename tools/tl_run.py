"""Run one instrumented launch (a -DSAT_TIMELINE build selected with
SAT_LIBRARY) of a given config and dump its timeline to argv[2]
(development tool; analyse with tools/tl3.py / tools/tl_bands.py).

usage: SAT_LIBRARY=.../libsat_tl.so python tools/tl_run.py PAIR:H:W:N OUT.txt"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch

import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

pair, H, W, N = (int(v) for v in sys.argv[1].split(":"))
out_path = sys.argv[2]
dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64}[pair]
shape = (N, H, W) if N > 1 else (H, W)
x = torch.empty(shape, dtype=dt, device="cuda")
satgen.fill_device(x, seed=1)
y = torch.empty(shape, dtype=sat.out_dtype(pair), device="cuda")
os.environ.pop("SAT_TIMELINE_OUT", None)
for _ in range(3):
    sat.sat(x, out=y)
torch.cuda.synchronize()
if os.path.exists(out_path):
    os.remove(out_path)
os.environ["SAT_TIMELINE_OUT"] = out_path
sat.sat(x, out=y)
torch.cuda.synchronize()
print("timeline written to", out_path)
