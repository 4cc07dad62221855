"""Small SATs for compute-sanitizer runs (memcheck / synccheck / racecheck)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

bad = 0
for cl in ("1", "4", "8"):
    os.environ["SAT_CLUSTER"] = cl
    for dt, H, W, N in [(torch.uint8, 300, 517, 1), (torch.float32, 200, 300, 1),
                        (torch.float64, 130, 129, 1), (torch.uint8, 70, 260, 3)]:
        shape = (N, H, W) if N > 1 else (H, W)
        x = torch.empty(shape, dtype=dt, device="cuda")
        satgen.fill_device(x, seed=H)
        y = sat.sat(x).cpu().numpy().reshape(N, H, W)
        xs = x.cpu().numpy().reshape(N, H, W)
        for n in range(N):
            ref = oracle.sat(np.ascontiguousarray(xs[n]))
            ok = np.array_equal(y[n], ref) if dt == torch.uint8 else np.allclose(y[n], ref, rtol=1e-4)
            bad += 0 if ok else 1
print("BAD", bad)
