"""Small SATs for compute-sanitizer runs (memcheck / synccheck / racecheck):
every product kernel variant of round 2 on small shapes -- cluster sizes 5 / 4
/ 8, for 8u both carry mechanisms (look-back and the counted reduction tree)
-- results checked against the oracle (BAD 0 = all match)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

bad = 0


def chk(ok, what):
    global bad
    if not ok:
        bad += 1
        print("MISMATCH", what, flush=True)


PAIR = {torch.uint8: sat.PAIR_8U_32S, torch.float32: sat.PAIR_32F_32F, torch.float64: sat.PAIR_64F_64F}
for cl in ("5", "4", "8"):
    os.environ["SAT_CLUSTER"] = cl  # read at plan creation: one plan per cluster size
    for dt, H, W, N in [(torch.uint8, 300, 517, 1), (torch.float32, 200, 300, 1),
                        (torch.float64, 130, 129, 1), (torch.uint8, 70, 260, 3)]:
        # integer pairs: both cross-cluster carry mechanisms (look-back, tree)
        for mode in (("lookback", "tree") if dt == torch.uint8 else ("auto",)):
            shape = (N, H, W) if N > 1 else (H, W)
            plan = sat.Plan(PAIR[dt], H, W, N)
            plan.set_carry(mode)
            x = torch.empty(shape, dtype=dt, device="cuda")
            satgen.fill_device(x, seed=H)
            y = sat.sat(x, plan=plan).cpu().numpy().reshape(N, H, W)
            xs = x.cpu().numpy().reshape(N, H, W)
            for n in range(N):
                ref = oracle.sat(np.ascontiguousarray(xs[n]))
                ok = np.array_equal(y[n], ref) if dt == torch.uint8 else np.allclose(y[n], ref, rtol=1e-4)
                chk(ok, f"sat CL={cl} {mode} {dt} {shape}")
os.environ.pop("SAT_CLUSTER")
# multi-channel pairs
x = torch.empty((150, 333), dtype=torch.uint8, device="cuda")
satgen.fill_device(x, seed=5)
chk(np.array_equal(sat.sat_sq(x).cpu().numpy(), oracle.sat_sq(x.cpu().numpy())), "sat_sq")
hst = sat.integral_histogram(x, bins=8).cpu().numpy()
ref = oracle.integral_histogram(x.cpu().numpy(), np.arange(256) * 8 // 256, 8)
chk(np.array_equal(np.moveaxis(hst, 3, 1).reshape(-1, 150, 333), ref), "histogram")
# chained bands (links, 2 epochs)
P, H, W = 3, 300, 517
links = [sat.new_chain_buffer(0, W) for _ in range(P)]
out = torch.empty((H, W), dtype=torch.int32, device="cuda")
for ep in (1, 2):
    xe = torch.empty((H, W), dtype=torch.uint8, device="cuda")
    satgen.fill_device(xe, seed=40 + ep)
    for r in range(P):
        a, b = sat.band_partition(H, P, r)
        sat.sat_band_chained(xe[a:b], links[r], links[r - 1] if r else None,
                             links[r + 1] if r < P - 1 else None, ep, out=out[a:b])
    chk(np.array_equal(out.cpu().numpy(), oracle.sat(xe.cpu().numpy())), f"chained epoch {ep}")
# exclusive layout and the BRLT ablation
xf = torch.empty((90, 700), dtype=torch.float32, device="cuda")
satgen.fill_device(xf, seed=4)
chk(np.allclose(sat.sat_exclusive(xf).cpu().numpy(), oracle.sat_exclusive(xf.cpu().numpy()), rtol=1e-4),
    "exclusive")
chk(np.array_equal(sat.sat_brlt(x).cpu().numpy(), oracle.sat(x.cpu().numpy())), "brlt")
torch.cuda.synchronize()
print("BAD", bad)
