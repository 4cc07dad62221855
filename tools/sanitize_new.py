"""Small runs of the session-3 entry points for compute-sanitizer
(exclusive layout, short-band kernels, chained bands, consumers, 8u->32f,
32s->32s, dist carry kernels); every result checked against the oracle."""
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


x8 = torch.empty((300, 517), dtype=torch.uint8, device="cuda")
satgen.fill_device(x8, seed=3)
A8 = x8.cpu().numpy()
# exclusive, both layouts, vector and scalar stores
for full in (True, False):
    J = sat.sat_exclusive(x8, full=full, nval=5)
    chk(np.array_equal(J.cpu().numpy(), oracle.sat_exclusive(A8, full=full, nval=5)), f"exclusive {full}")
big = torch.zeros((310, 530), dtype=torch.int32, device="cuda")
sat.sat_exclusive(x8, full=True, out=big[1:302, 1:519])
chk(np.array_equal(big[1:302, 1:519].cpu().numpy(), oracle.sat_exclusive(A8, full=True)), "exclusive unaligned")
# short-band kernels
os.environ["SAT_SHORT"] = "1"
chk(np.array_equal(sat.sat(x8).cpu().numpy(), oracle.sat(A8)), "short 8u")
xf = torch.empty((90, 700), dtype=torch.float64, device="cuda")
satgen.fill_device(xf, seed=4)
chk(np.allclose(sat.sat(xf).cpu().numpy(), oracle.sat(xf.cpu().numpy()), rtol=1e-12), "short 64f")
os.environ["SAT_SHORT"] = "0"
# chained bands
P, H, W = 3, 300, 517
links = [sat.new_chain_buffer(0, W) for _ in range(P)]
out = torch.empty((H, W), dtype=torch.int32, device="cuda")
for r in range(P):
    a, b = sat.band_partition(H, P, r)
    sat.sat_band_chained(x8[a:b], links[r], links[r - 1] if r else None,
                         links[r + 1] if r < P - 1 else None, 1, out=out[a:b])
chk(np.array_equal(out.cpu().numpy(), oracle.sat(A8)), "chained")
# dist carry kernels (virtual ranks)
spans = [sat.band_partition(H, P, r) for r in range(P)]
g = torch.stack([sat.dist_colsum(x8[a:b]) for a, b in spans])
for r, (a, b) in enumerate(spans):
    c = sat.dist_carry(g, r, 0)
    y = sat.sat_band(x8[a:b], carry_in=c if r else None)
    chk(np.array_equal(y.cpu().numpy(), oracle.sat(A8)[a:b]), f"dist rank {r}")
# consumers
S = sat.sat(x8)
chk(np.array_equal(sat.box_filter(S, 2, 3).cpu().numpy(), oracle.box_filter(A8, 2, 3)), "box")
rects = torch.tensor([[0, 0, 300, 517], [5, 6, 50, 60], [-3, 400, 10, 900]], dtype=torch.int32)
chk(np.array_equal(sat.rect_sums(S, rects.cuda()).cpu().numpy(), oracle.rect_sums(A8, rects.numpy())), "rects")
# 8u->32f and 32s->32s
F = sat.sat(x8, out_dtype=torch.float32)
chk(np.allclose(F.cpu().numpy(), oracle.sat_8u32f(A8), rtol=1e-4), "8u32f")
xi = torch.randint(-2**31, 2**31 - 1, (120, 300), dtype=torch.int32, device="cuda")
chk(np.array_equal(sat.sat(xi).cpu().numpy(), oracle.sat_32s(xi.cpu().numpy())), "32s")
torch.cuda.synchronize()
print("BAD", bad)
