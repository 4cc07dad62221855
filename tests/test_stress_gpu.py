"""Carry stress: the -DSAT_DEBUG_DELAY build sleeps a pseudo-random 0..4 us
before every carry publication, look-back round, tree update / query round and
DSMEM hand-off, so late predecessors, half-summed tree nodes, mixed
aggregate/inclusive windows and retries all occur (40 two-band frames put
several whole images in one cluster).  Both cross-cluster carry mechanisms run:
the decoupled look-back (SAT_TREE=0) and, for the integer pairs, the counted
reduction tree (SAT_TREE=1).  Run in a subprocess (the library is chosen at
import through SAT_LIBRARY)."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
DELAY_LIB = os.path.join(ROOT, "paper_conf_cluster_chenwttm18_b200", "libsat_delay.so")
# the look-back variant that reads payload words with per-lane ld.relaxed.gpu
# (8-byte single-copy atomicity guaranteed by PTX) instead of bulk copies
LDG_LIB = os.path.join(ROOT, "paper_conf_cluster_chenwttm18_b200", "libsat_delay_ldg.so")

SCRIPT = r'''
import numpy as np, torch, sys
sys.path.insert(0, sys.argv[1])
import oracle, satgen
import paper_conf_cluster_chenwttm18_b200 as sat
assert "libsat_delay" in sat.LIB_PATH, sat.LIB_PATH
bad = 0
for (dt, H, W, N) in [(torch.uint8, 4099, 2311, 1), (torch.float32, 2500, 3000, 1),
                      (torch.float64, 1800, 1700, 1), (torch.uint8, 1080, 900, 5),
                      (torch.uint8, 9001, 700, 1), (torch.float32, 8200, 500, 1),
                      (torch.uint8, 45, 300, 40)]:
    shape = (N, H, W) if N > 1 else (H, W)
    x = torch.empty(shape, dtype=dt, device="cuda")
    satgen.fill_device(x, seed=H + W)
    for rep in range(3):
        y = sat.sat(x).cpu().numpy()
        xs = x.cpu().numpy().reshape(N, H, W)
        ys = y.reshape(N, H, W)
        for n in range(N):
            ref = oracle.sat(np.ascontiguousarray(xs[n]))
            if dt == torch.uint8:
                ok = np.array_equal(ys[n], ref)
            else:
                tol = 1e-4 if dt == torch.float32 else 1e-12
                nz = ref != 0
                ok = np.all(np.abs(ys[n][nz] - ref[nz]) / np.abs(ref[nz]) <= tol)
            bad += 0 if ok else 1
print("BAD", bad)
'''


@pytest.mark.parametrize("cluster,tree", [("5", "0"), ("5", "1"), ("4", "0"), ("4", "1"),
                                          ("8", "-1")])
def test_carries_under_injected_delays(cluster, tree):
    if not os.path.exists(DELAY_LIB):
        pytest.skip("libsat_delay.so not built")
    env = dict(os.environ, SAT_LIBRARY=DELAY_LIB, SAT_CLUSTER=cluster, SAT_TREE=tree)
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], env=env, capture_output=True,
                         text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    assert "BAD 0" in out.stdout, out.stdout[-2000:]


@pytest.mark.parametrize("cluster,tree", [("5", "0"), ("4", "0"), ("5", "1")])
def test_carries_ldg_variant_under_injected_delays(cluster, tree):
    """The same stress on the SAT_LB_LDG=1 build (look-back words and tree node
    words read with ld.relaxed.gpu -- the variant whose per-word atomicity PTX
    guarantees)."""
    if not os.path.exists(LDG_LIB):
        pytest.skip("libsat_delay_ldg.so not built")
    env = dict(os.environ, SAT_LIBRARY=LDG_LIB, SAT_CLUSTER=cluster, SAT_TREE=tree)
    out = subprocess.run([sys.executable, "-c", SCRIPT, ROOT], env=env, capture_output=True,
                         text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-2000:]
    assert "BAD 0" in out.stdout, out.stdout[-2000:]
