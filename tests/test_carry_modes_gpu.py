"""Both cross-cluster carry mechanisms of the integer pairs against the oracle:
the decoupled look-back and the counted reduction tree (sat_plan_set_carry,
include/libsat.h; Sec. IV-C carries between blocks).  Shapes
span many cluster tickets (tree depth >= 7 nodes per query at 9001 rows),
ragged edges, and batches whose clusters straddle image boundaries (several
whole images inside one cluster at 45 rows); 32s inputs cover the full u32
range so every node word's value bits wrap."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

pytestmark = pytest.mark.gpu

SHAPES = [(9001, 700, 1), (4099, 2311, 1), (1080, 900, 5), (45, 300, 40), (257, 129, 3),
          (16384, 256, 1)]


def _input(dt, shape, seed):
    if dt == torch.int32:
        g = torch.Generator(device="cuda").manual_seed(seed)
        return torch.randint(-2**31, 2**31 - 1, shape, dtype=torch.int32, device="cuda", generator=g)
    x = torch.empty(shape, dtype=dt, device="cuda")
    satgen.fill_device(x, seed=seed)
    return x


@pytest.mark.parametrize("mode", ["lookback", "tree", "auto"])
@pytest.mark.parametrize("dt", [torch.uint8, torch.int32])
@pytest.mark.parametrize("H,W,N", SHAPES)
def test_integer_sat_by_carry_mode(mode, dt, H, W, N):
    pair = sat.PAIR_8U_32S if dt == torch.uint8 else sat.PAIR_32S_32S
    plan = sat.Plan(pair, H, W, N)
    plan.set_carry(mode)
    shape = (N, H, W) if N > 1 else (H, W)
    x = _input(dt, shape, seed=H * 7 + W + N)
    for _ in range(2):  # the second launch finds the tree zeroed by the first
        y = sat.sat(x, plan=plan)
    torch.cuda.synchronize()
    plan.status()
    xs = x.cpu().numpy().reshape(N, H, W)
    ys = y.cpu().numpy().reshape(N, H, W)
    ref_of = oracle.sat if dt == torch.uint8 else oracle.sat_32s
    for n in range(N):
        ref = ref_of(np.ascontiguousarray(xs[n]))
        assert np.array_equal(ys[n], ref), f"image {n}"


@pytest.mark.parametrize("mode", ["lookback", "tree"])
def test_multichannel_by_carry_mode(mode):
    H, W = 3001, 777
    x = _input(torch.uint8, (H, W), seed=5)
    plan = sat.Plan(sat.PAIR_8U_SQ, H, W, 1)
    plan.set_carry(mode)
    y = sat.sat_sq(x, plan=plan).cpu().numpy()
    assert np.array_equal(y, oracle.sat_sq(x.cpu().numpy()))


def test_tree_refused_for_float_pairs():
    plan = sat.Plan(sat.PAIR_32F_32F, 64, 64, 1)
    with pytest.raises(sat.SatError):
        plan.set_carry("tree")
    plan.set_carry("lookback")
    plan.set_carry("auto")
