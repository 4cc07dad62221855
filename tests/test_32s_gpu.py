"""GPU parity of the 32s->32s pair (int32 in, int32 out, exact mod 2^32 --
reading R2): bit-exact against oracle.sat_32s on full-range signed inputs
(every sum wraps), across shapes, launch variants, batches, the exclusive
layout, the row-banded and chained multi-GPU building blocks and the
consumers."""
import numpy as np
import pytest

import oracle

pytestmark = pytest.mark.gpu


def _t():
    import torch
    return torch


def _sat():
    import paper_conf_cluster_chenwttm18_b200 as sat
    return sat


def _img(shape, seed):
    torch = _t()
    g = torch.Generator(device="cuda").manual_seed(seed)
    return torch.randint(-2**31, 2**31 - 1, shape, dtype=torch.int32, device="cuda", generator=g)


SHAPES = [(1, 1), (1, 300), (300, 1), (33, 129), (32, 128), (999, 1001), (1080, 1920), (2049, 4099)]


@pytest.mark.parametrize("shape", SHAPES)
def test_32s_parity(shape):
    torch, sat = _t(), _sat()
    x = _img(shape, 401)
    y = sat.sat(x)
    torch.cuda.synchronize()
    assert y.dtype == torch.int32
    assert np.array_equal(y.cpu().numpy(), oracle.sat_32s(x.cpu().numpy()))


@pytest.mark.parametrize("env", [{"SAT_CLUSTER": "5"}, {"SAT_CLUSTER": "8"}, {"SAT_SHORT": "1"},
                                 {"SAT_FORCE_GENERIC": "1"}])
def test_32s_launch_variants(monkeypatch, env):
    torch, sat = _t(), _sat()
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    x = _img((777, 2050), 402)
    y = sat.sat(x)
    torch.cuda.synchronize()
    assert np.array_equal(y.cpu().numpy(), oracle.sat_32s(x.cpu().numpy()))


def test_32s_batched_exclusive_and_consumers():
    torch, sat = _t(), _sat()
    x = _img((4, 100, 300), 403)
    y = sat.sat(x)
    torch.cuda.synchronize()
    xs = x.cpu().numpy()
    for i in range(4):
        assert np.array_equal(y[i].cpu().numpy(), oracle.sat_32s(xs[i]))
    J = sat.sat_exclusive(x[0], full=True, nval=-5)
    torch.cuda.synchronize()
    ref = np.zeros((101, 301), dtype=np.int64)
    ref[1:, 1:] = oracle.sat_32s(xs[0]).view(np.uint32)
    ref = ((ref - 5) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
    assert np.array_equal(J.cpu().numpy(), ref)
    r = torch.tensor([[0, 0, 100, 300], [10, 20, 50, 70], [99, 299, 100, 300]], dtype=torch.int32)
    got = sat.rect_sums(y[0], r.cuda()).cpu().numpy()
    for k, (a, b, c, d) in enumerate(r.tolist()):
        want = int(xs[0][a:c, b:d].astype(np.int64).sum()) & 0xFFFFFFFF
        assert int(got[k].view(np.uint32)) == want


def test_32s_dist_virtual_ranks_and_chain():
    torch, sat = _t(), _sat()
    H, W = 1001, 1999
    x = _img((H, W), 404)
    ref = oracle.sat_32s(x.cpu().numpy())
    P = 3
    spans = [sat.band_partition(H, P, r) for r in range(P)]
    gathered = torch.stack([sat.dist_colsum(x[a:b]) for a, b in spans])
    for r, (a, b) in enumerate(spans):
        carry = sat.dist_carry(gathered, r, sat.PAIR_32S_32S)
        y = sat.sat_band(x[a:b], carry_in=carry if r > 0 else None)
        torch.cuda.synchronize()
        assert np.array_equal(y.cpu().numpy(), ref[a:b]), f"colsum rank {r}"
    links = [sat.new_chain_buffer(sat.PAIR_32S_32S, W) for _ in range(P)]
    out = torch.empty((H, W), dtype=torch.int32, device="cuda")
    for r, (a, b) in enumerate(spans):
        sat.sat_band_chained(x[a:b], links[r], links[r - 1] if r > 0 else None,
                             links[r + 1] if r < P - 1 else None, 1, out=out[a:b])
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), ref)
