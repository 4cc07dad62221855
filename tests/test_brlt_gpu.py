"""The BRLT-ScanRow x 2 ablation (PAPER.md:248-254,
Alg. 5): the paper's fastest method ported to sm_100a, kept beside the
single-pass kernel for the same-box comparison.  Parity with the oracle at the
same bars as the product path (bit-exact 8u, 1e-4 / 1e-12 relative)."""
import numpy as np
import pytest

import oracle
import satgen

pytestmark = pytest.mark.gpu
TOL = {np.uint8: 0.0, np.float32: 1e-4, np.float64: 1e-12}


def _check(got, ref, d, what):
    if TOL[d] == 0.0:
        assert np.array_equal(got, ref), f"{what}: {np.count_nonzero(got != ref)} mismatches"
    else:
        nz = ref != 0
        rel = np.max(np.abs(got[nz].astype(np.float64) - ref[nz]) / np.abs(ref[nz])) if nz.any() else 0.0
        assert rel <= TOL[d] and np.all(got[~nz] == 0), f"{what}: rel err {rel}"


@pytest.mark.parametrize("d", [np.uint8, np.float32, np.float64])
@pytest.mark.parametrize("shape", [(1, 1), (31, 33), (32, 1024), (33, 1025), (999, 1001),
                                   (1080, 1920), (2050, 4100)])
def test_brlt_parity(d, shape):
    import torch

    import paper_conf_cluster_chenwttm18_b200 as sat
    H, W = shape
    x = torch.empty((H, W), dtype={np.uint8: torch.uint8, np.float32: torch.float32,
                                   np.float64: torch.float64}[d], device="cuda")
    satgen.fill_device(x, seed=H + 3 * W)
    y = sat.sat_brlt(x)
    torch.cuda.synchronize()
    _check(y.cpu().numpy(), oracle.sat(x.cpu().numpy()), d, f"BRLT {d.__name__} {shape}")


def test_brlt_8u_wraps_at_8192sq():
    import torch

    import paper_conf_cluster_chenwttm18_b200 as sat
    x = torch.empty((8192, 8192), dtype=torch.uint8, device="cuda")
    satgen.fill_device(x, seed=1001)
    y = sat.sat_brlt(x)
    torch.cuda.synchronize()
    ref = oracle.sat(x.cpu().numpy())
    for r0 in range(0, 8192, 2048):
        assert np.array_equal(y[r0:r0 + 2048].cpu().numpy(), ref[r0:r0 + 2048])
