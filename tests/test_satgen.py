"""The seeded generator: numpy and C implementations agree bit for bit."""
import numpy as np
import pytest

import satgen


@pytest.mark.parametrize("kind", [satgen.KIND_U8, satgen.KIND_F32, satgen.KIND_F64])
@pytest.mark.parametrize("mode", [satgen.MODE_UNIFORM, satgen.MODE_DYADIC24, satgen.MODE_CONST])
def test_numpy_equals_c_host(kind, mode):
    H, W = 37, 301
    ref = satgen.generate(kind, H, W, seed=1234, img=5, y0=17, mode=mode, value=3.0)
    buf = np.zeros((H, W + 13), dtype=satgen.DTYPE_OF_KIND[kind])[:, :W]
    satgen.fill_host(buf, seed=1234, img0=5, y0=17, mode=mode, value=3.0)
    np.testing.assert_array_equal(buf, ref)


def test_batched_host_fill_uses_global_image_index():
    A = np.zeros((3, 20, 30), dtype=np.uint8)
    satgen.fill_host(A, seed=9, img0=10)
    for n in range(3):
        np.testing.assert_array_equal(A[n], satgen.generate(satgen.KIND_U8, 20, 30, seed=9, img=10 + n))


def test_distributions_have_expected_ranges():
    u8 = satgen.generate(satgen.KIND_U8, 256, 256, seed=1)
    assert u8.min() == 0 and u8.max() == 255 and abs(u8.mean() - 127.5) < 1.0
    f = satgen.generate(satgen.KIND_F32, 256, 256, seed=1)
    assert f.min() >= 0 and f.max() < 1 and abs(f.mean() - 0.5) < 0.01
    assert np.all(f * 2**24 == np.rint(f * 2**24))
    d = satgen.generate(satgen.KIND_F64, 256, 256, seed=1)
    assert d.min() >= 0 and d.max() < 1
