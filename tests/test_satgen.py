"""The seeded input generator: numpy and C implementations agree bit for bit, strips regenerate
the rows of the global matrix, and the distributions have the advertised ranges.  CPU only
(the device copy is checked in test_gpu_parity.py)."""
import numpy as np
import pytest

import satgen


@pytest.mark.parametrize("dist", ["u32", "u8", "u2", "f01", "fsym", "fu2"])
def test_numpy_equals_c(dist):
    a = satgen.gen_numpy(37, 53, seed=1447, dist=dist)
    b = satgen.gen_host(37, 53, seed=1447, dist=dist)
    assert a.dtype == b.dtype and (a.view(np.uint32) == b.view(np.uint32)).all()


def test_strips_and_pitch():
    full = satgen.gen_host(40, 30, seed=7)
    top = satgen.gen_host(15, 30, seed=7)
    bot = satgen.gen_host(25, 30, seed=7, row0=15)
    assert (np.concatenate([top, bot]) == full).all()
    padded = satgen.gen_host(40, 30, seed=7, pitch=36)
    assert (padded[:, :30] == full).all() and (padded[:, 30:] == 0).all()
    assert not (satgen.gen_host(40, 30, seed=8) == full).all()


def test_ranges():
    assert satgen.gen_host(64, 64, 1, "u8").max() <= 255
    u2 = satgen.gen_host(64, 64, 1, "u2")
    assert set(np.unique(u2)) <= {0, 1, 2, 3}
    f = satgen.gen_host(64, 64, 1, "f01")
    assert f.dtype == np.float32 and f.min() >= 0 and f.max() < 1
    s = satgen.gen_host(64, 64, 1, "fsym")
    assert s.min() >= -1 and s.max() < 1 and s.min() < -0.5
    full = satgen.gen_host(256, 256, 1, "u32")
    assert full.min() < -(2 ** 30) and full.max() > 2 ** 30
