"""Histogram on the GPU against oracle.histogram, bit-exact:
both sides decide each bin in fp64 with the same three correctly rounded
operations (R13).  Shared-memory and global-memory bin paths, ragged
head/tail, out-of-range values, NaN/inf, large inputs."""
import numpy as np
import pytest

import oracle
import synth
from tests._util import to_device

pytestmark = pytest.mark.gpu


def _rb():
    import paper_conf_cgo_gonzalohghmh19_b200 as rb
    return rb


@pytest.mark.parametrize("dtype", ["int32", "float32"])
@pytest.mark.parametrize("nbins", [1, 7, 256, 1000, 16384, 16385, 100000, 1 << 20])
def test_histogram_bit_exact(dtype, nbins):
    rb = _rb()
    for k, n in enumerate([0, 1, 13, 4097, (1 << 20) + 3]):
        if dtype == "int32":
            x = synth.make("int32", n, "int_small", 40 + k)
            lo, hi = -900.0, 1000.0 - 7 * k
        else:
            x = synth.make("float32", n, "uniform_pm1", 40 + k)
            lo, hi = -0.75, 0.8 + 0.01 * k
        t = to_device(x, k % 8)
        got = rb.histogram(t, lo, hi, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, lo, hi, nbins)
        assert (got == want).all(), (dtype, nbins, n, np.nonzero(got != want)[0][:5])


def test_histogram_special_values_and_big():
    rb = _rb()
    x = synth.make("float32", (1 << 24) + 5, "uniform01", 3)
    x[[0, 5, 99, -1]] = [np.nan, np.inf, -np.inf, -0.0]
    t = to_device(x, 3)
    for nbins in (10, 4096, 65536):
        got = rb.histogram(t, 0.0, 1.0, nbins).cpu().numpy().view(np.uint32)
        want = oracle.histogram(x, 0.0, 1.0, nbins)
        assert (got == want).all()
        assert int(got.sum()) == int(((x >= 0) & (x < 1)).sum())
