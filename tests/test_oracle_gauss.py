"""Pins of the float-variant oracle O-7 (oracle.gauss_taps / gauss_f32, reading A43)
against a library routine and closed forms."""
import numpy as np
import pytest

from oracle import oracle as O

scipy_ndimage = pytest.importorskip("scipy.ndimage")


def test_taps_closed_form():
    w = O.gauss_taps(1.0)
    assert w.dtype == np.float32 and len(w) == 7  # r = ceil(3 sigma) = 3
    assert np.array_equal(w, w[::-1])  # symmetric
    assert abs(float(w.astype(np.float64).sum()) - 1.0) < 4e-7  # normalised (up to f32 rounding)
    # exp(-k^2/2) ratios of a unit Gaussian
    assert abs(w[3] / w[2] - np.exp(0.5)) < 1e-6 and abs(w[3] / w[1] - np.exp(2.0)) < 1e-5
    assert len(O.gauss_taps(0.5)) == 5 and len(O.gauss_taps(1.3)) == 9


@pytest.mark.parametrize("sigma", [0.5, 1.0, 1.3])
def test_matches_scipy_correlate1d(sigma):
    """Library pin: two scipy correlate1d passes with mode='nearest' (= replicate)."""
    rng = np.random.default_rng(3)
    x = rng.random((2, 37, 53), dtype=np.float32)
    w = O.gauss_taps(sigma).astype(np.float64)
    ref = scipy_ndimage.correlate1d(x.astype(np.float64), w, axis=2, mode="nearest")
    ref = scipy_ndimage.correlate1d(ref, w, axis=1, mode="nearest")
    assert np.allclose(O.gauss_f32(x, sigma), ref, rtol=0, atol=1e-13)


def test_closed_forms():
    w = O.gauss_taps(1.0).astype(np.float64)
    # constant image -> the constant times the tap sum squared
    c = np.full((1, 20, 30), 0.7, dtype=np.float32)
    assert np.allclose(O.gauss_f32(c, 1.0), np.float64(np.float32(0.7)) * w.sum() ** 2, atol=1e-15)
    # impulse away from the border -> the outer product of the taps
    imp = np.zeros((1, 21, 21), dtype=np.float32)
    imp[0, 10, 10] = 1.0
    out = O.gauss_f32(imp, 1.0)[0]
    assert np.allclose(out[7:14, 7:14], np.outer(w, w), atol=1e-15)
    assert np.count_nonzero(out) == 49
    # a linear ramp is kept in the interior (symmetric taps), scaled by the tap sum
    ramp = np.tile(np.arange(40, dtype=np.float32) / 40, (1, 16, 1))
    got = O.gauss_f32(ramp, 1.0)[0, :, 3:-3]
    assert np.allclose(got, ramp[0, :, 3:-3].astype(np.float64) * w.sum() ** 2, atol=1e-12)


def test_replicate_border_closed_form():
    """Left border: out(x=0) of a horizontal step 0 | 1 at x = 2 is the taps reaching x >= 2."""
    w = O.gauss_taps(1.0).astype(np.float64)
    x = np.zeros((1, 9, 12), dtype=np.float32)
    x[:, :, 2:] = 1.0
    out = O.gauss_f32(x, 1.0)[0, 4]
    # at x = 0 the row reads clamp(x + j), j = -3..3: columns 0,0,0,0,1,2,3 -> ones at j >= 2
    assert abs(out[0] - w[5:].sum() * w.sum()) < 1e-15
