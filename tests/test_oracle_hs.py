"""Pins of the Horn–Schunck Jacobi oracle (O-14): a hand-worked example,
closed forms of the iteration, the HS projection identity, and the f32 evaluation against
an f64 twin (the GPU kernel must equal the f32 oracle bit for bit; tests/test_gpu_hs.py)."""
import os

import numpy as np
import pytest

from inputs import synth
from oracle import oracle as O

GOLD = os.path.join(os.path.dirname(__file__), "golden", "hs_3x3.txt")


def _fields(u, v, Ix, Iy, It):
    coef = np.stack([Ix, Iy, It, np.zeros_like(Ix)], axis=-1)[None].astype(np.float32)
    s0 = np.stack([u, v], axis=-1)[None].astype(np.float32)
    return coef, s0


def test_hand_worked_3x3():
    u = np.array([[0, 1, 0], [2, 5, 4], [0, 3, 0]], np.float32)
    v = np.array([[0, 0, 0], [1, 7, -1], [0, 2, 0]], np.float32)
    Ix, Iy, It = (np.zeros((3, 3), np.float32) for _ in range(3))
    Ix[1, 1], Iy[1, 1], It[1, 1] = 1.0, 2.0, 0.5
    coef, s0 = _fields(u, v, Ix, Iy, It)
    out = O.hs_jacobi(coef, s0, 3.0, 1)[0]
    for line in open(GOLD):
        if line.startswith("#") or not line.strip():
            continue
        y, x, uu, vv = line.split()
        assert out[int(y), int(x), 0] == np.float32(uu) and out[int(y), int(x), 1] == np.float32(vv)


def test_pure_smoothing_keeps_linear_fields():
    """Ix = Iy = It = 0: u' = the 4-neighbour mean, so a linear field is reproduced exactly
    away from the border (small integers: exact in f32) and a constant field everywhere."""
    H, W = 16, 24
    yy, xx = np.mgrid[0:H, 0:W].astype(np.float32)
    z = np.zeros((H, W), np.float32)
    coef, s0 = _fields(3 * xx - 2 * yy, np.full((H, W), 7.0, np.float32), z, z, z)
    out = O.hs_jacobi(coef, s0, 1.0, 1)[0]
    assert np.array_equal(out[1:-1, 1:-1, 0], (3 * xx - 2 * yy)[1:-1, 1:-1])
    assert np.array_equal(out[..., 1], np.full((H, W), 7.0, np.float32))


def test_fixed_point_of_a_consistent_flow():
    """A constant flow that satisfies the brightness constraint Ix*u + Iy*v + It = 0 at
    every pixel is a fixed point: it stays exactly, over many iterations."""
    H, W = 12, 20
    one = np.ones((H, W), np.float32)
    coef, s0 = _fields(3 * one, -1 * one, 1 * one, 2 * one, -1 * one)
    out = O.hs_jacobi(coef, s0, 0.25, 40)
    assert np.array_equal(out, s0)


def test_projection_identity_f64():
    """One update moves the neighbour mean along (Ix, Iy) so that the constraint residual
    shrinks by alpha^2 / (alpha^2 + Ix^2 + Iy^2) (Horn & Schunck's update), checked in f64."""
    coef, s0 = synth.hs_fields(5, 40, 24, 1)
    a2 = 0.7
    c, s = coef.astype(np.float64), s0.astype(np.float64)
    out = O.hs_jacobi(coef, s0, a2, 1, dtype=np.float64)
    u = s[..., 0]
    v = s[..., 1]
    pad = lambda a: np.pad(a, ((0, 0), (1, 1), (1, 1)), mode="edge")  # noqa: E731
    pu, pv = pad(u), pad(v)
    ub = (pu[:, 1:-1, :-2] + pu[:, 1:-1, 2:] + pu[:, :-2, 1:-1] + pu[:, 2:, 1:-1]) / 4
    vb = (pv[:, 1:-1, :-2] + pv[:, 1:-1, 2:] + pv[:, :-2, 1:-1] + pv[:, 2:, 1:-1]) / 4
    Ix, Iy, It = c[..., 0], c[..., 1], c[..., 2]
    res_mean = Ix * ub + Iy * vb + It
    res_new = Ix * out[..., 0] + Iy * out[..., 1] + It
    np.testing.assert_allclose(res_new, a2 / (a2 + Ix**2 + Iy**2) * res_mean, rtol=0, atol=1e-12)


@pytest.mark.parametrize("iters", [1, 10, 50])
def test_f32_close_to_f64(iters):
    """The f32 evaluation (the GPU's) stays within 1e-5 of the f64 one on the synthetic
    fields (|u|, |v| < 2.4): the iteration is a contraction, rounding errors do not grow."""
    coef, s0 = synth.hs_fields(9, 64, 48, 2)
    a = O.hs_jacobi(coef, s0, 0.5, iters)
    b = O.hs_jacobi(coef, s0, 0.5, iters, dtype=np.float64)
    assert a.dtype == np.float32
    assert np.abs(a - b).max() <= 1e-5
