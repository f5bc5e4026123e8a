"""The seeded input generators' row-band forms (inputs/synth.py) equal the slices of the
whole images, so full-size GPU parity (tests/test_gpu_fullsize.py) can run the oracle on
bands of images too large to generate whole on the host."""
import numpy as np

from inputs import synth


def test_scene_rows_is_a_slice():
    W, H = 301, 198
    for s in (0, 1234, 7):
        whole = synth.scene_frame(s, W, H)
        for y0, y1 in ((0, 10), (57, 133), (180, 198), (0, H)):
            assert np.array_equal(synth.scene_rows(s, W, H, y0, y1), whole[y0:y1])


def test_uniform_rows_is_a_slice():
    W, H, F = 130, 70, 3
    whole = synth.uniform(9, W, H, F)
    assert np.array_equal(synth.uniform_rows(9, W, H, 11, 40, F=2, f0=1), whole[1:3, 11:40])
    assert np.array_equal(synth.uniform_rows(9, W, H, 0, H, F=F), whole)
