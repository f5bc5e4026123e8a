"""Pins for the oracle (SURVEY §8(c) P1–P7): the oracle is checked against things
other than itself — library routines, closed forms, hand-worked fixtures — chosen so
a dropped term, a wrong sign or index, or a transposed operand fails one of them."""
import os

import numpy as np
import pytest

from inputs import synth
from oracle import oracle as O

cv2 = pytest.importorskip("cv2")
PIL = pytest.importorskip("PIL.Image")


def _read_golden(path):
    sec, out = None, {}
    for line in open(path):
        line = line.split("#")[0].strip()
        if not line:
            continue
        if line.replace("_", "").isalpha() and " " not in line:
            sec = line
            out[sec] = []
            continue
        out[sec].append([int(t) for t in line.split()])
    return out


# ---------------------------------------------------------------- P1 gray
def test_gray_equals_pillow_on_all_colours():
    """P1 (library): Pillow convert('L') on all 2^24 RGB colours, bit for bit."""
    v = np.arange(1 << 24, dtype=np.uint32)
    rgb = np.stack([(v >> 16) & 255, (v >> 8) & 255, v & 255], -1).astype(np.uint8).reshape(4096, 4096, 3)
    ours = O.gray(rgb)
    ref = np.asarray(PIL.fromarray(rgb, "RGB").convert("L"))
    assert np.array_equal(ours, ref)


def test_gray_closed_forms():
    """P1 (closed forms): gray(v,v,v) = v (weights sum to 2^16); primaries 76/150/29;
    within 1 of round(0.299R + 0.587G + 0.114B)."""
    v = np.arange(256, dtype=np.uint8)
    rgb = np.stack([v, v, v], -1)[None]
    assert np.array_equal(O.gray(rgb)[0], v)
    prim = np.array([[[255, 0, 0], [0, 255, 0], [0, 0, 255]]], np.uint8)
    assert O.gray(prim)[0].tolist() == [76, 150, 29]
    r = synth.uniform(5, 512, 512)[0]
    f = 0.299 * r[..., 0] + 0.587 * r[..., 1] + 0.114 * r[..., 2]
    assert np.abs(O.gray(r).astype(int) - np.floor(f + 0.5)).max() <= 1


# ---------------------------------------------------------------- P2 down2
def test_down2_hand_4x4(golden_dir):
    g = _read_golden(os.path.join(golden_dir, "hand_4x4.txt"))
    rgb = np.array(g["rgb"], np.uint8).reshape(4, 4, 3)
    assert O.gray(rgb).tolist() == g["gray"]
    assert O.down2(O.gray(rgb)).tolist() == g["down"]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_down2_equals_opencv_area_and_pil_reduce(seed):
    """P2 (library): cv2.resize(INTER_AREA) and PIL reduce(2) are the 2x2 mean with round-half-up."""
    a = synth.uniform(seed, 96, 64)[0, :, :, 0].copy()
    ours = O.down2(a)
    assert np.array_equal(ours, cv2.resize(a, (48, 32), interpolation=cv2.INTER_AREA))
    assert np.array_equal(ours, np.asarray(PIL.fromarray(a, "L").reduce(2)))


def test_down2_truncation_would_fail():
    """Negative control: 510/4 = 127.5 must round up to 128, so a truncating mean is caught."""
    a = np.array([[255, 255], [0, 0]], np.uint8)
    assert O.down2(a)[0, 0] == 128


# ---------------------------------------------------------------- P3 blur5
@pytest.mark.parametrize("seed,kind", [(0, "uniform"), (1, "scene"), (2, "uniform")])
def test_blur_equals_opencv_gaussian(seed, kind):
    """P3 (library): cv2.GaussianBlur(ksize 5x5, sigma 0 -> [1,4,6,4,1]/16, BORDER_REPLICATE)."""
    a = O.gray(synth.make(kind, seed, 77, 53)[0])
    ref = cv2.GaussianBlur(a, (5, 5), 0, borderType=cv2.BORDER_REPLICATE)
    assert np.array_equal(O.blur5(a), ref)


def test_blur_closed_forms():
    """P3 (closed forms): constants are fixed points; a 255 impulse gives the centre row
    (255*6*w + 128) >> 8 = [6, 24, 36, 24, 6]; separable u16 passes == the 2-D sum."""
    for c in (0, 1, 127, 255):
        a = np.full((9, 11), c, np.uint8)
        assert (O.blur5(a) == c).all()
    a = np.zeros((9, 9), np.uint8)
    a[4, 4] = 255
    b = O.blur5(a)
    assert b[4, 2:7].tolist() == [6, 24, 36, 24, 6]
    assert b[2:7, 4].tolist() == [6, 24, 36, 24, 6]
    assert b[4, 4] == (255 * 36 + 128) >> 8
    # separable identity on random data (integer arithmetic, exact)
    a = synth.uniform(3, 40, 30)[0, :, :, 1].astype(np.int64)
    w = np.array([1, 4, 6, 4, 1])
    p = np.pad(a, 2, mode="edge")
    h = sum(w[j] * p[:, j:j + a.shape[1]] for j in range(5))
    v = sum(w[i] * h[i:i + a.shape[0], :] for i in range(5))
    assert np.array_equal(O.blur5(a.astype(np.uint8)), ((v + 128) >> 8).astype(np.uint8))


# ---------------------------------------------------------------- P4 sobel3
@pytest.mark.parametrize("seed", [0, 1])
def test_sobel_equals_opencv(seed):
    """P4 (library): cv2.Sobel ksize 3 BORDER_REPLICATE gives gx, gy exactly; the magnitude is
    numpy's correctly rounded float32 sqrt of the exact integer sum (cv2.magnitude is NOT a
    valid pin: SURVEY A5)."""
    a = synth.uniform(seed, 70, 45)[0, :, :, 2].copy()
    gx = cv2.Sobel(a, cv2.CV_16S, 1, 0, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    gy = cv2.Sobel(a, cv2.CV_16S, 0, 1, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    ref = np.sqrt((gx * gx + gy * gy).astype(np.float32))
    ours = O.sobel3(a)
    assert ours.dtype == np.float32
    assert np.array_equal(ours.view(np.uint32), ref.view(np.uint32))


def test_sobel_closed_forms():
    """P4 (closed forms): ramp p = a x + b y -> interior gx = 8a, gy = 8b; first column under
    replicate gx = 4a; constants -> 0; a sign error or a transposed kernel fails here."""
    a, b = 3, 5
    y, x = np.mgrid[0:12, 0:20]
    p = (a * x + b * y).astype(np.uint8)
    m = O.sobel3(p)
    assert np.allclose(m[1:-1, 1:-1], np.float32(np.sqrt(np.float32(64 * a * a + 64 * b * b))))
    px = (a * x).astype(np.uint8)
    mx = O.sobel3(px)
    assert (mx[:, 1:-1] == 8 * a).all() and (mx[:, 0] == 4 * a).all() and (mx[:, -1] == 4 * a).all()
    py = (b * y).astype(np.uint8)
    my = O.sobel3(py)
    assert (my[1:-1, :] == 8 * b).all() and (my[0, :] == 4 * b).all()
    assert (O.sobel3(np.full((6, 6), 77, np.uint8)) == 0).all()


def test_sobel_asymmetric_orientation():
    """gx must respond to a vertical edge only, gy to a horizontal one (catches a swap)."""
    a = np.zeros((8, 8), np.uint8)
    a[:, 4:] = 100
    d = np.zeros((8, 8), np.uint8)
    d[4:, :] = 100
    # vertical edge: column 3 and 4 see gx = 4*100; rows identical, gy = 0
    assert O.sobel3(a)[2, 3] == 400 and O.sobel3(a)[2, 0] == 0
    assert O.sobel3(d)[3, 2] == 400 and O.sobel3(d)[0, 2] == 0


# ---------------------------------------------------------------- P5 thresh
def test_thresh_tie_and_integer_equivalence():
    """P5: gx=120, gy=160 -> mag = 200.0 exactly -> 0 under strict >; for integer T the mask
    equals [gx^2+gy^2 > T^2]."""
    assert O.thresh(np.array([[200.0, np.nextafter(np.float32(200), np.float32(300))]], np.float32)).tolist() == \
        [[0, 255]]
    a = synth.uniform(9, 64, 64)[0, :, :, 0].copy()
    m = O.sobel3(a)
    gx = cv2.Sobel(a, cv2.CV_16S, 1, 0, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    gy = cv2.Sobel(a, cv2.CV_16S, 0, 1, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    for T in (0, 1, 100, 200, 555, 1000):
        assert np.array_equal(O.thresh(m, float(T)) == 255, gx * gx + gy * gy > T * T)


# ---------------------------------------------------------------- P6 whole graph
def test_pipeline_hand_8x8(golden_dir):
    txt = [ln.split("#")[0].split() for ln in open(os.path.join(golden_dir, "hand_8x8.txt"))]
    rows = {t[0]: [int(v) for v in t[1:]] for t in txt if t}
    rgb = np.zeros((8, 8, 3), np.uint8)
    rgb[:, 4:] = 255
    out = O.pipeline(rgb)
    for r in range(8):
        assert out["gray"][r].tolist() == rows["gray_row"]
        assert out["blur"][r].tolist() == rows["blur_row"]
    for r in range(4):
        assert out["down"][r].tolist() == rows["down_row"]
        assert out["sob"][r].tolist() == rows["sob_row"]
        assert out["mask"][r].tolist() == rows["mask_row"]


def test_pipeline_equals_composed_libraries():
    """P6 (library chain): Pillow L -> cv2 GaussianBlur -> INTER_AREA -> cv2.Sobel magnitude -> > T."""
    rgb = synth.scene(4, 128, 96)[0]
    out = O.pipeline(rgb, T=150.0)
    g = np.asarray(PIL.fromarray(rgb, "RGB").convert("L"))
    b = cv2.GaussianBlur(g, (5, 5), 0, borderType=cv2.BORDER_REPLICATE)
    d = cv2.resize(b, (64, 48), interpolation=cv2.INTER_AREA)
    gx = cv2.Sobel(d, cv2.CV_16S, 1, 0, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    gy = cv2.Sobel(d, cv2.CV_16S, 0, 1, ksize=3, borderType=cv2.BORDER_REPLICATE).astype(np.int64)
    s = np.sqrt((gx * gx + gy * gy).astype(np.float32))
    assert np.array_equal(out["gray"], g) and np.array_equal(out["blur"], b) and np.array_equal(out["down"], d)
    assert np.array_equal(out["sob"].view(np.uint32), s.view(np.uint32))
    assert np.array_equal(out["mask"], np.where(s > 150.0, 255, 0).astype(np.uint8))


def test_pipeline_batch_is_per_frame():
    rgb = synth.scene(0, 64, 32, F=3)
    out = O.pipeline(rgb)
    for f in range(3):
        one = O.pipeline(rgb[f])
        for k in out:
            assert np.array_equal(out[k][f], one[k])


# ---------------------------------------------------------------- P7 motivational graph
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_motivational_equals_pillow_chain(seed):
    rgb = synth.scene(seed, 256, 256)[0]
    out = O.motivational(rgb)
    ref = np.asarray(PIL.fromarray(rgb, "RGB").convert("L").reduce(2))
    assert np.array_equal(out["down"], ref)
