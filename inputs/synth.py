"""Seeded synthetic RGB8 inputs (SURVEY §8(d) "Concrete synthetic inputs").

This module holds NONE of KTILER's arithmetic: it only produces the graph
input image (interleaved RGB8, dense pitch 3*W, frames contiguous) that both
the CPU oracle and the CUDA path consume.  The same counter-based generator is
implemented a second time in ``inputs/synth_gpu.cu`` so that multi-GB inputs
can be produced on the device without an upload; ``tests/test_gpu_parity.py::test_gpu_generator_matches_numpy``
checks the two byte for byte.

Generators (the recipe DESIGN.md §3 states):

* ``uniform(seed)``: byte(f, y, x, c) = splitmix64(i + seed * K_SEED) & 0xFF
  with i = ((f*H + y)*W + x)*3 + c.  Dense random texture -> worst case for
  edges (the threshold mask is dense).
* ``scene(seed)``: per frame f (frame seed s = seed + f) a gradient background
  R = 255*x // W, G = 255*y // H, B = 128, 64 axis-aligned rectangles of hashed
  colour, position and size painted in order k = 0..63 (later wins), then a
  hashed uniform noise in [-8, 7] per channel, clipped to [0, 255].  Natural-ish
  edge density: long straight edges plus texture.
* closed-form images: constant, ramp, checkerboard, half-black/half-white.
"""
from __future__ import annotations

import numpy as np

M64 = (1 << 64) - 1
K_SEED = 0xD1B54A32D192ED03
K_NOISE = 0x632BE59BD9B4E019
N_RECTS = 64


def splitmix64_int(z: int) -> int:
    """Scalar splitmix64 finaliser (Steele, Lea, Flood 2014), on Python ints."""
    z = (z + 0x9E3779B97F4A7C15) & M64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M64
    return z ^ (z >> 31)


def splitmix64_np(z: np.ndarray) -> np.ndarray:
    """Vectorised splitmix64 on uint64 arrays (wrap-around arithmetic)."""
    z = z.astype(np.uint64, copy=True)
    with np.errstate(over="ignore"):
        z += np.uint64(0x9E3779B97F4A7C15)
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def uniform(seed: int, W: int, H: int, F: int = 1) -> np.ndarray:
    """uint8 array [F, H, W, 3] of hashed bytes."""
    return uniform_rows(seed, W, H, 0, H, F)


def uniform_rows(seed: int, W: int, H: int, y0: int, y1: int, F: int = 1, f0: int = 0) -> np.ndarray:
    """Rows [y0, y1) of frames [f0, f0+F) of ``uniform(seed)`` (global size W x H): uint8
    [F, y1-y0, W, 3], byte for byte the same as the slice of the whole image."""
    out = np.empty((F, y1 - y0, W, 3), dtype=np.uint8)
    for k in range(F):
        base = (((f0 + k) * H + y0) * W) * 3
        i = np.arange(base, base + (y1 - y0) * W * 3, dtype=np.uint64)
        with np.errstate(over="ignore"):
            i += np.uint64((seed * K_SEED) & M64)
        out[k] = (splitmix64_np(i) & np.uint64(0xFF)).astype(np.uint8).reshape(y1 - y0, W, 3)
    return out


def scene_rects(s: int, W: int, H: int):
    """The 64 rectangles of frame seed ``s``: list of (x0, y0, x1, y1, r, g, b)."""
    out = []
    for k in range(N_RECTS):
        h = [splitmix64_int((s * 1000003 + k * 16 + j + 0x5EED) & M64) for j in range(5)]
        x0 = h[0] % W
        y0 = h[1] % H
        rw = 1 + h[2] % max(1, W // 4)
        rh = 1 + h[3] % max(1, H // 4)
        c = h[4]
        out.append((x0, y0, min(W, x0 + rw), min(H, y0 + rh), c & 0xFF, (c >> 8) & 0xFF, (c >> 16) & 0xFF))
    return out


def scene_frame(s: int, W: int, H: int) -> np.ndarray:
    return scene_rows(s, W, H, 0, H)


def scene_rows(s: int, W: int, H: int, y0: int, y1: int) -> np.ndarray:
    """Rows [y0, y1) of frame seed ``s`` of the scene (global size W x H): uint8
    [y1-y0, W, 3], byte for byte the same as the slice of the whole frame."""
    n = y1 - y0
    img = np.empty((n, W, 3), dtype=np.int32)
    img[:, :, 0] = (np.arange(W, dtype=np.int64) * 255 // W)[None, :]
    img[:, :, 1] = (np.arange(y0, y1, dtype=np.int64) * 255 // H)[:, None]
    img[:, :, 2] = 128
    for (x0, ry0, x1, ry1, r, g, b) in scene_rects(s, W, H):
        a, c = max(ry0, y0), min(ry1, y1)
        if a < c:
            img[a - y0:c - y0, x0:x1, 0] = r
            img[a - y0:c - y0, x0:x1, 1] = g
            img[a - y0:c - y0, x0:x1, 2] = b
    i = np.arange(y0 * W * 3, y1 * W * 3, dtype=np.uint64)
    with np.errstate(over="ignore"):
        i += np.uint64((s * K_NOISE) & M64)
    noise = (splitmix64_np(i) & np.uint64(15)).astype(np.int32).reshape(n, W, 3) - 8
    return np.clip(img + noise, 0, 255).astype(np.uint8)


def scene(seed: int, W: int, H: int, F: int = 1) -> np.ndarray:
    """uint8 array [F, H, W, 3]; frame f uses frame seed ``seed + f``."""
    return np.stack([scene_frame(seed + f, W, H) for f in range(F)])


# ---- closed-form images -------------------------------------------------------------
def constant(v, W: int, H: int, F: int = 1) -> np.ndarray:
    a = np.empty((F, H, W, 3), dtype=np.uint8)
    a[...] = np.asarray(v, dtype=np.uint8)
    return a


def ramp(a: int, b: int, W: int, H: int, F: int = 1) -> np.ndarray:
    """Gray-level ramp p = a*x + b*y on all three channels (caller keeps it < 256)."""
    y, x = np.mgrid[0:H, 0:W]
    p = (a * x + b * y).astype(np.int64)
    assert p.max() <= 255
    return np.repeat(np.broadcast_to(p.astype(np.uint8)[None, :, :, None], (F, H, W, 1)), 3, axis=3).copy()


def checkerboard(cell: int, W: int, H: int, F: int = 1) -> np.ndarray:
    y, x = np.mgrid[0:H, 0:W]
    p = (((x // cell) + (y // cell)) % 2 * 255).astype(np.uint8)
    return np.repeat(np.broadcast_to(p[None, :, :, None], (F, H, W, 1)), 3, axis=3).copy()


def half_black_white(W: int, H: int, F: int = 1) -> np.ndarray:
    p = np.zeros((H, W), dtype=np.uint8)
    p[:, W // 2:] = 255
    return np.repeat(np.broadcast_to(p[None, :, :, None], (F, H, W, 1)), 3, axis=3).copy()


def make(kind: str, seed: int, W: int, H: int, F: int = 1) -> np.ndarray:
    if kind == "uniform":
        return uniform(seed, W, H, F)
    if kind == "scene":
        return scene(seed, W, H, F)
    raise ValueError(kind)


def hs_fields(seed: int, W: int, H: int, F: int = 1):
    """Horn-Schunck JI inputs, seeded and synthetic: brightness
    derivatives Ix, Iy, It in [-1, 1) on a 1/64 grid, smooth-ish (a hashed value per 4x4
    cell plus a hashed per-pixel perturbation), and an initial flow (u, v) in [-2, 2) on a
    1/64 grid.  Returns (coef [F, H, W, 4] f32 with channel 3 = 0, s0 [F, H, W, 2] f32).
    Plain data generation: no part of the method's arithmetic."""
    z = np.arange(F * H * W, dtype=np.uint64).reshape(F, H, W)
    f = np.arange(F, dtype=np.uint64)[:, None, None]
    y = np.arange(H, dtype=np.uint64)[None, :, None]
    x = np.arange(W, dtype=np.uint64)[None, None, :]
    cell = (f * np.uint64(1 << 40)) + ((y >> np.uint64(2)) << np.uint64(20)) + (x >> np.uint64(2))
    base = np.uint64((seed * 0xD1B54A32D192ED03) & M64)
    out = []
    for ch in range(5):
        salt = np.uint64((ch + 1) * 0x9E3779B97F4A7C15 & M64)
        c = splitmix64_np(cell ^ base ^ salt)
        p = splitmix64_np(z ^ base ^ salt ^ np.uint64(0x5851F42D4C957F2D))
        v = ((c & np.uint64(0x7F)).astype(np.int32) - 64) + ((p & np.uint64(0xF)).astype(np.int32) - 8)
        out.append(np.clip(v, -64, 63).astype(np.float32) / np.float32(64.0))
    coef = np.stack([out[0], out[1], out[2], np.zeros_like(out[0])], axis=-1)
    s0 = np.stack([out[3] * np.float32(2.0), out[4] * np.float32(2.0)], axis=-1)
    return coef, s0
