"""Footprint discovery helpers: turn the records of
``ktiler_discover_footprint`` (per block: byte runs it writes, 128-B lines it depends on)
into per-buffer line sets and pixel rects, and fit the affine access map the planner takes
(``ktiler_access``: block (bx, by) -> [ax*bx + ox - hl, ax*(bx+1) + ox + hr) x ...).

This restores the paper's "function-oblivious" front end (the
block analyzer derives memory lines and dependencies from a trace of sample inputs) for
kernels whose footprints are not declared by hand.  Host-side bookkeeping only; the
discovery itself runs in libktiler."""
from __future__ import annotations

from . import ktiler as K

LINE = 128


def line_sets(recs, mode: int) -> dict:
    """{buf_id: set of line indices relative to the buffer base} of the records of `mode`."""
    out = {}
    for b, m, first, last in recs:
        if m == mode:
            out.setdefault(b, set()).update(range(first // LINE, (last - 1) // LINE + 1))
    return out


def byte_sets(recs, mode: int) -> dict:
    out = {}
    for b, m, first, last in recs:
        if m == mode:
            out.setdefault(b, set()).update(range(first, last))
    return out


def pixel_rect(runs, pitch: int, fstride: int, elem: int):
    """Bounding box (x0, y0, z0, x1, y1, z1) in pixels of byte runs [first, last) of a
    buffer laid out as frames x rows x pitch (elem bytes per pixel)."""
    xs0, xs1, ys, zs = [], [], [], []
    for first, last in runs:
        b = first
        while b < last:
            z, r = divmod(b, fstride)
            y, xb = divmod(r, pitch)
            e = min(last, b - xb + pitch)  # end of this row inside the run
            xs0.append(xb // elem)
            xs1.append(-(-(e - (b - xb)) // elem))
            ys.append(y)
            zs.append(z)
            b = e
    if not xs0:
        return None
    return (min(xs0), min(ys), min(zs), max(xs1), max(ys) + 1, max(zs) + 1)


def rects(recs, descs: dict, mode: int) -> dict:
    """{buf_id: pixel bbox} of the records of `mode`; descs: buf_id -> (pitch, fstride, elem)."""
    runs = {}
    for b, m, first, last in recs:
        if m == mode:
            runs.setdefault(b, []).append((first, last))
    return {b: pixel_rect(r, *descs[b]) for b, r in runs.items()}


def fit_access(samples: dict, buf_id: int, mode: int, W: int, H: int, ax: int | None = None,
               ay: int | None = None) -> dict:
    """Affine access map from discovered rects of several blocks of one node.

    samples: {(bx, by): pixel rect (x0, y0, z0, x1, y1, z1) of the block in buffer buf_id}.
    The step along an axis (ax / ay) is measured from two blocks whose rects are not
    clipped by the buffer edge, unless given (line-quantized read rects of tiles narrower
    than a 128-B line are not affine in x; pass the step the buffer shapes imply).  The
    halos are the largest deviation over all samples, so the map covers every sampled
    block (conservative for line-quantized reads); ox = oy = 0 (scale + halo, like every
    built-in op)."""
    def step(i0, i1, size, bidx):
        pts = sorted({(k[bidx], r[i0], r[i1]) for k, r in samples.items() if r and 0 < r[i0] and r[i1] < size})
        if len(pts) < 2:
            raise ValueError("need two unclipped blocks along each axis")
        (b0, lo0, hi0), (b1, lo1, hi1) = pts[0], pts[-1]
        a = (lo1 - lo0) // (b1 - b0)
        if a <= 0 or (lo1 - lo0) != a * (b1 - b0) or (hi1 - hi0) != a * (b1 - b0):
            raise ValueError("footprint is not affine in the block index")
        return a

    def halos(a, i0, i1, bidx):
        lo = max(a * k[bidx] - r[i0] for k, r in samples.items() if r)
        hi = max(r[i1] - a * (k[bidx] + 1) for k, r in samples.items() if r)
        return max(0, lo), max(0, hi)
    ax = ax or step(0, 3, W, 0)
    ay = ay or step(1, 4, H, 1)
    hl, hr = halos(ax, 0, 3, 0)
    ht, hb = halos(ay, 1, 4, 1)
    return dict(buf=buf_id, mode=mode, ax=ax, ay=ay, hl=hl, hr=hr, ht=ht, hb=hb)
