"""The north star's kernel graphs, declared through the C ABI (BASELINE.json configs).

* ``Pipeline`` — the 5-kernel image pipeline rgb -> gray -> blur5 -> down2 -> sobel3 ->
  thresh (configs[1..4]) on W x H x frames.
* ``Motivational`` — the paper's Fig. 1 graph: 256x256 RGB -> A (grayscale) -> B (2x
  downscale) (configs[0]), in the paper's geometry (A<<<(8x32),(32x8)>>>
  one thread per pixel, B = 64x1 threads per block) or the B200 geometry.

Buffers are torch CUDA tensors (PyTorch is only the allocator here); with
``device=None`` the graph is declared over synthetic 128-B-aligned addresses so the
planner can run without a GPU (planning never dereferences buffers).

B200 geometry: per-op tiles, see B200_GEOMETRY (gray 256x32, blur5 512x64,
half-resolution kernels down2 256x32, sobel3 / thresh 256x64); the planner derives the mixed-geometry
block dependencies in closed form from the declared footprints.

"""
from __future__ import annotations

import json
import os
import struct

from . import ktiler as K

# op -> (tile w, tile h, threads per block) for the vector variant
B200_GEOMETRY = {
    "gray": (256, 32, 128),    # 512 items of 16 px (4 per thread); 24.6 KB staged rgb
    "blur": (512, 64, 128),    # 128 column strips x 16 rows; 37 KB staged halo tile
    "down": (256, 32, 128),    # 512 items (4 per thread); 32 KB staged blur rows
    "sobel": (256, 64, 128),   # 128 strips x 8 rows; 19 KB halo tile
    "thresh": (256, 64, 128),  # 1024 items (8 per thread); 64 KB staged f32 = one sobel tile
                               # (DAG + PDL step 1.5% faster than 256x32, profiles/r02c_policy_sweep.txt)
}

# The persistent executors (FLOW, PERSISTENT) stage every op's tiles in one ring of slots of
# the largest staged tile: with 64 KB thresh tiles FLOW fits one CTA per SM (9.2 ms on
# 64 x 8K), with 32 KB ones three (6.9 ms; profiles/r02c_policy_sweep.txt).
FLOW_GEOMETRY = dict(B200_GEOMETRY, thresh=(256, 32, 128))


def _cdiv(a: int, b: int) -> int:
    return -(-a // b)


def _round(a: int, m: int) -> int:
    return _cdiv(a, m) * m


class _Store:
    """Buffer storage: torch tensors on a device, or fake addresses (planning only)."""

    def __init__(self, device, base: int = 1 << 30):
        self.device = device
        self.next = base
        self.tensors = {}

    def alloc(self, name: str, frames: int, height: int, pitch: int):
        nbytes = frames * height * pitch
        if self.device is None:
            addr = self.next
            self.next += _round(nbytes, 4096) + 4096
            return addr
        import torch
        t = torch.empty(nbytes + 128, dtype=torch.uint8, device=self.device)
        off = (-t.data_ptr()) % 128
        t = t[off:off + nbytes]
        self.tensors[name] = t
        return t.data_ptr()


class _GraphBuilder:
    def __init__(self, device, pitch_align: int, bases=None):
        self.store = _Store(device)
        self.g = K.Graph()
        self.bufs = {}  # name -> (id, W, H, F, elem, pitch)
        self.slots = {}  # name -> frames of storage (< F for a ring buffer)
        self.nodes = {}
        self.grids = {}
        self.pitch_align = pitch_align
        self.bases = bases or {}

    def buffer(self, name, W, H, F, elem, internal, ring=0):
        """ring > 0 (internal buffers): storage for `ring` frames, frame z in slot z mod ring
        (ktiler_buffer_desc.ring_frames)."""
        pitch = _round(W * elem, self.pitch_align)
        ring = ring if internal and 0 < ring < F else 0
        if name in self.bases:
            addr = self.bases[name]
        else:
            addr = self.store.alloc(name, ring or F, H, pitch)
        bid = self.g.add_buffer(addr, W, H, elem, frames=F, pitch_bytes=pitch, internal=internal, ring_frames=ring)
        self.bufs[name] = (bid, W, H, F, elem, pitch)
        self.slots[name] = ring or F  # frames of storage (views)
        return bid

    def kernel(self, name, op, src, dst, tile, threads, halo=0, scale=1, params=None):
        sid, sW, sH, F, _, _ = self.bufs[src]
        did, dW, dH, _, _, _ = self.bufs[dst]
        tw, th = tile
        grid = (_cdiv(dW, tw), _cdiv(dH, th), F)
        block = (threads, 1, 1) if not isinstance(threads, tuple) else threads
        acc = [dict(buf=sid, mode=K.READ, ax=tw * scale, ay=th * scale, hl=halo, hr=halo, ht=halo, hb=halo),
               dict(buf=did, mode=K.WRITE, ax=tw, ay=th)]
        nid = self.g.add_kernel(op, grid, block, acc, params)
        self.nodes[name] = nid
        self.grids[name] = grid
        return nid

    def view(self, name):
        """torch view [F, H, W(, 3)] of a buffer (device mode only)."""
        import torch
        bid, W, H, F, elem, pitch = self.bufs[name]
        F = self.slots.get(name, F)
        t = self.store.tensors[name].view(F, H, pitch)[:, :, :W * elem]
        if elem == 3:
            return t.view(F, H, W, 3) if pitch == W * 3 else t.unflatten(2, (W, 3))
        if elem == 4:
            return t.contiguous().view(torch.float32) if pitch % 4 else t.view(torch.float32)
        return t


class Pipeline:
    """rgb -> gray -> blur5 -> down2 -> sobel3 -> thresh on W x H x frames (W, H even)."""

    NODE_ORDER = ("gray", "blur", "down", "sobel", "thresh")

    def __init__(self, W: int, H: int, frames: int = 1, T: float = 200.0, device="cuda", geometry=None,
                 internal: bool = True, pitch_align: int = 128, bases=None, ring_frames: int = 0):
        if W % 2 or H % 2:
            raise ValueError("down2 needs even W and H (SURVEY A3)")
        self.W, self.H, self.F, self.T = W, H, frames, T
        geo = dict(B200_GEOMETRY)
        if os.environ.get("KTILER_GEOMETRY"):  # experiments: JSON {node: [tw, th, threads]}
            geo.update({k: tuple(v) for k, v in json.loads(os.environ["KTILER_GEOMETRY"]).items()})
        geo.update(geometry or {})
        self.geometry = geo
        b = _GraphBuilder(device, pitch_align, bases)
        self.b = b
        b.buffer("rgb", W, H, frames, 3, internal=False)
        # ring_frames > 0: the four intermediates are WAR-aware rings of that many frames
        b.buffer("gray", W, H, frames, 1, internal=internal, ring=ring_frames)
        b.buffer("blur", W, H, frames, 1, internal=internal, ring=ring_frames)
        b.buffer("down", W // 2, H // 2, frames, 1, internal=internal, ring=ring_frames)
        b.buffer("sob", W // 2, H // 2, frames, 4, internal=internal, ring=ring_frames)
        b.buffer("mask", W // 2, H // 2, frames, 1, internal=False)

        def thr(n):
            return geo[n][2]
        b.kernel("gray", K.OP_GRAY, "rgb", "gray", geo["gray"][:2], thr("gray"))
        b.kernel("blur", K.OP_BLUR5, "gray", "blur", geo["blur"][:2], thr("blur"), halo=2)
        b.kernel("down", K.OP_DOWN2, "blur", "down", geo["down"][:2], thr("down"), scale=2)
        b.kernel("sobel", K.OP_SOBEL3, "down", "sob", geo["sobel"][:2], thr("sobel"), halo=1)
        b.kernel("thresh", K.OP_THRESH, "sob", "mask", geo["thresh"][:2], thr("thresh"),
                 params=struct.pack("f", T))
        n = b.nodes
        bu = b.bufs
        # edge weights < 0: derived from the performance tables by Alg. 1 (include/ktiler.h)
        b.g.add_edge(n["gray"], n["blur"], bu["gray"][0], -1.0)
        b.g.add_edge(n["blur"], n["down"], bu["blur"][0], -1.0)
        b.g.add_edge(n["down"], n["sobel"], bu["down"][0], -1.0)
        b.g.add_edge(n["sobel"], n["thresh"], bu["sob"][0], -1.0)
        self.plan_obj = None

    @property
    def graph(self) -> K.Graph:
        return self.b.g

    def buf_id(self, name: str) -> int:
        return self.b.bufs[name][0]

    def plan(self, cache_bytes: int = 0, **policy) -> K.Plan:
        self.plan_obj = self.b.g.plan(cache_bytes, **policy)
        return self.plan_obj

    def calibrate(self, reps: int = 5, max_points: int = 8) -> dict:
        """Self-calibrated performance tables on the current
        device: each node's time for row bands of 1, 2, 4, ... block rows up to the whole
        grid, input cold and hot (ktiler_calibrate), installed with ktiler_set_perf_table.
        Returns {node name: (block counts, cold ms, hot ms)}."""
        out = {}
        for name in self.NODE_ORDER:
            gx, gy, gz = self.b.grids[name]
            total = gx * gy * gz
            pts, k = [], gx
            while k < total and len(pts) < max_points - 1:
                pts.append(k)
                k *= 4
            pts.append(total)
            nid = self.b.nodes[name]
            cold, hot = self.graph.calibrate(nid, pts, reps)
            self.graph.set_perf_table(nid, pts, cold, hot)
            out[name] = (pts, cold, hot)
        return out

    def run(self, stream: int | None = None) -> None:
        if self.plan_obj is None:
            raise RuntimeError("call plan() first")
        if stream is None:
            import torch
            stream = torch.cuda.current_stream().cuda_stream
        self.plan_obj.execute(stream)

    def view(self, name: str):
        return self.b.view(name)

    # --- algorithmic bytes ---
    @property
    def pixels(self) -> int:
        return self.W * self.H * self.F

    def compulsory_bytes(self) -> int:
        """Graph input + output: 3 B/px (rgb) + 0.25 B/px (mask)."""
        return self.pixels * 3 + (self.W // 2) * (self.H // 2) * self.F

    def untiled_bytes(self) -> int:
        """Every intermediate written once and read once: 9.75 B/px."""
        P, Q = self.pixels, (self.W // 2) * (self.H // 2) * self.F
        return (3 * P + P) + (P + P) + (P + Q) + (Q + 4 * Q) + (4 * Q + Q)


class Motivational:
    """Fig. 1 of the paper: A = gray (in -> intm), B = down2 (intm -> out).

    geometry="paper": A tiles 32x8 with 32x8 threads, B tiles 64x1 with 64x1 threads, one
    thread per pixel; geometry="b200": the vector variant."""

    def __init__(self, W: int = 256, H: int = 256, frames: int = 1, device="cuda", geometry: str = "paper",
                 internal: bool = True, pitch_align: int = 16, bases=None):
        self.W, self.H, self.F = W, H, frames
        b = _GraphBuilder(device, pitch_align, bases)
        self.b = b
        b.buffer("in", W, H, frames, 3, internal=False)
        b.buffer("intm", W, H, frames, 1, internal=internal)
        b.buffer("out", W // 2, H // 2, frames, 1, internal=False)
        if geometry == "paper":
            b.kernel("A", K.OP_GRAY, "in", "intm", (32, 8), (32, 8, 1))
            b.kernel("B", K.OP_DOWN2, "intm", "out", (64, 1), (64, 1, 1), scale=2)
        else:
            b.kernel("A", K.OP_GRAY, "in", "intm", B200_GEOMETRY["gray"][:2], B200_GEOMETRY["gray"][2])
            b.kernel("B", K.OP_DOWN2, "intm", "out", B200_GEOMETRY["down"][:2], B200_GEOMETRY["down"][2], scale=2)
        b.g.add_edge(b.nodes["A"], b.nodes["B"], b.bufs["intm"][0], -1.0)
        self.plan_obj = None

    @property
    def graph(self) -> K.Graph:
        return self.b.g

    def plan(self, cache_bytes: int = 0, **policy) -> K.Plan:
        self.plan_obj = self.b.g.plan(cache_bytes, **policy)
        return self.plan_obj

    def run(self, stream: int | None = None) -> None:
        if stream is None:
            import torch
            stream = torch.cuda.current_stream().cuda_stream
        self.plan_obj.execute(stream)

    def view(self, name: str):
        return self.b.view(name)
