"""The float variant of the blur: a chain of K separable f32 Gaussian
nodes (KTILER_OP_GAUSS_F32) on [frames][H][W] f32 images,

    x_0 --G_1--> x_1 --G_2--> ... --G_K--> x_K          (x_1 .. x_{K-1} internal)

declared through the C ABI and tiled by the planner like the image pipeline (each node
reads its predecessor with a halo of r = ceil(3 sigma) pixels).  The kernels compute in
f32; the oracle (oracle.gauss_f32) in f64 with the same f32 taps; they agree within 1e-5
on data in [0, 1] (BJ:5, reading A43).  Device buffers are torch tensors (allocator only)."""
from __future__ import annotations

import math
import struct

from . import ktiler as K
from .pipeline import _GraphBuilder


class GaussChain:
    def __init__(self, W: int, H: int, nodes: int = 2, frames: int = 1, sigma: float = 1.0, tile=(128, 64),
                 threads: int = 128, device="cuda", internal: bool = True):
        self.W, self.H, self.K, self.F, self.sigma = W, H, nodes, frames, sigma
        self.radius = math.ceil(3 * sigma)
        b = _GraphBuilder(device, 128)
        self.b = b
        for k in range(nodes + 1):
            b.buffer(f"x{k}", W, H, frames, 4, internal=internal and 0 < k < nodes)
        prev = None
        for k in range(1, nodes + 1):
            nid = b.kernel(f"G{k}", K.OP_GAUSS_F32, f"x{k - 1}", f"x{k}", tile, threads, halo=self.radius,
                           params=struct.pack("f", sigma))
            if prev is not None:
                b.g.add_edge(prev, nid, b.bufs[f"x{k - 1}"][0], 1.0)
            prev = nid
        self.plan_obj = None

    @property
    def graph(self) -> K.Graph:
        return self.b.g

    def view(self, name: str):
        """torch f32 view [F, H, W] of buffer x_k (device mode)."""
        return self.b.view(name)

    def plan(self, cache_bytes: int = 0, **policy) -> K.Plan:
        self.plan_obj = self.b.g.plan(cache_bytes, **policy)
        return self.plan_obj

    def run(self, stream: int = 0) -> None:
        self.plan_obj.execute(stream)
