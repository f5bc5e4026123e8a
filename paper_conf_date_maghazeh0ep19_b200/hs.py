"""The paper's own workload: the Jacobi-iteration chain of Horn–Schunck
optical flow, HSOpticalFlow's JI nodes (Fig. 4: 500 JI nodes per step,
98.5% of the application's time, the nodes KTILER tiles).

``HSJacobi`` declares K chained KTILER_OP_JACOBI nodes through the C ABI:

    s_0 --JI_1--> s_1 --JI_2--> ... --JI_K--> s_K        every JI_k also reads `coef`

  s_k   f32 [frames][H][2W]: (u, v) per pixel, the flow after k iterations;
  coef  f32 [frames][H][4W]: (Ix, Iy, It, unused) per pixel; alpha^2 = a2 is the op's parameter.

Each iterate is its own buffer (the paper's DFG has one vector per JI node; KTILER's
hazard model is RAW only), so s_1..s_{K-1} are internal (discardable) and the
whole chain is one KTILER cluster: Alg. 2 tiles across iterations with the halo growing
by one pixel per iteration, exactly as for the image pipeline.  Device buffers are torch
tensors (allocator only); every step of the chain runs in libktiler's sm_100a kernel."""
from __future__ import annotations

import struct

from . import ktiler as K
from .pipeline import _GraphBuilder


class HSJacobi:
    def __init__(self, W: int, H: int, iters: int, frames: int = 1, a2: float = 1.0, tile=(64, 16),
                 threads: int = 128, device="cuda", internal: bool = True):
        if W % 2 or tile[0] % 8:
            raise ValueError("HSJacobi needs an even width and a tile width that is a multiple of 8 pixels")
        self.W, self.H, self.K, self.F = W, H, iters, frames
        b = _GraphBuilder(device, 128)
        self.b = b
        b.buffer("coef", 4 * W, H, frames, 4, internal=False)
        for k in range(iters + 1):
            b.buffer(f"s{k}", 2 * W, H, frames, 4, internal=internal and 0 < k < iters)
        tw, th = tile
        grid = (-(-W // tw), -(-H // th), frames)
        cid = b.bufs["coef"][0]
        self.nodes = []
        for k in range(1, iters + 1):
            src, dst = b.bufs[f"s{k - 1}"][0], b.bufs[f"s{k}"][0]
            acc = [dict(buf=src, mode=K.READ, ax=2 * tw, ay=th, hl=2, hr=2, ht=1, hb=1),
                   dict(buf=cid, mode=K.READ, ax=4 * tw, ay=th),
                   dict(buf=dst, mode=K.WRITE, ax=2 * tw, ay=th)]
            nid = b.g.add_kernel(K.OP_JACOBI, grid, (threads, 1, 1), acc, struct.pack("f", a2))
            self.nodes.append(nid)
            if k > 1:
                b.g.add_edge(self.nodes[-2], nid, src, -1.0)
        self.grid = grid
        self.plan_obj = None

    @property
    def graph(self) -> K.Graph:
        return self.b.g

    def _rows(self, name: str):
        """uint8 view [F, H, row bytes] of a buffer (pitch padding excluded)."""
        bid, Wf, H, F, elem, pitch = self.b.bufs[name]
        return self.b.store.tensors[name].view(F, H, pitch)[:, :, :Wf * elem]

    def set(self, name: str, arr) -> None:
        """Copy a host float32 array ([F, H, W, 4] for coef, [F, H, W, 2] for s_k) in."""
        import numpy as np
        import torch
        r = self._rows(name)
        r.copy_(torch.from_numpy(np.ascontiguousarray(arr, dtype=np.float32).view(np.uint8).reshape(r.shape)))

    def get(self, name: str):
        """Host float32 copy of a buffer: [F, H, W, 4] for coef, [F, H, W, 2] for s_k."""
        import numpy as np
        r = self._rows(name).cpu().numpy()
        ch = 4 if name == "coef" else 2
        return np.ascontiguousarray(r).view(np.float32).reshape(self.F, self.H, self.W, ch)

    def plan(self, cache_bytes: int = 0, **policy) -> K.Plan:
        self.plan_obj = self.b.g.plan(cache_bytes, **policy)
        return self.plan_obj

    def run(self, stream: int = 0) -> None:
        self.plan_obj.execute(stream)


class HSPyramid:
    """The tiled part of Fig. 4: HSOpticalFlow's three steps work on
    frames of 256, 512 and 1024 pixels per side (coarse to fine), each with a chain of 500 JI
    nodes that starts from a zero vector ("{0}") and reads that step's derivative
    coefficients.  The steps' other nodes (DS, WP, DV, AD, US: 1.5% of the application's
    time) are not part of the north star (the SDK code that defines them is
    not in the paper), so each step's coefficients come from the caller and the steps'
    chains are independent graphs: one HSJacobi per step, planned by the same policy and
    executed in Fig. 4's order on one stream.

      steps[0]: (W >> (levels-1)) x (H >> (levels-1)),  ...,  steps[-1]: W x H."""

    def __init__(self, W: int = 1024, H: int = 1024, iters: int = 500, levels: int = 3, frames: int = 1,
                 a2: float = 1.0, tile=(64, 16), threads: int = 128, device="cuda", internal: bool = True):
        if W % (2 << (levels - 1)) or H % (1 << (levels - 1)):
            raise ValueError("HSPyramid needs W divisible by 2^levels and H by 2^(levels-1)")
        self.levels, self.K = levels, iters
        self.steps = [HSJacobi(W >> l, H >> l, iters, frames=frames, a2=a2, tile=tile, threads=threads, device=device,
                               internal=internal) for l in reversed(range(levels))]
        if device is not None:
            for h in self.steps:
                h.b.store.tensors["s0"].zero_()  # Fig. 4: every JI chain starts from {0}
        self.plans = None

    def set_coef(self, step: int, coef) -> None:
        """(Ix, Iy, It, unused) of step `step` (0 = coarsest), host f32 [F, H, W, 4]."""
        self.steps[step].set("coef", coef)

    def get(self, step: int):
        """The flow increment after the chain of step `step`: host f32 [F, H, W, 2]."""
        return self.steps[step].get(f"s{self.K}")

    def plan(self, cache_bytes: int = 0, **policy):
        self.plans = [h.plan(cache_bytes, **policy) for h in self.steps]
        return self.plans

    def run(self, stream: int = 0) -> None:
        for p in self.plans:
            p.execute(stream)
