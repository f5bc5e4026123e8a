"""Strip partitioning of one giant image across ranks (BASELINE configs[4]).

Rank r of n owns full-resolution rows [r*H/n, (r+1)*H/n) and the mask rows
[r*H/2n, (r+1)*H/2n).  Each rank runs the tiled pipeline on its *extended* strip: its own
rows plus HALO_ROWS rgb rows from each neighbour, received over NCCL (torch.distributed
send/recv — the one exchange step of the path).  HALO_ROWS = 4 is the reach of the chain
in full-resolution rows: mask row m needs sob row m, down rows m-1..m+1, blur rows
2m-2..2m+3, gray rows 2m-4..2m+5.  Rows past the *global* image edge are never invented:
there the kernels clamp (replicate border), exactly as the 1-GPU run does, and
inside the image the halo makes every owned output identical to the whole-image result.

This module holds only row bookkeeping; the compute is the ordinary Pipeline (libktiler)
on the extended strip.  The exchange itself runs in libktiler (comm.cpp:
ktiler_halo_exchange — ncclSend/ncclRecv in one group, or the 1-GPU loopback backend), and
``StripPipeline.attach`` puts it into the plan's CUDA graph ahead of the schedule.
``exchange_halo`` is the same row bookkeeping over torch.distributed, used by the CPU
(gloo) tests.
"""
from __future__ import annotations

HALO_ROWS = 4


def strip_rows(H: int, world: int, rank: int, halo: int = HALO_ROWS):
    """(o0, o1, e0, e1): owned full-res rows [o0, o1) and extended rows [e0, e1)."""
    if H % (2 * world):
        raise ValueError(f"H={H} must split into {world} strips of even height")
    hs = H // world
    if world > 1 and hs < halo:
        raise ValueError(f"strip height {hs} < halo {halo}")
    o0, o1 = rank * hs, (rank + 1) * hs
    return o0, o1, max(0, o0 - halo), min(H, o1 + halo)


def owned_mask_rows(o0: int, o1: int, e0: int):
    """Mask rows of the extended strip's output that this rank owns: [m0, m1)."""
    m0 = (o0 - e0) // 2
    return m0, m0 + (o1 - o0) // 2


def exchange_halo(ext, o0: int, o1: int, e0: int, e1: int, rank: int, world: int, group=None) -> int:
    """Fill the halo rows of ``ext`` (tensor [e1-e0, ...] of the extended strip, owned rows
    already in place) from the neighbours: send the first / last owned rows up / down,
    receive into [e0, o0) and [o1, e1).  Returns the bytes this rank received."""
    import torch.distributed as dist
    ops = []
    top, bot = o0 - e0, e1 - o1
    own0, own1 = top, top + (o1 - o0)
    if rank > 0:
        ops.append(dist.P2POp(dist.irecv, ext[0:top], rank - 1, group))
        # the rank above needs as many of my rows as its own bottom halo: HALO_ROWS
        ops.append(dist.P2POp(dist.isend, ext[own0:own0 + min(HALO_ROWS, o1 - o0)].contiguous(), rank - 1, group))
    if rank < world - 1:
        ops.append(dist.P2POp(dist.irecv, ext[own1:own1 + bot], rank + 1, group))
        ops.append(dist.P2POp(dist.isend, ext[own1 - min(HALO_ROWS, o1 - o0):own1].contiguous(), rank + 1, group))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()
    return (top + bot) * (ext[0].numel() * ext.element_size())


class StripPipeline:
    """The 5-kernel Pipeline over this rank's extended strip of a W x H image."""

    def __init__(self, W: int, H: int, world: int, rank: int, T: float = 200.0, device="cuda", **kw):
        from .pipeline import Pipeline
        self.W, self.H, self.world, self.rank = W, H, world, rank
        self.o0, self.o1, self.e0, self.e1 = strip_rows(H, world, rank)
        self.m0, self.m1 = owned_mask_rows(self.o0, self.o1, self.e0)
        self.pipe = Pipeline(W, self.e1 - self.e0, 1, T=T, device=device, **kw)

    @property
    def own_offset(self) -> int:
        """Row of the extended strip holding global row o0."""
        return self.o0 - self.e0

    def rgb_ext(self):
        return self.pipe.view("rgb")[0]  # [rows, W, 3]

    def mask_owned(self):
        return self.pipe.view("mask")[0, self.m0:self.m1]

    def exchange(self, group=None) -> int:
        """torch.distributed exchange (the gloo tests; kept for comparison)."""
        return exchange_halo(self.rgb_ext(), self.o0, self.o1, self.e0, self.e1, self.rank, self.world, group)

    def register(self, comm) -> None:
        """Register this rank's extended rgb strip with a libktiler comm (ktiler.Comm)."""
        bid, W, H, F, elem, pitch = self.pipe.b.bufs["rgb"]
        comm.register_strip(self.rank, self.rgb_ext().data_ptr(), pitch, W * elem, self.o0, self.o1, self.e0, self.e1)

    def attach(self, comm) -> None:
        """Register the strip and put the exchange into the current plan's graph, ahead of
        the schedule (ktiler_plan_attach_halo): one execute = exchange + tiled schedule."""
        self.register(comm)
        self.pipe.plan_obj.attach_halo(comm, self.rank, HALO_ROWS)

    def plan(self, cache_bytes: int = 0, **policy):
        return self.pipe.plan(cache_bytes, **policy)

    def run(self, stream: int | None = None, group=None) -> None:
        if self.world > 1:
            self.exchange(group)
        self.pipe.run(stream)


def nccl_comm(world: int, rank: int):
    """A libktiler NCCL comm over the ranks of the default torch.distributed group (the
    unique id travels through the process group's broadcast)."""
    import torch.distributed as dist
    from . import ktiler as K
    obj = [K.comm_unique_id() if rank == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return K.Comm.nccl(obj[0], world, rank)
