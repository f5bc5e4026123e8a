"""Host-to-host execution of a frame batch, chunked and double-buffered (the end-to-end
path bench.py times as ``e2e``).

A batch that starts in host memory is bounded by the host link, not by the kernels: on
B200 the 6.4 GB of RGB of 64 8K frames take ~120 ms over PCIe against ~3.3 ms of tiled
compute.  ``FrameStreamer`` splits the batch into chunks of ``chunk`` frames and runs
them through ``nbuf`` independent pipelines (each with its own device buffers, KTILER
plan and CUDA stream), so chunk i+1's host->device copy overlaps chunk i's kernels and
its device->host copy of the mask (copy engines run both directions at once).  Every
chunk goes through the C ABI's ``ktiler_execute_host`` (copies in, ``ktiler_execute``,
copies out, in stream order), so reusing a pipeline's buffers for chunk i+nbuf is
ordered after chunk i by its stream.  Nothing here computes: all arithmetic runs in
libktiler's kernels; torch provides the buffers and streams."""
from __future__ import annotations

from .pipeline import Pipeline


class FrameStreamer:
    def __init__(self, W: int, H: int, chunk: int, T: float = 200.0, nbuf: int = 2, cache_bytes: int = 0,
                 **policy):
        import torch
        self.W, self.H, self.chunk, self.nbuf = W, H, chunk, nbuf
        self.pipes = [Pipeline(W, H, chunk, T=T, internal=True) for _ in range(nbuf)]
        self.plans = [p.plan(cache_bytes, **policy) for p in self.pipes]
        self.streams = [torch.cuda.Stream() for _ in range(nbuf)]
        self.rgb_id = self.pipes[0].buf_id("rgb")
        self.mask_id = self.pipes[0].buf_id("mask")

    def run(self, rgb_host, mask_host, stream=None) -> None:
        """rgb_host: pinned uint8 [F, H, W, 3]; mask_host: pinned uint8 [F, H/2, W/2];
        F a multiple of ``chunk``.  Asynchronous; ordered after the work already on
        ``stream`` (a torch stream, default the current one), which in turn waits for the
        whole batch, so events on it time the batch end to end."""
        import torch
        caller = stream if stream is not None else torch.cuda.current_stream()
        start = torch.cuda.Event()
        start.record(caller)
        for st in self.streams:
            st.wait_event(start)
        F = rgb_host.shape[0]
        if F % self.chunk or tuple(rgb_host.shape[1:]) != (self.H, self.W, 3):
            raise ValueError("rgb_host must be [k*chunk, H, W, 3]")
        fin = self.H * self.W * 3
        fout = (self.H // 2) * (self.W // 2)
        for i, f0 in enumerate(range(0, F, self.chunk)):
            k = i % self.nbuf
            self.plans[k].execute_host([(self.rgb_id, rgb_host.data_ptr() + f0 * fin, 0, 0)],
                                       [(self.mask_id, mask_host.data_ptr() + f0 * fout, 0, 0)],
                                       self.streams[k].cuda_stream)
        for st in self.streams:
            done = torch.cuda.Event()
            done.record(st)
            caller.wait_event(done)

    def wait(self) -> None:
        for s in self.streams:
            s.synchronize()
