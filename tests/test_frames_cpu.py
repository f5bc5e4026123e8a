"""Multi-process (gloo, CPU) tests of the frame-batch sharding path (SURVEY §8(e),
BASELINE configs[3]): the one batch is split into contiguous frame ranges, each rank runs
the graph on its own frames with no data-path collective, timing is the max over ranks
and the job's throughput counts every rank's pixels.  The per-rank compute here is the
oracle (tests may use it); on GPUs bench.py runs the same bookkeeping through libktiler."""
import os
import socket
import time

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from inputs import synth
from oracle import oracle as O
from paper_conf_date_maghazeh0ep19_b200 import frames as FR


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, total, W, H, seed, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        f0, n = FR.frame_range(total, world, rank)
        # frame f of the batch is scene(seed + f): each rank generates only its own frames
        rgb = synth.scene(seed + f0, W, H, n)
        dist.barrier()
        t0 = time.perf_counter()
        mask = O.pipeline(rgb, T=30.0)["mask"]
        # a deliberately unequal per-rank time: the job time must be the slowest rank's
        time.sleep(0.05 * rank)
        ms = (time.perf_counter() - t0) * 1e3
        dist.barrier()
        job_ms = FR.max_over_ranks(ms, world)
        pix = [W * H * FR.frame_range(total, world, r)[1] for r in range(world)]
        value = FR.job_mpix_per_s(pix, job_ms)
        # gather the masks (frames of different ranks may differ in count: pad to the max)
        nmax = -(-total // world)
        buf = torch.zeros((nmax, H // 2, W // 2), dtype=torch.uint8)
        buf[:n] = torch.from_numpy(mask)
        parts = [torch.empty_like(buf) for _ in range(world)]
        dist.all_gather(parts, buf)
        mss = [torch.zeros(1, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(mss, torch.tensor([ms], dtype=torch.float64))
        if rank == 0:
            got = np.concatenate([parts[r][:FR.frame_range(total, world, r)[1]].numpy() for r in range(world)])
            np.save(os.path.join(out_dir, "got.npy"), got)
            np.save(os.path.join(out_dir, "t.npy"), np.array([job_ms, value] + [float(m) for m in mss]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,total", [(2, 4), (3, 5), (2, 3)])
def test_frames_gloo_equal_whole_batch(tmp_path, world, total):
    W, H, seed = 48, 32, 21
    port = _free_port()
    mp.spawn(_worker, args=(world, port, total, W, H, seed, str(tmp_path)), nprocs=world, join=True)
    got = np.load(tmp_path / "got.npy")
    want = O.pipeline(synth.scene(seed, W, H, total), T=30.0)["mask"]
    assert got.shape == want.shape == (total, H // 2, W // 2)
    assert np.array_equal(got, want)
    job_ms, value, *mss = np.load(tmp_path / "t.npy")
    assert job_ms == pytest.approx(max(mss))       # max over ranks
    assert job_ms >= 50.0 * (world - 1)            # the slowest rank slept longest
    assert value == pytest.approx(total * W * H / (job_ms / 1e3) / 1e6)


def test_frame_range_covers_the_batch():
    for total in (1, 3, 8, 63, 64):
        for world in range(1, min(total, 9) + 1):
            rs = [FR.frame_range(total, world, r) for r in range(world)]
            assert rs[0][0] == 0 and sum(n for _, n in rs) == total
            assert all(a[0] + a[1] == b[0] for a, b in zip(rs, rs[1:]))
            assert max(n for _, n in rs) - min(n for _, n in rs) <= 1
    assert FR.frame_range(64, 8, 3) == (24, 8)  # BASELINE configs[3] on 8 GPUs: 8 frames each
    with pytest.raises(ValueError):
        FR.frame_range(2, 3, 0)
