"""Multi-process (gloo, CPU) tests of the strip partitioning path: the halo
exchange over torch.distributed fills exactly the neighbour rows, and running the graph
on each extended strip then keeping the owned mask rows reproduces the whole-image
result bit for bit.  The per-strip compute here is the oracle (tests may use it); the
GPU variant of the same bookkeeping is in test_gpu_parity.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from inputs import synth
from oracle import oracle as O
from paper_conf_date_maghazeh0ep19_b200 import strips as S


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, W, H, seed, T, out_dir):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        full = synth.uniform(seed, W, H, 1)[0]  # [H, W, 3]; each rank uses only its own rows
        o0, o1, e0, e1 = S.strip_rows(H, world, rank)
        ext = torch.zeros((e1 - e0, W, 3), dtype=torch.uint8)
        ext[o0 - e0:o1 - e0] = torch.from_numpy(full[o0:o1])
        nbytes = S.exchange_halo(ext, o0, o1, e0, e1, rank, world)
        halo_ok = bool(np.array_equal(ext.numpy(), full[e0:e1]))
        mask = O.pipeline(ext.numpy()[None], T=T)["mask"][0]
        m0, m1 = S.owned_mask_rows(o0, o1, e0)
        own = torch.from_numpy(np.ascontiguousarray(mask[m0:m1]))
        parts = [torch.empty_like(own) for _ in range(world)]
        dist.all_gather(parts, own)
        if rank == 0:
            got = torch.cat(parts).numpy()
            want = O.pipeline(full[None], T=T)["mask"][0]
            np.save(os.path.join(out_dir, "got.npy"), got)
            np.save(os.path.join(out_dir, "want.npy"), want)
        np.save(os.path.join(out_dir, f"r{rank}.npy"), np.array([halo_ok, nbytes, o0, o1, e0, e1]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,W,H", [(2, 64, 40), (3, 48, 36), (4, 32, 48)])
def test_strips_gloo_equal_whole_image(tmp_path, world, W, H):
    port = _free_port()
    mp.spawn(_worker, args=(world, port, W, H, 11, 30.0, str(tmp_path)), nprocs=world, join=True)
    got, want = np.load(tmp_path / "got.npy"), np.load(tmp_path / "want.npy")
    assert got.shape == want.shape == (H // 2, W // 2)
    assert np.array_equal(got, want)
    for r in range(world):
        halo_ok, nbytes, o0, o1, e0, e1 = np.load(tmp_path / f"r{r}.npy")
        assert halo_ok
        halos = (r > 0) + (r < world - 1)
        assert nbytes == halos * S.HALO_ROWS * W * 3


def test_strip_rows_bookkeeping():
    H = 8192 * 8
    for world in (1, 2, 4, 8):
        cover = []
        for r in range(world):
            o0, o1, e0, e1 = S.strip_rows(H, world, r)
            assert o1 - o0 == H // world and e0 == max(0, o0 - 4) and e1 == min(H, o1 + 4)
            m0, m1 = S.owned_mask_rows(o0, o1, e0)
            assert m1 - m0 == (o1 - o0) // 2 and (e1 - e0) % 2 == 0
            cover.append((o0, o1))
        assert cover[0][0] == 0 and cover[-1][1] == H
        assert all(a[1] == b[0] for a, b in zip(cover, cover[1:]))
    with pytest.raises(ValueError):
        S.strip_rows(100, 3, 0)  # 100 rows do not split into 3 even strips
    with pytest.raises(ValueError):
        S.strip_rows(12, 6, 0)  # 2-row strips are shorter than the halo


def test_halo_reach_is_minimal():
    """Why HALO_ROWS = 4: the owned output of a strip with a 4-row halo equals the
    whole-image result; with a 2-row halo (the next even size down) it does not."""
    W, H = 32, 32
    full = synth.uniform(5, W, H, 1)[0]
    want = O.pipeline(full[None], T=30.0)
    o0, o1 = 16, 32  # the lower of two strips
    for halo, ok in ((4, True), (2, False)):
        e0 = o0 - halo
        got = O.pipeline(full[None, e0:o1], T=30.0)
        m0 = (o0 - e0) // 2
        assert np.array_equal(got["sob"][0, m0:], want["sob"][0, o0 // 2:]) == ok
