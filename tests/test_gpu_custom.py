"""§8(f) f3 on an opaque user kernel: the paper's block analyzer is
"oblivious to kernel functionalities" and finds dependencies from sample
runs.  Here a USER kernel the library knows nothing about
(tests/custom_ops/asym_box.cu: an asymmetric 2 x 5 box filter, launched through the
KTILER_OP_CUSTOM callback) sits between two built-ins:

    rgb -> gray (built-in) -> box (user kernel) -> down2 (built-in)

1. It is declared with a naive footprint (its own tile, no halo).
2. ktiler_discover_footprint finds what its blocks really write (exactly the tile) and read
   (rows y..y+1 — the asymmetric reach — and columns x-2..x+2, line-quantized).
3. footprint.fit_access turns that into the affine map; the graph is re-declared with it,
   planned into many fragments and run tiled in the default executor (GRAPH_DAG, the
   callback captured per sub-kernel) and in STREAM / GRAPH — bit-exact against an oracle
   of the chain (the built-ins' oracle + the box filter's plain definition below)."""
import ctypes
import os
import subprocess

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from inputs import synth  # noqa: E402
from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))
TW, TH = 64, 16


class BoxUser(ctypes.Structure):
    _fields_ = [("inp", ctypes.c_void_p), ("out", ctypes.c_void_p), ("W", ctypes.c_int64), ("H", ctypes.c_int64),
                ("pitch_in", ctypes.c_int64), ("pitch_out", ctypes.c_int64), ("fs_in", ctypes.c_int64),
                ("fs_out", ctypes.c_int64), ("tw", ctypes.c_int32), ("th", ctypes.c_int32)]


@pytest.fixture(scope="module")
def boxlib():
    import __graft_entry__ as ge
    from paper_conf_date_maghazeh0ep19_b200 import build as B
    ge.build()
    src = os.path.join(HERE, "custom_ops", "asym_box.cu")
    so = os.path.join(HERE, "custom_ops", "libasym_box.so")
    if not os.path.exists(so) or os.path.getmtime(so) < os.path.getmtime(src):
        subprocess.check_call([B.NVCC, *B.ARCH, "-O2", "-shared", "-Xcompiler", "-fPIC", "-cudart", "static", "-o", so, src])
    return ctypes.CDLL(so)


def box_oracle(g: np.ndarray) -> np.ndarray:
    """The user kernel's plain definition: (sum of in[min(y+dy,H-1)][clamp(x+dx)], dy in
    0..1, dx in -2..2, + 5) // 10 — replicate border."""
    F, H, W = g.shape
    a = g.astype(np.int32)
    yy = np.minimum(np.arange(H)[:, None] + np.arange(2)[None, :], H - 1)        # [H, 2]
    xx = np.clip(np.arange(W)[:, None] + np.arange(-2, 3)[None, :], 0, W - 1)   # [W, 5]
    s = a[:, yy][:, :, :, xx].sum(axis=(2, 4))
    return ((s + 5) // 10).astype(np.uint8)


def _alloc(nbytes):
    t = torch.empty(nbytes + 128, dtype=torch.uint8, device="cuda")
    off = (-t.data_ptr()) % 128
    return t[off:off + nbytes]


class Chain:
    def __init__(self, lib, W, H, F, read_access=None):
        from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
        self.W, self.H, self.F = W, H, F
        self.t = {"rgb": _alloc(F * H * W * 3), "gray": _alloc(F * H * W), "box": _alloc(F * H * W),
                  "down": _alloc(F * (H // 2) * (W // 2))}
        g = K.Graph()
        self.g = g
        self.id = {"rgb": g.add_buffer(self.t["rgb"].data_ptr(), W, H, 3, frames=F, frame_stride_bytes=H * W * 3),
                   "gray": g.add_buffer(self.t["gray"].data_ptr(), W, H, 1, frames=F, frame_stride_bytes=H * W,
                                        internal=True),
                   "box": g.add_buffer(self.t["box"].data_ptr(), W, H, 1, frames=F, frame_stride_bytes=H * W,
                                       internal=True),
                   "down": g.add_buffer(self.t["down"].data_ptr(), W // 2, H // 2, 1, frames=F,
                                        frame_stride_bytes=(H // 2) * (W // 2))}
        i = self.id
        cd = lambda a, b: -(-a // b)  # noqa: E731
        self.user = BoxUser(self.t["gray"].data_ptr(), self.t["box"].data_ptr(), W, H, W, W, H * W, H * W, TW, TH)
        self.n_gray = g.add_kernel(K.OP_GRAY, (cd(W, TW), cd(H, TH), F), (64, 1, 1),
                                   [dict(buf=i["rgb"], mode=K.READ, ax=TW, ay=TH), dict(buf=i["gray"], mode=K.WRITE, ax=TW, ay=TH)])
        ra = read_access or dict(buf=i["gray"], mode=K.READ, ax=TW, ay=TH)  # naive: its own tile
        self.n_box = g.add_kernel(K.OP_CUSTOM, (cd(W, TW), cd(H, TH), F), (256, 1, 1),
                                  [ra, dict(buf=i["box"], mode=K.WRITE, ax=TW, ay=TH)],
                                  launch=ctypes.cast(lib.asym_box_launch, ctypes.c_void_p).value,
                                  user=ctypes.addressof(self.user))
        self.n_down = g.add_kernel(K.OP_DOWN2, (cd(W // 2, 32), cd(H // 2, 8), F), (64, 1, 1),
                                   [dict(buf=i["box"], mode=K.READ, ax=64, ay=16), dict(buf=i["down"], mode=K.WRITE, ax=32, ay=8)])
        g.add_edge(self.n_gray, self.n_box, i["gray"], 1.0)
        g.add_edge(self.n_box, self.n_down, i["box"], 1.0)

    def view(self, name):
        F, H, W = self.F, self.H, self.W
        shape = {"rgb": (F, H, W, 3), "gray": (F, H, W), "box": (F, H, W), "down": (F, H // 2, W // 2)}[name]
        return self.t[name].view(*shape)


W, H, F = 512, 96, 2


def _discover(lib):
    from paper_conf_date_maghazeh0ep19_b200 import footprint as FP
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    c = Chain(lib, W, H, F)
    descs = {c.id["rgb"]: (W * 3, H * W * 3, 3), c.id["gray"]: (W, H * W, 1), c.id["box"]: (W, H * W, 1),
             c.id["down"]: (W // 2, (H // 2) * (W // 2), 1)}
    gx, gy = W // TW, H // TH
    blocks = [(0, 0, 0), (gx - 1, gy - 1, 1), (gx // 2, gy // 2, 0), (gx - 1, 0, 0), (0, gy - 1, 1), (3, 2, 1)]
    reads, writes = {}, {}
    for b in blocks:
        recs = c.g.discover_footprint(c.n_box, *b, trials=3, seed=5)
        rr = FP.rects(recs, descs, K.READ)
        ww = FP.rects(recs, descs, K.WRITE)
        assert set(rr) == {c.id["gray"]} and set(ww) == {c.id["box"]}  # touches only its own buffers
        reads[b[:2]] = rr[c.id["gray"]]
        writes[b[:2]] = ww[c.id["box"]]
    return c, reads, writes


def test_discover_user_kernel(boxlib):
    from paper_conf_date_maghazeh0ep19_b200 import footprint as FP
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    c, reads, writes = _discover(boxlib)
    for (bx, by), wr in writes.items():  # writes: exactly the block's tile
        assert wr[:2] == (bx * TW, by * TH) and wr[3:5] == (min(W, (bx + 1) * TW), min(H, (by + 1) * TH))
    for (bx, by), rd in reads.items():  # reads: rows y0 .. y1 (the +1 reach, clipped), x reach 2 px
        assert rd[1] == by * TH and rd[4] == min(H, (by + 1) * TH + 1)
        assert rd[0] <= max(0, bx * TW - 2) and rd[3] >= min(W, (bx + 1) * TW + 2)
    acc = FP.fit_access(reads, c.id["gray"], K.READ, W, H, ax=TW, ay=TH)
    assert (acc["ht"], acc["hb"]) == (0, 1)      # the asymmetric 2-row reach, found exactly
    assert acc["hl"] >= 2 and acc["hr"] >= 2     # >= the 2-px reach (128-B line quantized)


@pytest.mark.parametrize("mode", ["dag", "dag_pdl", "graph", "stream"])
def test_user_kernel_tiled_after_discovery(boxlib, mode):
    """dag_pdl: the bench's DAG policy (programmatic producer edges, dispatch-order edges from
    the source's consumers, A50) with a user kernel as the source's consumer: the
    order and PDL edges skip it (a child graph has no programmatic port)."""
    from paper_conf_date_maghazeh0ep19_b200 import footprint as FP
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    c0, reads, _ = _discover(boxlib)
    acc = FP.fit_access(reads, c0.id["gray"], K.READ, W, H, ax=TW, ay=TH)
    c = Chain(boxlib, W, H, F, read_access=acc)  # re-declared with the discovered map
    rgb = synth.scene(31, W, H, F)
    c.view("rgb").copy_(torch.from_numpy(rgb))
    for k in ("gray", "box", "down"):
        c.t[k].fill_(0xA5)
    if mode == "dag_pdl":
        plan = c.g.plan(48 * 1024, kind="budget", exec_mode="dag", pdl=True, resident_budget=True, window=2)
    else:
        plan = c.g.plan(48 * 1024, kind="budget", exec_mode=mode)
    assert plan.num_fragments() >= 4
    for _ in range(2):  # replays (DAG: the captured callback runs again)
        plan.execute(torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    g = O.gray(rgb)
    want = O.down2(box_oracle(g))
    assert np.array_equal(c.view("box").cpu().numpy(), box_oracle(g))
    assert np.array_equal(c.view("down").cpu().numpy(), want)
