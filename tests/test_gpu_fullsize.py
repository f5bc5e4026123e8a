"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(SURVEY §8(c) P12 at scale): the default fragment policy of ``bench.policy``, the B200
geometry, the bench's seeded input (``scene(1234)``, generated on the device by the input
generator's GPU twin, exactly as bench.py does).

The oracle cannot run 2.1 Gpx in seconds, so the checks are
  * sampled outputs the oracle computes one by one: whole 8K frames of the 64-frame batch,
    and row bands of the 16384^2 and 65536^2 images (the oracle runs on the band plus a
    margin of rows; the chain's reach is 4 full-res rows (strips.HALO_ROWS), so with a
    16-row margin the band's interior mask rows are exact, and bands touching the image
    edge clamp like the whole image);
  * a property that holds at any size: the tiled schedule's mask equals the untiled
    schedule's mask bit for bit on every frame / row (schedule invariance, P10).
Oracle inputs come from inputs/synth (CPU), never from the device."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from inputs import synth  # noqa: E402
from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu

SEED = 1234
MARGIN = 16  # full-res rows of context around a sampled band (> the chain's reach of 4)


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__ as ge
    ge.build()


def _bench_policy():
    import bench
    return bench.policy(bench.parse([]))


def _pipeline(W, H, F):
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    p = Pipeline(W, H, F, T=200.0, internal=True)
    G.fill("scene", SEED, p.view("rgb").data_ptr(), W * 3, W * 3 * H, W, H, F=F,
           stream=torch.cuda.current_stream().cuda_stream)
    p.b.store.tensors["mask"].fill_(0xA5)
    return p


def _run(p, **pol):
    plan = p.plan(0, **pol)
    p.run()
    torch.cuda.synchronize()
    return plan


def _band_oracle(s, W, H, m0, m1):
    """Oracle mask rows [m0, m1) of frame seed s, from an rgb row band with a margin."""
    y0, y1 = max(0, 2 * m0 - MARGIN), min(H, 2 * m1 + MARGIN)
    band = synth.scene_rows(s, W, H, y0, y1)[None]
    mask = O.pipeline(band)["mask"][0]
    return mask[m0 - y0 // 2:m1 - y0 // 2]


def test_batch64_8k_bench_config():
    """BASELINE configs[3] at full size (64 x 7680x4320) under the bench's default plan."""
    W, H, F = 7680, 4320, 64
    pol = _bench_policy()
    p = _pipeline(W, H, F)
    plan = _run(p, **pol)
    assert plan.num_fragments() > 1  # really tiled (at 1.25 x L2 a fragment spans ~1.5 frames)
    tiled = p.view("mask").clone()
    for f in (0, 37, 63):  # whole frames, one by one
        ref = O.pipeline(synth.scene_rows(SEED + f, W, H, 0, H)[None])["mask"][0]
        assert np.array_equal(tiled[f].cpu().numpy(), ref), f"frame {f}"
    p.b.store.tensors["mask"].fill_(0xA5)
    _run(p, kind="none", exec_mode="graph", discard=False)
    assert torch.equal(tiled, p.view("mask")), "tiled != untiled on some frame"


@pytest.mark.parametrize("W", [16384, 65536])
def test_giant_image_bench_config(W):
    """BASELINE configs[2] (16384^2) and configs[4] (65536^2 as one strip, N = 1) at full
    size: sampled mask row bands (top edge, interior, fragment-sized middle, bottom edge)
    against the oracle, and tiled == untiled on the whole image."""
    H = W
    pol = _bench_policy()
    p = _pipeline(W, H, 1)
    plan = _run(p, **pol)
    assert plan.num_fragments() > 1
    tiled = p.view("mask")[0].clone()
    hm = H // 2
    for m0, m1 in ((0, 24), (hm // 3 - 5, hm // 3 + 19), (hm // 2 - 12, hm // 2 + 12), (hm - 24, hm)):
        ref = _band_oracle(SEED, W, H, m0, m1)
        assert np.array_equal(tiled[m0:m1].cpu().numpy(), ref), f"mask rows [{m0}, {m1})"
    p.b.store.tensors["mask"].fill_(0xA5)
    _run(p, kind="none", exec_mode="graph", discard=False)
    assert torch.equal(tiled, p.view("mask")[0]), "tiled != untiled"


@pytest.mark.parametrize("name,pol,ring", [
    ("flow", dict(kind="rows", rows=1, exec_mode="flow", consumer_discard=True), 0),
    ("dag-ring4", dict(kind="budget", l2_fraction=0.85, exec_mode="dag", window=2, resident_budget=True,
                       consumer_discard=True), 4),
    ("dag-multirate", dict(kind="budget", l2_fraction=0.6, exec_mode="dag", window=3, resident_budget=True,
                           consumer_discard=True, multirate=True), 0)])
def test_batch64_8k_other_executors(name, pol, ring):
    """The round-2 variants at BASELINE configs[3]'s full size, as measured in DESIGN §6.6-6.8:
    the FLOW executor, ring intermediates (4 frames of storage for 64 frames) and multi-rate
    fragments.  One sampled frame against the oracle; every frame against the untiled mask."""
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 7680, 4320, 64
    p = Pipeline(W, H, F, T=200.0, internal=True, ring_frames=ring)
    G.fill("scene", SEED, p.view("rgb").data_ptr(), W * 3, W * 3 * H, W, H, F=F,
           stream=torch.cuda.current_stream().cuda_stream)
    p.b.store.tensors["mask"].fill_(0xA5)
    plan = _run(p, **pol)
    assert plan.num_fragments() > 1
    got = p.view("mask").clone()
    ref = O.pipeline(synth.scene_rows(SEED + 50, W, H, 0, H)[None])["mask"][0]
    assert np.array_equal(got[50].cpu().numpy(), ref)
    u = _pipeline(W, H, F)
    _run(u, kind="none", exec_mode="graph", discard=False)
    assert torch.equal(got, u.view("mask")), f"{name}: tiled != untiled on some frame"
