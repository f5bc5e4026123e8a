"""GPU parity: the CUDA path through the C ABI vs the CPU oracle,
element by element, on the same seeded inputs.  Integer/uint8 outputs and the Sobel f32
magnitude are compared bit for bit (every float in the canonical chain is
exact by construction).

Two tile geometries: the B200 geometry bench.py uses (pipeline.B200_GEOMETRY: 512x64 /
256x32 tiles) and a SMALL geometry whose tiles are small enough that images of a few
hundred pixels split into tens of fragments, so tiling, fragment edges, ragged Alg. 2
fragments and discards are exercised at sizes the oracle finishes in seconds."""
import os

import numpy as np
import pytest

torch = pytest.importorskip("torch")

from inputs import synth  # noqa: E402
from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu

KEYS = ("gray", "blur", "down", "sob", "mask")
SMALL = {"gray": (64, 16, 64), "blur": (64, 16, 64), "down": (32, 8, 64), "sobel": (32, 8, 64), "thresh": (32, 8, 64)}


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__ as ge
    ge.build()
    from paper_conf_date_maghazeh0ep19_b200 import ktiler
    ktiler.lib()


def _run(W, H, F, rgb, T=200.0, cache_bytes=0, internal=False, geometry=SMALL, **pol):
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    p = Pipeline(W, H, F, T=T, internal=internal, geometry=geometry)
    # poison intermediates and output so a skipped block cannot pass
    for k in KEYS:
        p.b.store.tensors[k].fill_(0xA5)
    p.view("rgb").copy_(torch.from_numpy(rgb))
    plan = p.plan(cache_bytes, **pol)
    p.run()
    torch.cuda.synchronize()
    out = {k: p.view(k).cpu().numpy() for k in KEYS}
    return out, plan


def _eq(a, b):
    return np.array_equal(a.view(np.uint8), b.view(np.uint8))


SIZES = [(512, 64, 1), (520, 102, 1), (1040, 256, 2), (2, 2, 1), (16, 4, 1), (34, 18, 3), (7680 // 8, 4320 // 8, 2),
         (1552, 136, 1)]


@pytest.mark.parametrize("W,H,F", SIZES)
@pytest.mark.parametrize("kind", ["uniform", "scene"])
@pytest.mark.parametrize("geo", ["b200", "small"])
def test_each_kernel_untiled(W, H, F, kind, geo):
    """Every kernel bit-exact: several tiles, ragged right/bottom tails, tiny images."""
    rgb = synth.make(kind, W + H, W, H, F)
    ref = O.pipeline(rgb, T=40.0)
    out, _ = _run(W, H, F, rgb, T=40.0, kind="none", exec_mode="stream", geometry=None if geo == "b200" else SMALL)
    for k in KEYS:
        assert _eq(out[k], ref[k]), k


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("kind", ["uniform", "scene"])
def test_parity_seeds_tiled(seed, kind):
    W, H, F = 1536, 320, 2
    rgb = synth.make(kind, seed, W, H, F)
    ref = O.pipeline(rgb, T=60.0)
    out, plan = _run(W, H, F, rgb, T=60.0, cache_bytes=120 * 1024, kind="budget", exec_mode="graph")
    assert plan.num_fragments() > 20
    for k in KEYS:
        assert _eq(out[k], ref[k]), k


def test_closed_form_images():
    W, H = 768, 256
    for rgb in (synth.constant((17, 200, 3), W, H), synth.ramp(0, 1, W, H), synth.checkerboard(5, W, H),
                synth.half_black_white(W, H)):
        ref = O.pipeline(rgb, T=100.0)
        out, _ = _run(W, H, 1, rgb, T=100.0, cache_bytes=100 * 1024, kind="budget", exec_mode="stream")
        for k in KEYS:
            assert _eq(out[k], ref[k]), k


MODES = [
    dict(exec_mode="stream"),
    dict(exec_mode="graph"),
    dict(exec_mode="graph", pdl=True),
    dict(exec_mode="persist_l2"),
    dict(exec_mode="persistent"),
    dict(exec_mode="persistent", skew=-1),
    dict(exec_mode="persistent", skew=3, persistent_ctas=7),
    dict(exec_mode="dag"),
    dict(exec_mode="dag", pdl=True),  # programmatic edges from each sub-kernel's producers
    dict(exec_mode="dag", consumer_discard=True),  # down2 / thresh drop their consumed lines
    dict(exec_mode="graph", consumer_discard=True),
    dict(exec_mode="dag", consumer_discard=True, halo_discard=True),  # + counted halo-reader discards
    dict(exec_mode="dag", window=1),
    dict(exec_mode="dag", window=4),
    dict(exec_mode="chain"),
    dict(exec_mode="wave"),
]
POLICIES = [
    dict(kind="none"),
    dict(kind="budget", cache_bytes=60 * 1024),
    dict(kind="budget", cache_bytes=300 * 1024, l2_fraction=0.5),
    dict(kind="rows", rows=1),
    dict(kind="rows", rows=3),
    dict(kind="balanced", cache_bytes=200 * 1024),
    dict(kind="budget", cache_bytes=60 * 1024, resident_budget=True),
]


@pytest.mark.parametrize("mode", MODES, ids=lambda m: "-".join(f"{k}={v}" for k, v in m.items()))
@pytest.mark.parametrize("pol", POLICIES, ids=lambda m: "-".join(f"{k}={v}" for k, v in m.items()))
@pytest.mark.parametrize("discard", [False, True])
def test_modes_policies(mode, pol, discard):
    """Whole graph in every exec mode x fragment policy x discard: mask bit-exact (and all
    intermediates when they are not discarded)."""
    W, H, F = 1040, 230, 2
    rgb = synth.scene(5, W, H, F)
    ref = O.pipeline(rgb, T=50.0)
    pol = dict(pol)
    cb = pol.pop("cache_bytes", 1 << 20)
    out, plan = _run(W, H, F, rgb, T=50.0, cache_bytes=cb, internal=discard, discard=discard, **mode, **pol)
    keys = ("mask",) if discard else KEYS
    for k in keys:
        assert _eq(out[k], ref[k]), k


@pytest.mark.parametrize("mode", ["graph", "persistent", "chain"])
def test_b200_geometry_tiled(mode):
    """The bench geometry itself, tiled into several fragments (budget just above one closure)."""
    W, H, F = 2048, 1024, 2
    rgb = synth.scene(17, W, H, F)
    ref = O.pipeline(rgb, T=45.0)
    out, plan = _run(W, H, F, rgb, T=45.0, cache_bytes=3 << 20, geometry=None, internal=True, discard=True,
                     kind="budget", exec_mode=mode)
    assert plan.num_fragments() >= 3
    assert _eq(out["mask"], ref["mask"])


BENCH_POLICY = dict(kind="budget", exec_mode="dag", window=2, resident_budget=True, consumer_discard=True, pdl=True)


@pytest.mark.parametrize("W,H,F", [(2000, 1082, 3), (1538, 770, 2), (4100, 520, 1)])
@pytest.mark.parametrize("mode", ["dag-bench", "flow", "persistent"])
def test_b200_geometry_ragged(W, H, F, mode):
    """The shipped geometry (thresh 256x64 tiles: one sobel tile) on ragged sizes (no axis a
    multiple of any tile), tiled into several fragments: the bench's own policy, and FLOW /
    PERSISTENT on their one-CTA-per-SM fallbacks for 64 KB tiles; intermediates too."""
    rgb = synth.scene(W + H + F, W, H, F)
    ref = O.pipeline(rgb, T=45.0)
    pol = dict(BENCH_POLICY) if mode == "dag-bench" else dict(kind="rows", rows=1, exec_mode=mode)
    cb = (2 << 20) if mode == "dag-bench" else (4 << 20)  # the resident budget counts intermediates only
    out, plan = _run(W, H, F, rgb, T=45.0, cache_bytes=cb, geometry=None, internal=False, **pol)
    assert plan.num_fragments() >= 3
    for k in KEYS:
        assert _eq(out[k], ref[k]), k


REPLAY = [("graph", dict(discard=True)), ("persistent", dict(discard=True)), ("chain", dict(discard=True)),
          ("wave", dict(discard=True)),
          # bench.py's executor and its discard variants: the halo-reader counters persist
          # across executes and must reset themselves
          ("dag", dict(window=2, resident_budget=True, consumer_discard=True)),
          ("dag", dict(window=2, resident_budget=True, consumer_discard=True, pdl=True)),  # bench default
          ("dag", dict(window=2, consumer_discard=True, halo_discard=True)),
          ("dag", dict(window=2, consumer_discard=True, halo_discard=True, discard=True)),
          ("flow", dict(kind="rows", rows=1, consumer_discard=True)),
          ("flow", dict(kind="rows", rows=2, consumer_discard=True, window=3))]


@pytest.mark.parametrize("mode,pol", REPLAY, ids=[f"{m}-{'-'.join(sorted(k))}" for m, k in REPLAY])
def test_replay_is_idempotent(mode, pol):
    """A plan executes many times (GRAPH replays, persistent epochs, per-execute counters)
    with identical output, alternating inputs."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 1024, 128, 1
    pol = dict(pol)
    kind = pol.pop("kind", "budget")
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL)
    a = synth.uniform(1, W, H, F)
    b = synth.scene(2, W, H, F)
    plan = p.plan(100 * 1024, kind=kind, exec_mode=mode, **pol)
    assert plan.num_fragments() > 1
    for it in range(6):
        x = a if it % 2 == 0 else b
        p.view("rgb").copy_(torch.from_numpy(x))
        p.run()
        torch.cuda.synchronize()
        assert np.array_equal(p.view("mask").cpu().numpy(), O.pipeline(x, T=40.0)["mask"]), (mode, it)


@pytest.mark.parametrize("geometry", ["paper", "b200"])
@pytest.mark.parametrize("lines", [36, 68, 2176, 0])
@pytest.mark.parametrize("mode", ["graph", "persistent"])
def test_motivational_graph(geometry, lines, mode):
    """configs[0]: 256x256 RGB -> A -> B, paper geometry and B200 geometry, budgets from
    the worked example (36 lines = 64 fragments, 2176 = untiled) and the device L2."""
    from paper_conf_date_maghazeh0ep19_b200 import Motivational
    rgb = synth.scene(1234, 256, 256)
    ref = O.motivational(rgb)
    m = Motivational(device="cuda", geometry=geometry, internal=False)
    m.b.store.tensors["intm"].fill_(0xA5)
    m.b.store.tensors["out"].fill_(0xA5)
    m.view("in").copy_(torch.from_numpy(rgb))
    try:
        plan = m.plan(lines * 128, kind="budget", exec_mode=mode)
    except Exception as e:  # b200 tiles are larger than 36 / 68 lines
        assert geometry == "b200" and "UNTILEABLE" in str(e)
        return
    if geometry == "paper" and lines == 36:
        assert plan.num_fragments() == 64
    m.run()
    torch.cuda.synchronize()
    assert np.array_equal(m.view("intm").cpu().numpy(), ref["gray"])
    assert np.array_equal(m.view("out").cpu().numpy(), ref["down"])


def test_schedule_invariance_rows():
    """P10 on the GPU: differently interleaved valid schedules (ROWS plans with different
    fragment heights, persistent skews) all give the untiled result."""
    W, H, F = 768, 192, 1
    rgb = synth.uniform(3, W, H, F)
    ref = O.pipeline(rgb, T=30.0)
    for rows in (1, 2, 5, 12):
        out, _ = _run(W, H, F, rgb, T=30.0, kind="rows", rows=rows, exec_mode="stream")
        for k in KEYS:
            assert _eq(out[k], ref[k]), (rows, k)
        for skew in (-1, 1, 4):
            out, _ = _run(W, H, F, rgb, T=30.0, kind="rows", rows=rows, exec_mode="persistent", skew=skew)
            for k in KEYS:
                assert _eq(out[k], ref[k]), (rows, skew, k)


def test_host_io_end_to_end():
    """ktiler_execute_host: pinned host rgb in, host mask out, through the C ABI."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 1024, 200, 3
    rgb = synth.scene(9, W, H, F)
    ref = O.pipeline(rgb, T=70.0)
    p = Pipeline(W, H, F, T=70.0, internal=True, geometry=SMALL)
    plan = p.plan(100 * 1024, kind="budget", exec_mode="graph", discard=True)
    hin = torch.from_numpy(rgb).pin_memory()
    hout = torch.empty((F, H // 2, W // 2), dtype=torch.uint8).pin_memory()
    s = torch.cuda.current_stream().cuda_stream
    plan.execute_host([(p.buf_id("rgb"), hin.data_ptr(), 0, 0)], [(p.buf_id("mask"), hout.data_ptr(), 0, 0)], s)
    torch.cuda.synchronize()
    assert np.array_equal(hout.numpy(), ref["mask"])


def test_frame_streamer_end_to_end():
    """The double-buffered host-to-host path (bench.py's e2e): chunks of frames through two
    pipelines on two streams, each via ktiler_execute_host, equal the oracle frame by frame."""
    from paper_conf_date_maghazeh0ep19_b200.streaming import FrameStreamer
    W, H, F = 520, 198, 6
    rgb = synth.scene(11, W, H, F)
    ref = O.pipeline(rgb)["mask"]
    fs = FrameStreamer(W, H, 2, cache_bytes=1 << 20, kind="budget", exec_mode="dag")
    assert fs.plans[0].num_fragments() > 1
    rgb_h = torch.from_numpy(rgb).pin_memory()
    mask_h = torch.full((F, H // 2, W // 2), 0xA5, dtype=torch.uint8).pin_memory()
    for _ in range(2):  # reuse of both pipelines' buffers across runs
        fs.run(rgb_h, mask_h)
        torch.cuda.current_stream().synchronize()
        assert np.array_equal(mask_h.numpy(), ref)


def test_gpu_generator_matches_numpy():
    from inputs import gpu as G
    for kind in ("uniform", "scene"):
        W, H, F = 200, 60, 2
        t = torch.empty((F, H, W, 3), dtype=torch.uint8, device="cuda")
        G.fill(kind, 11, t.data_ptr(), W * 3, W * H * 3, W, H, F=F)
        torch.cuda.synchronize()
        assert np.array_equal(t.cpu().numpy(), synth.make(kind, 11, W, H, F))
        # a strip of rows
        s = torch.empty((1, 20, W, 3), dtype=torch.uint8, device="cuda")
        G.fill(kind, 11, s.data_ptr(), W * 3, 20 * W * 3, W, H, y0=17, rows=20, f0=1, F=1)
        torch.cuda.synchronize()
        assert np.array_equal(s.cpu().numpy()[0], synth.make(kind, 11, W, H, F)[1, 17:37])


@pytest.mark.parametrize("mode", ["graph", "chain", "persistent"])
def test_trace_records(mode):
    """ktiler_trace_*: one record per CTA (launch modes) or two per tile (persistent), with
    ordered timestamps; tracing does not change the result."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 1024, 256, 2
    rgb = synth.scene(21, W, H, F)
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL)
    p.view("rgb").copy_(torch.from_numpy(rgb))
    plan = p.plan(100 * 1024, kind="budget", exec_mode=mode, discard=True)
    plan.trace_enable(1 << 16)
    p.run()
    rec, n = plan.trace_read()
    assert n == len(rec) > 0
    assert (rec["t1"] >= rec["t0"]).all()
    if mode == "persistent":
        tiles = sum(s["n_blocks"] for s in plan.subkernels())
        assert (rec["kind"] == 2).sum() == tiles and (rec["kind"] == 1).sum() == tiles
    else:
        assert set(rec["kind"].tolist()) == ({0, 3, 4} if mode == "chain" else {0, 5, 6})
        assert set(rec["id"].tolist()) <= set(range(len(plan.launches())))
        if mode != "chain":  # CTA phases: start -> ready -> staged, one pair per op-kernel CTA
            k5, k6 = rec[rec["kind"] == 5], rec[rec["kind"] == 6]
            assert len(k5) == len(k6) > 0 and np.array_equal(np.sort(k6["t0"]), np.sort(k5["t1"]))
            node_of = np.array([node for (_, node, _) in plan.launches()])
            assert len(k5) == int((node_of[rec[rec["kind"] == 0]["id"].astype(np.int64)] >= 0).sum())
    assert np.array_equal(p.view("mask").cpu().numpy(), O.pipeline(rgb, T=40.0)["mask"])
    with pytest.raises(Exception):
        plan.trace_enable(16)  # after the first execute


def test_trace_shards_overflow():
    """ktiler_trace_* keeps at most ceil(capacity / 256) records per shard (per-CTA-and-SM
    counters, no device-wide atomic): past a shard's capacity records are dropped and
    counted, what is kept is whole and valid, and the result is unchanged."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 1024, 256, 2
    rgb = synth.scene(22, W, H, F)
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL)
    p.view("rgb").copy_(torch.from_numpy(rgb))
    plan = p.plan(100 * 1024, kind="budget", exec_mode="dag", pdl=True, consumer_discard=True, resident_budget=True)
    plan.trace_enable(256)  # one record per shard
    p.run()
    rec, n = plan.trace_read()
    assert n > 256 >= len(rec) > 0  # more CTAs than kept records
    assert (rec["t1"] >= rec["t0"]).all() and (rec["t0"] > 0).all()
    assert set(rec["kind"].tolist()) <= {0, 5, 6}
    assert set(rec["id"].tolist()) <= set(range(len(plan.launches())))
    p.run()
    rec2, n2 = plan.trace_read()  # counters were reset by the read
    assert n2 == n and 0 < len(rec2) <= 256  # which records fit depends on the SMs the CTAs ran on
    assert np.array_equal(p.view("mask").cpu().numpy(), O.pipeline(rgb, T=40.0)["mask"])


@pytest.mark.parametrize("world", [2, 4])
@pytest.mark.parametrize("mode", ["graph", "dag", "wave", "stream", "flow"])
def test_strips_on_one_gpu(world, mode):
    """§8(e) strip path, GPU side, through the real exchange: every emulated rank holds only
    its OWN rows; the 1-GPU loopback comm (libktiler ktiler_halo_exchange, one
    cudaMemcpy2DAsync per halo) attached to each rank's plan fills the halo rows inside the
    plan's graph; concatenated owned masks == whole-image oracle.  The halo rows are
    poisoned first, so a missing exchange cannot pass."""
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    from paper_conf_date_maghazeh0ep19_b200.strips import StripPipeline
    W, H = 1024, 512
    full = synth.scene(77, W, H, 1)[0]
    want = O.pipeline(full[None], T=45.0)["mask"][0]
    comm = K.Comm.loopback(world)
    sps = []
    for r in range(world):
        sp = StripPipeline(W, H, world, r, T=45.0, geometry=SMALL, internal=True)
        sp.rgb_ext().fill_(0xA5)
        sp.rgb_ext()[sp.own_offset:sp.own_offset + (sp.o1 - sp.o0)].copy_(torch.from_numpy(full[sp.o0:sp.o1]))
        pol = dict(kind="rows", rows=1, consumer_discard=True) if mode == "flow" else dict(kind="budget", discard=True)
        sp.plan(64 * 1024, exec_mode=mode, **pol)
        sps.append(sp)
    for sp in sps:  # every strip registered before any exchange runs
        sp.register(comm)
    got = []
    for sp in sps:
        sp.pipe.plan_obj.attach_halo(comm, sp.rank, 4)
        sp.pipe.run()
        torch.cuda.synchronize()
        assert np.array_equal(sp.rgb_ext().cpu().numpy(), full[sp.e0:sp.e1])  # halo rows delivered
        got.append(sp.mask_owned().cpu().numpy())
    assert np.array_equal(np.concatenate(got), want)


def test_halo_exchange_nccl_single_rank():
    """The NCCL backend through the C ABI on one rank (the only NCCL world one GPU allows):
    unique id, communicator, strip registration, the exchange attached to a DAG plan (no
    neighbour: no rows move); the output equals the oracle."""
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    from paper_conf_date_maghazeh0ep19_b200.strips import StripPipeline
    W, H = 512, 128
    full = synth.scene(5, W, H, 1)[0]
    comm = K.Comm.nccl(K.comm_unique_id(), 1, 0)
    sp = StripPipeline(W, H, 1, 0, T=45.0, geometry=SMALL, internal=True)
    sp.rgb_ext().copy_(torch.from_numpy(full))
    sp.plan(64 * 1024, kind="budget", exec_mode="dag")
    sp.attach(comm)
    sp.pipe.run()
    torch.cuda.synchronize()
    comm.check()  # ncclCommGetAsyncError: no asynchronous error
    assert np.array_equal(sp.mask_owned().cpu().numpy(), O.pipeline(full[None], T=45.0)["mask"][0])


def test_selftest_sqrt_exhaustive():
    """The Sobel magnitude's fast sqrt equals __fsqrt_rn on every integer of its domain."""
    from paper_conf_date_maghazeh0ep19_b200 import ktiler
    assert ktiler.selftest(ktiler.SELFTEST_SQRT) == 0


def test_alg1_calibrated_plan():
    """§8(f) f1 on the device: self-calibrated performance tables (ktiler_calibrate), an
    Alg. 1 plan from them, executed bit-exact; cold times grow with the block count."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 1024, 256, 2
    rgb = synth.scene(31, W, H, F)
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL)
    p.view("rgb").copy_(torch.from_numpy(rgb))
    tabs = p.calibrate(reps=2, max_points=4)
    for name, (pts, cold, hot) in tabs.items():
        assert len(pts) == len(cold) == len(hot) and all(t > 0 for t in cold + hot)
        assert cold[-1] >= cold[0]
    for mode in ("graph", "dag"):
        plan = p.plan(64 * 1024, kind="alg1", exec_mode=mode, discard=True)
        assert sorted(v for c, _ in plan.clusters() for v in c) == [0, 1, 2, 3, 4]
        p.run()
        torch.cuda.synchronize()
        assert np.array_equal(p.view("mask").cpu().numpy(), O.pipeline(rgb, T=40.0)["mask"])


@pytest.mark.parametrize("ring", [1, 2, 3])
@pytest.mark.parametrize("mode,pol", [("stream", dict()), ("graph", dict(discard=True)),
                                      ("dag", dict(window=2, consumer_discard=True)),
                                      ("dag", dict(window=3, resident_budget=True))],
                         ids=["stream", "graph-discard", "dag-w2-cd", "dag-w3"])
def test_ring_intermediates(ring, mode, pol):
    """§8(f) f4: the four intermediates as WAR-aware rings of `ring` frames (frame z in slot
    z mod ring).  The executors order every write of frame z after every read of frame
    z - ring (GRAPH_DAG: WAR edges; total orders: checked at plan time), so the whole batch
    — 6 frames through 1..3 frames of intermediate storage — equals the oracle, over
    repeated executes with alternating inputs."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 512, 128, 6
    a, b = synth.scene(3, W, H, F), synth.uniform(4, W, H, F)
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL, ring_frames=ring)
    for k in ("gray", "blur", "down", "sob"):
        assert p.view(k).shape[0] == ring  # the storage really is a ring
    # 4 of a frame's 8 leaf block-rows per fragment: fragments never straddle two frames
    plan = p.plan(1 << 20, kind="rows", rows=4, exec_mode=mode, **pol)
    assert plan.num_fragments() == 2 * F
    for it in range(3):
        x = a if it % 2 == 0 else b
        p.view("rgb").copy_(torch.from_numpy(x))
        p.run()
        torch.cuda.synchronize()
        assert np.array_equal(p.view("mask").cpu().numpy(), O.pipeline(x, T=40.0)["mask"]), (ring, mode, it)


@pytest.mark.parametrize("mode,pol", [("dag", dict(kind="budget", window=2, resident_budget=True, consumer_discard=True)),
                                      ("graph", dict(kind="budget", discard=True)),
                                      ("flow", dict(kind="rows", rows=1, consumer_discard=True))],
                         ids=["dag", "graph-discard", "flow"])
def test_multirate_bit_exact(mode, pol):
    """KTILER_PF_MULTIRATE (down2 / sobel3 / thresh: one sub-kernel per two fragments) in
    the bench's executor and two others: bit-exact vs the oracle."""
    rgb = synth.scene(12, 1040, 256, 2)
    pol = dict(pol)
    kind = pol.pop("kind")
    out, plan = _run(1040, 256, 2, rgb, T=40.0, cache_bytes=200 * 1024, internal=True, kind=kind, exec_mode=mode,
                     multirate=True, **pol)
    assert plan.num_fragments() > 2
    assert np.array_equal(out["mask"], O.pipeline(rgb, T=40.0)["mask"])


@pytest.mark.parametrize("mode,discard", [("stream", True), ("graph", True), ("dag", False)])
def test_random_linear_extensions(mode, discard):
    """P10 on the GPU: random dependency-respecting total orders of the plan's
    sub-kernels (ktiler_plan_reorder; last readers and discard lists re-derived per order),
    replayed on poisoned intermediates, all give the oracle's result — including with
    dead-line discards, where a wrong last reader would drop lines still to be read."""
    import sys
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from test_abi_cpu import _sub_deps, random_topo_orders
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 640, 160, 2
    rgb = synth.scene(21, W, H, F)
    ref = O.pipeline(rgb, T=40.0)
    p = Pipeline(W, H, F, T=40.0, internal=True, geometry=SMALL)
    p.view("rgb").copy_(torch.from_numpy(rgb))
    subs = p.plan(150 * 1024, kind="budget", exec_mode=mode, discard=discard).subkernels()
    assert len(subs) > 20
    deps = _sub_deps(p.graph, subs)
    for order in random_topo_orders(deps, 6, seed=7):
        for k in KEYS:
            p.b.store.tensors[k].fill_(0xA5)
        plan = p.plan(150 * 1024, kind="budget", exec_mode=mode, discard=discard)  # same shapes -> same plan
        plan.reorder(order)
        p.run()
        torch.cuda.synchronize()
        assert np.array_equal(p.view("mask").cpu().numpy(), ref["mask"]), order[:12]
