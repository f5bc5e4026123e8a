"""CPU tests of the C ABI (no GPU): the library loads and exports every symbol declared in
include/ktiler.h; the C++ planner equals the literal Alg. 2 oracle;
analytic dependencies and memory lines equal the traced ones (P11); error paths."""
import os
import re

import pytest

from oracle import oracle as O

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def K():
    import __graft_entry__ as ge
    ge.build()
    from paper_conf_date_maghazeh0ep19_b200 import ktiler
    ktiler.lib()
    return ktiler


def test_exports_every_header_symbol(K):
    hdr = open(os.path.join(ROOT, "include", "ktiler.h")).read()
    names = sorted(set(re.findall(r"^[a-z0-9_ ]+\**\s*(ktiler_[a-z_]+)\(", hdr, re.M)))
    assert len(names) >= 18
    lib = K.lib()
    for n in names:
        assert hasattr(lib, n), n
    assert set(K.EXPORTS) <= set(names)
    assert lib.ktiler_abi_version() == 2
    assert lib.ktiler_status_str(3).decode() == "KTILER_E_UNTILEABLE"


def _paper_pipe(bases):
    from paper_conf_date_maghazeh0ep19_b200 import Motivational
    return Motivational(device=None, bases=bases)


@pytest.fixture(scope="module")
def fig1():
    g = O.motivational_graph()
    return g, O.trace(g)


def _blocks_by_sub(plan):
    out = []
    for sk in plan.subkernels():
        blocks = []
        for (x0, y0, z0, x1, y1, z1) in sk["rects"]:
            blocks += [(x, y, z) for z in range(z0, z1) for y in range(y0, y1) for x in range(x0, x1)]
        out.append((sk["node"], sorted(blocks), sk["fragment"]))
    return out


@pytest.mark.parametrize("lines", [36, 50, 68, 104, 136, 2175, 2176])
def test_planner_equals_oracle_alg2_fig1(K, fig1, lines):
    """P8/P9: the C++ planner reproduces the literal Alg. 2 schedule on the paper's example,
    sub-kernel by sub-kernel (same blocks, same order, same fragments)."""
    g, tr = fig1
    m = _paper_pipe(g.bases())
    plan = m.plan(lines * 128, kind="budget", exec_mode="stream")
    ours = _blocks_by_sub(plan)
    ref = O.cluster_tile(g, tr, lines * 128)
    assert [(n, b, f) for n, b, f in ours] == [(n, sorted(b), f) for (n, b), f in zip(ref.seq, ref.frag)]


def test_planner_untileable(K, fig1):
    g, _ = fig1
    m = _paper_pipe(g.bases())
    with pytest.raises(K.KtilerError) as e:
        m.plan(35 * 128, kind="budget", exec_mode="stream")
    assert e.value.status == K.E_UNTILEABLE
    # FORCE_MINIMAL commits the over-budget closures instead
    p = m.plan(35 * 128, kind="budget", exec_mode="stream", force_minimal=True)
    assert p.num_fragments() == 64


def _pipe_pair(W, H, F, geo):
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    og = O.pipeline_graph(W, H, F, full_tile=geo["gray"][:2], half_tile=geo["down"][:2])
    bases = og.bases()
    p = Pipeline(W, H, F, device=None, geometry=geo, pitch_align=1, bases=bases)
    return og, p


SMALL = {"gray": (16, 8, 32), "blur": (16, 8, 32), "down": (8, 4, 32), "sobel": (8, 4, 32), "thresh": (8, 4, 32)}
# tiles that leave ragged right and bottom tails (pitches must stay multiples of 16 B)
RAGGED = {"gray": (64, 8, 32), "blur": (64, 8, 32), "down": (32, 4, 32), "sobel": (32, 4, 32), "thresh": (32, 4, 32)}
GEOS = [(64, 96, 2, SMALL), (96, 38, 1, RAGGED), (32, 24, 3, SMALL), (160, 70, 1, RAGGED)]


@pytest.mark.parametrize("W,H,F,geo", GEOS, ids=lambda v: str(v) if not isinstance(v, dict) else "")
@pytest.mark.parametrize("budget", [6000, 9000, 20000, 1 << 30])
def test_planner_equals_oracle_alg2_pipeline(K, W, H, F, geo, budget):
    """P9: C++ planner == literal Alg. 2 on the 5-kernel chain (odd remainders included)."""
    og, p = _pipe_pair(W, H, F, geo)
    tr = O.trace(og)
    ref = O.cluster_tile(og, tr, budget)
    if ref.cost == O.INF:
        with pytest.raises(K.KtilerError):
            p.plan(budget, kind="budget", exec_mode="stream")
        return
    plan = p.plan(budget, kind="budget", exec_mode="stream")
    ours = _blocks_by_sub(plan)
    assert [(n, b, f) for n, b, f in ours] == [(n, sorted(b), f) for (n, b), f in zip(ref.seq, ref.frag)]
    assert not O.validate_schedule(og, tr, [(n, b) for n, b, _ in ours], budget, [f for _, _, f in ours])


@pytest.mark.parametrize("W,H,F,geo", GEOS[:2], ids=lambda v: str(v) if not isinstance(v, dict) else "")
def test_analytic_deps_equal_traced(K, W, H, F, geo):
    """P11: analytic (affine-footprint) dependencies == traced RAW dependencies (equality)
    and analytic memory lines == traced lines, for every block of every kernel."""
    og, p = _pipe_pair(W, H, F, geo)
    tr = O.trace(og)
    G = p.graph
    for i in range(len(og.nodes)):
        for b in og.blocks(i):
            gid = og.gid(i, b)
            want = sorted(og.block_of(q) for q in tr.deps[gid])
            got = sorted((n, (bx, by, bz)) for n, bx, by, bz in G.block_deps(i, *b))
            assert got == want, (i, b)
            assert sorted(G.block_lines(i, *b)) == sorted(tr.lines[gid]), (i, b)


def test_analytic_deps_paper_geometry(K, fig1):
    g, tr = fig1
    m = _paper_pipe(g.bases())
    for i in range(2):
        for b in g.blocks(i)[::7]:
            gid = g.gid(i, b)
            want = sorted(g.block_of(q) for q in tr.deps[gid])
            got = sorted((n, (bx, by, bz)) for n, bx, by, bz in m.graph.block_deps(i, *b))
            assert got == want
            assert sorted(m.graph.block_lines(i, *b)) == sorted(tr.lines[gid])


@pytest.mark.parametrize("kind,extra", [("rows", dict(rows=1)), ("rows", dict(rows=5)),
                                        ("balanced", dict(l2_fraction=1.0)), ("none", {})])
def test_policies_valid(K, kind, extra):
    """Every policy yields a valid partition in dependency order (O-11)."""
    og, p = _pipe_pair(64, 96, 2, SMALL)
    tr = O.trace(og)
    plan = p.plan(9000, kind=kind, exec_mode="stream", **extra)
    ours = _blocks_by_sub(plan)
    assert not O.validate_schedule(og, tr, [(n, b) for n, b, _ in ours])


def test_plan_is_deterministic_and_content_free(K):
    """T-R6: a plan depends on shapes only — planning twice gives the same
    schedule (the planner never dereferences buffers)."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    a = Pipeline(7680, 4320, 4, device=None).plan(126 << 20, kind="budget", l2_fraction=0.5, exec_mode="graph")
    b = Pipeline(7680, 4320, 4, device=None).plan(126 << 20, kind="budget", l2_fraction=0.5, exec_mode="graph")
    sa, sb = a.subkernels(), b.subkernels()
    assert [(s["node"], s["rects"]) for s in sa] == [(s["node"], s["rects"]) for s in sb]
    st = a.stats()
    assert st["n_fragments"] > 4 and st["max_footprint_bytes"] <= st["budget_bytes"]


def test_error_paths(K):
    g = K.Graph()
    with pytest.raises(K.KtilerError) as e:
        g.add_buffer(0x1000 + 4, 16, 16, 1)  # misaligned
    assert e.value.status == K.E_INVALID
    a = g.add_buffer(0x100000, 64, 64, 3)
    with pytest.raises(K.KtilerError):
        g.add_buffer(0x100000 + 128, 64, 64, 1)  # aliasing
    b = g.add_buffer(0x200000, 64, 64, 1)
    c = g.add_buffer(0x300000, 32, 32, 1)
    acc = lambda buf, mode, ax, ay, h=0: dict(buf=buf, mode=mode, ax=ax, ay=ay, hl=h, hr=h, ht=h, hb=h)
    # declared footprint smaller than a built-in's stencil (halo 1 < 2) -> rejected
    with pytest.raises(K.KtilerError):
        g.add_kernel(K.OP_BLUR5, (4, 4, 1), (64, 1, 1), [acc(b, K.READ, 16, 16, 1), acc(c, K.WRITE, 16, 16)])
    # wrong scale -> rejected; a covering (larger-halo) footprint is accepted: it only adds
    # dependencies (the line-quantized maps fitted from ktiler_discover_footprint)
    with pytest.raises(K.KtilerError):
        g.add_kernel(K.OP_BLUR5, (4, 4, 1), (64, 1, 1), [acc(b, K.READ, 32, 16, 2), acc(c, K.WRITE, 16, 16)])
    gc = K.Graph()
    bb = gc.add_buffer(0x200000, 64, 64, 1)
    cc = gc.add_buffer(0x300000, 64, 64, 1)
    gc.add_kernel(K.OP_BLUR5, (4, 4, 1), (64, 1, 1), [acc(bb, K.READ, 16, 16, 16), acc(cc, K.WRITE, 16, 16)])
    n0 = g.add_kernel(K.OP_GRAY, (4, 8, 1), (64, 1, 1), [acc(a, K.READ, 16, 8), acc(b, K.WRITE, 16, 8)])
    with pytest.raises(K.KtilerError):
        g.add_edge(n0, n0, b)
    with pytest.raises(K.KtilerError):  # grid does not cover the output
        g.add_kernel(K.OP_DOWN2, (1, 1, 1), (64, 1, 1), [acc(b, K.READ, 32, 16), acc(c, K.WRITE, 16, 8)])
    # odd-size down2 input
    g2 = K.Graph()
    x = g2.add_buffer(0x100000, 63, 64, 1, pitch_bytes=64)
    y = g2.add_buffer(0x200000, 31, 32, 1, pitch_bytes=32)
    with pytest.raises(K.KtilerError):
        g2.add_kernel(K.OP_DOWN2, (2, 4, 1), (64, 1, 1), [acc(x, K.READ, 32, 16), acc(y, K.WRITE, 16, 8)])


def test_cycle_detected(K):
    """A graph that is not a DAG is rejected at plan time (KTILER_E_CYCLE)."""
    g = K.Graph()
    x = g.add_buffer(0x100000, 64, 64, 1)
    y = g.add_buffer(0x200000, 64, 64, 1)
    acc = lambda buf, mode: dict(buf=buf, mode=mode, ax=16, ay=16)
    for src, dst in ((x, y), (y, x)):
        g.add_kernel(K.OP_CUSTOM, (4, 4, 1), (64, 1, 1), [acc(src, K.READ), acc(dst, K.WRITE)],
                     launch=lambda *a: None)
    with pytest.raises(K.KtilerError) as e:
        g.plan(1 << 20, kind="budget", exec_mode="stream")
    assert e.value.status == K.E_CYCLE


def test_plan_without_device_requires_cache_bytes(K):
    """cache_bytes = 0 queries the device L2; with no device that must fail loudly."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a device")
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    p = Pipeline(256, 256, 1, device=None)
    with pytest.raises(K.KtilerError) as e:
        p.plan(0, kind="budget", exec_mode="graph")
    assert e.value.status == K.E_CUDA


def test_smoke_configuration_is_tileable(K):
    """__graft_entry__.smoke()'s plans split the graph into several fragments (B200
    geometry; a budget below one leaf block's closure would be KTILER_E_UNTILEABLE)."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    p = Pipeline(520, 198, 2, T=60.0, internal=True, device=None)
    assert p.b.g.plan(800 * 1024, kind="budget", exec_mode="graph", discard=True, pdl=True).num_fragments() > 1
    assert p.b.g.plan(1 << 20, kind="rows", rows=1, exec_mode="persistent", discard=True).num_fragments() > 1
    assert p.b.g.plan(400 * 1024, kind="budget", exec_mode="dag", window=2, pdl=True, consumer_discard=True,
                      resident_budget=True).num_fragments() > 1  # the bench's policy shape
    assert p.b.g.plan(1 << 20, kind="rows", rows=1, exec_mode="flow", consumer_discard=True).num_fragments() > 1


def test_gauss_f32_params(K):
    """KTILER_OP_GAUSS_F32: sigma must be positive with ceil(3 sigma) <= 4, and the declared
    read halo must cover the radius."""
    import struct
    g = K.Graph()
    a = g.add_buffer(0x100000, 64, 32, 4)
    b = g.add_buffer(0x200000, 64, 32, 4)

    def acc(buf, mode, ax, ay, h=0):
        return dict(buf=buf, mode=mode, ax=ax, ay=ay, hl=h, hr=h, ht=h, hb=h)
    for sigma in (0.0, -1.0, 1.4):
        with pytest.raises(K.KtilerError):
            g.add_kernel(K.OP_GAUSS_F32, (1, 2, 1), (64, 1, 1), [acc(a, K.READ, 64, 16, 4), acc(b, K.WRITE, 64, 16)],
                         struct.pack("f", sigma))
    with pytest.raises(K.KtilerError):  # radius 3 > declared halo 2
        g.add_kernel(K.OP_GAUSS_F32, (1, 2, 1), (64, 1, 1), [acc(a, K.READ, 64, 16, 2), acc(b, K.WRITE, 64, 16)],
                     struct.pack("f", 1.0))
    g.add_kernel(K.OP_GAUSS_F32, (1, 2, 1), (64, 1, 1), [acc(a, K.READ, 64, 16, 3), acc(b, K.WRITE, 64, 16)],
                 struct.pack("f", 1.0))


def _crop_pair(W=256, H=256):
    """A graph that triggers reading A16b: A = gray (in -> intm, 32x8 tiles)
    and B = a 2x2-mean consumer whose output is only the TOP HALF of down2's (W/2 x H/4),
    so the bottom half of A's blocks feed no leaf block.  Oracle: B is down2 on the cropped
    output (its tracer records exactly which intm rows B reads).  C++: B is an OP_CUSTOM node
    declaring the same affine footprint (read 2x its 64x1 tile, write the tile), planned
    only (never launched on CPU)."""
    og = O.OGraph()
    og.add_buf("in", W, H, 1, 3, external=True)
    og.add_buf("intm", W, H, 1, 1)
    og.add_buf("out", W // 2, H // 4, 1, 1)
    og.add_node("A", O.GRAY, "in", "intm", 32, 8)
    og.add_node("B", O.DOWN2, "intm", "out", 64, 1)
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    bases = og.bases()
    g = K.Graph()
    bi = g.add_buffer(bases["in"], W, H, 3)
    bm = g.add_buffer(bases["intm"], W, H, 1, internal=True)
    bo = g.add_buffer(bases["out"], W // 2, H // 4, 1)
    a = g.add_kernel(K.OP_GRAY, (W // 32, H // 8, 1), (32, 8, 1),
                     [dict(buf=bi, mode=K.READ, ax=32, ay=8), dict(buf=bm, mode=K.WRITE, ax=32, ay=8)])
    b = g.add_kernel(K.OP_CUSTOM, (W // 2 // 64, H // 4, 1), (64, 1, 1),
                     [dict(buf=bm, mode=K.READ, ax=128, ay=2), dict(buf=bo, mode=K.WRITE, ax=64, ay=1)],
                     launch=lambda *args: None)
    g.add_edge(a, b, bm, 1.0)
    return og, g


@pytest.mark.parametrize("lines", [36, 68, 136, 1000])
def test_planner_equals_oracle_a16b(K, lines):
    """Reading A16b (blocks no leaf block depends on are picked as bottom blocks, last node
    first, once every leaf block is taken) is exercised: C++ == O-8 sub-kernel by sub-kernel,
    and the schedule has fragments of A blocks that no B block reads."""
    og, g = _crop_pair()
    tr = O.trace(og)
    ref = O.cluster_tile(og, tr, lines * 128)
    plan = g.plan(lines * 128, kind="budget", exec_mode="stream")
    ours = _blocks_by_sub(plan)
    assert [(n, b, f) for n, b, f in ours] == [(n, sorted(b), f) for (n, b), f in zip(ref.seq, ref.frag)]
    assert not O.validate_schedule(og, tr, [(n, b) for n, b, _ in ours], lines * 128, [f for _, _, f in ours])
    b_frags = {f for n, _, f in ours if n == 1}
    orphan = [f for n, b, f in ours if n == 0 and f not in b_frags]
    assert orphan, "A16b not triggered"
    assert all(by >= 16 for n, b, f in ours if f in orphan for (_, by, _) in b)


def test_comm_abi_host_paths(K):
    """Strip halo comm (include/ktiler.h, comm.cpp) host-side paths, no GPU: loopback
    registration checks, missing-neighbour and misuse errors, attaching to a plan."""
    c = K.Comm.loopback(3)
    with pytest.raises(K.KtilerError) as e:  # e0 <= o0 < o1 <= e1 violated
        c.register_strip(0, 1 << 20, 768, 768, 8, 4, 0, 12)
    assert e.value.status == K.E_INVALID
    with pytest.raises(K.KtilerError) as e:  # pitch < row bytes
        c.register_strip(0, 1 << 20, 512, 768, 0, 8, 0, 12)
    assert e.value.status == K.E_INVALID
    c.register_strip(0, 1 << 20, 768, 768, 0, 8, 0, 12)
    c.register_strip(1, 2 << 20, 768, 768, 8, 16, 4, 20)
    with pytest.raises(K.KtilerError) as e:  # rank 1's bottom neighbour (rank 2) not registered
        c.exchange(1, 4, 0)
    assert e.value.status == K.E_STATE
    with pytest.raises(K.KtilerError):
        c.register_strip(3, 1 << 20, 768, 768, 0, 8, 0, 12)  # rank out of range
    # a plan takes the exchange before its first execute (planning needs no GPU)
    og, p = _pipe_pair(64, 96, 1, SMALL)
    plan = p.plan(20000, kind="budget", exec_mode="dag")
    plan.attach_halo(c, 0, 4)
    uid = K.comm_unique_id()  # NCCL is loadable here (no GPU needed for the id)
    assert len(uid) == 128
    c.check()  # failure detection: a loopback comm never has an asynchronous error
    c.close()


def test_flow_roles_abi(K):
    """ktiler_plan_set_flow_roles validation (host side, before any execute)."""
    og, p = _pipe_pair(64, 96, 1, SMALL)
    plan = p.plan(20000, kind="rows", rows=1, exec_mode="flow", consumer_discard=True)
    plan.set_flow_roles([0, 0, 0, 0, 0], [0, 0, 0, 0])
    plan.set_flow_roles([0, 1, 2, 3, 4], [0, 1, 2, 3, 4])
    plan.set_flow_roles([], [])  # automatic roles
    for nr, sr in (([0, 1], [0, 1]),                    # one role per node
                   ([0, 1, 1, 1, 1], [0, 0, 0]),          # role 1 has no slot
                   ([0, 0, 0, 0, 0], [0]),                # < 2 slots
                   ([0, 0, 0, 0, 0], [0] * 6)):           # > 5 slots
        with pytest.raises(K.KtilerError) as e:
            plan.set_flow_roles(nr, sr)
        assert e.value.status == K.E_INVALID
    dag = p.plan(20000, kind="budget", exec_mode="dag")
    with pytest.raises(K.KtilerError) as e:
        dag.set_flow_roles([0] * 5, [0, 0])
    assert e.value.status == K.E_STATE


def _frames_of(sk):
    return {z for (x0, y0, z0, x1, y1, z1) in sk["rects"] for z in range(z0, z1)}


@pytest.mark.parametrize("ring", [1, 2, 3])
def test_ring_buffers_war_order(K, ring):
    """Ring intermediates (ktiler_buffer_desc.ring_frames): the total
    order of an accepted plan puts every read of frame z - R before every write of frame z
    (write-after-read, the hazard PAPER.md:193's RAW model lacks); a plan whose fragments
    span R frames or more is refused (KTILER_E_UNTILEABLE) instead of racing."""
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    W, H, F = 64, 32, 6
    geo = SMALL
    p = Pipeline(W, H, F, device=None, geometry=geo, internal=True, ring_frames=ring)
    names = ("gray", "blur", "down", "sobel", "thresh")
    reads = {1: "gray", 2: "blur", 3: "down", 4: "sob"}   # node -> ring buffer it reads
    writes = {0: "gray", 1: "blur", 2: "down", 3: "sob"}  # node -> ring buffer it writes
    accepted = 0
    for budget in (16000, 24000, 40000):
        try:
            plan = p.plan(budget, kind="budget", exec_mode="graph")
        except K.KtilerError as e:
            assert e.status == K.E_UNTILEABLE
            continue
        accepted += 1
        subs = plan.subkernels()
        for buf in ("gray", "blur", "down", "sob"):
            last_read, first_write = {}, {}
            for i, sk in enumerate(subs):
                for z in _frames_of(sk):
                    if reads.get(sk["node"]) == buf:
                        last_read[z] = i
                    if writes.get(sk["node"]) == buf:
                        first_write.setdefault(z, i)
            for z in range(ring, F):
                assert first_write[z] > last_read[z - ring], (buf, z, budget)
    assert accepted >= 2
    # a whole-batch fragment (budget = infinity) spans every frame: a ring must refuse it
    with pytest.raises(K.KtilerError) as e:
        p.plan(0 + (1 << 40), kind="budget", exec_mode="graph")
    assert e.value.status == K.E_UNTILEABLE
    with pytest.raises(K.KtilerError) as e:  # executors without WAR support
        p.plan(6000, kind="budget", exec_mode="chain")
    assert e.value.status in (K.E_UNSUPPORTED, K.E_UNTILEABLE)


def test_ring_buffer_validation(K):
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as KK
    g = KK.Graph()
    with pytest.raises(KK.KtilerError):  # a ring must be INTERNAL
        g.add_buffer(1 << 20, 64, 32, 1, frames=4, ring_frames=2)
    g.add_buffer(1 << 20, 64, 32, 1, frames=4, internal=True, ring_frames=2)


@pytest.mark.parametrize("W,H,F,geo", GEOS[:2], ids=lambda v: str(v) if not isinstance(v, dict) else "")
def test_multirate_schedule_valid(K, W, H, F, geo):
    """KTILER_PF_MULTIRATE: the cheap half-resolution nodes (down2, sobel3, thresh: 1/4 of
    gray's pixels, all consumers cheap) run one sub-kernel per two fragments; the schedule
    is still a partition whose order respects every traced RAW dependency (O-11), and the
    expensive nodes keep one sub-kernel per fragment."""
    og, p = _pipe_pair(W, H, F, geo)
    tr = O.trace(og)
    base = p.plan(1 << 20, kind="rows", rows=1, exec_mode="stream")
    mr = p.plan(1 << 20, kind="rows", rows=1, exec_mode="stream", multirate=True)
    subs0, subs1 = _blocks_by_sub(base), _blocks_by_sub(mr)
    nfrag = base.num_fragments()
    assert nfrag >= 3
    assert not O.validate_schedule(og, tr, [(n, b) for n, b, _ in subs1])
    for v in range(5):
        n0 = sum(1 for n, _, _ in subs0 if n == v)
        n1 = sum(1 for n, _, _ in subs1 if n == v)
        if v < 2:
            assert n1 == n0
        else:
            assert n1 == -(-n0 // 2)


def _sub_deps(graph, subs):
    """sub-kernel -> set of sub-kernels it depends on, from the library's block deps."""
    owner = {}
    for i, sk in enumerate(subs):
        for (x0, y0, z0, x1, y1, z1) in sk["rects"]:
            for z in range(z0, z1):
                for y in range(y0, y1):
                    for x in range(x0, x1):
                        owner[(sk["node"], x, y, z)] = i
    deps = []
    for i, sk in enumerate(subs):
        d = set()
        for (x0, y0, z0, x1, y1, z1) in sk["rects"]:
            for z in range(z0, z1):
                for y in range(y0, y1):
                    for x in range(x0, x1):
                        for (u, px, py, pz) in graph.block_deps(sk["node"], x, y, z):
                            d.add(owner[(u, px, py, pz)])
        d.discard(i)
        deps.append(d)
    return deps


def random_topo_orders(deps, k, seed):
    import random
    rnd = random.Random(seed)
    n = len(deps)
    succ = [[] for _ in range(n)]
    for i, d in enumerate(deps):
        for j in d:
            succ[j].append(i)
    out = []
    for _ in range(k):
        indeg = [len(d) for d in deps]
        ready = [i for i in range(n) if indeg[i] == 0]
        order = []
        while ready:
            i = ready.pop(rnd.randrange(len(ready)))
            order.append(i)
            for s in succ[i]:
                indeg[s] -= 1
                if indeg[s] == 0:
                    ready.append(s)
        out.append(order)
    return out


def test_plan_reorder_validation(K):
    """ktiler_plan_reorder: any dependency-respecting order is accepted (and becomes the
    plan's order), an order that runs a consumer before its producer is refused."""
    og, p = _pipe_pair(64, 96, 2, SMALL)
    plan = p.plan(20000, kind="budget", exec_mode="stream")
    subs = plan.subkernels()
    deps = _sub_deps(p.graph, subs)
    order = random_topo_orders(deps, 1, 5)[0]
    plan.reorder(order)
    got = plan.subkernels()
    assert [(s["node"], s["rects"]) for s in got] == [(subs[i]["node"], subs[i]["rects"]) for i in order]
    plan2 = p.plan(20000, kind="budget", exec_mode="stream")
    bad = list(range(len(subs)))
    i = next(i for i in range(len(subs)) if deps[i])
    j = min(deps[i])
    bad[i], bad[j] = bad[j], bad[i]  # consumer i now runs before its producer j
    with pytest.raises(K.KtilerError) as e:
        plan2.reorder(bad)
    assert e.value.status == K.E_INVALID
    with pytest.raises(K.KtilerError):
        plan2.reorder([0] * len(subs))  # not a permutation


def test_hs_pyramid_steps_plan(K):
    """Fig. 4's three steps (256, 512, 1024 pixels per side, 500 JI nodes
    each) plan on the host: one JI chain per step, coarse to fine, each tiled across
    iterations by FRAG_CHAIN clusters of 4 nodes (the measured HS policy)."""
    from paper_conf_date_maghazeh0ep19_b200.hs import HSPyramid
    hp = HSPyramid(1024, 1024, 500, device=None)
    assert [(h.W, h.H, h.K) for h in hp.steps] == [(256, 256, 500), (512, 512, 500), (1024, 1024, 500)]
    plans = hp.plan(126 << 20, kind="chain", rows=4, l2_fraction=0.5, exec_mode="dag")
    assert [len(p.clusters()) for p in plans] == [125, 125, 125]
    assert all(p.num_fragments() >= 125 for p in plans)
    with pytest.raises(ValueError):
        HSPyramid(1020, 1024, 8, device=None)
