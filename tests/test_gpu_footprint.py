"""§8(f) f3 footprint discovery on the GPU (include/ktiler.h ktiler_discover_footprint):
differential execution of single blocks vs the oracle's traced footprints (O-10, a CPU
re-enactment of the paper's SASSI block analyzer).

Parity: for every kernel of the pipeline and blocks at corners, edges and the interior,
  - the bytes the block writes == its declared output rect, byte for byte;
  - the 128-B lines it depends on == the lines O-10 traces it reading (PAPER.md:225
    blkMemLines), line for line.
Then the affine maps fitted from the discovered (line-quantized) footprints re-declare the
graph, and the planner's schedule on that graph still reproduces the oracle exactly."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from inputs import synth  # noqa: E402
from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu

SMALL = {"gray": (64, 16, 64), "blur": (64, 16, 64), "down": (32, 8, 64), "sobel": (32, 8, 64), "thresh": (32, 8, 64)}
NAMES = ("gray", "blur", "down", "sobel", "thresh")
BUFS = ("rgb", "gray", "blur", "down", "sob", "mask")
W, H, F = 512, 64, 2


@pytest.fixture(scope="module")
def setup():
    import __graft_entry__ as ge
    ge.build()
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    p = Pipeline(W, H, F, T=60.0, internal=False, geometry=SMALL)
    g = O.pipeline_graph(W, H, F, T=60.0, full_tile=(64, 16), half_tile=(32, 8))
    tr = O.trace(g)
    return p, g, tr


def _blocks(grid):
    gx, gy, gz = grid
    cand = {(0, 0, 0), (gx - 1, gy - 1, gz - 1), (gx // 2, gy // 2, 0), (gx - 1, 0, gz - 1), (0, gy // 2, 1 % gz)}
    return sorted(cand)


@pytest.mark.parametrize("i", range(5), ids=NAMES)
def test_discovered_equals_traced(setup, i):
    from paper_conf_date_maghazeh0ep19_b200 import footprint as FP
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    p, g, tr = setup
    node = p.b.nodes[NAMES[i]]
    bid = {name: p.b.bufs[name][0] for name in BUFS}
    name_of = {v: k for k, v in bid.items()}
    bases = g.bases()
    for b in _blocks(p.b.grids[NAMES[i]]):
        recs = p.b.g.discover_footprint(node, *b, trials=3, seed=11)
        # writes: exactly the declared output rect (bytes)
        wb = FP.byte_sets(recs, K.WRITE)
        n = g.nodes[i]
        o = g.bufs[n.dst]
        x0, y0, x1, y1, z = g.out_rect(i, b)
        want = {z * o.W * o.H * o.elem + y * o.W * o.elem + xb for y in range(y0, y1) for xb in range(x0 * o.elem, x1 * o.elem)}
        assert set(wb) == {bid[n.dst]} and wb[bid[n.dst]] == want, (NAMES[i], b)
        # reads: the lines O-10 traces (relative to each buffer's base)
        gid = g.gid(i, b)
        traced = {}
        for ln in tr.rlines[gid]:
            nm = max((k for k in bases if (bases[k] >> 7) <= ln), key=lambda k: bases[k])
            traced.setdefault(bid[nm], set()).add(ln - (bases[nm] >> 7))
        assert FP.line_sets(recs, K.READ) == traced, (NAMES[i], b, {name_of[k]: len(v) for k, v in traced.items()})


def test_fitted_maps_replan_to_oracle(setup):
    """Declare the graph from discovered footprints only (fitted affine maps, line-
    quantized reads) and run a tiled schedule: bit-exact vs the oracle."""
    from paper_conf_date_maghazeh0ep19_b200 import footprint as FP
    from paper_conf_date_maghazeh0ep19_b200 import ktiler as K
    p, g, tr = setup
    descs = {p.b.bufs[n][0]: (p.b.bufs[n][5], p.b.bufs[n][5] * p.b.bufs[n][2], p.b.bufs[n][4]) for n in BUFS}
    dims = {p.b.bufs[n][0]: (p.b.bufs[n][1], p.b.bufs[n][2]) for n in BUFS}
    fitted = {}
    for name in NAMES:
        node = p.b.nodes[name]
        gx, gy, gz = p.b.grids[name]
        samples_r, samples_w = {}, {}
        # a row and a column of blocks: every phase of the tiles against the 128-B lines
        for bx, by in sorted({(x, min(1, gy - 1)) for x in range(gx)} | {(min(1, gx - 1), y) for y in range(gy)}):
            recs = p.b.g.discover_footprint(node, bx, by, 0, trials=2, seed=5)
            rr, ww = FP.rects(recs, descs, K.READ), FP.rects(recs, descs, K.WRITE)
            assert len(rr) == 1 and len(ww) == 1
            (rb, r), = rr.items()
            (wbuf, w), = ww.items()
            samples_r[(bx, by)] = r
            samples_w[(bx, by)] = w
        wmap = FP.fit_access(samples_w, wbuf, K.WRITE, *dims[wbuf])
        # read step along x from the write step and the buffer shapes (line-quantized reads)
        rmap = FP.fit_access(samples_r, rb, K.READ, *dims[rb], ax=wmap["ax"] * dims[rb][0] // dims[wbuf][0])
        fitted[name] = (rmap, wmap)
        assert (wmap["ax"], wmap["ay"]) == SMALL[name][:2] and wmap["hl"] == wmap["hr"] == wmap["ht"] == wmap["hb"] == 0
    # re-declare: same buffers and kernels, accesses from the fitted maps
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    q = Pipeline(W, H, F, T=60.0, internal=False, geometry=SMALL)
    g2 = K.Graph()
    ids = {}
    for n in BUFS:
        bid_, Wn, Hn, Fn, elem, pitch = q.b.bufs[n]
        ids[bid_] = g2.add_buffer(q.b.store.tensors[n].data_ptr(), Wn, Hn, elem, frames=Fn, pitch_bytes=pitch)
    ops = {"gray": K.OP_GRAY, "blur": K.OP_BLUR5, "down": K.OP_DOWN2, "sobel": K.OP_SOBEL3, "thresh": K.OP_THRESH}
    import struct
    nodes = {}
    for name in NAMES:
        r, w = fitted[name]
        acc = [dict(buf=ids[r["buf"]], mode=K.READ, ax=r["ax"], ay=r["ay"], hl=r["hl"], hr=r["hr"], ht=r["ht"], hb=r["hb"]),
               dict(buf=ids[w["buf"]], mode=K.WRITE, ax=w["ax"], ay=w["ay"])]
        nodes[name] = g2.add_kernel(ops[name], p.b.grids[name], (SMALL[name][2], 1, 1), acc,
                                    struct.pack("f", 60.0) if name == "thresh" else None)
    rgb = synth.scene(9, W, H, F)
    q.view("rgb").copy_(torch.from_numpy(rgb))
    for n in BUFS[1:]:
        q.b.store.tensors[n].fill_(0xA5)
    plan = g2.plan(1 << 20, kind="rows", rows=1, exec_mode="graph")
    assert plan.num_fragments() > 1
    plan.execute(0)
    torch.cuda.synchronize()
    ref = O.pipeline(rgb, T=60.0)
    for k in ("gray", "blur", "down", "sob", "mask"):
        assert np.array_equal(q.view(k).cpu().numpy().view(np.uint8), ref[k].view(np.uint8)), k
