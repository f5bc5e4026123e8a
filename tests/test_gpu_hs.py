"""§8(f) f2 on the GPU: chains of KTILER_OP_JACOBI nodes (the paper's JI nodes,
PAPER.md:381–399) through libktiler vs the f32 oracle O-14, bit for bit, untiled and tiled
across iterations (Alg. 2 closures growing one pixel per iteration), in several executors."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from inputs import synth  # noqa: E402
from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__ as ge
    ge.build()


def _run(W, H, F, K, a2, seed, internal, **pol):
    from paper_conf_date_maghazeh0ep19_b200.hs import HSJacobi
    h = HSJacobi(W, H, K, frames=F, a2=a2, internal=internal)
    coef, s0 = synth.hs_fields(seed, W, H, F)
    for k in range(1, K + 1):
        h.b.store.tensors[f"s{k}"].fill_(0xFF)  # NaN poison: a skipped block cannot pass
    h.set("coef", coef)
    h.set("s0", s0)
    cb = pol.pop("cache_bytes", 1 << 20)
    plan = h.plan(cb, **pol)
    h.run()
    torch.cuda.synchronize()
    return h.get(f"s{K}"), plan, coef, s0, h


CASES = [(128, 64, 1, 1), (256, 160, 1, 5), (512, 256, 2, 8), (200, 120, 1, 3)]


@pytest.mark.parametrize("W,H,F,K", CASES)
@pytest.mark.parametrize("pol", [dict(kind="none", exec_mode="graph"),
                                 dict(kind="rows", rows=1, exec_mode="graph", discard=True),
                                 dict(kind="rows", rows=2, exec_mode="dag", discard=True),
                                 dict(kind="budget", cache_bytes=4 << 20, exec_mode="stream"),
                                 dict(kind="rows", rows=1, exec_mode="wave", discard=True)],
                         ids=lambda d: "-".join(f"{k}={v}" for k, v in d.items()))
def test_jacobi_chain_bit_exact(W, H, F, K, pol):
    got, plan, coef, s0, _ = _run(W, H, F, K, 0.5, W + K, internal=bool(pol.get("discard")), **dict(pol))
    ref = O.hs_jacobi(coef, s0, 0.5, K)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))
    if pol["kind"] == "rows" and K > 1:
        assert plan.num_fragments() > 1


def test_every_iterate_bit_exact():
    """Intermediates too (not discarded): s_k == k oracle iterations for every k."""
    W, H, K = 192, 96, 4
    _, plan, coef, s0, h = _run(W, H, 1, K, 2.0, 3, internal=False, kind="rows", rows=1, exec_mode="graph")
    for k in range(1, K + 1):
        got = h.get(f"s{k}")
        assert np.array_equal(got.view(np.uint32), O.hs_jacobi(coef, s0, 2.0, k).view(np.uint32)), k


@pytest.mark.parametrize("rows", [2, 3])
def test_frag_chain_bit_exact(rows):
    """KTILER_FRAG_CHAIN (DESIGN A40, the policy the HS measurements use): clusters of
    `rows` consecutive JI nodes, each tiled by Alg. 2, bit-exact vs O-14."""
    W, H, K = 256, 128, 8
    got, plan, coef, s0, _ = _run(W, H, 1, K, 0.5, 17, internal=True, kind="chain", rows=rows, exec_mode="dag",
                                  cache_bytes=2 << 20)
    assert len(plan.clusters()) == -(-K // rows) and plan.num_fragments() > 1
    assert np.array_equal(got.view(np.uint32), O.hs_jacobi(coef, s0, 0.5, K).view(np.uint32))


def test_paper_shape_500_iterations():
    """The paper's finest pyramid level (Fig. 4): 500 JI iterations on
    a 1024^2 frame, tiled across iterations by the measured configuration (FRAG_CHAIN
    clusters of 4 nodes under half the device L2, GRAPH_DAG), bit-exact vs the f32 oracle
    after all 500 iterations (parity stopped at K = 8)."""
    W = H = 1024
    K = 500
    got, plan, coef, s0, _ = _run(W, H, 1, K, 0.5, 2024, internal=True, kind="chain", rows=4, exec_mode="dag",
                                  cache_bytes=0, l2_fraction=0.5)
    assert len(plan.clusters()) == K // 4
    ref = O.hs_jacobi(coef, s0, 0.5, K)
    assert np.array_equal(got.view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("K,W,H,pol", [(8, 256, 160, dict(kind="none")), (8, 256, 160, dict(kind="rows", rows=2)),
                                       (500, 1024, 1024, dict(kind="none"))],
                         ids=["k8-one-fragment", "k8-rows2", "k500-1024"])
def test_jacobi_chain_flow(K, W, H, pol):
    """The JI chain under the persistent per-tile-flag executor (FLOW): a tile of iteration
    k+1 starts as soon as the iteration-k tiles covering its 1-pixel halo are published —
    a wavefront across iterations with no launch per iteration (the paper's inter-launch
    gap, removed inside one launch).  Bit-exact vs O-14."""
    got, plan, coef, s0, _ = _run(W, H, 1, K, 0.5, 99 + K, internal=True, exec_mode="flow", consumer_discard=True,
                                  **dict(pol))
    assert plan.stats()["n_launches"] == 1
    assert np.array_equal(got.view(np.uint32), O.hs_jacobi(coef, s0, 0.5, K).view(np.uint32))


def test_pyramid_fig4_steps():
    """Fig. 4's tiled nodes end to end: the three steps' JI chains (256,
    512, 1024 pixels per side, 500 iterations each, every chain starting from {0}) executed
    in order by HSPyramid under the measured HS policy; each step's result bit-exact vs the
    f32 oracle O-14."""
    from paper_conf_date_maghazeh0ep19_b200.hs import HSPyramid
    K = 500
    hp = HSPyramid(1024, 1024, K, a2=0.5)
    coefs = []
    for i, h in enumerate(hp.steps):
        coef, _ = synth.hs_fields(700 + i, h.W, h.H, 1)
        hp.set_coef(i, coef)
        coefs.append(coef)
        h.b.store.tensors[f"s{K}"].fill_(0xFF)  # NaN poison
    hp.plan(0, kind="chain", rows=4, l2_fraction=0.5, exec_mode="dag")
    hp.run()
    torch.cuda.synchronize()
    for i, h in enumerate(hp.steps):
        zero = np.zeros((1, h.H, h.W, 2), np.float32)
        ref = O.hs_jacobi(coefs[i], zero, 0.5, K)
        assert np.array_equal(hp.get(i).view(np.uint32), ref.view(np.uint32)), i
