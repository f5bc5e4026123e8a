"""The float variant (reading A43) on the GPU: chains of
KTILER_OP_GAUSS_F32 nodes through libktiler vs the f64 oracle O-7, max-abs <= 1e-5 on
seeded uniform f32 data in [0, 1] (BJ:5), untiled and tiled (fragment edges, ragged tails,
replicate borders), in several executors."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")

from oracle import oracle as O  # noqa: E402

pytestmark = pytest.mark.gpu
TOL = 1e-5


@pytest.fixture(scope="module", autouse=True)
def _lib():
    import __graft_entry__ as ge
    ge.build()


def _run(W, H, F, nodes, sigma, seed, cache_bytes=1 << 20, **pol):
    from paper_conf_date_maghazeh0ep19_b200.gauss import GaussChain
    g = GaussChain(W, H, nodes=nodes, frames=F, sigma=sigma, tile=(64, 16))  # small tiles: many fragments
    x = np.random.default_rng(seed).random((F, H, W), dtype=np.float32)
    for k in range(1, nodes + 1):
        g.b.store.tensors[f"x{k}"].fill_(0xFF)  # NaN poison: a skipped block cannot pass
    g.view("x0").copy_(torch.from_numpy(x))
    plan = g.plan(cache_bytes, **pol)
    g.run()
    torch.cuda.synchronize()
    return g.view(f"x{nodes}").cpu().numpy(), x, plan


CASES = [(200, 70, 1, 2, 1.0), (256, 128, 2, 3, 0.5), (130, 45, 1, 1, 1.3), (18, 5, 1, 2, 1.0), (512, 96, 1, 4, 0.8)]


@pytest.mark.parametrize("W,H,F,nodes,sigma", CASES)
@pytest.mark.parametrize("pol", [dict(kind="none", exec_mode="graph"),
                                 dict(kind="budget", exec_mode="stream", cache_bytes=256 * 1024),
                                 dict(kind="budget", exec_mode="dag", cache_bytes=256 * 1024, discard=True),
                                 dict(kind="rows", rows=1, exec_mode="graph")],
                         ids=["untiled", "stream", "dag", "rows1"])
def test_gauss_chain_within_tolerance(W, H, F, nodes, sigma, pol):
    pol = dict(pol)
    cb = pol.pop("cache_bytes", 1 << 20)
    got, x, plan = _run(W, H, F, nodes, sigma, seed=W + H + nodes, cache_bytes=cb, **pol)
    ref = O.gauss_f32(x, sigma, passes=nodes)
    assert np.isfinite(got).all()
    err = float(np.abs(got.astype(np.float64) - ref).max())
    assert err <= TOL, f"max abs error {err:.3g} > {TOL}"


def test_gauss_is_really_tiled():
    got, x, plan = _run(512, 96, 1, 4, 1.0, seed=5, cache_bytes=256 * 1024, kind="budget", exec_mode="dag")
    assert plan.num_fragments() > 1
    assert float(np.abs(got - O.gauss_f32(x, 1.0, passes=4)).max()) <= TOL
