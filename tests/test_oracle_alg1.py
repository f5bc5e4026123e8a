"""Pins of the Alg. 1 oracle (O-13) against hand-worked costs and the
paper's definitions, and parity of the C++ planner's
KTILER_FRAG_ALG1 with it."""
import math

import pytest

from oracle import oracle as O


def linear_table(n_max, overhead, rate_cold, rate_hot):
    """t(n) = overhead + rate * n at n = 1 and n = n_max (exact under linear interpolation)."""
    return ([1, n_max], [overhead + rate_cold, overhead + rate_cold * n_max],
            [overhead + rate_hot, overhead + rate_hot * n_max])


@pytest.fixture(scope="module")
def fig1():
    g = O.motivational_graph()
    return g, O.trace(g)


def test_et_lookup_definition():
    t = ([10, 100], [1.0, 5.0], [0.5, 2.0])
    assert O.et_lookup(t, 1, False) == 1.0  # below the table: first point
    assert O.et_lookup(t, 55, False) == pytest.approx(3.0)  # midpoint
    assert O.et_lookup(t, 55, True) == pytest.approx(1.25)
    assert O.et_lookup(t, 200, False) == pytest.approx(10.0)  # above: last per-block rate


@pytest.mark.parametrize("overhead,merged", [(0.001, True), (0.1, False)])
def test_alg1_fig1_merge_decision_hand_worked(fig1, overhead, merged):
    """Fig. 1 graph, budget 36 lines -> Alg. 2 gives 64 fragments of {4 A, 4 B} blocks.
    Linear tables t = o + rate*n (A: 0.01 ms/block; B: 0.02 cold, 0.005 hot):
      merged   = 64 * (o + 0.04 + o + 0.02)
      separate = (o + 2.56) + (o + 5.12).
    o = 0.001: 3.968 < 7.682 -> one cluster; o = 0.1: 16.64 > 7.88 -> two clusters."""
    g, tr = fig1
    tables = {0: linear_table(256, overhead, 0.01, 0.01), 1: linear_table(256, overhead, 0.02, 0.005)}
    clusters, costs, sched = O.application_tiling(g, tr, 36 * 128, tables, {(0, 1): None}, 0.0)
    exp_m = 64 * (2 * overhead + 0.06)
    exp_s = 2 * overhead + 7.68
    if merged:
        assert clusters == [[0, 1]] and costs[0] == pytest.approx(exp_m)
        assert len(sched) == 128 and sched[0] == (0, [(0, 0, 0), (1, 0, 0), (2, 0, 0), (3, 0, 0)], 0)
    else:
        assert clusters == [[0], [1]] and sum(costs) == pytest.approx(exp_s)
        assert [(v, len(b)) for v, b, _ in sched] == [(0, 256), (1, 256)]


def test_alg1_threshold_excludes_edges(fig1):
    """Only edges with weight > thld are candidates (A22 strict)."""
    g, tr = fig1
    tables = {0: linear_table(256, 0.001, 0.01, 0.01), 1: linear_table(256, 0.001, 0.02, 0.005)}
    w = 5.12 - 1.28  # the derived weight of A -> B: ET_cold(256) - ET_hot(256)
    c1, _, _ = O.application_tiling(g, tr, 36 * 128, tables, {(0, 1): None}, w - 1e-9)
    c2, _, _ = O.application_tiling(g, tr, 36 * 128, tables, {(0, 1): None}, w + 1e-9)
    assert c1 == [[0, 1]] and c2 == [[0], [1]]


def test_alg1_untileable_merge_is_rejected(fig1):
    """ClusterTile returns inf (l.23) below the closure size, so the merge never wins."""
    g, tr = fig1
    tables = {0: linear_table(256, 0.0, 0.01, 0.01), 1: linear_table(256, 0.0, 0.02, 0.0)}
    clusters, costs, _ = O.application_tiling(g, tr, 35 * 128, tables, {(0, 1): None}, 0.0)
    assert clusters == [[0], [1]] and all(math.isfinite(c) for c in costs)


def test_valid_partition_is_acyclic_quotient():
    """clusters must be totally orderable with no back-dependency."""
    edges = [(0, 1), (1, 2), (0, 2)]  # a diamond-free triangle 0 -> 1 -> 2, 0 -> 2
    assert not O.quotient_is_acyclic(edges, {0: 0, 1: 1, 2: 0})  # {0,2} <-> {1}
    assert O.quotient_is_acyclic(edges, {0: 0, 1: 0, 2: 2})
    assert O.quotient_is_acyclic(edges, {0: 0, 1: 1, 2: 2})
    assert O.quotient_is_acyclic(edges, {0: 0, 1: 0, 2: 0})


def _pipe(W=64, H=96, F=2):
    g = O.pipeline_graph(W, H, F, full_tile=(16, 8), half_tile=(8, 4))
    return g, O.trace(g)


def test_alg1_takes_heaviest_edge_first():
    """Edge order (l.6–7): with user weights making down -> sobel the heaviest, the first
    merge is {down, sobel}; a cost model where only that pair gains keeps it alone."""
    g, tr = _pipe()
    n = {v: g.nblocks(v) for v in range(5)}
    tables = {v: linear_table(n[v], 1.0, 0.01, 0.01) for v in range(5)}  # tiling never pays...
    tables[3] = linear_table(n[3], 0.0, 1.0, 0.0)  # ...except sobel with down's output hot
    tables[2] = linear_table(n[2], 0.0, 0.01, 0.01)
    weights = {(0, 1): 1.0, (1, 2): 2.0, (2, 3): 9.0, (3, 4): 3.0}
    clusters, costs, sched = O.application_tiling(g, tr, 9000, tables, weights, 0.0)
    assert [2, 3] in clusters
    assert sorted(v for c in clusters for v in c) == [0, 1, 2, 3, 4]
    assert not O.validate_schedule(g, tr, [(v, b) for v, b, _ in sched])


# ---- C++ planner (KTILER_FRAG_ALG1) == oracle -------------------------------------------
@pytest.fixture(scope="module")
def K():
    import __graft_entry__ as ge
    ge.build()
    from paper_conf_date_maghazeh0ep19_b200 import ktiler
    ktiler.lib()
    return ktiler


SMALL = {"gray": (16, 8, 32), "blur": (16, 8, 32), "down": (8, 4, 32), "sobel": (8, 4, 32), "thresh": (8, 4, 32)}


def _both(W, H, F):
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    og = O.pipeline_graph(W, H, F, full_tile=(16, 8), half_tile=(8, 4))
    p = Pipeline(W, H, F, device=None, geometry=SMALL, pitch_align=1, bases=og.bases())
    return og, O.trace(og), p


TABLE_SETS = {
    "tiling_pays": lambda n: {v: linear_table(n[v], 0.0005, 0.01, 0.004 if v else 0.01) for v in range(5)},
    "tiling_never": lambda n: {v: linear_table(n[v], 0.5, 0.01, 0.009) for v in range(5)},
    "mixed": lambda n: {0: linear_table(n[0], 0.01, 0.02, 0.02), 1: linear_table(n[1], 0.01, 0.01, 0.0099),
                        2: linear_table(n[2], 0.0, 0.03, 0.001), 3: linear_table(n[3], 0.0, 0.02, 0.002),
                        4: linear_table(n[4], 0.0, 0.03, 0.0005)},
}


@pytest.mark.parametrize("tables", sorted(TABLE_SETS))
@pytest.mark.parametrize("budget", [6000, 20000])
def test_planner_alg1_equals_oracle(K, tables, budget):
    W, H, F = 64, 96, 2
    og, tr, p = _both(W, H, F)
    n = {v: og.nblocks(v) for v in range(5)}
    tab = TABLE_SETS[tables](n)
    for v in range(5):
        p.graph.set_perf_table(v, *tab[v])
    want_c, want_cost, want_s = O.application_tiling(og, tr, budget, tab, {}, 0.0)
    g2 = p.graph  # its edges carry weight -1: derived from the performance tables
    plan = g2.plan(budget, kind="alg1", exec_mode="stream", alg1_thld=0.0)
    got_c = plan.clusters()
    assert [c for c, _ in got_c] == want_c
    assert [c for _, c in got_c] == pytest.approx(want_cost, rel=1e-9)
    got_s = []
    for sk in plan.subkernels():
        blocks = sorted((x, y, z) for (x0, y0, z0, x1, y1, z1) in sk["rects"]
                        for z in range(z0, z1) for y in range(y0, y1) for x in range(x0, x1))
        got_s.append((sk["node"], blocks, sk["cluster"]))
    assert got_s == [(v, sorted(b), c) for v, b, c in want_s]


@pytest.mark.parametrize("rows", [1, 2, 3, 5])
@pytest.mark.parametrize("budget", [6000, 20000])
def test_planner_frag_chain_equals_oracle(K, rows, budget):
    """KTILER_FRAG_CHAIN (DESIGN A40): the fixed partition into consecutive groups of `rows`
    nodes (topological order), each group tiled by the literal Alg. 2 (O-8 with cluster=the
    group) under the budget and the groups run one after another.  C++ == O-8 per cluster,
    sub-kernel by sub-kernel (FRAG_CHAIN had no tests)."""
    W, H, F = 64, 96, 2
    og, tr, p = _both(W, H, F)
    want, inf = [], False
    for c, lo in enumerate(range(0, 5, rows)):
        t = O.cluster_tile(og, tr, budget, cluster=list(range(lo, min(5, lo + rows))))
        inf |= t.cost == O.INF
        want += [(v, sorted(b), c) for (v, b) in t.seq]
    if inf:  # a group's leaf closure exceeds the budget: the paper's infinity (A18)
        with pytest.raises(K.KtilerError) as e:
            p.graph.plan(budget, kind="chain", rows=rows, exec_mode="stream")
        assert e.value.status == K.E_UNTILEABLE
        return
    plan = p.graph.plan(budget, kind="chain", rows=rows, exec_mode="stream")
    got = []
    for sk in plan.subkernels():
        blocks = sorted((x, y, z) for (x0, y0, z0, x1, y1, z1) in sk["rects"]
                        for z in range(z0, z1) for y in range(y0, y1) for x in range(x0, x1))
        got.append((sk["node"], blocks, sk["cluster"]))
    assert got == want
    assert [c for c, _ in plan.clusters()] == [list(range(lo, min(5, lo + rows))) for lo in range(0, 5, rows)]
