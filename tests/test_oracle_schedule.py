"""Pins for the schedule side of the oracle: O-8 (Alg. 2), O-9 (block executor), O-10
(traced deps), O-11 (validator), O-12 (LRU model) — SURVEY §8(c) P8, P10, T-R1..T-R7."""
import itertools
import os
import random

import numpy as np
import pytest

from inputs import synth
from oracle import oracle as O


def _fig1_golden(golden_dir):
    deps, first = {}, {}
    for ln in open(os.path.join(golden_dir, "fig1_block_deps.txt")):
        ln = ln.split("#")[0].strip()
        if not ln:
            continue
        lhs, rhs = ln.split(":")
        lhs = lhs.split()
        if lhs[0] == "first_fragment":
            first[lhs[1]] = sorted(tuple(int(t) for t in p.split()) for p in rhs.split(","))
        else:
            deps[(lhs[0], int(lhs[1]), int(lhs[2]))] = sorted(
                (p.split()[0], int(p.split()[1]), int(p.split()[2])) for p in rhs.split(","))
    return deps, first


@pytest.fixture(scope="module")
def fig1():
    g = O.motivational_graph()
    return g, O.trace(g)


def test_fig1_grids(fig1):
    g, _ = fig1
    assert g.grid(0) == (8, 32, 1)  # A<<<(8x32),(32x8)>>>
    assert g.grid(1) == (2, 128, 1)


def test_fig1_block_deps_printed_in_paper(fig1, golden_dir):
    """T-R1: B(0,0..3) depend exactly on A(0..3,0)."""
    g, tr = fig1
    deps, _ = _fig1_golden(golden_dir)
    names = {0: "A", 1: "B"}
    for (n, bx, by), want in deps.items():
        gid = g.gid(1 if n == "B" else 0, (bx, by, 0))
        got = sorted((names[g.block_of(p)[0]], g.block_of(p)[1][0], g.block_of(p)[1][1]) for p in tr.deps[gid])
        assert got == want


def test_no_intra_kernel_deps(fig1):
    """T-R4: dependencies exist only between blocks of different kernels."""
    g, tr = fig1
    for c, ps in tr.deps.items():
        for p in ps:
            assert g.block_of(c)[0] != g.block_of(p)[0]


def test_alg2_first_fragment_printed_in_paper(fig1, golden_dir):
    """T-R2: first iteration -> delta1_A = A(0..3,0), delta1_B = B(0,0..3)."""
    g, tr = fig1
    _, first = _fig1_golden(golden_dir)
    t = O.cluster_tile(g, tr, 36 * 128)
    (na, ba), (nb, bb) = t.seq[0], t.seq[1]
    assert (na, nb) == (0, 1)
    assert sorted((b[0], b[1]) for b in ba) == first["A"]
    assert sorted((b[0], b[1]) for b in bb) == first["B"]
    assert t.footprint_lines[0] == 36  # 24 rgb + 8 intm + 4 out lines


@pytest.mark.parametrize("lines,nfrag", [(36, 64), (50, 64), (67, 64), (68, 32), (103, 32), (104, 22), (136, 16),
                                         (2175, 2), (2176, 1), (100000, 1)])
def test_alg2_fragment_counts(fig1, lines, nfrag):
    """P8 derived values: 36–67 lines -> 64 fragments of 4A+4B, 68 -> 32,
    136 -> 16, >= 2176 (= whole graph 278,528 B) -> 1 fragment = the untiled schedule."""
    g, tr = fig1
    t = O.cluster_tile(g, tr, lines * 128)
    assert t.cost != O.INF
    assert len(set(t.frag)) == nfrag
    assert not O.validate_schedule(g, tr, t.seq, lines * 128, t.frag)
    if nfrag == 1:
        assert [(i, len(b)) for i, b in t.seq] == [(0, 256), (1, 256)]


def test_alg2_untileable_is_inf(fig1):
    """T-R7 / A18 (PAPER.md:305 l.23): a budget below the first closure (36 lines) -> INF."""
    g, tr = fig1
    assert O.cluster_tile(g, tr, 35 * 128).cost == O.INF
    assert O.cluster_tile(g, tr, 0).cost == O.INF


def test_alg2_tail_imbalance(fig1):
    """A19: the literal greedy leaves a tail fragment (2175 lines -> 252+252 blocks, then 4+4)."""
    g, tr = fig1
    t = O.cluster_tile(g, tr, 2175 * 128)
    assert [len(b) for _, b in t.seq] == [252, 252, 4, 4]


def test_plan_independent_of_pixel_values():
    """T-R6: same input size -> identical block deps -> same schedule."""
    g = O.pipeline_graph(64, 48, 1, full_tile=(16, 4), half_tile=(8, 4))
    t1 = O.trace(g, {"rgb": synth.uniform(0, 64, 48)})
    t2 = O.trace(g, {"rgb": synth.scene(7, 64, 48)})
    assert t1.deps == t2.deps and t1.lines == t2.lines
    a = O.cluster_tile(g, t1, 2048)
    b = O.cluster_tile(g, t2, 2048)
    assert a.seq == b.seq


@pytest.fixture(scope="module")
def small_pipe():
    g = O.pipeline_graph(64, 96, 2, full_tile=(16, 8), half_tile=(8, 4), T=40.0)
    return g, O.trace(g)


def test_pipeline_deps_shape(small_pipe):
    """Closed forms of the 5-kernel deps: blur -> gray 3x3 (interior), down -> blur 1,
    sobel -> down 3x3, thresh -> sob 1 (SURVEY §8 tile geometry)."""
    g, tr = small_pipe
    def dset(i, b):
        return sorted(g.block_of(p)[1] for p in tr.deps[g.gid(i, b)])
    assert len(dset(1, (1, 1, 0))) == 9
    assert dset(2, (1, 1, 1)) == [(1, 1, 1)]
    assert len(dset(3, (1, 1, 0))) == 9
    assert dset(4, (2, 3, 1)) == [(2, 3, 1)]
    assert len(dset(1, (0, 0, 0))) == 4  # corner: clamp stays inside the image


@pytest.mark.parametrize("budget,nfrag", [(8000, 0), (10000, 12), (14000, 8), (20000, 5), (60000, 2), (1 << 30, 1)])
def test_alg2_pipeline_valid_and_exact(small_pipe, budget, nfrag):
    """O-8 schedules are valid partitions in dependency order within the budget (O-11) and
    executing them block by block on poisoned buffers reproduces the untiled graph (O-9)."""
    g, tr = small_pipe
    t = O.cluster_tile(g, tr, budget)
    if nfrag == 0:
        assert t.cost == O.INF
        return
    assert len(set(t.frag)) == nfrag
    assert not O.validate_schedule(g, tr, t.seq, budget, t.frag)
    rgb = synth.scene(3, 64, 96, 2)
    ref = O.pipeline(rgb, T=40.0)
    mem = O.run_schedule(g, t.seq, {"rgb": rgb})
    for k in ("gray", "blur", "down", "sob", "mask"):
        assert np.array_equal(mem[k].view(np.uint8), ref[k].view(np.uint8)), k


def _linear_extensions(items, deps):
    """All topological orders of ``items`` (list of keys) under deps[k] = set of predecessors."""
    if not items:
        yield []
        return
    for k in items:
        if not (deps[k] & set(items)):
            rest = [x for x in items if x != k]
            for tail in _linear_extensions(rest, deps):
                yield [k] + tail


def test_bruteforce_all_orders_a4_b1():
    """P10 (brute force): A with 4 blocks, B with 1 block depending on all 4 -> 24 linear
    extensions; every one reproduces the untiled result."""
    g = O.motivational_graph(128, 8, 1, a_tile=(32, 8), b_tile=(64, 4))
    assert g.nblocks(0) == 4 and g.nblocks(1) == 1
    tr = O.trace(g)
    keys = list(range(5))
    deps = {k: set(tr.deps[k]) for k in keys}
    rgb = synth.uniform(1, 128, 8)
    ref = O.motivational(rgb)
    n = 0
    for order in _linear_extensions(keys, deps):
        sched = [g.block_of(k) for k in order]
        mem = O.run_schedule(g, [(i, [b]) for i, b in sched], {"in": rgb})
        assert np.array_equal(mem["out"][0], ref["down"][0])
        n += 1
    assert n == 24


def test_bruteforce_all_orders_a4_b4():
    """P10: 4 A blocks x 4 B blocks each depending on all A blocks -> 4! * 4! = 576 orders."""
    g = O.motivational_graph(128, 8, 1, a_tile=(32, 8), b_tile=(64, 1))
    assert g.nblocks(0) == 4 and g.nblocks(1) == 4
    tr = O.trace(g)
    keys = list(range(8))
    deps = {k: set(tr.deps[k]) for k in keys}
    rgb = synth.scene(2, 128, 8)
    ref = O.motivational(rgb)
    n = 0
    for order in _linear_extensions(keys, deps):
        mem = O.run_schedule(g, [(g.block_of(k)[0], [g.block_of(k)[1]]) for k in order], {"in": rgb})
        assert np.array_equal(mem["out"][0], ref["down"][0])
        n += 1
    assert n == 576


def _random_topo(keys, deps, rng):
    indeg = {k: len(deps[k]) for k in keys}
    succ = {k: [] for k in keys}
    for k in keys:
        for p in deps[k]:
            succ[p].append(k)
    ready = [k for k in keys if indeg[k] == 0]
    out = []
    while ready:
        k = ready.pop(rng.randrange(len(ready)))
        out.append(k)
        for s in succ[k]:
            indeg[s] -= 1
            if indeg[s] == 0:
                ready.append(s)
    return out


@pytest.mark.parametrize("seed", range(4))
def test_random_topological_orders_pipeline(small_pipe, seed):
    """P10 (beyond exhaustive): random linear extensions of the 5-kernel block DAG all
    reproduce the untiled graph (250 orders per seed x 4 seeds = 1000)."""
    g, tr = small_pipe
    rgb = synth.uniform(seed, 64, 96, 2)
    ref = O.pipeline(rgb, T=40.0)
    assert 0 < (ref["mask"] == 255).mean() < 1
    keys = list(tr.deps)
    rng = random.Random(seed)
    for _ in range(250):
        order = _random_topo(keys, tr.deps, rng)
        mem = O.run_schedule(g, [(g.block_of(k)[0], [g.block_of(k)[1]]) for k in order], {"rgb": rgb})
        assert np.array_equal(mem["mask"], ref["mask"])
        assert np.array_equal(mem["sob"].view(np.uint32), ref["sob"].view(np.uint32))


def test_negative_control_swapped_pair_changes_output(small_pipe):
    """P10 negative control: moving one block before its producer on poisoned buffers must
    change the output — proves the invariance tests can fail."""
    g, tr = small_pipe
    rgb = synth.uniform(11, 64, 96, 2)
    ref = O.pipeline(rgb, T=40.0)
    order = [g.gid(i, b) for i in range(len(g.nodes)) for b in g.blocks(i)]
    c = g.gid(3, (3, 2, 1))  # a sobel block
    first = min(order.index(p) for p in tr.deps[c])
    order.remove(c)
    order.insert(first, c)  # consumer now runs before its producers
    sched = [(g.block_of(k)[0], [g.block_of(k)[1]]) for k in order]
    mem = O.run_schedule(g, sched, {"rgb": rgb})
    assert not np.array_equal(mem["sob"].view(np.uint32), ref["sob"].view(np.uint32))
    assert O.validate_schedule(g, tr, sched)


def test_validator_catches_overlap_and_gap(small_pipe):
    g, tr = small_pipe
    sched = O.untiled_schedule(g)
    assert not O.validate_schedule(g, tr, sched)
    bad = [(i, list(b)) for i, b in sched]
    bad[2][1].append(bad[2][1][0])
    assert any("two sub-kernels" in e for e in O.validate_schedule(g, tr, bad))
    bad = [(i, list(b)) for i, b in sched]
    bad[3][1].pop()
    assert any("cover" in e for e in O.validate_schedule(g, tr, bad))


def test_lru_model_tiling_reduces_dram(small_pipe):
    """O-12 (expectation): with a cache smaller than the graph, the Alg. 2 schedule moves
    fewer DRAM bytes than the untiled one, and discarding dead intermediates removes their
    write-back.  Model only — no parity claim rests on it."""
    g, tr = small_pipe
    cache = 8 * 1024
    un = O.lru_dram_bytes(g, tr, O.untiled_schedule(g), cache)
    t = O.cluster_tile(g, tr, cache)
    ti = O.lru_dram_bytes(g, tr, t.seq, cache)
    td = O.lru_dram_bytes(g, tr, t.seq, cache, discard_dead=True)
    assert ti["read"] < un["read"]
    assert td["write_incl_tail"] < ti["write_incl_tail"]
    compulsory = g.bufs["rgb"].nbytes + g.bufs["mask"].nbytes
    assert td["read"] + td["write_incl_tail"] >= compulsory


def _lru_tiny():
    """Fig. 1's A -> B on a 128 x 2 image: A tiles 128 x 1 (2 blocks, one image row each),
    B tile 64 x 1 (1 block, reads both intm rows).  Every buffer row is a whole number of
    128-B lines at 128-B-aligned bases: in rows are 3 lines each (384 B),
    intm rows 1 line each, out 1 line (64 B)."""
    g = O.motivational_graph(W=128, H=2, a_tile=(128, 1), b_tile=(64, 1))
    return g, O.trace(g)


def test_lru_model_exact_hand_trace():
    """O-12 pinned to a hand-worked trace (O-12 was parity-unpinned).  Untiled
    order A0, A1, B0; each block reads its lines in ascending order, then writes.

    cache 4 lines:
      A0  miss in0 in1 in2 (rd 3)               LRU [in0 in1 in2]; write i0* -> [in0 in1 in2 i0*]
      A1  miss in3 in4 in5 (rd 6), evicting in0 in1 in2 (clean)   -> [i0* in3 in4 in5]
          write i1*: evicts i0* DIRTY (wr 1)                        -> [in3 in4 in5 i1*]
      B0  i0 misses again (rd 7), evicts in3; i1 hits               -> [in4 in5 i0 i1*]
          write o0*: evicts in4                                     -> [in5 i0 i1* o0*]
      => read 7 lines, write 1 line, dirty tail {i1, o0} = 2 lines.
      With the discard of dead intermediates, i0 and i1 die after B0 (their last reader):
      the write-back of i0 already happened, i1's never does -> tail {o0} = 1 line.
    cache 64 lines (everything fits): read 6, write 0, tail {i0, i1, o0} = 3 lines;
      with discard: tail {o0} = 1 line."""
    g, tr = _lru_tiny()
    L = 128
    s = O.untiled_schedule(g)
    assert O.lru_dram_bytes(g, tr, s, 4 * L) == {"read": 7 * L, "write": 1 * L, "write_incl_tail": 3 * L}
    assert O.lru_dram_bytes(g, tr, s, 4 * L, discard_dead=True) == {"read": 7 * L, "write": 1 * L,
                                                                     "write_incl_tail": 2 * L}
    assert O.lru_dram_bytes(g, tr, s, 64 * L) == {"read": 6 * L, "write": 0, "write_incl_tail": 3 * L}
    assert O.lru_dram_bytes(g, tr, s, 64 * L, discard_dead=True) == {"read": 6 * L, "write": 0,
                                                                      "write_incl_tail": 1 * L}


def test_lru_model_exact_reordered_trace():
    """Same graph, cache 4 lines, order A1, A0, B0 (another valid order):
      A1  miss in3 in4 in5 (rd 3); write i1*       -> [in3 in4 in5 i1*]
      A0  miss in0 (rd 4) evicts in3; in1 evicts in4; in2 evicts in5 (all clean)
                                                   -> [i1* in0 in1 in2]
          write i0*: evicts i1* DIRTY (wr 1)       -> [in0 in1 in2 i0*]
      B0  i0 hits; i1 misses (the 7th line read), evicts in0
                                                   -> [in1 in2 i0* i1]
          write o0*: evicts in1                    -> [in2 i0* i1 o0*]
      => read 7, write 1, dirty tail {i0, o0} = 2 lines (i1 was re-read clean)."""
    g, tr = _lru_tiny()
    L = 128
    s = [(0, [(0, 1, 0)]), (0, [(0, 0, 0)]), (1, [(0, 0, 0)])]
    assert O.lru_dram_bytes(g, tr, s, 4 * L) == {"read": 7 * L, "write": 1 * L, "write_incl_tail": 3 * L}
