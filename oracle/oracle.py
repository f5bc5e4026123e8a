"""KTILER oracle — Python side (TEST INFRASTRUCTURE ONLY).

Only tests/, ``__graft_entry__.smoke()`` and bench.py's ``cpu_baseline`` /
``--impl reference`` legs may import this module.  It shares no code with the
product package and never imports it.

Contents (ids O-n):

* O-1..O-6  numpy wrappers over the C kernels in ktiler_oracle.c (whole images).
* ``OGraph`` the oracle's OWN description of a kernel graph: buffers, nodes
  and each node's block geometry (output tile tw x th per block, grid =
  ceil(W/tw) x ceil(H/th) x frames; "threads in one block
  process a small fragment of the input image ... and produce a small fragment
  of the output image").
* O-9  ``run_schedule``: runs any schedule block by block on poisoned buffers
  (0xA5 bytes / NaN floats), so an order that violates a dependency changes the
  output.
* O-10 ``trace``: exact RAW block dependencies and per-block 128-B memory lines
  by instrumented execution.
* O-8  ``cluster_tile``: Alg. 2 (ClusterTile) transcribed step
  by step in the paper's order and notation, with readings A11–A19.
* O-11 ``validate_schedule``: partition, dependency order
  (PAPER.md:171, 271), cache constraint.
* O-12 ``lru_dram_bytes``: fully-associative LRU line model, write-back,
  write-allocate, optional discard; pinned to hand-worked traces (every read miss,
  dirty eviction and dirty tail counted by hand, tests/test_oracle_schedule.py).  What
  it predicts for a real B200 (whose L2 is neither fully associative nor LRU) is an
  expectation, not a parity claim.
* O-13 ``application_tiling``: Alg. 1 with performance tables.
* O-14 ``hs_jacobi``: K Horn–Schunck Jacobi iterations, the paper's JI nodes
  (SURVEY §8(f) f2), in f32 (the GPU's exact operation order) or f64.
* O-7  ``gauss_taps`` / ``gauss_f32``: the float variant of the blur (SURVEY §8(c) O-7,
  reading A43): separable Gaussian with f64-normalised taps rounded to f32, evaluated in
  f64 with replicate border, as the plain definition.
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ktiler_oracle.c")
_SO = os.path.join(_HERE, "libktiler_oracle.so")
CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-std=c99", "-shared", "-fPIC"]

GRAY, BLUR5, DOWN2, SOBEL3, THRESH = 0, 1, 2, 3, 4
OP_NAMES = {GRAY: "gray", BLUR5: "blur5", DOWN2: "down2", SOBEL3: "sobel3", THRESH: "thresh"}
LINE = 128  # memory-line size in bytes


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", *CFLAGS, "-o", _SO, _SRC, "-lm"])
    return _SO


class KoBuf(ctypes.Structure):
    _fields_ = [("data", ctypes.c_void_p), ("W", ctypes.c_int64), ("H", ctypes.c_int64), ("F", ctypes.c_int64),
                ("elem", ctypes.c_int64), ("base", ctypes.c_int64), ("id", ctypes.c_int32), ("pad", ctypes.c_int32)]


_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        L = ctypes.CDLL(build())
        L.ko_run_rect.argtypes = [ctypes.c_int, ctypes.POINTER(KoBuf), ctypes.POINTER(KoBuf)] + \
            [ctypes.c_int64] * 5 + [ctypes.c_float]
        L.ko_run_rect.restype = ctypes.c_int
        L.ko_pipeline.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_float] + \
            [ctypes.c_void_p] * 5
        L.ko_pipeline.restype = ctypes.c_int
        L.ko_trace_begin.argtypes = [ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)]
        L.ko_trace_set_block.argtypes = [ctypes.c_int64]
        L.ko_trace_ndeps.restype = ctypes.c_int64
        L.ko_trace_nlines.restype = ctypes.c_int64
        L.ko_trace_get.argtypes = [ctypes.c_void_p, ctypes.c_void_p]
        _LIB = L
    return _LIB


# ---------------------------------------------------------------------------------------
# O-1 .. O-6: whole-image kernels
# ---------------------------------------------------------------------------------------
def _kobuf(arr: np.ndarray, W: int, H: int, F: int, elem: int, base: int = 0, bid: int = 0) -> KoBuf:
    assert arr.flags["C_CONTIGUOUS"]
    return KoBuf(arr.ctypes.data, W, H, F, elem, base, bid, 0)


def _run_whole(op: int, src: np.ndarray, out_shape, out_dtype, W_in, H_in, elem_in, W_out, H_out, T=200.0):
    F = src.shape[0]
    out = np.empty(out_shape, dtype=out_dtype)
    bi = _kobuf(src, W_in, H_in, F, elem_in, 0, 0)
    bo = _kobuf(out, W_out, H_out, F, np.dtype(out_dtype).itemsize, 0, 1)
    for z in range(F):
        rc = lib().ko_run_rect(op, ctypes.byref(bi), ctypes.byref(bo), z, 0, 0, W_out, H_out, T)
        assert rc == 0
    return out


def _as_batch(a: np.ndarray, nd: int) -> np.ndarray:
    a = np.ascontiguousarray(a)
    return a[None] if a.ndim == nd else a


def gray(rgb: np.ndarray) -> np.ndarray:
    """O-1: rgb uint8 [F,]H,W,3 -> uint8 [F,]H,W."""
    squeeze = rgb.ndim == 3
    r = _as_batch(rgb, 3)
    F, H, W, _ = r.shape
    out = _run_whole(GRAY, r, (F, H, W), np.uint8, W, H, 3, W, H)
    return out[0] if squeeze else out


def blur5(g: np.ndarray) -> np.ndarray:
    """O-2: uint8 [F,]H,W -> uint8 same shape."""
    squeeze = g.ndim == 2
    a = _as_batch(g, 2)
    F, H, W = a.shape
    out = _run_whole(BLUR5, a, (F, H, W), np.uint8, W, H, 1, W, H)
    return out[0] if squeeze else out


def down2(g: np.ndarray) -> np.ndarray:
    """O-3: uint8 [F,]H,W (even) -> uint8 [F,]H/2,W/2."""
    squeeze = g.ndim == 2
    a = _as_batch(g, 2)
    F, H, W = a.shape
    assert H % 2 == 0 and W % 2 == 0, "down2 needs even sizes (SURVEY A3)"
    out = _run_whole(DOWN2, a, (F, H // 2, W // 2), np.uint8, W, H, 1, W // 2, H // 2)
    return out[0] if squeeze else out


def sobel3(d: np.ndarray) -> np.ndarray:
    """O-4: uint8 [F,]h,w -> float32 magnitude."""
    squeeze = d.ndim == 2
    a = _as_batch(d, 2)
    F, H, W = a.shape
    out = _run_whole(SOBEL3, a, (F, H, W), np.float32, W, H, 1, W, H)
    return out[0] if squeeze else out


def thresh(s: np.ndarray, T: float = 200.0) -> np.ndarray:
    """O-5: float32 -> uint8 {0,255}, strict >."""
    squeeze = s.ndim == 2
    a = _as_batch(np.asarray(s, dtype=np.float32), 2)
    F, H, W = a.shape
    out = _run_whole(THRESH, a, (F, H, W), np.uint8, W, H, 4, W, H, T)
    return out[0] if squeeze else out


def pipeline(rgb: np.ndarray, T: float = 200.0) -> dict:
    """O-6: the untiled 5-kernel graph over a batch [F,H,W,3] (or one [H,W,3] image)."""
    squeeze = rgb.ndim == 3
    r = _as_batch(rgb, 3)
    F, H, W, _ = r.shape
    g = np.empty((F, H, W), np.uint8)
    b = np.empty((F, H, W), np.uint8)
    d = np.empty((F, H // 2, W // 2), np.uint8)
    s = np.empty((F, H // 2, W // 2), np.float32)
    m = np.empty((F, H // 2, W // 2), np.uint8)
    rc = lib().ko_pipeline(r.ctypes.data, W, H, F, T, g.ctypes.data, b.ctypes.data, d.ctypes.data, s.ctypes.data,
                           m.ctypes.data)
    assert rc == 0
    out = {"gray": g, "blur": b, "down": d, "sob": s, "mask": m}
    if squeeze:
        out = {k: v[0] for k, v in out.items()}
    return out


def motivational(rgb: np.ndarray) -> dict:
    """The paper's Fig. 1 graph: A = gray, B = down2 (no blur)."""
    g = gray(rgb)
    return {"gray": g, "down": down2(g)}


# ---------------------------------------------------------------------------------------
# The oracle's own graph description and block geometry
# ---------------------------------------------------------------------------------------
@dataclass
class OBuf:
    name: str
    W: int
    H: int
    F: int
    elem: int  # bytes per pixel (3 for rgb, 1 for u8, 4 for f32)
    dtype: object = np.uint8
    external: bool = False  # graph input (never written)

    @property
    def nbytes(self) -> int:
        return self.W * self.H * self.F * self.elem


@dataclass
class ONode:
    name: str
    op: int
    src: str
    dst: str
    tw: int  # output pixels per block in x
    th: int  # output pixels per block in y
    T: float = 200.0


@dataclass
class OGraph:
    bufs: dict = field(default_factory=dict)  # name -> OBuf, insertion order = address order
    nodes: list = field(default_factory=list)  # topological order

    def add_buf(self, *a, **k):
        b = OBuf(*a, **k)
        self.bufs[b.name] = b
        return b

    def add_node(self, *a, **k):
        n = ONode(*a, **k)
        self.nodes.append(n)
        return n

    # -- geometry --
    def grid(self, i: int):
        n = self.nodes[i]
        o = self.bufs[n.dst]
        return (-(-o.W // n.tw), -(-o.H // n.th), o.F)

    def nblocks(self, i: int) -> int:
        gx, gy, gz = self.grid(i)
        return gx * gy * gz

    def gid(self, i: int, b) -> int:
        """Global block id: nodes in order, blocks in (x, y, z) linear order (A12)."""
        off = sum(self.nblocks(j) for j in range(i))
        gx, gy, _ = self.grid(i)
        bx, by, bz = b
        return off + (bz * gy + by) * gx + bx

    def block_of(self, gid: int):
        for i in range(len(self.nodes)):
            n = self.nblocks(i)
            if gid < n:
                gx, gy, _ = self.grid(i)
                return i, (gid % gx, (gid // gx) % gy, gid // (gx * gy))
            gid -= n
        raise IndexError

    def blocks(self, i: int):
        gx, gy, gz = self.grid(i)
        return [(bx, by, bz) for bz in range(gz) for by in range(gy) for bx in range(gx)]

    def out_rect(self, i: int, b):
        """Output pixel rect of block b of node i: [x0,x1) x [y0,y1), frame z."""
        n = self.nodes[i]
        o = self.bufs[n.dst]
        bx, by, bz = b
        return (n.tw * bx, n.th * by, min(n.tw * (bx + 1), o.W), min(n.th * (by + 1), o.H), bz)

    def producers(self, i: int):
        return [j for j, m in enumerate(self.nodes) if m.dst == self.nodes[i].src]

    def consumers(self, i: int):
        return [j for j, m in enumerate(self.nodes) if m.src == self.nodes[i].dst]

    def bases(self):
        """Simulated 128-B-aligned byte addresses, one buffer after another."""
        out, a = {}, 1 << 20
        for name, b in self.bufs.items():
            out[name] = a
            a += -(-b.nbytes // 4096) * 4096 + 4096
        return out

    # -- storage --
    def alloc(self, inputs: dict, poison: bool = True) -> dict:
        mem = {}
        for name, b in self.bufs.items():
            shape = (b.F, b.H, b.W, 3) if b.elem == 3 else (b.F, b.H, b.W)
            if name in inputs:
                a = np.ascontiguousarray(inputs[name]).reshape(shape).copy()
            elif b.dtype == np.float32:
                a = np.full(shape, np.nan if poison else 0.0, dtype=np.float32)
            else:
                a = np.full(shape, 0xA5 if poison else 0, dtype=np.uint8)
            mem[name] = a
        return mem

    def _kobufs(self, mem: dict):
        bases = self.bases()
        return {name: _kobuf(mem[name], b.W, b.H, b.F, b.elem, bases[name], k)
                for k, (name, b) in enumerate(self.bufs.items())}

    def run_block(self, kb: dict, i: int, b) -> None:
        n = self.nodes[i]
        x0, y0, x1, y1, z = self.out_rect(i, b)
        rc = lib().ko_run_rect(n.op, ctypes.byref(kb[n.src]), ctypes.byref(kb[n.dst]), z, x0, y0, x1, y1, n.T)
        assert rc == 0


def pipeline_graph(W: int, H: int, F: int = 1, T: float = 200.0, full_tile=(256, 16), half_tile=(128, 8)) -> OGraph:
    """The north star's 5-kernel chain (BASELINE.json configs[1..4]) in the oracle's terms."""
    g = OGraph()
    g.add_buf("rgb", W, H, F, 3, external=True)
    g.add_buf("gray", W, H, F, 1)
    g.add_buf("blur", W, H, F, 1)
    g.add_buf("down", W // 2, H // 2, F, 1)
    g.add_buf("sob", W // 2, H // 2, F, 4, dtype=np.float32)
    g.add_buf("mask", W // 2, H // 2, F, 1)
    g.add_node("gray", GRAY, "rgb", "gray", *full_tile)
    g.add_node("blur", BLUR5, "gray", "blur", *full_tile)
    g.add_node("down", DOWN2, "blur", "down", *half_tile)
    g.add_node("sobel", SOBEL3, "down", "sob", *half_tile)
    g.add_node("thresh", THRESH, "sob", "mask", *half_tile, T=T)
    return g


def motivational_graph(W: int = 256, H: int = 256, F: int = 1, a_tile=(32, 8), b_tile=(64, 1)) -> OGraph:
    """Fig. 1: A<<<(8x32),(32x8)>>> one thread per pixel; B = 64x1
    threads, grid 2x128, one thread per output pixel (the reading that reproduces
    PAPER.md:43/291/307)."""
    g = OGraph()
    g.add_buf("in", W, H, F, 3, external=True)
    g.add_buf("intm", W, H, F, 1)
    g.add_buf("out", W // 2, H // 2, F, 1)
    g.add_node("A", GRAY, "in", "intm", *a_tile)
    g.add_node("B", DOWN2, "intm", "out", *b_tile)
    return g


# ---------------------------------------------------------------------------------------
# O-9 block-granular executor, O-10 tracer
# ---------------------------------------------------------------------------------------
def run_schedule(g: OGraph, schedule, inputs: dict, poison: bool = True) -> dict:
    """Execute ``schedule`` = iterable of (node_index, blocks) in order, each block computing
    only its own output rect, on buffers pre-filled with poison.  Returns all buffers."""
    mem = g.alloc(inputs, poison)
    kb = g._kobufs(mem)
    for i, blocks in schedule:
        for b in blocks:
            g.run_block(kb, i, tuple(b))
    return mem


def untiled_schedule(g: OGraph):
    """PAPER.md:41 normal execution mode: each kernel over all its blocks, in order."""
    return [(i, g.blocks(i)) for i in range(len(g.nodes))]


@dataclass
class Trace:
    deps: dict  # gid -> set of producer gids (direct, RAW)
    lines: dict  # gid -> set of 128-B line ids (read or written)
    rlines: dict  # gid -> set of lines read
    wlines: dict  # gid -> set of lines written


def trace(g: OGraph, inputs: dict | None = None) -> Trace:
    """O-10: run the untiled schedule block by block with instrumented accessors.  Block
    deps do not depend on pixel values for these kernels, so any input
    works; default is zeros."""
    if inputs is None:
        inputs = {n: np.zeros((b.F, b.H, b.W, 3) if b.elem == 3 else (b.F, b.H, b.W), np.uint8)
                  for n, b in g.bufs.items() if b.external}
    mem = g.alloc(inputs, poison=False)
    kb = g._kobufs(mem)
    sizes = (ctypes.c_int64 * len(g.bufs))(*[b.nbytes for b in g.bufs.values()])
    L = lib()
    L.ko_trace_begin(len(g.bufs), sizes)
    try:
        for i in range(len(g.nodes)):
            for b in g.blocks(i):
                L.ko_trace_set_block(g.gid(i, b))
                g.run_block(kb, i, b)
    finally:
        L.ko_trace_stop()
    nd, nl = L.ko_trace_ndeps(), L.ko_trace_nlines()
    deps_a = np.empty((nd, 2), np.int64)
    lines_a = np.empty((nl, 2), np.int64)
    L.ko_trace_get(deps_a.ctypes.data if nd else None, lines_a.ctypes.data if nl else None)
    total = sum(g.nblocks(i) for i in range(len(g.nodes)))
    deps = {k: set() for k in range(total)}
    for c, p in np.unique(deps_a, axis=0) if nd else []:
        deps[int(c)].add(int(p))
    lines = {k: set() for k in range(total)}
    rl = {k: set() for k in range(total)}
    wl = {k: set() for k in range(total)}
    for b, lw in np.unique(lines_a, axis=0) if nl else []:
        b, ln, w = int(b), int(lw) >> 1, int(lw) & 1
        lines[b].add(ln)
        (wl if w else rl)[b].add(ln)
    return Trace(deps, lines, rl, wl)


# ---------------------------------------------------------------------------------------
# O-8: Alg. 2 ClusterTile, literally
# ---------------------------------------------------------------------------------------
INF = math.inf


@dataclass
class Tiling:
    """T_i of Alg. 2: the tiling sequence (list of sub-kernels, each (node, sorted blocks)),
    the fragment index of each sub-kernel, and the cost (here: #sub-kernels, or INF)."""
    seq: list
    frag: list
    cost: float
    footprint_lines: list  # per fragment: |lines(newSubKBlks)|


def cluster_tile(g: OGraph, tr: Trace, budget_bytes: int, cluster=None, et=None) -> Tiling:
    """Alg. 2 for the cluster ``cluster`` (default: all nodes).

    Readings: A11 CheckCacheConst counts |union of lines read or written by
    the blocks in toBeAssigned| * 128 <= budget_bytes; A12 one next block per leaf node per
    iteration, (x,y,z) linear order, "unassigned" = not in assigned or toBeAssigned; A13
    FindAllDeps = transitive closure over intra-cluster producers, assigned blocks skipped;
    A14 FindMoreBlks = unassigned blocks of non-source nodes whose non-empty intra-cluster
    dependency set is inside toBeAssigned U assigned, iterated to a fixpoint; A15
    toBeAssigned accumulates across successful iterations and is emptied only at l.24; A16
    when no leaf block is left, newSubKBlks is committed; A17 one sub-kernel per node per
    commit, in topological order, empty ones omitted; A18 l.23 -> INF.  Cost (l.19):
    ``et(v, n_blocks, hot)`` = the performance-table time of a sub-kernel of node v with n
    blocks, hot iff one of v's producers is in the cluster; without ``et``
    CO_i counts sub-kernels (it then only matters for the INF signal).
    """
    nodes = list(range(len(g.nodes))) if cluster is None else sorted(cluster)
    in_cluster = set(nodes)
    node_of = {}
    blocks_of = {}
    for v in nodes:
        blocks_of[v] = [g.gid(v, b) for b in g.blocks(v)]
        for b in blocks_of[v]:
            node_of[b] = v
    allb = set(node_of)
    # intra-cluster direct deps (blkDepGraph restricted to the cluster)
    dep = {b: {p for p in tr.deps[b] if p in allb} for b in allb}
    has_consumer_in_cluster = {v: any(c in in_cluster for c in g.consumers(v)) for v in nodes}
    leaves = [v for v in nodes if not has_consumer_in_cluster[v]]
    sources = {v for v in nodes if not any(p in in_cluster for p in g.producers(v))}
    budget_lines = budget_bytes // LINE

    def find_all_deps(b, assigned):  # l.6 (A13)
        out, stack, seen = [], list(dep[b]), set()
        while stack:
            d = stack.pop()
            if d in seen or d in assigned:
                continue
            seen.add(d)
            out.append(d)
            stack.extend(dep[d])
        return out

    def find_more_blks(covered, assigned):  # l.11 (A14)
        ready = []
        cov = set(covered)
        changed = True
        while changed:
            changed = False
            for v in nodes:  # topological order
                if v in sources:
                    continue
                for b in blocks_of[v]:
                    if b in cov or b in assigned:
                        continue
                    if dep[b] and dep[b] <= cov:
                        cov.add(b)
                        ready.append(b)
                        changed = True
        return ready

    def check_cache_const(tba):  # l.13 (A11)
        lines = set()
        for b in tba:
            lines |= tr.lines[b]
        return len(lines) <= budget_lines, len(lines)

    # l.1-2
    CO = 0.0
    T, frag = [], []
    assigned = set()
    toBe = {v: [] for v in nodes}  # toBeAssigned[v] (ordered, set semantics)
    toBe_set = set()
    newSub = {v: set() for v in nodes}  # newSubKBlks[v]
    new_lines = 0
    fps = []
    nfrag = 0

    def push_tba(b):
        if b not in toBe_set:
            toBe_set.add(b)
            toBe[node_of[b]].append(b)

    def commit():  # l.17-22
        nonlocal CO, nfrag
        changed = False
        for v in nodes:
            if newSub[v]:
                T.append((v, sorted(g.block_of(b)[1] for b in newSub[v])))
                frag.append(nfrag)
                if et is None:
                    CO += 1
                else:  # l.19: ET(subKer_v, C_i, perfTables)
                    CO += et(v, len(newSub[v]), any(p in in_cluster for p in g.producers(v)))
                assigned.update(newSub[v])
                changed = True
        if changed:
            fps.append(new_lines)
            nfrag += 1
        return changed

    def pick(pool):
        out = []
        for v in pool:  # l.4 (A12)
            for b in blocks_of[v]:
                if b not in assigned and b not in toBe_set:
                    out.append(b)
                    break
        return out

    while assigned != allb:  # l.3
        # ---- bottom-up round (l.4-10) ----
        picked = pick(leaves)
        if not picked:
            # A16b: blocks no leaf block depends on act as bottom blocks, last node first
            rest = [v for v in reversed(nodes) if any(b not in assigned and b not in toBe_set for b in blocks_of[v])]
            picked = pick(rest[:1])
        if not picked:
            # A16: every block is in assigned U toBeAssigned -> commit newSubKBlks
            if not commit():
                return Tiling(T, frag, INF, fps)
            break
        for b in picked:
            push_tba(b)  # l.5
            for d in find_all_deps(b, assigned):  # l.6-10
                if d not in assigned:
                    push_tba(d)
        # ---- top-down round (l.11-12) ----
        for b in find_more_blks(toBe_set, assigned):
            push_tba(b)
        # ---- l.13 ----
        ok, nl = check_cache_const(toBe_set)
        if ok:  # l.14-15
            for v in nodes:
                newSub[v].update(toBe[v])
            new_lines = nl
        else:  # l.16-24
            if not commit():
                return Tiling(T, frag, INF, fps)  # l.23 (A18)
            toBe = {v: [] for v in nodes}  # l.24
            toBe_set = set()
            newSub = {v: set() for v in nodes}
            new_lines = 0
    return Tiling(T, frag, CO, fps)


# ---------------------------------------------------------------------------------------
# O-13: Alg. 1 Application Tiling with performance tables
# ---------------------------------------------------------------------------------------
def et_lookup(table, n: int, hot: bool) -> float:
    """Performance-table lookup ("for the missing points, the duration is
    obtained by interpolation"; reading A35): ``table`` = (block counts, cold ms, hot ms);
    linear between points, the first point's time below the table, the last point's
    per-block rate above it."""
    ns, cold, hot_t = table
    t = hot_t if hot else cold
    if n <= ns[0]:
        return t[0]
    for k in range(1, len(ns)):
        if n <= ns[k]:
            return t[k - 1] + (t[k] - t[k - 1]) * (n - ns[k - 1]) / (ns[k] - ns[k - 1])
    return t[-1] * n / ns[-1]


def quotient_is_acyclic(edges, cluster_of) -> bool:
    """A partition is valid iff its clusters can be totally ordered with no back-dependency
    (PAPER.md:247–257): the graph of clusters (edges between different clusters) is
    acyclic."""
    nodes = set(cluster_of.values())
    adj = {c: set() for c in nodes}
    for u, v in edges:
        if cluster_of[u] != cluster_of[v]:
            adj[cluster_of[u]].add(cluster_of[v])
    state = {}

    def dfs(c):
        state[c] = 1
        for d in adj[c]:
            if state.get(d) == 1 or (d not in state and not dfs(d)):
                return False
        state[c] = 2
        return True
    return all(c in state or dfs(c) for c in nodes)


def application_tiling(g: OGraph, tr: Trace, budget_bytes: int, tables: dict, weights: dict, thld: float):
    """Alg. 1, line by line.  ``tables[v]`` = performance table of node v
    (see et_lookup); ``weights[(u, v)]`` = edge weight (None: derived as the time v saves
    when that input is cached, ET_cold(N) - ET_hot(N)).  Reading A22: weight
    > thld strict; ties by (src, dst); an edge whose ends already share a cluster is dropped.
    Returns (clusters in execution order, their costs, schedule [(node, blocks, cluster)])."""
    n = len(g.nodes)
    et = lambda v, k, hot: et_lookup(tables[v], k, hot)  # noqa: E731
    P = {i: [i] for i in range(n)}  # l.1–5: C_i = {v_i}
    T = {i: None for i in range(n)}  # None = the kernel untiled (T_i = {kernel(v_i)})
    CO = {i: et(i, g.nblocks(i), False) for i in range(n)}  # kerExeTimes
    cluster_of = {i: i for i in range(n)}
    edges = [(u, v) for v in range(n) for u in g.producers(v)]
    w = {}
    for (u, v) in edges:
        wv = weights.get((u, v))
        w[(u, v)] = et(v, g.nblocks(v), False) - et(v, g.nblocks(v), True) if wv is None else wv
    cand = sorted([e for e in edges if w[e] > thld], key=lambda e: (-w[e], e[0], e[1]))  # l.6–7
    eix = 0
    while eix < len(cand):  # l.8
        u, v = cand[eix]  # l.9
        a, b = cluster_of[u], cluster_of[v]  # l.10
        if a == b:
            cand.pop(eix)
            eix = 0
            continue
        merged = sorted(P[a] + P[b])  # l.11 (node ids are in topological order)
        tmp_of = dict(cluster_of)  # l.12
        for x in P[b]:
            tmp_of[x] = a
        if quotient_is_acyclic(edges, tmp_of):  # l.13
            til = cluster_tile(g, tr, budget_bytes, cluster=merged, et=et)  # l.14
            if til.cost < CO[a] + CO[b]:  # l.15
                cluster_of = tmp_of
                P[a] = merged
                del P[b]
                T[a], CO[a] = til, til.cost
                del T[b], CO[b]
            cand.pop(eix)  # l.16
            eix = 0
        else:
            eix += 1  # l.18
    # l.21–23: the clusters' tiling sequences in a topological order of the clusters
    order, done = [], set()
    while len(order) < len(P):
        ready = [c for c in P if c not in done and all(cluster_of[p] in done or cluster_of[p] == c
                                                       for x in P[c] for p in g.producers(x))]
        c = min(ready, key=lambda c: P[c][0])
        order.append(c)
        done.add(c)
    sched = []
    for k, c in enumerate(order):
        if T[c] is None:
            v = P[c][0]
            sched.append((v, g.blocks(v), k))
        else:
            sched.extend((v, blocks, k) for (v, blocks) in T[c].seq)
    return [P[c] for c in order], [CO[c] for c in order], sched


# ---------------------------------------------------------------------------------------
# O-11 schedule validator
# ---------------------------------------------------------------------------------------
def validate_schedule(g: OGraph, tr: Trace, schedule, budget_bytes: int | None = None, frags=None) -> list:
    """Returns a list of violations (empty = valid).  ``schedule`` = [(node, blocks)]."""
    errs = []
    seen = {}
    pos = {}
    for s, (i, blocks) in enumerate(schedule):
        for b in blocks:
            gid = g.gid(i, tuple(b))
            if gid in seen:
                errs.append(f"block {i}{tuple(b)} in two sub-kernels")  # disjoint
            seen[gid] = s
            pos[gid] = s
    total = sum(g.nblocks(i) for i in range(len(g.nodes)))
    if len(seen) != total:
        errs.append(f"sub-kernels cover {len(seen)} of {total} blocks")  # cover
    for c, ps in tr.deps.items():
        for p in ps:
            if c in pos and p in pos and not pos[p] < pos[c]:
                errs.append(f"block {g.block_of(c)} scheduled before its producer {g.block_of(p)}")
                break
    if budget_bytes is not None and frags is not None:
        by_frag = {}
        for s, (i, blocks) in enumerate(schedule):
            for b in blocks:
                by_frag.setdefault(frags[s], set()).update(tr.lines[g.gid(i, tuple(b))])
        for f, ls in by_frag.items():
            if len(ls) * LINE > budget_bytes:
                errs.append(f"fragment {f}: footprint {len(ls) * LINE} B > budget {budget_bytes}")
    return errs


# ---------------------------------------------------------------------------------------
# O-12 LRU line model (expectation only)
# ---------------------------------------------------------------------------------------
def lru_dram_bytes(g: OGraph, tr: Trace, schedule, cache_bytes: int, discard_dead: bool = False,
                   internal=None) -> dict:
    """Fully associative LRU over 128-B lines, write-back, write-allocate without fetch.
    Each block reads its read-lines then writes its write-lines.  With ``discard_dead``,
    a line of an internal buffer is dropped (no write-back) after its last reader."""
    from collections import OrderedDict
    cap = cache_bytes // LINE
    cache = OrderedDict()  # line -> dirty
    rd = wr = 0
    order = [g.gid(i, tuple(b)) for i, blocks in schedule for b in blocks]
    last_reader = {}
    if discard_dead:
        bases = g.bases()
        if internal is None:
            internal = [n for n, b in g.bufs.items() if not b.external and any(m.src == n for m in g.nodes)]
        ranges = [(bases[n] // LINE, (bases[n] + g.bufs[n].nbytes + LINE - 1) // LINE) for n in internal]
        for k, b in enumerate(order):
            for ln in tr.rlines[b]:
                if any(lo <= ln < hi for lo, hi in ranges):
                    last_reader[ln] = k
    dead_at = {}
    for ln, k in last_reader.items():
        dead_at.setdefault(k, []).append(ln)
    for k, b in enumerate(order):
        for ln in sorted(tr.rlines[b]):
            if ln in cache:
                cache.move_to_end(ln)
            else:
                rd += LINE
                cache[ln] = False
                if len(cache) > cap:
                    _, d = cache.popitem(last=False)
                    wr += LINE if d else 0
        for ln in sorted(tr.wlines[b]):
            cache[ln] = True
            cache.move_to_end(ln)
            if len(cache) > cap:
                _, d = cache.popitem(last=False)
                wr += LINE if d else 0
        for ln in dead_at.get(k, []):
            cache.pop(ln, None)
    wr_tail = sum(LINE for d in cache.values() if d)
    return {"read": rd, "write": wr, "write_incl_tail": wr + wr_tail}


# ---------------------------------------------------------------------------------------
# O-14: Horn–Schunck Jacobi iterations (the JI nodes of Fig. 4)
# ---------------------------------------------------------------------------------------
def hs_jacobi(coef: np.ndarray, s0: np.ndarray, a2: float, iters: int, dtype=np.float32) -> np.ndarray:
    """K Jacobi iterations of the Horn–Schunck equations (Horn & Schunck 1981, the method
    HSOpticalFlow implements): with ub, vb the mean of the 4 neighbours
    (replicate border, reading A39),
        t  = (Ix*ub + Iy*vb + It) / (alpha^2 + Ix^2 + Iy^2)
        u' = ub - Ix*t,   v' = vb - Iy*t.
    coef [F, H, W, 4] = (Ix, Iy, It, -); s0 [F, H, W, 2] = (u, v); a2 = alpha^2.  Every
    operation is evaluated in the order written in include/ktiler.h (KTILER_OP_JACOBI),
    one numpy op at a time in ``dtype`` (float32: each op IEEE-rounded, no contraction)."""
    c = coef.astype(dtype)
    Ix, Iy, It = c[..., 0], c[..., 1], c[..., 2]
    a2 = dtype(a2)
    quarter = dtype(0.25)
    den = (a2 + Ix * Ix) + Iy * Iy
    s = s0.astype(dtype).copy()
    for _ in range(iters):
        u, v = s[..., 0], s[..., 1]

        def mean4(a):
            left = np.concatenate([a[:, :, :1], a[:, :, :-1]], axis=2)
            right = np.concatenate([a[:, :, 1:], a[:, :, -1:]], axis=2)
            up = np.concatenate([a[:, :1], a[:, :-1]], axis=1)
            down = np.concatenate([a[:, 1:], a[:, -1:]], axis=1)
            return ((left + right) + (up + down)) * quarter
        ub, vb = mean4(u), mean4(v)
        t = ((Ix * ub + Iy * vb) + It) / den
        s = np.stack([ub - Ix * t, vb - Iy * t], axis=-1)
    return s


def gauss_taps(sigma: float) -> np.ndarray:
    """O-7 weights (reading A43): radius r = ceil(3 sigma); w_k = exp(-k^2 / (2 sigma^2))
    for k = -r..r, normalised to sum 1 in f64, then rounded to f32 (the values both sides
    use).  Returned as float32 [2r+1]."""
    r = int(np.ceil(3.0 * np.float64(np.float32(sigma))))
    s = np.float64(np.float32(sigma))
    k = np.arange(-r, r + 1, dtype=np.float64)
    w = np.exp(-k * k / (2.0 * s * s))
    return (w / w.sum()).astype(np.float32)


def gauss_f32(x: np.ndarray, sigma: float, passes: int = 1) -> np.ndarray:
    """O-7: ``passes`` applications of the separable Gaussian to f32 images x [F, H, W],
    out[y][x] = sum_i w_i sum_j w_j in[clamp(y+i)][clamp(x+j)] (replicate border), written
    out in f64 (the definition; the GPU computes it in f32 FMA chains, tolerance 1e-5 on
    data in [0, 1], BJ:5).  Returns float64 [F, H, W]."""
    w = gauss_taps(sigma).astype(np.float64)
    r = (len(w) - 1) // 2
    a = x.astype(np.float64)
    for _ in range(passes):
        F, H, W = a.shape
        p = np.pad(a, ((0, 0), (0, 0), (r, r)), mode="edge")
        h = np.zeros_like(a)
        for j in range(2 * r + 1):
            h += w[j] * p[:, :, j:j + W]
        p = np.pad(h, ((0, 0), (r, r), (0, 0)), mode="edge")
        a = np.zeros_like(h)
        for i in range(2 * r + 1):
            a += w[i] * p[:, i:i + H, :]
    return a
