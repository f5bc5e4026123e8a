"""Thin ctypes binding of libktiler.so (include/ktiler.h) — argument marshalling only.

Every step of the hot path (planning, dependency analysis, partitioning, emission,
launching, the kernels themselves) runs inside libktiler.so.  There is no Python or
CPU fallback: if the shared library is missing this module raises on import of the
library, and every ABI error is raised as KtilerError with the library's message.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libktiler.so")

# ---- enums (mirror include/ktiler.h) ----
OK, E_INVALID, E_CYCLE, E_UNTILEABLE, E_NOMEM, E_CUDA, E_STATE, E_UNSUPPORTED = range(8)
BUF_INTERNAL = 1
READ, WRITE = 1, 2
OP_GRAY, OP_BLUR5, OP_DOWN2, OP_SOBEL3, OP_THRESH, OP_CUSTOM, OP_JACOBI, OP_GAUSS_F32 = range(8)
FRAG_BUDGET, FRAG_ROWS, FRAG_BALANCED, FRAG_NONE, FRAG_ALG1, FRAG_CHAIN = range(6)
EXEC_STREAM, EXEC_GRAPH, EXEC_GRAPH_PERSIST_L2, EXEC_PERSISTENT, EXEC_GRAPH_DAG, EXEC_GRAPH_CHAIN, EXEC_GRAPH_WAVE, \
    EXEC_FLOW = range(8)
PF_DISCARD_DEAD, PF_PDL, PF_FORCE_MINIMAL, PF_RESIDENT_BUDGET, PF_CONSUMER_DISCARD, PF_HALO_DISCARD = 1, 2, 4, 8, 16, 32
PF_MULTIRATE = 64

EXEC_MODES = {"stream": EXEC_STREAM, "graph": EXEC_GRAPH, "persist_l2": EXEC_GRAPH_PERSIST_L2,
              "persistent": EXEC_PERSISTENT, "dag": EXEC_GRAPH_DAG, "chain": EXEC_GRAPH_CHAIN,
              "wave": EXEC_GRAPH_WAVE, "flow": EXEC_FLOW}
FRAG_KINDS = {"budget": FRAG_BUDGET, "rows": FRAG_ROWS, "balanced": FRAG_BALANCED, "none": FRAG_NONE,
              "alg1": FRAG_ALG1, "chain": FRAG_CHAIN}


SELFTEST_SQRT = 0
COMM_NCCL, COMM_LOOPBACK = 0, 1


def selftest(which: int = SELFTEST_SQRT) -> int:
    """ktiler_selftest: number of failing inputs (0 = pass)."""
    n = ctypes.c_int64()
    _check(lib().ktiler_selftest(which, ctypes.byref(n)))
    return n.value


class KtilerError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__(f"{_status_name(status)}: {msg}")


class BufferDesc(ctypes.Structure):
    _fields_ = [("base", ctypes.c_void_p), ("width", ctypes.c_int64), ("height", ctypes.c_int64),
                ("frames", ctypes.c_int64), ("pitch_bytes", ctypes.c_int64), ("frame_stride_bytes", ctypes.c_int64),
                ("elem_bytes", ctypes.c_int32), ("flags", ctypes.c_uint32), ("ring_frames", ctypes.c_int64)]


class Access(ctypes.Structure):
    _fields_ = [("buf_id", ctypes.c_int32), ("mode", ctypes.c_int32), ("ax", ctypes.c_int64), ("ay", ctypes.c_int64),
                ("ox", ctypes.c_int64), ("oy", ctypes.c_int64), ("halo_l", ctypes.c_int32),
                ("halo_r", ctypes.c_int32), ("halo_t", ctypes.c_int32), ("halo_b", ctypes.c_int32)]


LAUNCH_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.POINTER(ctypes.c_int32), ctypes.c_int32, ctypes.c_void_p)


class KernelDesc(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int32), ("grid", ctypes.c_uint32 * 3), ("block", ctypes.c_uint32 * 3),
                ("n_access", ctypes.c_int32), ("access", ctypes.POINTER(Access)), ("params", ctypes.c_void_p),
                ("params_bytes", ctypes.c_size_t), ("launch", LAUNCH_FN), ("user", ctypes.c_void_p)]


class Policy(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("l2_fraction", ctypes.c_double), ("rows", ctypes.c_int64),
                ("exec_mode", ctypes.c_int32), ("flags", ctypes.c_uint32), ("persistent_ctas", ctypes.c_int32),
                ("pipeline_skew", ctypes.c_int32), ("window", ctypes.c_int32), ("alg1_thld", ctypes.c_double)]


class SubKernelInfo(ctypes.Structure):
    _fields_ = [("node", ctypes.c_int32), ("fragment", ctypes.c_int32), ("n_blocks", ctypes.c_int64),
                ("n_rects", ctypes.c_int32), ("cluster", ctypes.c_int32), ("footprint_bytes", ctypes.c_int64)]


class FootprintRec(ctypes.Structure):
    _fields_ = [("buf_id", ctypes.c_int32), ("mode", ctypes.c_int32), ("first", ctypes.c_int64), ("last", ctypes.c_int64)]


class PlanStats(ctypes.Structure):
    _fields_ = [("n_subkernels", ctypes.c_int64), ("n_fragments", ctypes.c_int64), ("n_launches", ctypes.c_int64),
                ("n_discard_lines", ctypes.c_int64), ("budget_bytes", ctypes.c_int64),
                ("max_footprint_bytes", ctypes.c_int64), ("plan_ms", ctypes.c_double), ("exec_mode", ctypes.c_int32),
                ("pad", ctypes.c_int32)]


class TraceRecord(ctypes.Structure):
    _fields_ = [("id", ctypes.c_uint64), ("smid", ctypes.c_uint32), ("kind", ctypes.c_uint32),
                ("t0_ns", ctypes.c_uint64), ("t1_ns", ctypes.c_uint64)]


class Strip(ctypes.Structure):
    _fields_ = [("base", ctypes.c_void_p), ("pitch_bytes", ctypes.c_int64), ("row_bytes", ctypes.c_int64),
                ("o0", ctypes.c_int64), ("o1", ctypes.c_int64), ("e0", ctypes.c_int64), ("e1", ctypes.c_int64)]


class HostCopy(ctypes.Structure):
    _fields_ = [("buf_id", ctypes.c_int32), ("pad", ctypes.c_int32), ("host", ctypes.c_void_p),
                ("frame0", ctypes.c_int64), ("frames", ctypes.c_int64)]


EXPORTS = ["ktiler_status_str", "ktiler_last_error", "ktiler_abi_version", "ktiler_graph_create",
           "ktiler_graph_destroy", "ktiler_add_buffer", "ktiler_add_kernel", "ktiler_add_edge",
           "ktiler_graph_block_deps", "ktiler_graph_block_lines", "ktiler_plan", "ktiler_plan_destroy",
           "ktiler_plan_num_subkernels", "ktiler_plan_num_fragments", "ktiler_plan_get_subkernel",
           "ktiler_plan_get_stats", "ktiler_execute", "ktiler_execute_host", "ktiler_trace_enable",
           "ktiler_trace_read", "ktiler_plan_get_launch", "ktiler_selftest", "ktiler_plan_num_clusters",
           "ktiler_plan_get_cluster", "ktiler_set_perf_table", "ktiler_calibrate", "ktiler_discover_footprint",
           "ktiler_plan_set_flow_roles", "ktiler_comm_unique_id", "ktiler_comm_init_nccl",
           "ktiler_comm_init_loopback", "ktiler_comm_destroy", "ktiler_comm_register_strip", "ktiler_halo_exchange",
           "ktiler_plan_attach_halo", "ktiler_plan_reorder", "ktiler_comm_check"]

_LIB = None


def lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} is missing: build it with `python -c 'import __graft_entry__ as g; g.build()'` "
                           "(there is no fallback path)")
    L = ctypes.CDLL(LIB_PATH)
    vp, i32, i64, P = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.POINTER
    st = ctypes.c_int
    sig = {
        "ktiler_status_str": ([st], ctypes.c_char_p),
        "ktiler_last_error": ([], ctypes.c_char_p),
        "ktiler_abi_version": ([], i32),
        "ktiler_graph_create": ([P(vp)], st),
        "ktiler_graph_destroy": ([vp], None),
        "ktiler_add_buffer": ([vp, P(BufferDesc), P(i32)], st),
        "ktiler_add_kernel": ([vp, P(KernelDesc), P(i32)], st),
        "ktiler_add_edge": ([vp, i32, i32, i32, ctypes.c_float], st),
        "ktiler_graph_block_deps": ([vp, i32, i32, i32, i32, P(i32), i64, P(i64)], st),
        "ktiler_graph_block_lines": ([vp, i32, i32, i32, i32, P(i64), i64, P(i64)], st),
        "ktiler_plan": ([vp, ctypes.c_size_t, P(Policy), P(vp)], st),
        "ktiler_plan_destroy": ([vp], None),
        "ktiler_plan_num_subkernels": ([vp, P(i64)], st),
        "ktiler_plan_num_fragments": ([vp, P(i64)], st),
        "ktiler_plan_get_subkernel": ([vp, i64, P(SubKernelInfo), P(i32), i32], st),
        "ktiler_plan_get_stats": ([vp, P(PlanStats)], st),
        "ktiler_execute": ([vp, vp], st),
        "ktiler_execute_host": ([vp, P(HostCopy), i32, P(HostCopy), i32, vp], st),
        "ktiler_trace_enable": ([vp, i64], st),
        "ktiler_trace_read": ([vp, vp, i64, P(i64)], st),
        "ktiler_plan_get_launch": ([vp, i64, P(i32), P(i32), P(i64)], st),
        "ktiler_selftest": ([i32, P(i64)], st),
        "ktiler_plan_num_clusters": ([vp, P(i32)], st),
        "ktiler_plan_get_cluster": ([vp, i32, P(i32), i32, P(i32), P(ctypes.c_double)], st),
        "ktiler_set_perf_table": ([vp, i32, i32, P(i64), P(ctypes.c_double), P(ctypes.c_double)], st),
        "ktiler_calibrate": ([vp, i32, i32, P(i64), i32, P(ctypes.c_double), P(ctypes.c_double)], st),
        "ktiler_discover_footprint": ([vp, i32, i32, i32, i32, i32, ctypes.c_uint64, P(FootprintRec), i32, P(i32)], st),
        "ktiler_plan_set_flow_roles": ([vp, P(i32), i32, P(i32), i32], st),
        "ktiler_comm_unique_id": ([P(ctypes.c_uint8)], st),
        "ktiler_comm_init_nccl": ([P(ctypes.c_uint8), i32, i32, P(vp)], st),
        "ktiler_comm_init_loopback": ([i32, P(vp)], st),
        "ktiler_comm_destroy": ([vp], None),
        "ktiler_comm_register_strip": ([vp, i32, P(Strip)], st),
        "ktiler_halo_exchange": ([vp, i32, i32, vp], st),
        "ktiler_plan_attach_halo": ([vp, vp, i32, i32], st),
        "ktiler_plan_reorder": ([vp, P(i64), i64], st),
        "ktiler_comm_check": ([vp], st),
    }
    for name, (args, res) in sig.items():
        f = getattr(L, name)
        f.argtypes = args
        f.restype = res
    if L.ktiler_abi_version() != 2:
        raise RuntimeError("libktiler ABI version mismatch")
    _LIB = L
    return L


def _status_name(s: int) -> str:
    try:
        return lib().ktiler_status_str(s).decode()
    except Exception:  # pragma: no cover
        return str(s)


def _check(s: int) -> None:
    if s != OK:
        raise KtilerError(s, lib().ktiler_last_error().decode())


class Graph:
    """Owning wrapper of a ktiler_graph_t."""

    def __init__(self):
        h = ctypes.c_void_p()
        _check(lib().ktiler_graph_create(ctypes.byref(h)))
        self._h = h
        self._keep = []

    def close(self):
        if self._h:
            lib().ktiler_graph_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def add_buffer(self, base: int, width: int, height: int, elem_bytes: int, frames: int = 1,
                   pitch_bytes: int | None = None, frame_stride_bytes: int = 0, internal: bool = False,
                   ring_frames: int = 0) -> int:
        pitch = pitch_bytes if pitch_bytes is not None else width * elem_bytes
        d = BufferDesc(base, width, height, frames, pitch, frame_stride_bytes, elem_bytes,
                       BUF_INTERNAL if internal else 0, ring_frames)
        out = ctypes.c_int32()
        _check(lib().ktiler_add_buffer(self._h, ctypes.byref(d), ctypes.byref(out)))
        return out.value

    def add_kernel(self, op: int, grid, block, accesses, params: bytes | None = None, launch=None,
                   user: int | None = None) -> int:
        """launch (OP_CUSTOM): a Python callable, or the integer address of a C function with
        the ktiler_launch_fn signature (a user's compiled kernel launcher); user: its
        opaque pointer."""
        acc = (Access * len(accesses))()
        for i, a in enumerate(accesses):
            acc[i] = Access(a["buf"], a["mode"], a["ax"], a["ay"], a.get("ox", 0), a.get("oy", 0),
                            a.get("hl", 0), a.get("hr", 0), a.get("ht", 0), a.get("hb", 0))
        pbuf = ctypes.create_string_buffer(params) if params else None
        fn = LAUNCH_FN(launch) if launch is not None else LAUNCH_FN()
        if launch is not None:
            self._keep.append(fn)
        d = KernelDesc(op, (ctypes.c_uint32 * 3)(*grid), (ctypes.c_uint32 * 3)(*block), len(accesses), acc,
                       ctypes.cast(pbuf, ctypes.c_void_p) if pbuf else None, len(params) if params else 0, fn, user)
        out = ctypes.c_int32()
        _check(lib().ktiler_add_kernel(self._h, ctypes.byref(d), ctypes.byref(out)))
        return out.value

    def add_edge(self, src: int, dst: int, buf: int, weight: float = 1.0) -> None:
        _check(lib().ktiler_add_edge(self._h, src, dst, buf, weight))

    def block_deps(self, node: int, bx: int, by: int, bz: int = 0):
        n = ctypes.c_int64()
        _check(lib().ktiler_graph_block_deps(self._h, node, bx, by, bz, None, 0, ctypes.byref(n)))
        arr = (ctypes.c_int32 * (4 * max(1, n.value)))()
        _check(lib().ktiler_graph_block_deps(self._h, node, bx, by, bz, arr, n.value, ctypes.byref(n)))
        return [tuple(arr[4 * i:4 * i + 4]) for i in range(n.value)]

    def block_lines(self, node: int, bx: int, by: int, bz: int = 0):
        n = ctypes.c_int64()
        _check(lib().ktiler_graph_block_lines(self._h, node, bx, by, bz, None, 0, ctypes.byref(n)))
        arr = (ctypes.c_int64 * max(1, n.value))()
        _check(lib().ktiler_graph_block_lines(self._h, node, bx, by, bz, arr, n.value, ctypes.byref(n)))
        return list(arr[:n.value])

    def set_perf_table(self, node: int, nblocks, ms_cold, ms_hot) -> None:
        """Performance table of a node for the ALG1 policy."""
        n = len(nblocks)
        _check(lib().ktiler_set_perf_table(self._h, node, n, (ctypes.c_int64 * n)(*nblocks),
                                           (ctypes.c_double * n)(*ms_cold), (ctypes.c_double * n)(*ms_hot)))

    def discover_footprint(self, node: int, bx: int, by: int, bz: int = 0, trials: int = 3, seed: int = 1):
        """Dependency footprint of one block by differential execution (include/ktiler.h,
        SURVEY §8(f) f3) -> list of (buf_id, mode, first_byte, last_byte_exclusive)."""
        n = ctypes.c_int32()
        _check(lib().ktiler_discover_footprint(self._h, node, bx, by, bz, trials, seed, None, 0, ctypes.byref(n)))
        arr = (FootprintRec * max(1, n.value))()
        _check(lib().ktiler_discover_footprint(self._h, node, bx, by, bz, trials, seed, arr, n.value, ctypes.byref(n)))
        return [(r.buf_id, r.mode, r.first, r.last) for r in arr[:n.value]]

    def calibrate(self, node: int, nblocks, reps: int = 5):
        """Measure a node's performance table on the current device -> (cold, hot) lists (ms)."""
        n = len(nblocks)
        c, h = (ctypes.c_double * n)(), (ctypes.c_double * n)()
        _check(lib().ktiler_calibrate(self._h, node, n, (ctypes.c_int64 * n)(*nblocks), reps, c, h))
        return list(c), list(h)

    def plan(self, cache_bytes: int = 0, kind: str | int = "budget", l2_fraction: float = 1.0, rows: int = 1,
             exec_mode: str | int = "graph", discard: bool = False, pdl: bool = False, force_minimal: bool = False,
             persistent_ctas: int = 0, skew: int = 0, window: int = 0, resident_budget: bool = False,
             alg1_thld: float = 0.0, consumer_discard: bool = False, halo_discard: bool = False,
             multirate: bool = False) -> "Plan":
        k = FRAG_KINDS[kind] if isinstance(kind, str) else kind
        m = EXEC_MODES[exec_mode] if isinstance(exec_mode, str) else exec_mode
        flags = (PF_DISCARD_DEAD if discard else 0) | (PF_PDL if pdl else 0) | (PF_FORCE_MINIMAL if force_minimal else 0) \
            | (PF_RESIDENT_BUDGET if resident_budget else 0) | (PF_CONSUMER_DISCARD if consumer_discard else 0) \
            | (PF_HALO_DISCARD if halo_discard else 0) | (PF_MULTIRATE if multirate else 0)
        pol = Policy(k, l2_fraction, rows, m, flags, persistent_ctas, skew, window, alg1_thld)
        h = ctypes.c_void_p()
        _check(lib().ktiler_plan(self._h, cache_bytes, ctypes.byref(pol), ctypes.byref(h)))
        return Plan(h, self)


class Plan:
    """Owning wrapper of a ktiler_plan_t.  Keeps its graph's Python objects alive (custom
    launch callbacks)."""

    def __init__(self, h, graph: Graph):
        self._h = h
        self._graph_keep = graph._keep

    def close(self):
        if self._h:
            lib().ktiler_plan_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def num_subkernels(self) -> int:
        n = ctypes.c_int64()
        _check(lib().ktiler_plan_num_subkernels(self._h, ctypes.byref(n)))
        return n.value

    def num_fragments(self) -> int:
        n = ctypes.c_int64()
        _check(lib().ktiler_plan_num_fragments(self._h, ctypes.byref(n)))
        return n.value

    def subkernels(self):
        """List of dicts: node, fragment, n_blocks, footprint_bytes, rects [(x0,y0,z0,x1,y1,z1)]."""
        out = []
        for i in range(self.num_subkernels()):
            info = SubKernelInfo()
            _check(lib().ktiler_plan_get_subkernel(self._h, i, ctypes.byref(info), None, 0))
            arr = (ctypes.c_int32 * (6 * max(1, info.n_rects)))()
            _check(lib().ktiler_plan_get_subkernel(self._h, i, ctypes.byref(info), arr, info.n_rects))
            out.append({"node": info.node, "fragment": info.fragment, "n_blocks": info.n_blocks, "cluster": info.cluster,
                        "footprint_bytes": info.footprint_bytes,
                        "rects": [tuple(arr[6 * k:6 * k + 6]) for k in range(info.n_rects)]})
        return out

    def clusters(self):
        """[(node ids, estimated cost ms)] in execution order (Alg. 1 partition)."""
        n = ctypes.c_int32()
        _check(lib().ktiler_plan_num_clusters(self._h, ctypes.byref(n)))
        out = []
        for i in range(n.value):
            cnt, cost = ctypes.c_int32(), ctypes.c_double()
            _check(lib().ktiler_plan_get_cluster(self._h, i, None, 0, ctypes.byref(cnt), ctypes.byref(cost)))
            arr = (ctypes.c_int32 * max(1, cnt.value))()
            _check(lib().ktiler_plan_get_cluster(self._h, i, arr, cnt.value, ctypes.byref(cnt), ctypes.byref(cost)))
            out.append((list(arr[:cnt.value]), cost.value))
        return out

    def stats(self) -> dict:
        s = PlanStats()
        _check(lib().ktiler_plan_get_stats(self._h, ctypes.byref(s)))
        return {f: getattr(s, f) for f, _ in PlanStats._fields_ if f != "pad"}

    def trace_enable(self, capacity: int = 1 << 20) -> None:
        """Device-side timeline records (include/ktiler.h, ktiler_trace_enable); call before
        the first execute."""
        _check(lib().ktiler_trace_enable(self._h, capacity))
        self._trace_cap = capacity

    def trace_read(self):
        """numpy structured array of the records written since the last read (synchronizes)."""
        import numpy as np
        n = ctypes.c_int64()
        cap = self._trace_cap
        buf = (TraceRecord * cap)()
        _check(lib().ktiler_trace_read(self._h, ctypes.cast(buf, ctypes.c_void_p), cap, ctypes.byref(n)))
        dt = np.dtype([("id", "<u8"), ("smid", "<u4"), ("kind", "<u4"), ("t0", "<u8"), ("t1", "<u8")])
        k = min(n.value, cap)
        rec = np.frombuffer(bytes(buf)[:k * dt.itemsize], dtype=dt).copy()
        # the library gathers its shards; a full shard drops its excess records, so fewer
        # than k may have been copied (the rest of buf stays zero: t1 is never 0 in a record)
        return rec[rec["t1"] != 0], n.value

    def launches(self):
        """[(sub, node, tiles)] of the plan's launch list (trace ids index it)."""
        out, i = [], 0
        while True:
            sub, node, tiles = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64()
            if lib().ktiler_plan_get_launch(self._h, i, ctypes.byref(sub), ctypes.byref(node), ctypes.byref(tiles)):
                break
            out.append((sub.value, node.value, tiles.value))
            i += 1
        return out

    def set_flow_roles(self, node_role, slot_role) -> None:
        """KTILER_EXEC_FLOW roles (include/ktiler.h ktiler_plan_set_flow_roles): node_role[v]
        = role of node v, slot_role[s] = role of the s-th CTA on every SM (2..5 slots);
        empty lists restore the automatic roles.  Before the first execute."""
        nr, sr = list(node_role), list(slot_role)
        _check(lib().ktiler_plan_set_flow_roles(self._h, (ctypes.c_int32 * max(1, len(nr)))(*nr), len(nr),
                                                (ctypes.c_int32 * max(1, len(sr)))(*sr), len(sr)))

    def reorder(self, order) -> None:
        """Run the sub-kernels in another dependency-respecting total order
        (include/ktiler.h ktiler_plan_reorder); order[k] = current index of the k-th."""
        o = list(order)
        _check(lib().ktiler_plan_reorder(self._h, (ctypes.c_int64 * max(1, len(o)))(*o), len(o)))

    def attach_halo(self, comm: "Comm", rank: int, halo_rows: int) -> None:
        """Run rank's strip exchange first in every execute, inside the plan's CUDA graph
        (include/ktiler.h ktiler_plan_attach_halo).  Before the first execute."""
        _check(lib().ktiler_plan_attach_halo(self._h, comm._h, rank, halo_rows))
        self._comm_keep = comm

    def execute(self, stream: int = 0) -> None:
        _check(lib().ktiler_execute(self._h, ctypes.c_void_p(stream)))

    def execute_host(self, inputs, outputs, stream: int = 0) -> None:
        """inputs/outputs: lists of (buf_id, host_ptr, frame0, frames)."""
        ci = (HostCopy * max(1, len(inputs)))(*[HostCopy(b, 0, p, f0, nf) for b, p, f0, nf in inputs])
        co = (HostCopy * max(1, len(outputs)))(*[HostCopy(b, 0, p, f0, nf) for b, p, f0, nf in outputs])
        _check(lib().ktiler_execute_host(self._h, ci, len(inputs), co, len(outputs), ctypes.c_void_p(stream)))


def comm_unique_id() -> bytes:
    """128 opaque bytes (an ncclUniqueId) for Comm.nccl, made on one rank."""
    buf = (ctypes.c_uint8 * 128)()
    _check(lib().ktiler_comm_unique_id(buf))
    return bytes(buf)


class Comm:
    """Owning wrapper of a ktiler_comm_t (strip halo exchange, include/ktiler.h)."""

    def __init__(self, h):
        self._h = h

    @classmethod
    def nccl(cls, uid: bytes, nranks: int, rank: int) -> "Comm":
        h = ctypes.c_void_p()
        buf = (ctypes.c_uint8 * 128)(*uid)
        _check(lib().ktiler_comm_init_nccl(buf, nranks, rank, ctypes.byref(h)))
        return cls(h)

    @classmethod
    def loopback(cls, nranks: int) -> "Comm":
        h = ctypes.c_void_p()
        _check(lib().ktiler_comm_init_loopback(nranks, ctypes.byref(h)))
        return cls(h)

    def register_strip(self, rank: int, base: int, pitch_bytes: int, row_bytes: int, o0: int, o1: int, e0: int,
                       e1: int) -> None:
        st = Strip(base, pitch_bytes, row_bytes, o0, o1, e0, e1)
        _check(lib().ktiler_comm_register_strip(self._h, rank, ctypes.byref(st)))

    def check(self) -> None:
        """Raise KtilerError if the NCCL communicator hit an asynchronous error."""
        _check(lib().ktiler_comm_check(self._h))

    def exchange(self, rank: int, halo_rows: int, stream: int = 0) -> None:
        _check(lib().ktiler_halo_exchange(self._h, rank, halo_rows, ctypes.c_void_p(stream)))

    def close(self):
        if self._h:
            lib().ktiler_comm_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass
