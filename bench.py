"""bench.py — Mpix/s of the KTILER-tiled kernel graph on B200 (BASELINE.json metric).

Workload (default ``batch64_8k`` = BASELINE configs[3]): 64 frames of 8K (7680x4320) RGB
through the 5-kernel pipeline gray -> blur5 -> down2 -> sobel3 -> thresh, the
configuration the north star's 1-GPU target is stated on ("8K-class images on one B200")
and the one its multi-GPU scaling target uses ("frame batches").  With --gpus N (one
process per GPU, launched by torchrun) the batch is sharded by frames — frame
sharding with no data-path collective: by default the one 64-frame batch is split into
contiguous frame ranges (64/N frames per GPU, "scaling": "strong"; frames.frame_range);
--scaling weak gives every rank a whole batch of its own instead.  Workload
``strip_65536`` (configs[4]) splits one 65536x65536 image into row strips whose 4 halo
rows per side move over NCCL send/recv (libktiler's ktiler_halo_exchange, captured into
the plan's graph ahead of the schedule) in each step.

A step = one ktiler_execute of the plan over the rank's whole share (all five kernels).
Timing: W untimed warm-up steps, then exactly K steps bracketed by a barrier + cuda
synchronize, CUDA events on the launching stream, max over ranks.  Inputs (6.4 GB of
RGB per 64-frame batch) are far larger than L2 (126 MB): no flush is needed between
steps, and every step re-reads its input from HBM.

Keys beyond the driver contract:
  untiled       the same graph under the untiled schedule (KTILER_FRAG_NONE: one launch
                per kernel over the whole batch, the paper's "normal execution mode")
  roofline      the step against HBM: compulsory bytes (3.25 B/px) / step time; traffic
                = ncu-measured DRAM bytes per step when profiles/ holds them for this
                configuration
  trace         per-kernel share of CTA time in the tiled and untiled steps, from the
                library's device-side tracer (ktiler_trace_*)
  e2e           host buffers in, host mask out: FrameStreamer (chunks of --e2e-chunk frames
                through two pipelines on two streams, each ktiler_execute_host), so the
                PCIe copies of one chunk overlap the kernels of the previous one
  cpu_baseline  the oracle (oracle/ktiler_oracle.c, one thread) on a bounded sample
  clocks        NVML SM clock + event reasons sampled during the timed region
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "Mpix/s end-to-end kernel graph, tiled vs untiled; DRAM bytes & L2 hit rate"
WORKLOADS = {
    # name: (W, H, frames, BASELINE config index, sharding)
    "batch64_8k": (7680, 4320, 64, 3, "frames"),
    "pipeline_4096": (4096, 4096, 1, 1, "replicas"),
    "pipeline_16384": (16384, 16384, 1, 2, "strips"),
    "strip_65536": (65536, 65536, 1, 4, "strips"),
}


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ktiler", choices=["ktiler", "reference"])
    ap.add_argument("--workload", default="batch64_8k", choices=sorted(WORKLOADS))
    ap.add_argument("--mode", default="dag", choices=["stream", "graph", "persist_l2", "persistent", "dag", "chain", "wave", "flow"])
    ap.add_argument("--kind", default="budget", choices=["budget", "rows", "balanced", "none"])
    ap.add_argument("--rows", type=int, default=2)
    ap.add_argument("--l2-fraction", type=float, default=1.0)
    ap.add_argument("--no-resident", action="store_true",
                    help="paper-literal budget (count graph input/output lines too; SURVEY A11)")
    ap.add_argument("--scaling", default="strong", choices=["weak", "strong"],
                    help="frames: strong (default) = the one batch split into contiguous frame ranges "
                         "(BASELINE configs[3]); weak = every rank runs a whole batch of its own")
    ap.add_argument("--window", type=int, default=2)
    ap.add_argument("--ring-frames", type=int, default=0,
                    help="intermediates as WAR-aware rings of this many frames (SURVEY f4; 0 = full batch)")
    ap.add_argument("--discard", action="store_true",
                    help="discard dead intermediate lines (DRAM -55%% but slower on B200: DESIGN.md §6)")
    ap.add_argument("--no-discard", action="store_true", help="(default) keep dead lines")
    ap.add_argument("--halo-discard", action="store_true",
                    help="also drop gray / down lines via per-block reader counts (DRAM -62%%, ~15%% slower: A44)")
    ap.add_argument("--no-consumer-discard", action="store_true",
                    help="keep the lines down2 / thresh consume (default: drop them once staged, DESIGN A44)")
    ap.add_argument("--pdl", action="store_true", default=True,
                    help="(default) programmatic-dependent-launch edges from each sub-kernel's producers (DESIGN §6.10)")
    ap.add_argument("--no-pdl", dest="pdl", action="store_false")
    ap.add_argument("--ctas", type=int, default=0)
    ap.add_argument("--skew", type=int, default=0)
    ap.add_argument("--T", type=float, default=200.0)
    ap.add_argument("--seed", type=int, default=1234)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-chunk", type=int, default=8,
                    help="frames per chunk of the double-buffered host-to-host path (0: one ktiler_execute_host)")
    ap.add_argument("--no-untiled", action="store_true")
    ap.add_argument("--no-trace", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-ncu", action="store_true", help="skip the in-run ncu DRAM / L2-hit capture")
    ap.add_argument("--cpu-seconds", type=float, default=12.0, help="target CPU time of the oracle sample")
    return ap.parse_args(argv)


class Clocks:
    """NVML sampler (SM clock, clock-event reasons) running during the timed region."""

    NAMES = {"SwPowerCap": "sw_power_cap", "HwSlowdown": "hw_slowdown", "SwThermalSlowdown": "sw_thermal_slowdown",
             "HwThermalSlowdown": "hw_thermal_slowdown", "HwPowerBrakeSlowdown": "hw_power_brake_slowdown",
             "ApplicationsClocksSetting": "applications_clocks_setting"}

    def __init__(self, idx: int):
        self.samples, self.stop = [], threading.Event()
        try:
            import pynvml as N
            N.nvmlInit()
            self.N, self.h = N, N.nvmlDeviceGetHandleByIndex(idx)
            self.max = N.nvmlDeviceGetMaxClockInfo(self.h, N.NVML_CLOCK_SM)
        except Exception:
            self.N = None
        self.t = threading.Thread(target=self.run, daemon=True)

    def run(self):
        N = self.N
        while N is not None and not self.stop.is_set():
            try:
                self.samples.append((N.nvmlDeviceGetClockInfo(self.h, N.NVML_CLOCK_SM),
                                     N.nvmlDeviceGetCurrentClocksEventReasons(self.h)))
            except Exception:
                pass
            self.stop.wait(0.002)

    def __enter__(self):
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=5)

    def summary(self):
        if self.N is None or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        N = self.N
        reasons = set()
        for _, r in self.samples:
            for k, name in self.NAMES.items():
                if r & getattr(N, "nvmlClocksEventReason" + k, 0):
                    reasons.add(name)
        return {"sm_mhz": statistics.median(s[0] for s in self.samples), "sm_max_mhz": self.max,
                "reasons": sorted(reasons), "samples": len(self.samples)}


def peaks():
    try:
        d = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
        return float(d["hbm_gbs"]), "measured: MEASURED_PEAKS.json hbm_gbs (torch copy, read+write)"
    except Exception:
        return 6650.0, "fallback: B200_PROFILING.md"


def l2_ceiling():
    """Measured L2 read / write-to-resident throughput (tools/l2bw.cu, 64 MiB resident
    buffer) from profiles/, or None."""
    try:
        rows = [json.loads(l) for l in open(os.path.join(ROOT, "profiles", "r02_l2bw.jsonl"))]
        r = {d["mode"]: d["GBps"] for d in rows if d["mb"] == 64}
        return {"read": r["read"], "write": r["write"], "source": "profiles/r02_l2bw.jsonl (tools/l2bw, 64 MiB resident)"}
    except Exception:
        return None


def traffic_for(cfg: dict):
    """ncu DRAM bytes per step for this exact configuration, if profiles/ has them."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
    except Exception:
        return None, None
    for e in d.get("entries", []):
        if all(e["config"].get(k, False if k == "pdl" else None) == v for k, v in cfg.items()):
            return e["dram_bytes_per_step"], e["source"]
    return None, None


def _oracle_frame(job):
    """One worker of the all-cores oracle: frame f of the workload through O-6."""
    W, rows, T, seed, f = job
    from inputs import synth
    from oracle import oracle as O
    t0 = time.perf_counter()
    O.pipeline(synth.scene(seed + f, W, rows, 1), T=T)
    return time.perf_counter() - t0


def cpu_baseline(W, H, T, seed, target_s):
    """The oracle as it stands (single-threaded C, O-6) on a bounded sample: whole frames
    of the workload, as many as fit ~target_s seconds (at least one; a row band for
    images larger than one 8K frame), on ONE core (the process pinned to CPU 0 for the
    duration); then the all-cores figure: nproc processes x one frame each,
    wall time of the whole set (BASELINE configs[3] "the oracle timed on the box's own host
    cores")."""
    from inputs import synth
    from oracle import oracle as O
    rows = H if W * H <= 7680 * 4320 else max(64, (7680 * 4320 // W) // 16 * 16)
    rgb = synth.scene(seed, W, rows, 1)
    old_aff = None
    try:
        old_aff = os.sched_getaffinity(0)
        os.sched_setaffinity(0, {min(old_aff)})
    except (AttributeError, OSError):
        pass
    try:
        t0 = time.perf_counter()
        O.pipeline(rgb, T=T)
        one = time.perf_counter() - t0
        n, dt = 1, one
        while dt + one <= target_s:
            t1 = time.perf_counter()
            O.pipeline(rgb, T=T)
            dt += time.perf_counter() - t1
            n += 1
    finally:
        if old_aff:
            os.sched_setaffinity(0, old_aff)
    out = {"value": W * rows * n / dt / 1e6, "unit": "Mpix/s", "cores": 1, "kind": "oracle",
           "sample": f"{n} x {W}x{rows} scene image(s) through the untiled oracle graph, 1 thread pinned to "
                     f"CPU {min(old_aff) if old_aff else '?'}, {dt:.1f} s",
           "host": host_cpu()}
    ncores = len(old_aff) if old_aff else (os.cpu_count() or 1)
    if ncores > 1:
        import concurrent.futures as cf
        import multiprocessing as mp
        jobs = [(W, rows, T, seed, f) for f in range(ncores)]
        t0 = time.perf_counter()
        with cf.ProcessPoolExecutor(ncores, mp_context=mp.get_context("spawn")) as ex:
            list(ex.map(_oracle_frame, jobs))
        wall = time.perf_counter() - t0
        out["all_cores"] = {"value": W * rows * ncores / wall / 1e6, "unit": "Mpix/s", "cores": ncores,
                            "sample": f"{ncores} processes x one {W}x{rows} frame each (frames seed+0..{ncores - 1}), "
                                      f"wall {wall:.1f} s including process start"}
    return out


def host_cpu() -> dict:
    """The oracle's host: CPU model name (/proc/cpuinfo) and the cores the OS exposes."""
    name = "unknown"
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                name = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return {"model": name, "nproc": os.cpu_count()}


def run_reference(args):
    """--impl reference: the oracle, as it stands, is the reference arm (rank 0 only).

    Frame batches (configs[3]): each step is the WHOLE batch, frame f on host core
    f mod ncores (one process per core, each frame through the oracle's untiled graph), so
    the line has the same workload as the GPU arm.  The run stops after ~150 s of steps
    (the line reports the steps actually run).  Other workloads: one row band / frame per
    step, one thread (a bounded sample, stated in `sample`)."""
    W, H, Ftot, cfg, shard = WORKLOADS[args.workload]
    if int(os.environ.get("RANK", "0")) != 0:
        return
    from inputs import synth
    from oracle import oracle as O
    budget_s = 150.0
    ts = []
    if shard == "frames":
        import concurrent.futures as cf
        import multiprocessing as mp
        try:
            ncores = len(os.sched_getaffinity(0))
        except (AttributeError, OSError):
            ncores = os.cpu_count() or 1
        jobs = [(W, H, args.T, args.seed, f) for f in range(Ftot)]
        with cf.ProcessPoolExecutor(ncores, mp_context=mp.get_context("spawn")) as ex:
            list(ex.map(_oracle_frame, [(W, 16, args.T, args.seed, f) for f in range(ncores)]))  # warm-up: workers up
            for k in range(max(1, args.steps)):
                t0 = time.perf_counter()
                list(ex.map(_oracle_frame, jobs))
                ts.append(time.perf_counter() - t0)
                if sum(ts) + statistics.mean(ts) > budget_s:
                    break
        pix, cores = W * H * Ftot, ncores
        sample = (f"the whole {Ftot}-frame batch per step ({W}x{H} frames scene(seed+f)), frame f on one of {ncores} "
                  f"host cores (one process per core, untiled oracle graph each)")
        scaling = "strong"
    else:
        rows = H if W * H <= 7680 * 4320 else max(64, (7680 * 4320 // W) // 16 * 16)
        rgb = synth.scene(args.seed, W, rows, 1)
        for _ in range(min(args.warmup, 1)):
            O.pipeline(rgb[:, : max(16, rows // 8)], T=args.T)
        for k in range(max(1, args.steps)):
            t0 = time.perf_counter()
            O.pipeline(rgb, T=args.T)
            ts.append(time.perf_counter() - t0)
            if sum(ts) + statistics.mean(ts) > budget_s:
                break
        pix, cores = W * rows, 1
        sample = f"1 {W}x{rows} image per step (bounded sample of the {args.workload} workload), 1 thread"
        scaling = "weak"
    steps = len(ts)
    ms = 1000 * statistics.mean(ts)
    v = pix / (ms / 1000) / 1e6
    print(json.dumps({
        "metric": METRIC, "value": v, "unit": "Mpix/s", "n_gpus": args.gpus, "steps": steps, "warmup": args.warmup,
        "ms_per_step": ms, "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u8",
        "data": "synthetic", "config": {"workload": args.workload, "W": W, "H": H, "frames": Ftot, "baseline_config": cfg},
        "impl": "reference",
        "cpu_baseline": {"value": v, "unit": "Mpix/s", "cores": cores, "kind": "oracle", "sample": sample,
                         "host": host_cpu()},
        "e2e": {"value": v, "unit": "Mpix/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}), flush=True)


# algorithmic bytes per OUTPUT pixel of each kernel (input bytes it must read + output bytes)
NODE_BYTES = {"gray": 3 + 1, "blur": 1 + 1, "down": 4 + 1, "sobel": 1 + 4, "thresh": 4 + 1}


def trace_shares(pipe, pol):
    """Per-kernel share of CTA time in one traced execute of a fresh plan of ``pol``, and
    per kernel the mean device span of its launches (first CTA start -> last CTA end) with
    the algorithmic bytes those launches move."""
    import numpy as np
    pl = pipe.b.g.plan(0, **pol)
    pl.trace_enable(1 << 22)
    pl.execute(0)
    pl.trace_read()
    pl.execute(0)
    rec, _ = pl.trace_read()
    names = ("gray", "blur", "down", "sobel", "thresh")
    launches = pl.launches()
    k0 = rec[rec["kind"] == 0]
    node = np.array([launches[i][1] for i in k0["id"]])
    dur = (k0["t1"].astype(np.int64) - k0["t0"].astype(np.int64)).astype(np.float64)
    tot = dur.sum()
    out = {names[v] if v >= 0 else "discard": round(float(dur[node == v].sum() / tot), 3) for v in sorted(set(node.tolist()))}
    span = int(k0["t1"].max() - k0["t0"].min())
    per = {}
    ids = k0["id"].astype(np.int64)
    for lid in np.unique(ids):
        v = launches[int(lid)][1]
        if v < 0:
            continue
        m = ids == lid
        sp = float(k0["t1"][m].max() - k0["t0"][m].min())
        tw, th = pipe.geometry[names[v]][:2]
        d = per.setdefault(names[v], {"launches": 0, "span_ns": 0.0, "bytes": 0.0})
        d["launches"] += 1
        d["span_ns"] += sp
        d["bytes"] += launches[int(lid)][2] * tw * th * NODE_BYTES[names[v]]
    del pl
    return out, span / 1e6, per


def ktiler_env() -> dict:
    """Every KTILER_* variable of the environment (experiment knobs the library reads):
    echoed into the line so a stray knob can never silently change the measured config."""
    return {k: v for k, v in sorted(os.environ.items()) if k.startswith("KTILER_")}


def ncu_traffic(args, pols, timeout_s=420, ring=0):
    """DRAM bytes and L2 sector hit rate of one execute of each policy in `pols`, measured
    in THIS run by ncu (graph-level ranges, caches flushed before each, 3rd execute of
    tools/sweep.py's 2 warm-ups + 1), on the workload's own shape.  None if ncu is absent
    or fails (then profiles/traffic.json, if it matches, is reported instead)."""
    import shutil
    import subprocess
    import tempfile
    ncu = shutil.which("ncu") or ("/usr/local/cuda/bin/ncu" if os.path.exists("/usr/local/cuda/bin/ncu") else None)
    if not ncu:
        return None
    W, H, Ftot, _, _ = WORKLOADS[args.workload]
    with tempfile.TemporaryDirectory() as d:
        csv_path = os.path.join(d, "t.csv")
        cmd = [ncu, "--graph-profiling", "graph", "--cache-control", "all", "--clock-control", "none", "--metrics",
               "dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum", "--csv",
               "--log-file", csv_path, sys.executable, os.path.join(ROOT, "tools", "sweep.py"), "--W", str(W), "--H",
               str(H), "--F", str(Ftot), "--reps", "1", "--ring", str(ring), "--configs", json.dumps(pols)]
        try:
            r = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout_s, cwd=ROOT)
            if r.returncode:
                return None
            rows = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "traffic_summary.py"), csv_path],
                                  capture_output=True, text=True, check=True).stdout.splitlines()
        except Exception:
            return None
    rows = [json.loads(x) for x in rows]
    per = len(rows) // max(1, len(pols))
    if per < 3:
        return None
    out = []
    for i in range(len(pols)):
        g = rows[i * per:(i + 1) * per]
        r3 = g[2]  # the 3rd execute (2 warm-ups)
        if per > 3:  # non-graph executors (several ranges per execute): sum the last execute's ranges
            k = (per) // 3
            last = g[2 * k:3 * k]
            r3 = {"read_GB": sum(x["read_GB"] for x in last), "write_GB": sum(x["write_GB"] for x in last),
                  "dram_GB": sum(x["dram_GB"] for x in last), "l2_hit_pct": None,
                  "ms": sum(x["ms"] for x in last)}
        out.append({"dram_bytes": r3["dram_GB"] * 1e9, "dram_read": r3["read_GB"] * 1e9,
                    "dram_write": r3["write_GB"] * 1e9, "lts_sector_hit_rate_pct": r3["l2_hit_pct"],
                    "ncu_duration_ms": r3["ms"],
                    "source": "ncu in this bench run (--graph-profiling graph --cache-control all --clock-control none, "
                              "tools/sweep.py 3rd execute; serialised under the profiler: bytes, not time)"})
    return out


def policy(args) -> dict:
    """The fragment policy of the timed step (also used by tests/test_gpu_fullsize.py)."""
    return dict(kind=args.kind, rows=args.rows, l2_fraction=args.l2_fraction, exec_mode=args.mode,
                discard=args.discard and not args.no_discard, pdl=args.pdl, persistent_ctas=args.ctas, skew=args.skew,
                window=args.window, resident_budget=not args.no_resident, consumer_discard=not args.no_consumer_discard,
                halo_discard=args.halo_discard)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    from paper_conf_date_maghazeh0ep19_b200 import frames as FR
    from paper_conf_date_maghazeh0ep19_b200.strips import StripPipeline

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # KTILER_BENCH_BACKEND=gloo (test only, echoed in config.env): ranks may share a GPU, so
    # the multi-rank path (barriers, max over ranks, rank-0 line) runs on a 1-GPU box
    backend = os.environ.get("KTILER_BENCH_BACKEND", "nccl")
    if backend == "gloo":
        local %= max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    coll_dev = "cuda" if backend == "nccl" else "cpu"
    W, H, Ftot, cfg_idx, shard = WORKLOADS[args.workload]
    import __graft_entry__ as ge
    ge.build()
    stream = torch.cuda.current_stream()
    s = stream.cuda_stream

    sp = None
    if shard == "strips":
        sp = StripPipeline(W, H, world, rank, T=args.T, internal=True)
        p = sp.pipe
        # each rank generates only the rows it owns; the halo rows come from the neighbours
        G.fill("scene", args.seed, sp.rgb_ext()[sp.own_offset:].data_ptr(), W * 3, 0, W, H, y0=sp.o0,
               rows=sp.o1 - sp.o0, F=1, stream=s)
        pix_rank = W * (sp.o1 - sp.o0)
        pix_ranks = [pix_rank] * world
        per = 1
    else:
        strong = shard == "frames" and args.scaling == "strong"
        if strong:  # contiguous frame ranges, the first Ftot % world ranks one frame more
            f0, per = FR.frame_range(Ftot, world, rank)
            pix_ranks = [W * H * FR.frame_range(Ftot, world, r)[1] for r in range(world)]
        else:  # weak: every rank its own whole batch (frames Ftot*rank ...)
            f0, per = (rank * Ftot if shard == "frames" else 0), Ftot
            pix_ranks = [W * H * Ftot] * world
        p = Pipeline(W, H, per, T=args.T, internal=True, ring_frames=args.ring_frames)
        G.fill("scene", args.seed, p.view("rgb").data_ptr(), W * 3, W * 3 * H, W, H, f0=f0, F=per, stream=s)
        pix_rank = W * H * per
    torch.cuda.synchronize()
    pol = policy(args)
    discard, resident = pol["discard"], pol["resident_budget"]
    plan = p.plan(0, **pol)
    st = plan.stats()

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    step_ms = []  # per-step event times of the last timed() with per_step=True (this rank)

    def timed(fn, steps, warm, clocks=None, per_step=False):
        for _ in range(warm):
            fn()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        marks = [torch.cuda.Event(enable_timing=True) for _ in range(steps)] if per_step else []
        if clocks:
            clocks.__enter__()
        e0.record(stream)
        for k in range(steps):
            fn()
            if per_step:
                marks[k].record(stream)
        e1.record(stream)
        barrier()
        if clocks:
            clocks.__exit__()
        ms = e0.elapsed_time(e1) / steps
        if per_step:
            step_ms[:] = [(e0 if k == 0 else marks[k - 1]).elapsed_time(marks[k]) for k in range(steps)]
        return FR.max_over_ranks(ms, world, device=coll_dev)

    comm = None
    if sp is not None and world > 1:
        # the strip halo exchange runs inside libktiler (ncclSend/ncclRecv in one group),
        # captured into the plan's graph ahead of the schedule: one execute per step
        from paper_conf_date_maghazeh0ep19_b200 import strips as SM
        comm = SM.nccl_comm(world, rank)
        sp.register(comm)
        plan.attach_halo(comm, rank, SM.HALO_ROWS)

    def step():
        plan.execute(s)

    clk = Clocks(local)
    ms = timed(step, args.steps, args.warmup, clocks=clk, per_step=True)
    pix = sum(pix_ranks)
    value = FR.job_mpix_per_s(pix_ranks, ms)
    peak, peak_src = peaks()
    comp_bytes = pix * 3.25  # rgb in + mask out: the method's algorithmic bytes
    achieved = comp_bytes / world / (ms / 1000) / 1e9  # per GPU, against one GPU's peak
    tcfg = {"workload": args.workload, "mode": args.mode, "policy": args.kind, "l2_fraction": args.l2_fraction,
            "discard": discard, "window": args.window, "resident_budget": resident,
            "consumer_discard": pol["consumer_discard"], "halo_discard": pol["halo_discard"], "pdl": bool(args.pdl)}
    traffic, traffic_src = traffic_for(tcfg)
    line = {
        "metric": METRIC,
        "value": value,
        "unit": "Mpix/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": ms,
        "step_ms": {q: round(statistics.quantiles(step_ms, n=10)[i] if len(step_ms) >= 2 else ms, 4)
                    for q, i in (("p10", 0), ("p50", 4), ("p90", 8))},
        "higher_is_better": True,
        "scaling": "strong" if (shard == "strips" or (shard == "frames" and args.scaling == "strong")) else "weak",
        "vs_baseline": None,
        "dtype": "u8",
        "data": "synthetic",
        "config": {"workload": args.workload, "baseline_config": cfg_idx, "W": W, "H": H, "frames": Ftot,
                   "frames_per_gpu": per if sp is None else None,
                   "sharding": shard if world > 1 else "none", "pixels_per_gpu": pix_rank, "mode": args.mode,
                   "policy": args.kind, "rows": args.rows, "l2_fraction": args.l2_fraction, "window": args.window,
                   "resident_budget": resident, "discard": discard, "consumer_discard": pol["consumer_discard"],
                   "halo_discard": pol["halo_discard"], "ring_frames": args.ring_frames,
                   "pdl": args.pdl,
                   "l2_flush": "not needed: each step reads >= 6.4 GB of input (>> 126 MB L2)" if Ftot > 1 or W >= 16384
                   else "none (input smaller than L2: steady-state replay)",
                   "fragments": st["n_fragments"], "subkernels": st["n_subkernels"],
                   "plan_ms": round(st["plan_ms"], 1), "input": f"scene(seed={args.seed}) per frame",
                   "env": ktiler_env()},
        "gpu_launches": int(st["n_launches"]) * args.steps,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": traffic, "traffic_source": traffic_src,
                     "kernel": f"one ktiler_execute ({args.mode}: {st['n_launches']} sub-kernel launches)",
                     "algorithmic_bytes": "3.25 B/px compulsory (rgb 3 in + mask 0.25 out) x pixels per step",
                     "peak_source": peak_src},
        "clocks": clk.summary(),
    }
    l2 = l2_ceiling()
    if l2:
        # secondary ceiling: every byte the kernels read or write passes the L2 slices;
        # writes into L2 are capped near the HBM write rate on B200 (dirty lines are written
        # back within microseconds), reads of resident lines at ~2.6x HBM
        rd, wr = 6.25 * pix, 3.5 * pix
        floor_ms = (rd / (l2["read"] * 1e9) + wr / (l2["write"] * 1e9)) * 1e3
        line["roofline"]["l2"] = {"bound": "l2", "read_peak": l2["read"], "write_peak": l2["write"], "unit": "GB/s",
                                  "algorithmic_bytes": "6.25 B/px read + 3.5 B/px written (all five kernels)",
                                  "floor_ms": floor_ms, "frac": floor_ms / ms, "source": l2["source"]}
    pu = p  # the untiled baseline's pipeline (full-batch intermediates when the tiled one uses rings)
    if args.ring_frames and sp is None:
        pu = Pipeline(W, H, per, T=args.T, internal=True)
        pu.view("rgb").copy_(p.view("rgb"))
    if not args.no_untiled:
        un = pu.b.g.plan(0, kind="none", exec_mode="graph", discard=False)
        if comm is not None:
            un.attach_halo(comm, rank, SM.HALO_ROWS)
        ms_un = timed(lambda: un.execute(s), max(3, args.steps // 2), 2)
        unp = pu.b.g.plan(0, kind="none", exec_mode="graph", discard=False, pdl=True)
        if comm is not None:
            unp.attach_halo(comm, rank, SM.HALO_ROWS)
        ms_unp = timed(lambda: unp.execute(s), max(3, args.steps // 2), 2)
        del unp
        line["untiled"] = {"value": pix / (ms_un / 1000) / 1e6, "ms_per_step": ms_un,
                           "pdl_ms_per_step": ms_unp, "tiled_speedup_vs_pdl": ms_unp / ms,
                           "tiled_speedup": ms_un / ms,
                           "achieved_gbs": 9.75 * pix / (ms_un / 1000) / 1e9,
                           "roofline_frac": 9.75 * pix / (ms_un / 1000) / 1e9 / peak,
                           "algorithmic_bytes": "9.75 B/px (every intermediate written and read once)"}
        del un
    if not args.no_untiled and sp is None and not args.ring_frames and args.mode != "flow":
        # the persistent executor driven by per-tile dependency flags (north star's variant,
        # KTILER_EXEC_FLOW, its measured-best defaults) on the same batch, for comparison
        try:
            from paper_conf_date_maghazeh0ep19_b200.pipeline import FLOW_GEOMETRY
            pf = Pipeline(W, H, per, T=args.T, internal=True, geometry=FLOW_GEOMETRY)  # FLOW's best tiles
            pf.view("rgb").copy_(p.view("rgb"))
            fl = pf.plan(0, kind="rows", rows=1, exec_mode="flow", consumer_discard=True)
            ms_fl = timed(lambda: fl.execute(s), max(3, args.steps // 4), 2)
            line["flow"] = {"value": pix / (ms_fl / 1000) / 1e6, "ms_per_step": ms_fl,
                            "vs_untiled": line["untiled"]["ms_per_step"] / ms_fl,
                            "policy": "rows=1 fragments, 3 CTAs/SM one role, skew 32, consumer discard; "
                                      "pipeline.FLOW_GEOMETRY (thresh 256x32)"}
            del fl, pf
        except Exception as e:  # diagnostics only
            line["flow"] = {"error": str(e)}
    if not args.no_trace and rank == 0:
        try:
            tiled_sh, tiled_span, per_node = trace_shares(p, pol) if args.mode != "persistent" else (None, None, None)
            un_sh, un_span, _ = trace_shares(pu, dict(kind="none", exec_mode="graph"))
            line["trace"] = {"tiled_cta_share": tiled_sh, "tiled_span_ms": tiled_span, "untiled_cta_share": un_sh,
                             "untiled_span_ms": un_span}
            if per_node:
                # the dominant kernel of the tiled step (largest CTA-time share): its
                # algorithmic bytes per launch / its mean launch span (device-side tracer)
                dom = max(tiled_sh, key=lambda k: tiled_sh[k] if k in per_node else -1)
                d = per_node[dom]
                ach = d["bytes"] / d["launches"] / (d["span_ns"] / d["launches"])  # B/ns = GB/s
                dtraffic = None
                try:
                    dt = json.load(open(os.path.join(ROOT, "profiles", "r02j_dominant_traffic.json")))
                    if dom in dt["kernels"] and all(line["config"].get(k) == v for k, v in dt["config"].items()):
                        kd = dt["kernels"][dom]
                        dtraffic = {"bytes": kd["dram_bytes_per_launch_mean"], "source": kd["source"]}
                except Exception:
                    pass
                # the bytes of it that must come from HBM in the tiled step: its graph input
                # (gray: 3 B of rgb per pixel; its 1 B output stays in L2 for blur)
                hbm_b = {"gray": 3}.get(dom)
                line["roofline"]["dominant_kernel"] = {
                    "kernel": dom, "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s", "frac": ach / peak,
                    "hbm_bytes_frac": (ach * hbm_b / NODE_BYTES[dom] / peak) if hbm_b else None,
                    "hbm_bytes_note": "frac on the bytes that must come from HBM (gray: its 3 B/px rgb read; "
                                      "the 1 B/px gray store lands in L2)",
                    "launches_per_step": d["launches"], "mean_launch_us": d["span_ns"] / d["launches"] / 1e3,
                    "traffic": dtraffic["bytes"] if dtraffic else None,
                    "traffic_source": dtraffic["source"] if dtraffic else None,
                    "algorithmic_bytes": f"{NODE_BYTES[dom]} B per output pixel x output pixels per launch",
                    "timing": "device-side tracer (%globaltimer, first CTA start -> last CTA end per launch); "
                              "launches of the DAG overlap, so this is a per-launch rate, not a share of the step"}
        except Exception as e:  # diagnostics only
            line["trace"] = {"error": str(e)}
    if not args.no_e2e:
        e2e_path = None
        if sp is None:
            rgb_h = torch.empty((per, H, W, 3), dtype=torch.uint8).pin_memory()
            rgb_h.copy_(p.view("rgb"))
            mask_h = torch.empty((per, H // 2, W // 2), dtype=torch.uint8).pin_memory()
            chunk = args.e2e_chunk if args.e2e_chunk > 0 and per % args.e2e_chunk == 0 and per > args.e2e_chunk else 0
            if chunk:
                from paper_conf_date_maghazeh0ep19_b200.streaming import FrameStreamer
                fs = FrameStreamer(W, H, chunk, T=args.T, **pol)
                ms_e2e = timed(lambda: fs.run(rgb_h, mask_h, stream), args.e2e_steps, 1)
                fs.wait()
                ref = torch.empty_like(mask_h).pin_memory()
                ref.copy_(p.view("mask"))
                if not torch.equal(ref, mask_h):
                    raise RuntimeError("e2e: the streamed batch's mask differs from the device run")
                e2e_path = (f"FrameStreamer: {per // chunk} chunks of {chunk} frames through 2 pipelines on 2 streams, "
                            "each ktiler_execute_host (pinned host rgb -> device -> plan -> host mask)")
                del fs
            else:
                ins = [(p.buf_id("rgb"), rgb_h.data_ptr(), 0, 0)]
                outs = [(p.buf_id("mask"), mask_h.data_ptr(), 0, 0)]
                ms_e2e = timed(lambda: plan.execute_host(ins, outs, s), args.e2e_steps, 1)
            h2d, d2h = rgb_h.numel(), mask_h.numel()
        else:
            own = sp.rgb_ext()[sp.own_offset:sp.own_offset + (sp.o1 - sp.o0)]
            rgb_h = own.cpu().pin_memory()
            mask_h = torch.empty(tuple(sp.mask_owned().shape), dtype=torch.uint8).pin_memory()

            def e2e_step():
                own.copy_(rgb_h, non_blocking=True)
                step()
                mask_h.copy_(sp.mask_owned(), non_blocking=True)
            ms_e2e = timed(e2e_step, args.e2e_steps, 1)
            h2d, d2h = rgb_h.numel(), mask_h.numel()
        line["e2e"] = {"value": pix / (ms_e2e / 1000) / 1e6, "unit": "Mpix/s", "ms_per_step": ms_e2e,
                       "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                       "path": (e2e_path or "ktiler_execute_host (pinned host rgb -> device -> plan -> host mask)")
                       if sp is None else "pinned host rows -> device, halo exchange, ktiler_execute, mask -> host"}
    if rank == 0 and world == 1 and not args.no_ncu:  # (a one-rank strip is the whole image)
        # DRAM bytes and L2 hit rate of the tiled step and of the untiled one, measured by
        # ncu on this run's exact configuration (the metric's "DRAM bytes & L2 hit rate")
        if args.ring_frames:  # the untiled schedule needs full-batch intermediates
            mt = ncu_traffic(args, [pol], ring=args.ring_frames)
            mu = ncu_traffic(args, [dict(kind="none", exec_mode="graph")])
            meas = mt + mu if mt and mu else None
        else:
            meas = ncu_traffic(args, [pol, dict(kind="none", exec_mode="graph")])
        if meas:
            t, u = meas
            line["roofline"]["traffic"] = t["dram_bytes"]
            line["roofline"]["traffic_source"] = t["source"]
            line["dram"] = {"tiled_bytes": t["dram_bytes"], "tiled_read": t["dram_read"], "tiled_write": t["dram_write"],
                            "untiled_bytes": u["dram_bytes"], "untiled_read": u["dram_read"],
                            "untiled_write": u["dram_write"], "reduction": 1.0 - t["dram_bytes"] / u["dram_bytes"],
                            "compulsory_bytes": comp_bytes, "source": t["source"]}
            line["l2_hit_rate"] = {"tiled_pct": t["lts_sector_hit_rate_pct"], "untiled_pct": u["lts_sector_hit_rate_pct"],
                                   "metric": "lts__t_sector_hit_rate.pct", "source": t["source"]}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(W, H, args.T, args.seed, args.cpu_seconds)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
