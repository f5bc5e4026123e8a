"""bench.py — Mpix/s of the tiled kernel graph on B200 (BASELINE.json metric).

Default workload: configs[3], a batch of 64 8K (7680x4320) RGB frames through the
5-kernel pipeline (gray -> blur5 -> down2 -> sobel3 -> thresh), the configuration the
north star's targets are stated on (">= 1.3x ... on 8K-class images on one B200, scaling
>= 7x on 8 GPUs for frame batches").  With --gpus N the 64 frames are split across N
ranks (one process per GPU, frame sharding, no data-path collective).

Timing (per the driver contract): W untimed warm-up steps, then K timed steps bracketed by
a barrier + cuda synchronize, CUDA events on the launching stream, max over ranks.  The
input (6.4 GB of RGB) is far larger than L2 (126 MB) — no L2 flush is needed between
steps.  A step = one ktiler_execute over the whole batch (all five kernels).

Extra keys: roofline (dominant kernel: the persistent executor = the whole step),
cpu_baseline (the oracle on host cores, bounded sample), e2e (host buffers through
ktiler_execute_host), untiled (the same graph with the KTILER_FRAG_NONE schedule),
clocks (nvidia-smi sampled during the timed region).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (W, H, frames_total, BASELINE config index)
    "batch64_8k": (7680, 4320, 64, 3),
    "pipeline_4096": (4096, 4096, 1, 1),
    "pipeline_16384": (16384, 16384, 1, 2),
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ktiler", choices=["ktiler", "reference"])
    ap.add_argument("--workload", default="batch64_8k", choices=sorted(WORKLOADS))
    ap.add_argument("--mode", default="persistent", choices=["stream", "graph", "persist_l2", "persistent"])
    ap.add_argument("--kind", default="rows", choices=["budget", "rows", "balanced", "none"])
    ap.add_argument("--rows", type=int, default=2)
    ap.add_argument("--l2-fraction", type=float, default=0.5)
    ap.add_argument("--no-discard", action="store_true")
    ap.add_argument("--pdl", action="store_true")
    ap.add_argument("--ctas", type=int, default=0)
    ap.add_argument("--skew", type=int, default=0)
    ap.add_argument("--T", type=float, default=200.0)
    ap.add_argument("--seed", type=int, default=1234)
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-untiled", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-frames", type=int, default=2)
    ap.add_argument("--sweep", action="store_true", help="extra lines: fragment-size / mode sweep (not the headline)")
    return ap.parse_args()


class Clocks:
    """nvidia-smi sampler for the timed region."""

    def __init__(self, idx: int):
        self.idx, self.samples, self.stop = idx, [], threading.Event()
        self.t = threading.Thread(target=self.run, daemon=True)

    def run(self):
        q = "clocks.sm,clocks.max.sm,clocks_event_reasons.active"
        while not self.stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", "-i", str(self.idx), f"--query-gpu={q}", "--format=csv,noheader,nounits"],
                                     capture_output=True, text=True, timeout=5).stdout.strip()
                if out:
                    a = [x.strip() for x in out.split(",")]
                    self.samples.append((float(a[0]), float(a[1]), int(a[2], 16) if a[2].startswith("0x") else 0))
            except Exception:
                pass
            self.stop.wait(0.2)

    def __enter__(self):
        self.t.start()
        return self

    def __exit__(self, *a):
        self.stop.set()
        self.t.join(timeout=10)

    def summary(self):
        names = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
                 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        load = [s for s in self.samples if not (s[2] & 0x1)] or self.samples
        reasons = sorted({n for s in load for b, n in names.items() if s[2] & b and b != 0x1})
        return {"sm_mhz": statistics.median(s[0] for s in load), "sm_max_mhz": max(s[1] for s in load),
                "reasons": reasons, "samples": len(load)}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def cpu_baseline(W, H, frames, T, seed):
    """The oracle as it stands (oracle/ktiler_oracle.c, single thread) on a bounded sample."""
    from inputs import synth
    from oracle import oracle as O
    rgb = synth.scene(seed, W, H, frames)
    t0 = time.perf_counter()
    O.pipeline(rgb, T=T)
    dt = time.perf_counter() - t0
    return {"value": W * H * frames / dt / 1e6, "unit": "Mpix/s", "cores": 1, "kind": "oracle",
            "sample": f"{frames} of the workload's {W}x{H} scene frames, untiled oracle graph, 1 thread, {dt:.1f} s"}


def run_reference(args):
    """--impl reference: the oracle timed as the reference arm (rank 0 only)."""
    W, H, Ftot, cfg = WORKLOADS[args.workload]
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from inputs import synth
    from oracle import oracle as O
    frames = 1
    rgb = synth.scene(args.seed, W, H, frames)
    for _ in range(max(0, min(args.warmup, 1))):
        O.pipeline(rgb[:, : H // 8], T=args.T)
    ts = []
    steps = max(1, min(args.steps, 3))
    for _ in range(steps):
        t0 = time.perf_counter()
        O.pipeline(rgb, T=args.T)
        ts.append(time.perf_counter() - t0)
    ms = 1000 * statistics.mean(ts)
    v = W * H * frames / (ms / 1000) / 1e6
    line = {"metric": "Mpix/s end-to-end kernel graph", "value": v, "unit": "Mpix/s", "n_gpus": args.gpus,
            "steps": steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": {"workload": args.workload, "W": W, "H": H, "frames": Ftot, "baseline_config": cfg},
            "impl": "reference",
            "cpu_baseline": {"value": v, "unit": "Mpix/s", "cores": 1, "kind": "oracle",
                             "sample": f"1 {W}x{H} frame per step (bounded sample of the {Ftot}-frame batch)"},
            "e2e": {"value": v, "unit": "Mpix/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    if args.impl == "reference":
        run_reference(args)
        return
    import torch
    import torch.distributed as dist

    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    W, H, Ftot, cfg = WORKLOADS[args.workload]
    per = Ftot // world if Ftot >= world else 1
    f0 = rank * per
    import __graft_entry__ as ge
    ge.build()

    p = Pipeline(W, H, per, T=args.T, internal=True)
    G.fill("scene", args.seed, p.view("rgb").data_ptr(), W * 3, W * 3 * H, W, H, f0=f0, F=per,
           stream=torch.cuda.current_stream().cuda_stream)
    torch.cuda.synchronize()
    discard = not args.no_discard
    pol = dict(kind=args.kind, rows=args.rows, l2_fraction=args.l2_fraction, exec_mode=args.mode, discard=discard,
               pdl=args.pdl, persistent_ctas=args.ctas, skew=args.skew)
    plan = p.plan(0, **pol)
    st = plan.stats()
    stream = torch.cuda.current_stream()
    s = stream.cuda_stream

    def barrier():
        if world > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def timed(fn, steps, warm):
        for _ in range(warm):
            fn()
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(steps):
            fn()
        e1.record(stream)
        barrier()
        ms = e0.elapsed_time(e1) / steps
        if world > 1:
            t = torch.tensor([ms], device="cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        return ms

    def step():
        plan.execute(s)

    for _ in range(args.warmup):
        step()
    barrier()
    with Clocks(local) as clk:
        ms = timed(step, args.steps, 0)
    pix = W * H * per * world
    value = pix / (ms / 1000) / 1e6
    peak, peak_src = peaks()
    comp = p.compulsory_bytes() * world
    achieved = comp / (ms / 1000) / 1e9
    line = {
        "metric": "Mpix/s end-to-end kernel graph (tiled)",
        "value": value,
        "unit": "Mpix/s",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": ms,
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": "u8",
        "data": "synthetic",
        "config": {"workload": args.workload, "baseline_config": cfg, "W": W, "H": H, "frames": Ftot,
                   "frames_per_gpu": per, "mode": args.mode, "policy": args.kind, "rows": args.rows,
                   "l2_fraction": args.l2_fraction, "discard": discard, "pdl": args.pdl,
                   "l2_flush": "none: input 6.4 GB >> 126 MB L2", "fragments": st["n_fragments"],
                   "subkernels": st["n_subkernels"], "plan_ms": round(st["plan_ms"], 1)},
        "gpu_launches": int(st["n_launches"]) * args.steps,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": None, "kernel": "persistent_kernel" if args.mode == "persistent" else "whole graph",
                     "bytes": "compulsory 3.25 B/px (rgb in + mask out)", "peak_source": peak_src},
        "clocks": clk.summary(),
    }
    if not args.no_untiled:
        un = p.b.g.plan(0, kind="none", exec_mode="graph", discard=False)
        ms_un = timed(lambda: un.execute(s), max(3, args.steps // 2), 2)
        line["untiled"] = {"value": pix / (ms_un / 1000) / 1e6, "ms_per_step": ms_un,
                           "speedup_tiled_vs_untiled": ms_un / ms,
                           "achieved_gbs_untiled_bytes": p.untiled_bytes() * world / (ms_un / 1000) / 1e9}
        del un
    if not args.no_e2e:
        rgb_h = torch.empty((per, H, W, 3), dtype=torch.uint8).pin_memory()
        rgb_h.copy_(p.view("rgb"))
        mask_h = torch.empty((per, H // 2, W // 2), dtype=torch.uint8).pin_memory()
        ins = [(p.buf_id("rgb"), rgb_h.data_ptr(), 0, 0)]
        outs = [(p.buf_id("mask"), mask_h.data_ptr(), 0, 0)]
        ms_e2e = timed(lambda: plan.execute_host(ins, outs, s), args.e2e_steps, 1)
        line["e2e"] = {"value": pix / (ms_e2e / 1000) / 1e6, "unit": "Mpix/s", "ms_per_step": ms_e2e,
                       "h2d_bytes_per_step": rgb_h.numel(), "d2h_bytes_per_step": mask_h.numel()}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(W, H if args.workload != "pipeline_16384" else 2048, args.cpu_frames if Ftot > 1 else 1,
                                            args.T, args.seed)
    if rank == 0:
        print(json.dumps(line), flush=True)
    if args.sweep and rank == 0:
        sweep(p, s, timed, pix)
    if world > 1:
        dist.destroy_process_group()


def sweep(p, s, timed, pix):
    """Fragment-size / mode sweep (BASELINE configs[2] analogue) — extra lines, not headline."""
    cfgs = [dict(kind="none", exec_mode="graph"), dict(kind="none", exec_mode="graph", discard=True)]
    for fr in (0.25, 0.5, 1.0):
        cfgs.append(dict(kind="budget", l2_fraction=fr, exec_mode="graph", discard=True))
        cfgs.append(dict(kind="budget", l2_fraction=fr, exec_mode="graph", discard=True, pdl=True))
    for rows in (1, 2, 4, 8):
        for skew in (0, 1, 4, -1):
            cfgs.append(dict(kind="rows", rows=rows, exec_mode="persistent", discard=True, skew=skew))
        cfgs.append(dict(kind="rows", rows=rows, exec_mode="persistent", discard=False))
    cfgs.append(dict(kind="none", exec_mode="persistent", discard=False))
    cfgs.append(dict(kind="budget", l2_fraction=0.5, exec_mode="persistent", discard=True))
    for c in cfgs:
        try:
            pl = p.b.g.plan(0, **c)
            ms = timed(lambda: pl.execute(s), 5, 2)
            print(json.dumps({"sweep": c, "ms": ms, "Mpix/s": pix / (ms / 1000) / 1e6,
                              "fragments": pl.stats()["n_fragments"], "launches": pl.stats()["n_launches"]}), flush=True)
            del pl
        except Exception as e:  # report and continue
            print(json.dumps({"sweep": c, "error": str(e)}), flush=True)


if __name__ == "__main__":
    main()
