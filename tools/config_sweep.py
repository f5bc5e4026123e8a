"""Every BASELINE config on one B200, tiled vs untiled (SURVEY §8(d) per-config runs).

  [0] 256x256 motivational graph (paper geometry and B200 geometry), cache_bytes in
      {8 KiB, 278,528 B = whole graph, device L2}: a launch-bound worked example;
  [1] 4096^2 pipeline: the whole graph (~109 MB) fits L2, so the planner returns one
      fragment = the untiled schedule ("tiled must not regress");
  [2] 16384^2 pipeline: the fragment-size sweep (ROWS and BUDGET fractions, with and
      without discard) — the B200 analogue of the paper's Fig. 3;
  [3] is bench.py's workload; [4] is the strip workload (bench.py --workload strip_65536).
Prints one JSON line per configuration (CUDA events, median of reps; L2 flushed by a 2xL2
memset before each timed execute for the configs whose input is smaller than L2)."""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def timeit(torch, s, fn, reps, flush=None):
    for _ in range(2):
        fn()
    ts = []
    for _ in range(reps):
        if flush is not None:
            flush.fill_(1)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--only", default="0,1,2")
    args = ap.parse_args()
    import torch

    import __graft_entry__ as ge
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Motivational, Pipeline
    ge.build()
    s = torch.cuda.current_stream()
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    flush = torch.empty(2 * l2, dtype=torch.uint8, device="cuda")
    only = {int(x) for x in args.only.split(",")}

    def run(tag, obj, W, H, F, cfg, flush_l2):
        cfg = dict(cfg)
        try:
            pl = obj.b.g.plan(cfg.get("cache_bytes", 0), **{k: v for k, v in cfg.items() if k != "cache_bytes"})
            ms = timeit(torch, s, lambda: pl.execute(s.cuda_stream), args.reps, flush if flush_l2 else None)
            st = pl.stats()
            print(json.dumps({"config": tag, "cfg": cfg, "ms": round(ms, 4), "Mpix/s": round(W * H * F / ms / 1e3, 1),
                              "fragments": st["n_fragments"], "launches": st["n_launches"]}), flush=True)
        except Exception as e:
            print(json.dumps({"config": tag, "cfg": cfg, "error": str(e)}), flush=True)

    if 0 in only:
        for geo in ("paper", "b200"):
            m = Motivational(256, 256, 1, geometry=geo, internal=True)
            G.fill("scene", 1234, m.b.store.tensors["in"].data_ptr(), 256 * 3, 0, 256, 256, F=1, stream=s.cuda_stream)
            for cb in (8 * 1024, 278528, 0):
                for mode in ("graph", "stream"):
                    run(f"[0] 256x256 motivational, {geo} geometry", m, 256, 256, 1,
                        dict(cache_bytes=cb, kind="budget", exec_mode=mode, discard=True), True)
            run(f"[0] 256x256 motivational, {geo} geometry", m, 256, 256, 1, dict(kind="none", exec_mode="graph"), True)
    if 1 in only:
        p = Pipeline(4096, 4096, 1, internal=True)
        G.fill("scene", 1234, p.view("rgb").data_ptr(), 4096 * 3, 0, 4096, 4096, F=1, stream=s.cuda_stream)
        for cfg in (dict(kind="none", exec_mode="graph"), dict(kind="budget", l2_fraction=1.0, exec_mode="graph", discard=True),
                    dict(kind="budget", l2_fraction=0.5, exec_mode="dag", discard=True, resident_budget=True),
                    dict(kind="budget", l2_fraction=0.25, exec_mode="dag", discard=True, resident_budget=True)):
            run("[1] 4096^2 pipeline", p, 4096, 4096, 1, cfg, True)
        del p
    if 2 in only:
        N = 16384
        p = Pipeline(N, N, 1, internal=True)
        G.fill("scene", 1234, p.view("rgb").data_ptr(), N * 3, 0, N, N, F=1, stream=s.cuda_stream)
        run("[2] 16384^2 pipeline", p, N, N, 1, dict(kind="none", exec_mode="graph"), False)
        for rows in (1, 2, 4, 8, 16, 32):
            for disc in (True, False):
                run("[2] 16384^2 pipeline, ROWS sweep", p, N, N, 1,
                    dict(kind="rows", rows=rows, exec_mode="dag", discard=disc, window=2), False)
        for fr in (0.125, 0.25, 0.5, 0.75, 1.0, 1.5, 2.0):
            for disc in (True, False):
                run("[2] 16384^2 pipeline, BUDGET sweep", p, N, N, 1,
                    dict(kind="budget", l2_fraction=fr, exec_mode="dag", discard=disc, resident_budget=True, window=2), False)
            run("[2] 16384^2 pipeline, BUDGET sweep (GRAPH)", p, N, N, 1,
                dict(kind="budget", l2_fraction=fr, exec_mode="graph", discard=True), False)


if __name__ == "__main__":
    main()
