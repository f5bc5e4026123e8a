"""Calibrate the 64x8K pipeline's performance tables on this B200 (ktiler_calibrate), run
Alg. 1 (KTILER_FRAG_ALG1) at several thresholds / budgets / executors, and time the
schedules it picks beside the untiled and Alg. 2-only ones.  Writes the tables to --out."""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="")
    ap.add_argument("--reps", type=int, default=9)
    args = ap.parse_args()
    import torch

    import __graft_entry__ as ge
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    ge.build()
    W, H, F = 7680, 4320, 64
    p = Pipeline(W, H, F, internal=True)
    s = torch.cuda.current_stream()
    G.fill("scene", 1234, p.view("rgb").data_ptr(), W * 3, W * 3 * H, W, H, F=F, stream=s.cuda_stream)
    torch.cuda.synchronize()
    tabs = p.calibrate(reps=5)
    print(json.dumps({"perf_tables_ms": tabs}), flush=True)
    if args.out:
        json.dump({"workload": "64 x 7680x4320", "tables": tabs}, open(args.out, "w"), indent=1)
    pix = W * H * F
    cfgs = [dict(kind="none", exec_mode="graph"), dict(kind="budget", l2_fraction=1.0, exec_mode="dag", discard=True)]
    for fr in (0.5, 1.0):
        for mode in ("graph", "dag", "persistent"):
            for rb in (False, True):
                cfgs.append(dict(kind="alg1", l2_fraction=fr, exec_mode=mode, discard=True, resident_budget=rb))
    for c in cfgs:
        try:
            pl = p.b.g.plan(0, **c)
            for _ in range(2):
                pl.execute(s.cuda_stream)
            ts = []
            for _ in range(args.reps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(s)
                pl.execute(s.cuda_stream)
                e1.record(s)
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            ms = statistics.median(ts)
            print(json.dumps({"cfg": c, "ms": round(ms, 4), "Mpix/s": round(pix / ms / 1e3, 1),
                              "clusters": [[v for v in cl] for cl, _ in pl.clusters()],
                              "est_ms": [round(x, 4) for _, x in pl.clusters()],
                              "fragments": pl.stats()["n_fragments"]}), flush=True)
            del pl
        except Exception as e:
            print(json.dumps({"cfg": c, "error": str(e)}), flush=True)


if __name__ == "__main__":
    main()
