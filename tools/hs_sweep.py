"""Horn–Schunck JI chain on one B200: untiled vs tiled across iterations
(KTILER_FRAG_CHAIN clusters of c consecutive JI nodes, each tiled by Alg. 2).  Prints one
JSON line per configuration: ms per execute (CUDA events, median), Mpix x iterations / s,
fragments, launches.  Workloads: the paper's finest HS level (1024^2, 500 JI nodes,
PAPER.md:391–399) and an 8K frame (whose fields exceed L2)."""
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
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--workloads", default="1024x1024x500,7680x4320x40")
    ap.add_argument("--configs", default="")
    ap.add_argument("--tile", default="64x16", help="JI tile (pixels) WxH")
    ap.add_argument("--pyramid", action="store_true",
                    help="Fig. 4's three steps instead (256^2, 512^2, 1024^2 x 500 JI, HSPyramid): ms per step and total")
    args = ap.parse_args()
    if args.pyramid:
        return pyramid(args)
    import numpy as np
    import torch

    import __graft_entry__ as ge
    from inputs import synth
    from paper_conf_date_maghazeh0ep19_b200.hs import HSJacobi
    ge.build()
    s = torch.cuda.current_stream()
    for wl in args.workloads.split(","):
        W, H, K = (int(v) for v in wl.split("x"))
        tw, th = (int(v) for v in args.tile.split("x"))
        h = HSJacobi(W, H, K, a2=1.0, internal=True, tile=(tw, th))
        coef, s0 = synth.hs_fields(1234, W, H, 1)
        h.set("coef", coef)
        h.set("s0", s0)
        del coef, s0
        if args.configs:
            cfgs = json.loads(args.configs)
        else:
            cfgs = [dict(kind="none", exec_mode="graph")]
            for c in (4, 8, 16):
                for fr, mode in ((0.5, "graph"), (0.5, "dag"), (1.0, "dag")):
                    cfgs.append(dict(kind="chain", rows=c, l2_fraction=fr, exec_mode=mode, discard=True, resident_budget=True))
        for cfg in cfgs:
            try:
                pl = h.plan(0, **cfg)
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
                st = pl.stats()
                print(json.dumps({"workload": wl, "tile": args.tile, "cfg": cfg, "ms": round(ms, 4), "Mpix_iter_per_s": round(W * H * K / ms / 1e3, 1),
                                  "fragments": st["n_fragments"], "launches": st["n_launches"]}), flush=True)
                del pl
            except Exception as e:
                print(json.dumps({"workload": wl, "cfg": cfg, "error": str(e)}), flush=True)
        del h
        torch.cuda.empty_cache()


def pyramid(args):
    """Fig. 4's JI part (the paper's ~25% gain is on this application,
    98.5% of whose time is in these nodes): the three steps' chains executed in order,
    untiled vs tiled, CUDA events around each step and around the whole."""
    import torch

    import __graft_entry__ as ge
    from inputs import synth
    from paper_conf_date_maghazeh0ep19_b200.hs import HSPyramid
    ge.build()
    s = torch.cuda.current_stream()
    tw, th = (int(v) for v in args.tile.split("x"))
    hp = HSPyramid(1024, 1024, 500, tile=(tw, th))
    for i, h in enumerate(hp.steps):
        hp.set_coef(i, synth.hs_fields(1234 + i, h.W, h.H, 1)[0])
    cfgs = json.loads(args.configs) if args.configs else [
        dict(kind="none", exec_mode="graph"),
        dict(kind="chain", rows=4, l2_fraction=0.5, exec_mode="dag", discard=True, resident_budget=True),
        dict(kind="chain", rows=4, l2_fraction=0.5, exec_mode="dag", discard=True, resident_budget=True, pdl=True)]
    for cfg in cfgs:
        plans = hp.plan(0, **cfg)
        for _ in range(2):
            hp.run(s.cuda_stream)
        tot, per = [], [[] for _ in plans]
        for _ in range(args.reps):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(len(plans) + 1)]
            ev[0].record(s)
            for i, p in enumerate(plans):
                p.execute(s.cuda_stream)
                ev[i + 1].record(s)
            ev[-1].synchronize()
            for i in range(len(plans)):
                per[i].append(ev[i].elapsed_time(ev[i + 1]))
            tot.append(ev[0].elapsed_time(ev[-1]))
        print(json.dumps({"workload": "fig4_steps_256_512_1024_x500", "tile": args.tile, "cfg": cfg,
                          "ms": round(statistics.median(tot), 4),
                          "ms_per_step": [round(statistics.median(x), 4) for x in per],
                          "fragments": [p.stats()["n_fragments"] for p in plans],
                          "launches": [p.stats()["n_launches"] for p in plans]}), flush=True)
        del plans


if __name__ == "__main__":
    main()
