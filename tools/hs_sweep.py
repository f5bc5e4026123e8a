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
    args = ap.parse_args()
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


if __name__ == "__main__":
    main()
