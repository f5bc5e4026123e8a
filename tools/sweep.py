"""Plan/exec-mode sweep on one pipeline instance (BASELINE configs[2]/[3] fragment-size
sweep).  Prints one JSON line per configuration: ms per execute (CUDA events, median of
reps), Mpix/s, fragments, launches.  Not the headline bench (bench.py is)."""
from __future__ import annotations

import argparse
import itertools
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--W", type=int, default=7680)
    ap.add_argument("--H", type=int, default=4320)
    ap.add_argument("--F", type=int, default=64)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--configs", default="default", help="default | json list of plan kwargs")
    ap.add_argument("--geom", default="", help='json {op: [tile_w, tile_h, threads]} overriding B200_GEOMETRY')
    ap.add_argument("--check", action="store_true", help="compare every config's mask with the untiled graph's")
    ap.add_argument("--ring", type=int, default=0, help="intermediates as rings of this many frames (f4)")
    args = ap.parse_args()
    import torch

    import __graft_entry__ as ge
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    ge.build()
    geom = None
    if args.geom:
        from paper_conf_date_maghazeh0ep19_b200.pipeline import B200_GEOMETRY
        geom = dict(B200_GEOMETRY)
        geom.update({k: tuple(v) for k, v in json.loads(args.geom).items()})
    p = Pipeline(args.W, args.H, args.F, internal=True, geometry=geom, ring_frames=args.ring)
    s = torch.cuda.current_stream()
    G.fill("scene", 1234, p.view("rgb").data_ptr(), args.W * 3, args.W * 3 * args.H, args.W, args.H, F=args.F,
           stream=s.cuda_stream)
    torch.cuda.synchronize()
    if args.configs == "default":
        cfgs = [dict(kind="none", exec_mode="graph")]
        for rows, skew in itertools.product((1, 2, 4, 8), (0, 2, 6)):
            cfgs.append(dict(kind="rows", rows=rows, exec_mode="persistent", discard=True, skew=skew))
        cfgs.append(dict(kind="none", exec_mode="persistent"))
        cfgs.append(dict(kind="budget", l2_fraction=0.5, exec_mode="persistent", discard=True))
        cfgs.append(dict(kind="budget", l2_fraction=1.0, exec_mode="graph", discard=True))
    else:
        cfgs = json.loads(args.configs)
    pix = args.W * args.H * args.F
    ref = None
    if args.check:
        ref_pipe = Pipeline(args.W, args.H, args.F, internal=True, geometry=geom) if args.ring else p
        if args.ring:
            ref_pipe.view("rgb").copy_(p.view("rgb"))
        pl = ref_pipe.b.g.plan(0, kind="none", exec_mode="graph")
        pl.execute(s.cuda_stream)
        torch.cuda.synchronize()
        ref = ref_pipe.view("mask").clone()
        del pl, ref_pipe
    for c in cfgs:
        try:
            c = dict(c)
            roles = c.pop("roles", None)
            pl = p.b.g.plan(0, **c)
            if roles:
                pl.set_flow_roles(roles[0], roles[1])
            if ref is not None:
                p.view("mask").fill_(77)
            c["roles"] = roles
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
            ok = None
            if ref is not None:
                torch.cuda.synchronize()
                ok = bool(torch.equal(p.view("mask"), ref))
            print(json.dumps({"cfg": c, "geom": args.geom or "default", "minb": os.environ.get("KTILER_PERSIST_MINB", "default"), "ms": round(ms, 4),
                              "Mpix/s": round(pix / ms / 1e3, 1), "fragments": st["n_fragments"],
                              "launches": st["n_launches"], "match": ok}), flush=True)
            del pl
        except Exception as e:
            print(json.dumps({"cfg": c, "error": str(e)}), flush=True)


if __name__ == "__main__":
    main()
