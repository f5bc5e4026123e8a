"""Device timeline of one KTILER_EXEC_FLOW execute (ktiler_trace_enable, flow.cuh kinds
5/6/7): per node, how long a tile waits between its claim and its TMA issue, between
issue and compute start (staging latency), how long it computes, and how long its flag
waits for publication; plus each node's compute-busy fraction of the step.  Diagnostic
tool, not product code.

  python tools/flow_trace.py --F 16 --geom '{...}' --cfg '{"kind":"rows",...,"roles":[[...],[...]]}'
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--W", type=int, default=7680)
    ap.add_argument("--H", type=int, default=4320)
    ap.add_argument("--F", type=int, default=16)
    ap.add_argument("--geom", default="")
    ap.add_argument("--cfg", required=True)
    args = ap.parse_args()
    import numpy as np
    import torch

    import __graft_entry__ as ge
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    from paper_conf_date_maghazeh0ep19_b200.pipeline import B200_GEOMETRY
    ge.build()
    geom = dict(B200_GEOMETRY)
    if args.geom:
        geom.update({k: tuple(v) for k, v in json.loads(args.geom).items()})
    p = Pipeline(args.W, args.H, args.F, internal=True, geometry=geom)
    s = torch.cuda.current_stream()
    G.fill("scene", 1234, p.view("rgb").data_ptr(), args.W * 3, args.W * 3 * args.H, args.W, args.H, F=args.F,
           stream=s.cuda_stream)
    c = json.loads(args.cfg)
    roles = c.pop("roles", None)
    pl = p.b.g.plan(0, **c)
    if roles:
        pl.set_flow_roles(roles[0], roles[1])
    pl.trace_enable(1 << 23)
    pl.execute(s.cuda_stream)
    pl.trace_read()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(s)
    pl.execute(s.cuda_stream)
    e1.record(s)
    torch.cuda.synchronize()
    rec, n = pl.trace_read()
    print(json.dumps({"cfg": c, "roles": roles, "ms": e0.elapsed_time(e1), "records": int(n)}))
    names = ("gray", "blur", "down", "sobel", "thresh")
    t_all0 = rec["t0"][rec["t0"] > 0].min()
    t_all1 = rec["t1"].max()
    span = float(t_all1 - t_all0)
    by = {}
    for k in (5, 6, 7):
        r = rec[rec["kind"] == k]
        by[k] = {int(i): (int(a), int(b)) for i, a, b in zip(r["id"], r["t0"], r["t1"])}
    for v, nm in enumerate(names):
        ids = [i for i in by[6] if (i >> 59) == v]
        if not ids:
            continue
        claim = np.array([by[5][i][1] - by[5][i][0] for i in ids if i in by[5]], dtype=np.float64)
        stage = np.array([by[6][i][0] - by[5][i][1] for i in ids if i in by[5]], dtype=np.float64)
        comp = np.array([by[6][i][1] - by[6][i][0] for i in ids], dtype=np.float64)
        pub = np.array([by[7][i][0] - by[6][i][1] for i in ids if i in by[7]], dtype=np.float64)
        nsm = len(set(rec["smid"][(rec["kind"] == 6) & ((rec["id"] >> 59) == v)].tolist()))
        busy = comp.sum() / span
        print(f"{nm:7s} tiles {len(ids):7d}  claim->issue {np.median(claim)/1e3:7.2f} us  issue->compute {np.median(stage)/1e3:6.2f} us"
              f"  compute {np.median(comp)/1e3:6.2f} us (mean {comp.mean()/1e3:6.2f})  done->publish {np.median(pub)/1e3:6.2f} us"
              f"  busy CTAs {busy:6.1f} on {nsm} SMs")
    # progress curve: fraction of each node's tiles published by time t (10 samples)
    print("published fraction over the step (10 points):")
    for v, nm in enumerate(names):
        ts = np.sort(np.array([by[7][i][0] for i in by[7] if (i >> 59) == v], dtype=np.float64))
        if len(ts) == 0:
            continue
        pts = [float(np.searchsorted(ts, t_all0 + span * q / 10) / len(ts)) for q in range(1, 11)]
        print(f"  {nm:7s} " + " ".join(f"{x:4.2f}" for x in pts))


if __name__ == "__main__":
    main()
