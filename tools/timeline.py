"""Device-side timeline of one execute (ktiler_trace_*): where the time of a schedule goes.

For each configuration: plan, enable tracing, warm up, run once traced, then summarise
  - span: first CTA start -> last CTA end (ns, %globaltimer);
  - per node: CTA-time (sum of CTA durations) and its share, wall span of its launches;
  - occupancy: time-weighted mean number of resident CTAs (op kernels) or busy compute
    groups (persistent), and the fraction of the span with less than half the peak;
  - persistent: control-warp time per tile (dependency check + staging issue), compute
    time per tile, and the gap between a buffer's arrival and the previous tile's end.
Raw records go to --out (npz) when given.  Diagnostic tool, not the bench."""
from __future__ import annotations

import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
NODES = ("gray", "blur", "down", "sobel", "thresh")


def occupancy(t0, t1):
    """Time-weighted mean of the number of open intervals, its max, and the fraction of
    the span with fewer than half the max open."""
    ev = np.concatenate([np.stack([t0, np.ones_like(t0, dtype=np.int64)], 1),
                         np.stack([t1, -np.ones_like(t1, dtype=np.int64)], 1)])
    ev = ev[np.lexsort((ev[:, 1], ev[:, 0]))]
    cnt = np.cumsum(ev[:, 1])
    dt = np.diff(ev[:, 0])
    span = ev[-1, 0] - ev[0, 0]
    mean = float((cnt[:-1] * dt).sum() / max(span, 1))
    peak = int(cnt.max())
    low = float(dt[cnt[:-1] < peak / 2].sum() / max(span, 1))
    return mean, peak, low


def summarise(rec, launches, pix):
    out = {}
    k0 = rec[rec["kind"] == 0]
    if len(k0):  # kind 0: one record per CTA
        t0, t1 = k0["t0"].astype(np.int64), k0["t1"].astype(np.int64)
        base = t0.min()
        span = int(t1.max() - base)
        node = np.array([launches[i][1] for i in k0["id"]])
        dur = t1 - t0
        out["span_us"] = span / 1e3
        out["ctas"] = int(len(k0))
        per = {}
        for v in sorted(set(node.tolist())):
            m = node == v
            name = NODES[v] if 0 <= v < len(NODES) else ("discard" if v < 0 else str(v))
            per[name] = {"cta_ms": round(float(dur[m].sum()) / 1e6, 3), "ctas": int(m.sum()),
                         "mean_cta_us": round(float(dur[m].mean()) / 1e3, 2)}
        tot = sum(x["cta_ms"] for x in per.values())
        for x in per.values():
            x["share"] = round(x["cta_ms"] / max(tot, 1e-9), 3)
        out["nodes"] = per
        mean, peak, low = occupancy(t0, t1)
        out["occ_mean"], out["occ_peak"], out["occ_low_frac"] = round(mean, 1), peak, round(low, 3)
        # launch gaps: per launch (first start, last end) in launch order
        lid = k0["id"].astype(np.int64)
        order = np.unique(lid)
        starts = np.array([t0[lid == i].min() for i in order])
        ends = np.array([t1[lid == i].max() for i in order])
        out["launch_span_us_median"] = round(float(np.median(ends - starts)) / 1e3, 2)
        gaps = starts[1:] - ends[:-1]
        out["launch_gap_us_median"] = round(float(np.median(gaps)) / 1e3, 2) if len(gaps) else 0.0
        out["launch_overlap_frac"] = round(float((gaps < 0).mean()), 3) if len(gaps) else 0.0
        # per node: median launch span and median gap from the previous launch's end
        lnode = np.array([launches[i][1] for i in order])
        per_span, per_gap = {}, {}
        for v in sorted(set(lnode.tolist())):
            m = lnode == v
            name = NODES[v] if 0 <= v < len(NODES) else "discard"
            per_span[name] = round(float(np.median((ends - starts)[m])) / 1e3, 2)
            gm = m[1:]
            if gm.any():
                per_gap[name] = round(float(np.median(gaps[gm])) / 1e3, 2)
        out["node_launch_span_us"] = per_span
        out["node_gap_before_us"] = per_gap
    # op-kernel CTA phases (kinds 5, 6): start -> producers ready (PDL wait, discards),
    # ready -> first tile staged (TMA latency), rest = compute + stores + exit
    k5, k6 = rec[rec["kind"] == 5], rec[rec["kind"] == 6]
    if len(k5) and len(k6) and len(k0):
        phases = {}
        node5 = np.array([launches[i][1] for i in k5["id"]])
        d5 = k5["t1"].astype(np.int64) - k5["t0"].astype(np.int64)
        d6 = k6["t1"].astype(np.int64) - k6["t0"].astype(np.int64)
        node0 = np.array([launches[i][1] for i in k0["id"]])
        d0 = k0["t1"].astype(np.int64) - k0["t0"].astype(np.int64)
        for v in sorted(set(node5.tolist())):
            if not 0 <= v < len(NODES):
                continue
            m5, m0 = node5 == v, node0 == v
            w, l, c = float(d5[m5].mean()), float(d6[m5].mean()), float(d0[m0].mean())
            phases[NODES[v]] = {"wait_us": round(w / 1e3, 2), "stage_us": round(l / 1e3, 2),
                                "rest_us": round((c - w - l) / 1e3, 2),
                                "stage_us_p10_50_90": [round(float(np.percentile(d6[m5], q)) / 1e3, 2) for q in (10, 50, 90)]}
        out["cta_phases"] = phases
    for kind, name in ((3, "ready_to_computed"), (4, "publish")):
        kk = rec[rec["kind"] == kind]
        if len(kk):
            d = kk["t1"].astype(np.int64) - kk["t0"].astype(np.int64)
            node = np.array([launches[i][1] for i in kk["id"]])
            out[name + "_us"] = {NODES[v]: round(float(d[node == v].mean()) / 1e3, 3) for v in sorted(set(node.tolist()))}
    if len(k0) and (rec["kind"] == 3).any():
        # CTA start -> first tile's producers ready (spin + launch latency), per node
        k3 = rec[rec["kind"] == 3]
        first_ready = {}
        for i, t in zip(k3["id"].tolist(), k3["t0"].tolist()):
            first_ready.setdefault(i, []).append(t)
        # approximate: mean over launches of (median ready time - median CTA start)
        lat = {}
        for lid in set(k0["id"].tolist()):
            if lid in first_ready:
                st0 = np.median(k0["t0"][k0["id"] == lid].astype(np.int64))
                lat.setdefault(launches[lid][1], []).append(np.median(first_ready[lid]) - st0)
        out["start_to_ready_us_median"] = {NODES[v]: round(float(np.mean(x)) / 1e3, 2) for v, x in sorted(lat.items())}
    k2 = rec[rec["kind"] == 2]
    if len(k2):
        k1 = rec[rec["kind"] == 1]
        t0, t1 = k2["t0"].astype(np.int64), k2["t1"].astype(np.int64)
        base = min(t0.min(), k1["t0"].min() if len(k1) else t0.min())
        span = int(t1.max() - base)
        out["span_us"] = span / 1e3
        out["tiles"] = int(len(k2))
        node = (k2["id"] >> np.uint64(60)).astype(np.int64)
        dur = t1 - t0
        per = {}
        for v in sorted(set(node.tolist())):
            m = node == v
            per[NODES[v]] = {"compute_ms": round(float(dur[m].sum()) / 1e6, 3), "tiles": int(m.sum()),
                             "mean_tile_us": round(float(dur[m].mean()) / 1e3, 2)}
        out["nodes"] = per
        mean, peak, low = occupancy(t0, t1)
        out["busy_mean"], out["busy_peak"], out["busy_low_frac"] = round(mean, 1), peak, round(low, 3)
        if len(k1):
            c = (k1["t1"].astype(np.int64) - k1["t0"].astype(np.int64))
            out["ctl_us_mean"] = round(float(c.mean()) / 1e3, 3)
            out["ctl_us_p90"] = round(float(np.percentile(c, 90)) / 1e3, 3)
            cn = (k1["id"] >> np.uint64(60)).astype(np.int64)
            out["ctl_us_by_node"] = {NODES[v]: round(float(c[cn == v].mean()) / 1e3, 3) for v in sorted(set(cn.tolist()))}
            # staging issued -> compute start, per node (TMA latency + queueing behind earlier tiles)
            i1 = {int(i): int(t) for i, t in zip(k1["id"], k1["t1"])}
            lat = np.array([t - i1.get(int(i), t) for i, t in zip(k2["id"], k2["t0"])], dtype=np.int64)
            out["issue_to_start_us_by_node"] = {NODES[v]: [round(float(np.percentile(lat[node == v], q)) / 1e3, 2)
                                                           for q in (10, 50, 90)] for v in sorted(set(node.tolist()))}
        # per SM: idle between consecutive compute intervals (all CTAs of the SM merged)
        sm = k2["smid"].astype(np.int64)
        idle = []
        for s in np.unique(sm):
            m = sm == s
            a, b = np.sort(t0[m]), np.sort(t1[m])
            mean_s, _, _ = occupancy(a, b)
            idle.append(mean_s)
        out["per_sm_busy_mean"] = round(float(np.mean(idle)), 2)
    if "span_us" in out:
        out["Mpix_per_s_span"] = round(pix / out["span_us"], 1)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--W", type=int, default=7680)
    ap.add_argument("--H", type=int, default=4320)
    ap.add_argument("--F", type=int, default=64)
    ap.add_argument("--configs", required=True, help="json list of plan kwargs")
    ap.add_argument("--out", default="")
    ap.add_argument("--cap", type=int, default=1 << 22)
    args = ap.parse_args()
    import torch

    import __graft_entry__ as ge
    from inputs import gpu as G
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    ge.build()
    p = Pipeline(args.W, args.H, args.F, internal=True)
    s = torch.cuda.current_stream()
    G.fill("scene", 1234, p.view("rgb").data_ptr(), args.W * 3, args.W * 3 * args.H, args.W, args.H, F=args.F,
           stream=s.cuda_stream)
    torch.cuda.synchronize()
    raw = {}
    for ci, c in enumerate(json.loads(args.configs)):
        try:
            pl = p.b.g.plan(0, **c)
            pl.trace_enable(args.cap)
            for _ in range(2):
                pl.execute(s.cuda_stream)
            pl.trace_read()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s)
            pl.execute(s.cuda_stream)
            e1.record(s)
            e1.synchronize()
            rec, n = pl.trace_read()
            res = summarise(rec, pl.launches(), args.W * args.H * args.F)
            res.update({"cfg": c, "event_ms": round(e0.elapsed_time(e1), 4), "records": n,
                        "fragments": pl.stats()["n_fragments"]})
            print(json.dumps(res), flush=True)
            if args.out:
                raw[f"c{ci}"] = rec
                raw[f"c{ci}_launch"] = np.array(pl.launches(), dtype=np.int64).reshape(-1, 3)
            del pl
        except Exception as e:
            print(json.dumps({"cfg": c, "error": repr(e)}), flush=True)
    if args.out:
        np.savez_compressed(args.out, **raw)


if __name__ == "__main__":
    main()
