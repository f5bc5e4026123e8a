"""Which dependency releases each sub-kernel of a traced GRAPH_DAG execute (diagnostic).

Input: the npz of tools/timeline.py --out (per-CTA records + the plan's launch list).  Per
launch: node, fragment (sub-kernel index // nodes, the pipeline's fragment-major order),
first CTA start, last CTA end.  Then, for each node: the fraction of the span during which
one of its launches runs, the median gap between its consecutive launches, and how often
its start follows (a) the previous sub-kernel of the same node (chain edge), (b) its
producer in the same fragment, (c) the window edge (leaf of fragment f - window) — the
edge whose end is latest before the start is the binding one.
Usage: python tools/critical_path.py trace.npz [config-key c0] [window 2]"""
from __future__ import annotations

import collections
import json
import sys

import numpy as np

NODES = ("gray", "blur", "down", "sobel", "thresh")


def main():
    z = np.load(sys.argv[1])
    key = sys.argv[2] if len(sys.argv) > 2 else "c0"
    window = int(sys.argv[3]) if len(sys.argv) > 3 else 2
    rec, L = z[key], z[key + "_launch"]
    k0 = rec[rec["kind"] == 0]
    ids = k0["id"].astype(np.int64)
    t0, t1 = k0["t0"].astype(np.int64), k0["t1"].astype(np.int64)
    base = t0.min()
    span = (t1.max() - base) / 1e3
    st, en = {}, {}
    for li in np.unique(ids):
        m = ids == li
        sub, node, _ = L[li]
        if node < 0:
            continue
        k = (int(node), int(sub) // 5)
        st[k] = min(st.get(k, 1 << 62), (t0[m].min() - base) / 1e3)
        en[k] = max(en.get(k, -1), (t1[m].max() - base) / 1e3)
    nfrag = max(f for _, f in st) + 1
    out = {"span_us": round(span, 1), "fragments": nfrag, "nodes": {}}
    for v in range(5):
        iv = sorted((st[(v, f)], en[(v, f)]) for f in range(nfrag) if (v, f) in st)
        busy, cur0, cur1 = 0.0, None, None
        for a, b in iv:
            if cur1 is None or a > cur1:
                if cur1 is not None:
                    busy += cur1 - cur0
                cur0, cur1 = a, b
            else:
                cur1 = max(cur1, b)
        busy += cur1 - cur0
        durs = [b - a for a, b in iv]
        gaps = [iv[i + 1][0] - iv[i][1] for i in range(len(iv) - 1)]
        bind = collections.Counter()
        lag = []
        for f in range(nfrag):
            if (v, f) not in st:
                continue
            cand = {}
            if (v, f - 1) in en:
                cand["chain"] = en[(v, f - 1)]
            if v > 0 and (v - 1, f) in en:
                cand["producer"] = en[(v - 1, f)]
            if v == 0 and (4, f - window) in en:
                cand["window"] = en[(4, f - window)]
            if not cand:
                continue
            which = max(cand, key=cand.get)
            bind[which] += 1
            lag.append(st[(v, f)] - cand[which])
        out["nodes"][NODES[v]] = {
            "busy_frac": round(busy / span, 3), "launch_us_median": round(float(np.median(durs)), 1),
            "gap_us_median": round(float(np.median(gaps)), 2) if gaps else None,
            "binding_edge": dict(bind), "start_after_binding_us_median": round(float(np.median(lag)), 2) if lag else None}
    # fragment chain: gray start -> thresh end
    ch = [en[(4, f)] - st[(0, f)] for f in range(nfrag) if (0, f) in st and (4, f) in en]
    out["fragment_chain_us_median"] = round(float(np.median(ch)), 1)
    print(json.dumps(out))
    if "-v" in sys.argv:
        for f in range(nfrag):
            print(f, " ".join(f"{NODES[v]}[{st.get((v, f), -1):8.1f},{en.get((v, f), -1):8.1f}]" for v in range(5)))


if __name__ == "__main__":
    main()
