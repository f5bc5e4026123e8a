"""Float-variant chain (KTILER_OP_GAUSS_F32, O-7) timing sweep on one B200: K nodes on
F frames of W x H f32, untiled vs tiled configurations (median of reps, CUDA events).
Diagnostic tool (the bench's headline workload is the image pipeline)."""
import argparse, json, os, statistics, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import __graft_entry__ as ge
from paper_conf_date_maghazeh0ep19_b200.gauss import GaussChain
ap = argparse.ArgumentParser()
ap.add_argument("--W", type=int, default=7680); ap.add_argument("--H", type=int, default=4320)
ap.add_argument("--F", type=int, default=8); ap.add_argument("--K", type=int, default=4)
ap.add_argument("--configs", required=True)
a = ap.parse_args()
ge.build()
g = GaussChain(a.W, a.H, nodes=a.K, frames=a.F, sigma=1.0)
g.view("x0").copy_(torch.rand((a.F, a.H, a.W), device="cuda"))
s = torch.cuda.current_stream()
for cfg in json.loads(a.configs):
    try:
        pl = g.plan(0, **cfg)
        for _ in range(3):
            pl.execute(s.cuda_stream)
        ts = []
        for _ in range(9):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(s); pl.execute(s.cuda_stream); e1.record(s); e1.synchronize(); ts.append(e0.elapsed_time(e1))
        ms = statistics.median(ts)
        print(json.dumps({"cfg": cfg, "ms": round(ms, 4), "fragments": pl.num_fragments(),
                          "untiled_bytes_GBps": round(8 * a.W * a.H * a.F * a.K / ms / 1e6, 1)}))
    except Exception as e:
        print(json.dumps({"cfg": cfg, "error": str(e)[:120]}))
