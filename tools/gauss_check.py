"""Float variant (O-7, KTILER_OP_GAUSS_F32) on one B200: max-abs error vs the f64 oracle on
a small case, and time per execute of a K-node chain on a large f32 image, untiled vs
tiled (median of reps, CUDA events).  Diagnostic tool."""
import json, os, statistics, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np
import torch
import __graft_entry__ as ge
from oracle import oracle as O
from paper_conf_date_maghazeh0ep19_b200.gauss import GaussChain
ge.build()
for (W, H, K, sig) in [(512, 256, 4, 1.0), (640, 200, 2, 1.3)]:
    g = GaussChain(W, H, nodes=K, sigma=sig, tile=(64, 16))
    x = np.random.default_rng(1).random((1, H, W), dtype=np.float32)
    g.view("x0").copy_(torch.from_numpy(x))
    g.plan(256 * 1024, kind="budget", exec_mode="dag")
    g.run(); torch.cuda.synchronize()
    err = float(np.abs(g.view(f"x{K}").cpu().numpy().astype(np.float64) - O.gauss_f32(x, sig, passes=K)).max())
    print(json.dumps({"check": f"{W}x{H} K={K} sigma={sig}", "max_abs_err": err}))
W, H, K = 7680, 4320, 4
g = GaussChain(W, H, nodes=K, sigma=1.0)
g.view("x0").copy_(torch.rand((1, H, W), device="cuda"))
s = torch.cuda.current_stream()
for cfg in [dict(kind="none", exec_mode="graph"), dict(kind="budget", l2_fraction=1.0, exec_mode="dag", resident_budget=True),
            dict(kind="budget", l2_fraction=0.5, exec_mode="dag", resident_budget=True)]:
    pl = g.plan(0, **cfg)
    for _ in range(3):
        pl.execute(s.cuda_stream)
    ts = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s); pl.execute(s.cuda_stream); e1.record(s); e1.synchronize(); ts.append(e0.elapsed_time(e1))
    ms = statistics.median(ts)
    print(json.dumps({"cfg": cfg, "W": W, "H": H, "nodes": K, "ms": round(ms, 4), "fragments": pl.num_fragments(),
                      "GBps_untiled_bytes": round(8 * W * H * K / ms / 1e6, 1)}))
