"""Diagnostic (profiles/r02e_instantiation_states.txt): time DAG + PDL plans
created back to back, then re-created after deleting others, in one process.  Not product
code."""
import os, sys, statistics, json
sys.path.insert(0, os.getcwd())
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
pol = dict(kind="budget", exec_mode="dag", resident_budget=True, window=2, pdl=True, consumer_discard=True, l2_fraction=1.0)

def t(pl, reps=9):
    for _ in range(2):
        pl.execute(s.cuda_stream)
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s); pl.execute(s.cuda_stream); e1.record(s); e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return round(statistics.median(ts), 4)

plans = []
for i in range(6):
    plans.append(p.b.g.plan(0, **pol))
    print("create", i, t(plans[i]), flush=True)
print("again", [t(x) for x in plans], flush=True)
for i in (0, 2, 4):
    plans[i] = None
import gc; gc.collect()
for i in (0, 2, 4):
    plans[i] = p.b.g.plan(0, **pol)
    print("recreate", i, t(plans[i]), flush=True)
print("again", [t(x) for x in plans], flush=True)
# untiled plan in between
plans = None; gc.collect()
for i in range(4):
    u = p.b.g.plan(0, kind="none", exec_mode="graph"); tu = t(u); del u
    d = p.b.g.plan(0, **pol); td = t(d); del d
    print("untiled, dag", tu, td, flush=True)
