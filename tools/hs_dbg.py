import sys, os; sys.path.insert(0, os.getcwd())
import numpy as np, torch
import __graft_entry__ as ge; ge.build()
from inputs import synth
from paper_conf_date_maghazeh0ep19_b200.hs import HSJacobi
W,H,K=128,64,1
h = HSJacobi(W, H, K, a2=0.5)
coef, s0 = synth.hs_fields(1, W, H, 1)
h.set("coef", coef); h.set("s0", s0)
pl = h.plan(1<<20, kind="none", exec_mode="stream")
h.run(); torch.cuda.synchronize(); print("ok")
