"""Small-config run of every executor for compute-sanitizer (SURVEY
§4.2 / §5): memcheck, racecheck, synccheck and initcheck over the same replay of each
exec mode (with discards and the flag / counter synchronisation paths on), each output
checked against the oracle.  Usage (GPU box):

  compute-sanitizer --tool memcheck python tools/sanitize.py [modes...]

Exit status 0 iff every mode's mask equals the oracle's.  Diagnostic tool, not product
code."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

MODES = {
    "stream": dict(kind="budget", discard=True),
    "graph": dict(kind="budget", discard=True, pdl=True),
    "persist_l2": dict(kind="budget", discard=True),
    "dag": dict(kind="budget", window=2, resident_budget=True, consumer_discard=True, halo_discard=True, discard=True),
    # the bench default: programmatic (PDL) producer edges, consumer discards
    "dag_pdl": dict(kind="budget", window=2, resident_budget=True, consumer_discard=True, pdl=True),
    "chain": dict(kind="budget", discard=True, consumer_discard=True),
    "wave": dict(kind="budget", discard=True),
    "persistent": dict(kind="rows", rows=1, discard=True),
    "flow": dict(kind="rows", rows=1, consumer_discard=True),
}
SMALL = {"gray": (64, 16, 64), "blur": (64, 16, 64), "down": (32, 8, 64), "sobel": (32, 8, 64), "thresh": (32, 8, 64)}


def main(argv):
    import numpy as np
    import torch

    import __graft_entry__ as ge
    from inputs import synth
    from oracle import oracle as O
    from paper_conf_date_maghazeh0ep19_b200 import Pipeline
    ge.build()
    W, H, F = 520, 198, 2
    rgb = synth.scene(7, W, H, F)
    ref = O.pipeline(rgb, T=60.0)["mask"]
    bad = 0
    for mode in (argv or list(MODES)):
        pol = dict(MODES[mode])
        kind = pol.pop("kind")
        geo = None if mode in ("persistent", "flow") else SMALL
        p = Pipeline(W, H, F, T=60.0, internal=True, geometry=geo)
        p.view("rgb").copy_(torch.from_numpy(rgb))
        plan = p.plan(256 * 1024 if geo else 1 << 20, kind=kind, exec_mode=mode.split("_")[0] if mode != "persist_l2" else mode, **pol)
        for _ in range(2):
            p.run()
        torch.cuda.synchronize()
        ok = np.array_equal(p.view("mask").cpu().numpy(), ref)
        print(f"sanitize {mode}: fragments {plan.num_fragments()} match {ok}", flush=True)
        bad += not ok
        del plan, p
    return 1 if bad else 0


if __name__ == "__main__":
    sys.exit(main(sys.argv[1:]))
