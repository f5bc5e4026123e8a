"""bench.py's host-side contract pieces that need no GPU: the default policy is the one
profiles/ has measured (so the bench line carries its DRAM traffic), and the reference arm
(the oracle) prints one well-formed JSON line."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def test_default_policy_has_measured_traffic():
    import bench
    args = bench.parse([])
    pol = bench.policy(args)
    cfg = {"workload": args.workload, "mode": args.mode, "policy": args.kind, "l2_fraction": args.l2_fraction,
           "discard": pol["discard"], "window": args.window, "resident_budget": pol["resident_budget"],
           "consumer_discard": pol["consumer_discard"], "halo_discard": pol["halo_discard"], "pdl": bool(args.pdl)}
    traffic, src = bench.traffic_for(cfg)
    assert traffic and traffic > 0 and src.startswith("profiles/")
    assert bench.l2_ceiling() is not None


def test_reference_arm_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--steps", "1",
                          "--warmup", "1", "--workload", "pipeline_4096"], capture_output=True, text=True, timeout=300,
                         cwd=ROOT)
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["value"] > 0 and line["steps"] == 1
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] == 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0
