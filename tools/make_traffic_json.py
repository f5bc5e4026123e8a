"""Build profiles/traffic.json (DRAM bytes per step per configuration, read by bench.py)
from ncu captures of tools/sweep.py: each configuration ran 2 warm-ups + 1 execute; the
3rd profiled range of each is kept.  Usage: make_traffic_json.py OUT (CSV CFG_JSON NAME)..."""
import json
import subprocess
import sys

out = sys.argv[1]
entries = []
args = sys.argv[2:]
for k in range(0, len(args), 3):
    csv_path, cfgs, name = args[k], json.loads(open(args[k + 1]).read()), args[k + 2]
    rows = [json.loads(l) for l in subprocess.run([sys.executable, "tools/traffic_summary.py", csv_path],
                                                   capture_output=True, text=True, check=True).stdout.splitlines()]
    for i, c in enumerate(cfgs):
        if 3 * i + 2 >= len(rows):
            break
        r = rows[3 * i + 2]
        cfg = {"workload": "batch64_8k", "mode": c.get("exec_mode", "graph"), "policy": c.get("kind", "budget"),
               "l2_fraction": c.get("l2_fraction", 1.0), "discard": bool(c.get("discard", False)),
               "window": c.get("window", 2), "resident_budget": bool(c.get("resident_budget", False)),
               "consumer_discard": bool(c.get("consumer_discard", False)),
               "halo_discard": bool(c.get("halo_discard", False))}
        if c.get("skew"):
            cfg["skew"] = c["skew"]
        entries.append({"config": cfg, "dram_bytes_per_step": r["dram_GB"] * 1e9, "dram_read": r["read_GB"] * 1e9,
                        "dram_write": r["write_GB"] * 1e9, "lts_sector_hit_rate_pct": r["l2_hit_pct"],
                        "ncu_duration_ms": r["ms"],
                        "source": f"profiles/{name} (ncu --cache-control all --clock-control none, 3rd execute)"})
json.dump({"round": 1, "workload": "batch64_8k (64 x 7680x4320)", "pixels": 2123366400,
           "compulsory_bytes_per_step": 3.25 * 2123366400, "entries": entries}, open(out, "w"), indent=1)
print(len(entries), "entries")
