"""Run one entry of tools/sweeps.json (the round-1 GPU experiment scripts and sweep
configurations, kept as one manifest).  Diagnostic tool, not product code.

  python tools/run_sweep.py <script-name>        # e.g. gpu_s5c: bash body, from the repo root
  python tools/run_sweep.py --config <cfg-name>  # print a config list (tools/sweep.py --configs)
"""
import json
import os
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
MAN = json.load(open(os.path.join(ROOT, "tools", "sweeps.json")))


def main(argv):
    if argv[:1] == ["--config"]:
        print(json.dumps(MAN["configs"][argv[1]]))
        return 0
    body = MAN["scripts"][argv[0]]
    d = tempfile.mkdtemp(prefix="ktiler_cfg_")
    for name, cfg in MAN["configs"].items():  # the scripts read tools/cfg_<name>.json
        with open(os.path.join(d, name + ".json"), "w") as f:
            json.dump(cfg, f)
    body = body.replace("tools/cfg_", d + "/cfg_")
    return subprocess.call(["bash", "-c", body], cwd=ROOT)


if __name__ == "__main__":
    sys.exit(main(sys.argv[1:]))
