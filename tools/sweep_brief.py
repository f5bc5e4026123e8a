"""Condense tools/sweep.py JSON lines to `kind l2_fraction ms match fragments` (for sweep logs)."""
import json
import sys

for line in sys.stdin:
    if not line.startswith("{"):
        sys.stdout.write(line)
        continue
    d = json.loads(line)
    c = d["cfg"]
    print(f'  {c.get("exec_mode")}/{c.get("kind")} l2={c.get("l2_fraction")} pdl={c.get("pdl", False)} '
          f'ms={d["ms"]} match={d.get("match")} frags={d.get("fragments")}')
