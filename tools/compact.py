"""Compact view of tools/sweep.py JSON lines: mode, budget, ms, fragments (stdin -> stdout)."""
import json, sys
for l in sys.stdin:
    l = l.strip()
    if not l.startswith("{"):
        if l: print(l)
        continue
    try:
        d = json.loads(l)
    except Exception:
        print("?", l[:100]); continue
    c = d.get("cfg", {})
    print(f"  {c.get('exec_mode','?'):10s} {c.get('kind','?'):7s} r={c.get('rows','-')} f={c.get('l2_fraction','-')} w={c.get('window','-')} "
          f"ms={d.get('ms','-')} frags={d.get('fragments','-')} {d.get('error','')[:80]}")
