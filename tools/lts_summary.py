"""Summarise an ncu --csv capture (graph-level or per-kernel) of LTS sector counters:
per ID, the time and the sector traffic by source / op in GB."""
import csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10 and not r[0].startswith("{")]
h = rows[0]
ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
by = {}
for r in rows[1:]:
    by.setdefault(r[0], [r[ki][:40], {}])[1][r[mi]] = r[vi]
for k, (name, v) in by.items():
    out = []
    for m, x in sorted(v.items()):
        x = float(x.replace(",", ""))
        if "sectors" in m:
            out.append(f"{m.replace('lts__t_sectors', '').replace('.sum', '') or 'all'}={x * 32 / 1e9:.2f}")
        elif "bytes" in m:
            out.append(f"{m.replace('.sum', '')}={x / 1e9:.2f}")
        elif "duration" in m:
            out.append(f"t={x / 1e6:.3f}ms")
    print(k, name, " ".join(out))
