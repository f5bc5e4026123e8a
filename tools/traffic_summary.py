"""Summarise an ncu --csv metrics capture of tools/sweep.py (graph-level profiling): per
profiled range (graph or kernel launch) DRAM bytes, L2 hit rate, duration.  The sweep runs
2 warm-ups + reps executes per configuration, so ranges come in groups of 2 + reps."""
import csv, sys, json
lines = [l for l in open(sys.argv[1]) if l.startswith('"')]
rows = list(csv.reader(lines))
h = rows[0]
K, order = {}, []
for r in rows[1:]:
    d = dict(zip(h, r))
    i = int(d["ID"])
    if i not in K:
        K[i] = {"name": d["Kernel Name"]}
        order.append(i)
    v = d["Metric Value"].replace(",", "")
    K[i][d["Metric Name"]] = float(v) * ({"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3}.get(d["Metric Unit"], 1.0)
                                         if "bytes" in d["Metric Name"] else 1.0)
out = []
for i in order:
    v = K[i]
    if "gen_" in v["name"]:
        continue
    out.append({"id": i, "name": v["name"][:40], "dram_GB": round((v["dram__bytes_read.sum"] + v["dram__bytes_write.sum"]) / 1e9, 3),
                "read_GB": round(v["dram__bytes_read.sum"] / 1e9, 3), "write_GB": round(v["dram__bytes_write.sum"] / 1e9, 3),
                "l2_hit_pct": round(v["lts__t_sector_hit_rate.pct"], 1), "ms": round(v["gpu__time_duration.sum"] / 1e6, 3)})
for o in out:
    print(json.dumps(o))
