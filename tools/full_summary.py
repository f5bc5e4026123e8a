"""Summarise ncu --set full details CSVs (tools/round_profile.sh): for each file, the profiled
launch with the largest grid (a full-size sub-kernel, not a ragged remainder) and its
throughput / occupancy / issue metrics.  Diagnostic tool, not product code.

  python tools/full_summary.py HEADER name1=file1.csv name2=file2.csv ..."""
import csv
import sys

WANT = ["Memory Throughput", "DRAM Throughput", "Duration", "L2 Cache Throughput", "Compute (SM) Throughput",
        "Executed Ipc Active", "Issue Slots Busy", "L2 Hit Rate", "Block Size", "Grid Size", "Registers Per Thread",
        "Dynamic Shared Memory Per Block", "Waves Per SM", "Block Limit Registers", "Block Limit Shared Mem",
        "Theoretical Occupancy", "Achieved Occupancy"]


def main(argv):
    print("# " + argv[0])
    for arg in argv[1:]:
        name, path = arg.split("=", 1)
        rows = list(csv.reader(open(path)))
        h = rows[0]
        per = {}
        for r in rows[1:]:
            d = dict(zip(h, r))
            per.setdefault(d["ID"], {}).setdefault((d["Metric Name"], d["Metric Unit"]), d["Metric Value"])
        def grid(m):
            for (k, u), v in m.items():
                if k == "Grid Size":
                    return float(v.replace(",", ""))
            return 0.0
        best_id = max(per, key=lambda i: grid(per[i]))
        m = per[best_id]
        print(f"## {name} (profiled launch {best_id} of {len(per)}: the largest grid)")
        for w in WANT:
            for (k, u), v in m.items():
                if k == w:
                    print(f"{k}: {v} {u}".rstrip())


if __name__ == "__main__":
    main(sys.argv[1:])
