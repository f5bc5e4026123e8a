"""Summarise an ncu source page (--page source --csv --print-source sass): per kernel,
instruction totals by opcode and the hottest instructions by executed count / samples."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
kern = None; hdr = None; data = collections.OrderedDict()
for r in rows:
    if r and r[0] == "Kernel Name":
        kern = r[1]; data[kern] = []; hdr = None; continue
    if r and r[0] == "Address":
        hdr = r; continue
    if hdr and kern and len(r) == len(hdr):
        d = dict(zip(hdr, r)); data[kern].append(d)
for k, ins in data.items():
    tot = sum(int(d["Instructions Executed"] or 0) for d in ins)
    smp = sum(int(d["Warp Stall Sampling (All Samples)"] or 0) for d in ins)
    print(f"=== {k[:60]}  warp-inst {tot/1e6:.1f}M  samples {smp}  ninstr {len(ins)}")
    ops = collections.Counter()
    for d in ins:
        op = d["Source"].split()[0] if d["Source"].split() else "?"
        if op.startswith("@"): op = d["Source"].split()[1]
        ops[op.split(".")[0]] += int(d["Instructions Executed"] or 0)
    print("  by opcode:", ", ".join(f"{o} {v/1e6:.1f}M" for o, v in ops.most_common(18)))
    hot = sorted(ins, key=lambda d: -int(d["Warp Stall Sampling (All Samples)"] or 0))[:top]
    for d in hot:
        print(f"  {d['Address'][-5:]} smp {d['Warp Stall Sampling (All Samples)']:>6} ex {int(d['Instructions Executed'] or 0)/1e6:7.2f}M  {d['Source'].strip()[:70]}")

if len(sys.argv) > 3:  # top PCs for one stall reason: sass_hot.py file N reason
    col = sys.argv[3]
    for k, ins in data.items():
        tot = sum(int(d.get(col, 0) or 0) for d in ins)
        print(f"--- {k[:50]} {col} total {tot}")
        for d in sorted(ins, key=lambda d: -int(d.get(col, 0) or 0))[:top]:
            print(f"  {d['Address'][-5:]} {d.get(col)} ex {int(d['Instructions Executed'] or 0)/1e6:7.2f}M  {d['Source'].strip()[:80]}")
