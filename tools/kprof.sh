#!/bin/bash
# Per-kernel ncu counters of the untiled 64x8K graph (one launch per kernel): time,
# warp instructions, issue-active %, warps-active %, registers.  Usage: tools/kprof.sh [tag]
tag=${1:-k}
KTILER_TILES_PER_CTA=${TPC:-2} timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,sm__warps_active.avg.pct_of_peak_sustained_active,launch__registers_per_thread,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control ${KP_CACHE:-all} -k regex:op_kernel -c 5 --csv python tools/sweep.py --W ${W:-7680} --H ${H:-4320} --F ${F:-64} --reps 1 --configs '[{"kind":"none","exec_mode":"stream"}]' > gpurun_out/kprof_$tag.csv 2>/dev/null
python3 - "$tag" <<'PY'
import csv, sys
rows=[r for r in csv.reader(open(f'gpurun_out/kprof_{sys.argv[1]}.csv')) if len(r)>10]
h=rows[0]; K={}
for r in rows[1:]:
    d=dict(zip(h,r)); K.setdefault(d['ID'],{'k':d['Kernel Name'][16:31]})[d['Metric Name']]=d['Metric Value']
names=['gray','blur','down','sobel','thresh']
for i,(k,v) in enumerate(K.items()):
    print(f"{names[i] if i<5 else v['k']:7s} {float(v['gpu__time_duration.sum'])/1e3:8.1f} us  inst {float(v['smsp__inst_executed.sum'])/1e6:7.1f}M  issue {float(v['smsp__issue_active.avg.pct_of_peak_sustained_active']):5.1f}%  warps {float(v['sm__warps_active.avg.pct_of_peak_sustained_active']):5.1f}%  regs {v['launch__registers_per_thread']}  dram {(float(v['dram__bytes_read.sum'])+float(v['dram__bytes_write.sum']))/1e9:6.2f} GB")
PY
