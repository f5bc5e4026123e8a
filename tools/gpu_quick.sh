#!/bin/bash
# quick GPU check: parity tests, a short mode sweep, per-kernel instruction counts (untiled graph)
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -3
KTILER_PERSIST_MINB=${MINB:-4} timeout 300 python tools/sweep.py --configs "$(cat ${SWEEP:-tools/cfg_quick.json})" 2>&1 | grep -v "^$" | cut -c1-150
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:op_kernel -c 5 --csv python tools/sweep.py --reps 1 --configs "$(cat tools/cfg_graph_none.json)" > gpurun_out/ncu_quick.csv 2>&1
python3 - <<'PY'
import csv
rows=[r for r in csv.reader(open('gpurun_out/ncu_quick.csv')) if len(r)>10]
h=rows[0]
for r in rows[1:]:
    d=dict(zip(h,r)); print(d['Kernel Name'][16:30], d['Metric Name'][:40], d['Metric Value'])
PY
