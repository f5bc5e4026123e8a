#!/bin/bash
# One GPU call's worth of round evidence (run under gpurun from the repo root); tag = round:
#   gpurun_out/${TAG}_bench.json             python bench.py (defaults: the driver's command)
#   gpurun_out/${TAG}_bench_reference.json   python bench.py --impl reference
#   gpurun_out/${TAG}_launches_bench.csv     ncu launch list (gpu__time_duration per launch) of a short bench run
#   gpurun_out/${TAG}_dag_op{0,1}_details.csv ncu --set full of four gray / blur sub-kernel launches of the
#                                             default DAG plan (shipped geometry), serialised
#                                             (tools/full_summary.py keeps the largest grid of each)
#   gpurun_out/${TAG}_dominant_launches.csv  DRAM bytes of every gray sub-kernel launch of one execute
set -u
TAG=${1:-r02}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${TAG}_bench_reference.json 2>&1; echo "ref rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/${TAG}_launches_bench.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e --no-trace --no-untiled --no-ncu > gpurun_out/${TAG}_launches_bench.log 2>&1
echo "launches rc=$?"
C='[{"kind":"budget","l2_fraction":1.0,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true,"pdl":true}]'
for K in 0 1; do
  timeout 900 ncu --set full --import-source on --cache-control none --clock-control none --kernel-name-base mangled \
    -k regex:"op_kernelILi${K}ELb0" --launch-skip 120 -c 4 -f -o gpurun_out/${TAG}_dag_op${K}_full \
    python tools/sweep.py --reps 1 --configs "$C" > /dev/null 2>&1
  ncu -i gpurun_out/${TAG}_dag_op${K}_full.ncu-rep --page details --csv > gpurun_out/${TAG}_dag_op${K}_details.csv 2>/dev/null
done
N=$(python - <<'PY'
import sys; sys.path.insert(0, '.')
import bench, __graft_entry__ as ge
ge.build()
from paper_conf_date_maghazeh0ep19_b200 import Pipeline
p = Pipeline(7680, 4320, 64, internal=True)
pl = p.plan(0, **bench.policy(bench.parse([])))
import torch; pl.execute(0); torch.cuda.synchronize()
print(sum(1 for (sub, node, tiles) in pl.launches() if node == 0))
PY
)
echo "gray launches per execute: $N"
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct \
  --cache-control none --clock-control none --kernel-name-base mangled -k regex:"op_kernelILi0ELb0" --launch-skip $((2*N)) -c $N \
  --csv python tools/sweep.py --reps 1 --configs "$C" > gpurun_out/${TAG}_dominant_launches.csv 2> /dev/null
echo "dominant rc=$?"
