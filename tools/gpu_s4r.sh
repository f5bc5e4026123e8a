# Final round evidence for the default plan (DAG 0.85 x L2 resident, window 2, consumer discard)
bash tools/round_profile.sh
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
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --kernel-name-base mangled -k regex:"op_kernelILi0ELb0" --launch-skip $((2*N)) -c $N --csv python tools/sweep.py --reps 1 --configs '[{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]' > gpurun_out/gray_dag_launches.csv 2> /dev/null
timeout 300 python tools/timeline.py --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]' 2>&1 | grep span_us > gpurun_out/timeline_final.jsonl
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q 2>&1 | tail -1
