C='[{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]'
for K in 0 1; do
timeout 900 ncu --set full --import-source on --cache-control none --clock-control none --kernel-name-base mangled -k regex:"op_kernelILi${K}ELb0" --launch-skip 140 -c 1 -f -o gpurun_out/dag_op${K}_full python tools/sweep.py --reps 1 --configs "$C" > /dev/null 2>&1
ncu -i gpurun_out/dag_op${K}_full.ncu-rep --page details --csv > gpurun_out/dag_op${K}_details.csv 2>/dev/null
done
ls -la gpurun_out | grep dag_op
