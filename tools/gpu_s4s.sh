N=62
for K in 1; do
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --kernel-name-base mangled -k regex:"op_kernelILi${K}ELb0" --launch-skip $((2*N)) -c $N --csv python tools/sweep.py --reps 1 --configs '[{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]' > gpurun_out/op${K}_dag_launches.csv 2> /dev/null
done
