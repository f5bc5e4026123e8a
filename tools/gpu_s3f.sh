export KTILER_STAGE_POINTWISE=1
./tools/l2bw 2>&1
ncu --query-metrics --chip gb100 2>/dev/null | grep -E "^lts__t_(sectors|requests|bytes)" | head -80 > gpurun_out/lts_metrics.txt
wc -l gpurun_out/lts_metrics.txt
CFG='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.5,"exec_mode":"dag","discard":true,"resident_budget":true,"window":2},{"kind":"budget","l2_fraction":0.5,"exec_mode":"dag","discard":false,"resident_budget":true,"window":2}]'
M=gpu__time_duration.sum,lts__t_bytes.sum,lts__t_sectors.sum,lts__t_sectors_op_read.sum,lts__t_sectors_op_write.sum,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,lts__t_sectors_srcunit_tex.sum,lts__t_sectors_srcunit_ltcfabric.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__throughput.avg.pct_of_peak_sustained_elapsed
timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none --metrics $M --csv \
  python tools/sweep.py --reps 1 --configs "$CFG" > gpurun_out/lts_break.csv 2> gpurun_out/lts_break.err
echo "rc=$?"; tail -3 gpurun_out/lts_break.err
