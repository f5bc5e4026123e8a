./tools/l2bw 2>&1 | grep -v '"mb": 16,'
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3g.json)" 2>&1 | python tools/compact.py
CFG='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.5,"exec_mode":"dag","discard":false,"resident_budget":true,"window":2}]'
M=gpu__time_duration.sum,lts__t_sectors.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_ltcfabric.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none --metrics $M --csv \
  python tools/sweep.py --reps 1 --configs "$CFG" > gpurun_out/lts_break2.csv 2> gpurun_out/lts_break2.err
echo "rc=$?"
