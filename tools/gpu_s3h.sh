CFG='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.0,"exec_mode":"dag","discard":false,"resident_budget":true,"window":2}]'
for P in 256 0 128; do
echo "PROMOTION $P"
KTILER_TMA_PROMOTION=$P timeout 300 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3g.json)" 2>&1 | python tools/compact.py
M=gpu__time_duration.sum,lts__t_sectors.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_ltcfabric.sum,dram__bytes_read.sum,dram__bytes_write.sum
KTILER_TMA_PROMOTION=$P timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none --metrics $M --csv \
  python tools/sweep.py --reps 1 --configs "$CFG" > gpurun_out/lts_p$P.csv 2> gpurun_out/lts_p$P.err
done
# per-kernel SM read sectors of the untiled graph
KTILER_TMA_PROMOTION=256 timeout 600 ncu --metrics lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,gpu__time_duration.sum --clock-control none -k regex:op_kernel -c 5 --csv python tools/sweep.py --reps 1 --configs '[{"kind":"none","exec_mode":"stream"}]' > gpurun_out/lts_kern.csv 2>/dev/null
