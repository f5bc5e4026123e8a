bash tools/round_profile.sh
timeout 300 python tools/timeline.py --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.25,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true}]' 2>&1 | grep span_us > gpurun_out/timeline_s4d.jsonl
M=gpu__time_duration.sum,lts__t_sectors.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_ltcfabric.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct
timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none --metrics $M --csv \
  python tools/sweep.py --reps 1 --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.25,"exec_mode":"dag","discard":false,"resident_budget":true,"window":2}]' > gpurun_out/lts_s4d.csv 2> gpurun_out/lts_s4d.err
