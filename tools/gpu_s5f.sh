timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "consumer_discard or halo or dag" 2>&1 | tail -1
C='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true,"halo_discard":true},{"kind":"budget","l2_fraction":0.75,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true,"halo_discard":true}]'
timeout 600 python tools/sweep.py --reps 11 --configs "$C" 2>&1 | python tools/compact.py
timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum --csv \
  python tools/sweep.py --reps 1 --configs "$C" > gpurun_out/traffic_hd3.csv 2> /dev/null
python3 tools/traffic_summary.py gpurun_out/traffic_hd3.csv 2>/dev/null | awk 'NR%3==2'
