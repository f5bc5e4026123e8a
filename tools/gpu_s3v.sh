bash tools/round_profile.sh
bash tools/prof_full.sh s3v
ncu -i gpurun_out/prof_s3v.ncu-rep --page raw --csv > gpurun_out/prof_s3v_raw.csv 2>/dev/null
timeout 300 python tools/timeline.py --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.75,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true}]' 2>&1 | grep span_us > gpurun_out/timeline_s3v.jsonl
timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3j.json)" 2>&1 | python tools/compact.py
