timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -1
bash tools/round_profile.sh > /dev/null 2>&1; echo "round rc=$?"
timeout 300 python tools/timeline.py --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]' 2>&1 | grep span_us > gpurun_out/timeline_final.jsonl
bash tools/prof_full.sh s5a > /dev/null 2>&1
ncu -i gpurun_out/prof_s5a.ncu-rep --page raw --csv > gpurun_out/prof_s5a_raw.csv 2>/dev/null
python3 tools/traffic_summary.py gpurun_out/traffic_cfg.csv | head -6
