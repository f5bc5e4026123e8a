timeout 900 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s5c.json)" 2>&1 | tee gpurun_out/executors_final.jsonl | python tools/compact.py
