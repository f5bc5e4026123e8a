timeout 1200 python tools/hs_sweep.py --reps 5 2>&1 | tee gpurun_out/hs_sweep.jsonl | tail -40
