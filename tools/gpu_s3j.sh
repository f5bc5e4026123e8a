timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3j.json)" 2>&1 | python tools/compact.py
timeout 300 python tools/timeline.py --configs '[{"kind":"budget","l2_fraction":0.75,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true}]' --out gpurun_out/tl_s3j.npz 2>&1 | tail -3
