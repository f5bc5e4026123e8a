timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3k.json)" 2>&1 | python tools/compact.py
