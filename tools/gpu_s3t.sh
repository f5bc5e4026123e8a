timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
bash tools/kprof.sh s3t
timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3k.json)" 2>&1 | python tools/compact.py
