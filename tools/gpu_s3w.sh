for B in 0 1 2 3; do echo "WINDOW_BACK=$B"; KTILER_DAG_WINDOW_BACK=$B timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3w.json)" 2>&1 | python tools/compact.py; done
