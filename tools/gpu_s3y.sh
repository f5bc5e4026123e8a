timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2
TPC=1 bash tools/kprof.sh s3y
timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3k.json)" 2>&1 | python tools/compact.py
