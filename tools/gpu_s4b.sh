timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for i in 1 2; do timeout 600 python tools/sweep.py --reps 9 --configs "$(cat tools/cfg_s4b.json)" 2>&1 | python tools/compact.py; done
