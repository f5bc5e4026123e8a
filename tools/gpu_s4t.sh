timeout 600 python tools/sweep.py --reps 11 --configs "$(cat tools/cfg_s4t.json)" 2>&1 | python tools/compact.py
