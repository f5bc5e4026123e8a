KTILER_EVICT_READS=1 timeout 600 python tools/sweep.py --reps 9 --configs "$(cat tools/cfg_s4a.json)" 2>&1 | python tools/compact.py
