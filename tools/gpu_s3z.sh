for E in 0 1; do echo "EVICT_READS=$E"; KTILER_EVICT_READS=$E timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3z.json)" 2>&1 | python tools/compact.py; done
