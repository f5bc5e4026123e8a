timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3i.json)" 2>&1 | python tools/compact.py
echo TPC2; KTILER_TILES_PER_CTA=2 timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3i.json)" 2>&1 | python tools/compact.py
