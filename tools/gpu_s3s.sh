for T in 2 1; do echo "TPC=$T"; TPC=$T bash tools/kprof.sh tpc$T; done
KTILER_TILES_PER_CTA=1 timeout 300 python tools/sweep.py --reps 7 --configs '[{"kind":"none","exec_mode":"graph"}]' 2>&1 | python tools/compact.py
