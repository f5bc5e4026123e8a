for T in "" "2,1,1,1,1" "2,2,1,1,1" "2,1,2,1,2" "4,1,1,1,1" "2,2,2,2,2" "1,2,1,1,1"; do
echo "TPC_OPS=$T"; KTILER_TPC_OPS=$T timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3k.json)" 2>&1 | python tools/compact.py
done
