KTILER_PERSIST_GROUPS=0 timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "persistent" 2>&1 | tail -3
echo LITE; KTILER_PERSIST_GROUPS=0 timeout 600 python tools/sweep.py --reps 5 --configs "$(cat tools/cfg_s3o.json)" 2>&1 | python tools/compact.py
echo LITE_SMALL; KTILER_PERSIST_GROUPS=0 timeout 600 python tools/sweep.py --reps 5 --geom '{"gray":[256,16,128],"down":[256,16,128],"thresh":[256,16,128],"blur":[256,32,64],"sobel":[256,32,128]}' --configs "$(cat tools/cfg_s3o.json)" 2>&1 | python tools/compact.py
