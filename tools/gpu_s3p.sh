timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "modes_policies or b200_geometry" 2>&1 | tail -2
timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3p.json)" 2>&1 | python tools/compact.py
echo ALLEDGES; KTILER_DAG_PDL_EDGES=all timeout 600 python tools/sweep.py --reps 7 --configs "$(cat tools/cfg_s3p.json)" 2>&1 | python tools/compact.py
