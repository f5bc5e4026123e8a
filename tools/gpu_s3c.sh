timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
bash tools/kprof.sh s3c
timeout 300 python tools/sweep.py --configs "$(cat tools/cfg_s3.json)" 2>&1 | grep -v "^$" | cut -c1-150
echo STAGED; KTILER_STAGE_POINTWISE=1 timeout 300 python tools/sweep.py --configs "$(cat tools/cfg_s3.json)" 2>&1 | grep -v "^$" | cut -c1-150
for g in '{"blur":[256,64,128]}' '{"blur":[256,64,32]}' '{"sobel":[256,64,64]}' '{"gray":[256,32,256],"down":[256,32,256],"thresh":[256,32,256]}' '{"gray":[256,64,128],"down":[256,64,128],"thresh":[256,64,128]}'; do
  echo "geom $g"; timeout 300 python tools/sweep.py --geom "$g" --configs "$(cat tools/cfg_s3.json)" 2>&1 | grep -v "^$" | cut -c1-150
done
