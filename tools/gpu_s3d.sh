S="timeout 300 python tools/sweep.py --reps 7"
$S --configs "$(cat tools/cfg_s3.json)" 2>&1 | python tools/compact.py
echo STAGED; KTILER_STAGE_POINTWISE=1 $S --configs "$(cat tools/cfg_s3.json)" 2>&1 | python tools/compact.py
echo STAGED64; KTILER_STAGE_POINTWISE=1 $S --geom '{"gray":[256,32,64],"down":[256,32,64],"thresh":[256,32,64]}' --configs "$(cat tools/cfg_s3.json)" 2>&1 | python tools/compact.py
for g in '{"blur":[256,64,128]}' '{"sobel":[256,64,64]}' '{"gray":[256,64,128],"down":[256,64,128],"thresh":[256,64,128]}'; do
  echo "geom $g"; $S --geom "$g" --configs "$(cat tools/cfg_s3.json)" 2>&1 | python tools/compact.py
done
