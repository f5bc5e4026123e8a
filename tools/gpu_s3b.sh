timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
bash tools/kprof.sh s3b
timeout 300 python tools/sweep.py --configs "$(cat tools/cfg_s3.json)" 2>&1 | grep -v "^$" | cut -c1-200
for g in '{"blur":[256,64,32],"sobel":[256,64,32]}' '{"gray":[256,32,128],"down":[256,32,128],"thresh":[256,32,128]}' '{"blur":[256,64,64],"sobel":[256,64,128]}'; do
  echo "geom $g"; timeout 300 python tools/sweep.py --geom "$g" --configs "$(cat tools/cfg_s3.json)" 2>&1 | grep -v "^$" | cut -c1-200
done
