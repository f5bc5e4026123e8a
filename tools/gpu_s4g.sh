C='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.25,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true}]'
for g in '{}' '{"blur":[256,64,128]}' '{"blur":[256,32,64]}' '{"sobel":[256,32,128]}' '{"gray":[256,16,128]}' '{"thresh":[256,16,128],"down":[256,16,128]}' '{"gray":[512,16,128]}' '{"blur":[512,32,64]}'; do
  echo "geom $g"; timeout 300 python tools/sweep.py --reps 7 --geom "$g" --configs "$C" 2>&1 | python tools/compact.py
done
