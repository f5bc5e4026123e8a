C='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]'
for g in '{}' '{"blur":[256,64,128]}' '{"blur":[256,128,64]}' '{"blur":[512,64,128]}' '{"sobel":[256,64,64]}' '{"sobel":[256,128,128]}' '{"gray":[256,64,128]}'; do
  echo "geom $g"; timeout 300 python tools/sweep.py --reps 9 --geom "$g" --configs "$C" 2>&1 | python tools/compact.py
done
