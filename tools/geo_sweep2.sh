CFG='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.5,"exec_mode":"dag","discard":true,"resident_budget":true,"window":2}]'
for g in '{}' '{"thresh":[256,32,128],"down":[256,32,128]}' '{"thresh":[256,32,64],"down":[256,32,64]}' '{"thresh":[256,32,128],"down":[256,32,128],"gray":[256,64,128]}' '{"thresh":[512,32,128],"down":[512,32,128]}' '{"thresh":[256,32,128],"down":[256,32,128],"gray":[256,32,64]}' '{"thresh":[256,64,128],"down":[256,64,128],"sobel":[256,128,256]}'; do
  echo "geom $g"; KTILER_GEOMETRY="$g" timeout 300 python tools/sweep.py --configs "$CFG" 2>&1 | grep -o '"ms": [0-9.]*' | tr '\n' ' '; echo
done
