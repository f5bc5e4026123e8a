C='[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":0.85,"exec_mode":"dag","discard":false,"window":2,"resident_budget":true,"consumer_discard":true}]'
for i in 1 2; do timeout 600 python tools/sweep.py --reps 11 --configs "$C" 2>&1 | python tools/compact.py; done
