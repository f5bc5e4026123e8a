#!/bin/bash
# Geometry experiments: per-kernel counters (untiled) + end-to-end times for each
# KTILER_GEOMETRY override given as arguments (JSON objects).
i=0
for G in "$@"; do
  i=$((i+1))
  echo "=== geometry $G"
  KTILER_GEOMETRY="$G" ./tools/kprof.sh g$i
  KTILER_GEOMETRY="$G" KTILER_TILES_PER_CTA=${TPC:-2} timeout 300 python tools/sweep.py --reps 7 --configs '[{"kind":"none","exec_mode":"graph"},{"kind":"budget","l2_fraction":1.0,"exec_mode":"graph","discard":true},{"kind":"budget","l2_fraction":1.0,"exec_mode":"dag","discard":true,"window":2}]' 2>&1 | grep -v "^$" | python3 -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l); print('   ', d['cfg'].get('exec_mode'), d['cfg'].get('kind'), d['ms'])
    except Exception: pass"
done
