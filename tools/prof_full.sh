#!/bin/bash
# Full ncu capture (source-correlated) of the five untiled op kernels, plus per-kernel
# counters at 4096^2 (the whole graph fits L2: every input but rgb is an L2 hit).
# Usage: tools/prof_full.sh [tag]
tag=${1:-full}
W=${W:-7680} H=${H:-4320} F=${F:-64}
timeout 900 ncu --set full --import-source on --clock-control none -k regex:op_kernel -c 5 -f -o gpurun_out/prof_$tag \
  python tools/sweep.py --W $W --H $H --F $F --reps 1 --configs '[{"kind":"none","exec_mode":"stream"}]' > gpurun_out/prof_$tag.log 2>&1
echo "ncu rc=$?"
