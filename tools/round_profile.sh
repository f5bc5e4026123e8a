#!/bin/bash
# One GPU call's worth of round evidence (run under gpurun from the repo root):
#   gpurun_out/bench.json        python bench.py (defaults), the driver's command
#   gpurun_out/launches.csv      ncu launch list (gpu__time_duration per launch) of a short bench run
#   gpurun_out/traffic_cfg.csv   ncu graph-level DRAM bytes / L2 hit / duration of the bench's tiled
#                                 configuration and the untiled one (tools/traffic_summary.py)
set -u
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu --no-e2e --no-trace --no-untiled > gpurun_out/launches_bench.log 2>&1
echo "launches rc=$?"
CFG="$(python tools/run_sweep.py --config cfg_traffic_r01s3)"
timeout 900 ncu --graph-profiling graph --cache-control all --clock-control none \
  --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum --csv \
  python tools/sweep.py --reps 1 --configs "$CFG" > gpurun_out/traffic_cfg.csv 2> gpurun_out/traffic_cfg.err
echo "traffic rc=$?"
python3 tools/traffic_summary.py gpurun_out/traffic_cfg.csv
