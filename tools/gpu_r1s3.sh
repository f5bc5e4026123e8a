nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 600 python bench.py > gpurun_out/bench_s3.json 2> gpurun_out/bench_s3.err; tail -2 gpurun_out/bench_s3.err
cat gpurun_out/bench_s3.json
bash tools/prof_full.sh s3
for k in 0 1 2 3 4; do :; done
ncu -i gpurun_out/prof_s3.ncu-rep --page source --csv --print-source sass > gpurun_out/prof_s3_src.csv 2>/dev/null; ls -la gpurun_out
