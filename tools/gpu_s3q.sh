timeout 900 python tools/config_sweep.py > gpurun_out/configs_s3.jsonl 2> gpurun_out/configs_s3.err; echo "cfg rc=$?"; wc -l gpurun_out/configs_s3.jsonl
timeout 900 python bench.py --workload strip_65536 --steps 5 --no-cpu > gpurun_out/bench_strip_s3.json 2> gpurun_out/bench_strip_s3.err; echo "strip rc=$?"
timeout 600 python bench.py --workload pipeline_16384 --steps 10 --no-cpu > gpurun_out/bench_16384_s3.json 2> gpurun_out/bench_16384_s3.err; echo "16k rc=$?"
