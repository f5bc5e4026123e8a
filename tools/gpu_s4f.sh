timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "frame_streamer or host_io" 2>&1 | tail -2
timeout 900 python bench.py --no-cpu > gpurun_out/bench_s4f.json 2> gpurun_out/bench_s4f.err; tail -3 gpurun_out/bench_s4f.err
python -c "
import json; d=json.load(open('gpurun_out/bench_s4f.json')); print('value',round(d['value']),'ms',d['ms_per_step']); print(d['e2e'])"
for c in 4 16; do timeout 900 python bench.py --no-cpu --no-untiled --no-trace --e2e-chunk $c | python -c "import json,sys; d=json.loads(sys.stdin.read()); print($c, d['e2e']['value'], d['e2e']['ms_per_step'])"; done
