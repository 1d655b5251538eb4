export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python bench.py --scheme walk --steps 50 --warmup 3 --cpu-seconds 8 > gpurun_out/bench_walk_r01k.json 2> gpurun_out/bench_walk_r01k.err; echo "walk rc=$?"; tail -3 gpurun_out/bench_walk_r01k.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_walk_r01k.json').read().strip().splitlines()[-1]); print(d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], d['e2e']['value']/1e9, d['cpu_baseline']['value']/1e6)"
timeout 300 python -m pytest tests/test_gpu_parity.py -q -k walk 2>&1 | tail -2
