export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 python bench.py --steps 200 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_r01i.json 2> gpurun_out/bench_r01i.err; echo rc=$?; tail -3 gpurun_out/bench_r01i.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_r01i.json').read().strip().splitlines()[-1]); print(round(d['value']/1e9,3), d['ms_per_step'], d['roofline']['frac'], 'e2e', d['e2e'], 'sync', d['e2e_sync']['value']/1e9)"
MODES=sample timeout 300 python tools/phases.py 12 2>&1 | tail -14
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
