export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_layerwise.py -x -q 2>&1 | tail -3
for rep in 1 2; do
timeout 600 python bench.py --scheme layer --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('pers', d['value']/1e6, 'M edges/s', d['ms_per_step'], 'host', d['host_issue_ms_per_step'])"
DSP_LW_STAGED=1 timeout 600 python bench.py --scheme layer --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('staged', d['value']/1e6, 'M edges/s', d['ms_per_step'], 'host', d['host_issue_ms_per_step'])"
done
