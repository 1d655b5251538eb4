export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests -m gpu -x -q -k "biased" 2>&1 | tail -2
for rep in 1 2; do timeout 600 python bench.py --scheme biased --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('biased', d['value']/1e9, d['ms_per_step'], d['roofline']['frac'])"; done
MODES=biased timeout 300 python tools/phases.py 12 2>&1 | grep -E "total|sample"
