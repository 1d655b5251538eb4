#!/bin/bash
# quick perf loop: GPU parity (fast), sample-only phases, sampling-alone
# throughput (DIM=4 => no gather), bench headline
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
MODES=sample timeout 200 python tools/phases.py 12 2>&1 | head -12
DIM=4 KS=1,4 timeout 300 python tools/instances.py 2>&1 | grep "K="
timeout 300 python bench.py --steps 200 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('BENCH GEPS %.3f ms/step %.4f frac %.3f' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac']))"
