#!/bin/bash
# fast GPU loop: parity (fast subset), phases, bench headline
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -4
timeout 300 python tools/phases.py 12 2>&1 | tail -24
timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('GEPS', d['value']/1e9, 'ms/step', d['ms_per_step'], 'roofline', d['roofline']['frac']); print(d['breakdown'])"
