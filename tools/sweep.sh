#!/bin/bash
# env-knob sweep: phases (sample-only, full GPU) + 2-stream pipelined throughput
# usage: VAR=DSP_LANE_ROUNDS VALUES="0 1 2 4 8" bash tools/sweep.sh
export PYTHONUNBUFFERED=1
for v in $VALUES; do
  echo "=== $VAR=$v"
  env $VAR=$v MODES=sample timeout 200 python tools/phases.py 12 2>&1 | head -12
  env $VAR=$v timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('GEPS %.3f ms/step %.4f frac %.3f' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac']))"
done
