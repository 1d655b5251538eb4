#!/bin/bash
# One GPU session: smoke, GPU tests, bench, launch list.  Each step bounded by timeout.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -5
echo "== pytest gpu (fast)"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -15
echo "== bench"; timeout 900 python bench.py --steps 30 --warmup 5 --cpu-seconds 10 > gpurun_out/bench.json 2> gpurun_out/bench.err; tail -3 gpurun_out/bench.err; cat gpurun_out/bench.json
echo "== pytest gpu (slow)"; timeout 1200 python -m pytest tests -m "gpu and slow" -x -q 2>&1 | tail -15
