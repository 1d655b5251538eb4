#!/bin/bash
# One GPU session: smoke, GPU tests, bench, launch list.  Each step bounded by timeout.
# TAG=<name> names the outputs under gpurun_out/.
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
T=${TAG:-check}
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build()" || exit 1
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -5
echo "== pytest gpu (fast)"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -15
echo "== bench"; timeout 900 python bench.py --steps ${STEPS:-100} --warmup 5 --cpu-seconds 10 > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err; tail -3 gpurun_out/bench_$T.err; cat gpurun_out/bench_$T.json
if [ -z "$NOSLOW" ]; then echo "== pytest gpu (slow)"; timeout 1500 python -m pytest tests -m "gpu and slow" -x -q 2>&1 | tail -15; fi
