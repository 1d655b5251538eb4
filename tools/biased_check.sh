#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build()" || exit 1
echo "== pytest biased"; timeout 600 python -m pytest tests -m gpu -x -q -k "biased" 2>&1 | tail -3
echo "== pytest gpu fast"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
echo "== biased phases"; MODES=biased timeout 300 python tools/phases.py 12 2>&1 | tee gpurun_out/phases_biased_s3.txt
echo "== bench biased"; timeout 600 python bench.py --scheme biased --steps 100 --warmup 5 --no-cpu-baseline > gpurun_out/bench_biased_s3.json 2>&1; tail -1 gpurun_out/bench_biased_s3.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('GEPS', d['value']/1e9, 'ms/step', d['ms_per_step'], 'roofline', d['roofline']['frac'], d['breakdown'])"
