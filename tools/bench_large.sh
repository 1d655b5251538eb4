#!/bin/bash
# bench lines at BASELINE configs[3]/[4] shapes on one GPU (P = 1: the whole graph on one B200)
export PYTHONUNBUFFERED=1
tag=${1:-r01}
for c in papers friendster; do
  timeout 1500 python bench.py --config $c --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${c}_$tag.json 2> gpurun_out/bench_${c}_$tag.err; echo "$c rc=$?"
  python -c "
import json; d=json.loads(open('gpurun_out/bench_${c}_$tag.json').read().strip().splitlines()[-1]); print('$c', round(d['value']/1e9,3), 'G edges/s', round(d['ms_per_step'],4), 'ms', 'frac', round(d['roofline']['frac'],3), 'cpu', d['cpu_baseline'] and round(d['cpu_baseline']['value']/1e6,2))"
done
