#!/bin/bash
# bench lines of the secondary workloads (products graph): biased, layer-wise (Table 7), cold tier
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
tag=${1:-r01}
timeout 900 python bench.py --steps 100 --warmup 5 --scheme biased > gpurun_out/bench_biased_$tag.json 2> gpurun_out/bench_biased_$tag.err; echo "biased rc=$?"
timeout 900 python bench.py --steps 100 --warmup 5 --scheme layer > gpurun_out/bench_layer_$tag.json 2> gpurun_out/bench_layer_$tag.err; echo "layer rc=$?"
timeout 900 python bench.py --steps 100 --warmup 5 --hot-frac 0.25 --cpu-seconds 5 > gpurun_out/bench_hot25_$tag.json 2> gpurun_out/bench_hot25_$tag.err; echo "hot rc=$?"
for f in gpurun_out/bench_*_$tag.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', round(d['value']/1e9,3), 'G edges/s', round(d['ms_per_step'],4), 'ms', 'frac', round(d['roofline']['frac'],3), 'cpu', d['cpu_baseline'] and round(d['cpu_baseline']['value']/1e6,2))"; done
