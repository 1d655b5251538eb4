#!/bin/bash
# the round-end checks at the current build: smoke, the whole GPU suite, the default bench line
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${TAG:-final}
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -1
echo "== pytest gpu"; timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -2 | tee gpurun_out/gputest_$T.txt
echo "== bench"; timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err
tail -1 gpurun_out/bench_$T.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('GEPS %.3f ms/step %.4f frac %.3f e2e %.3f traffic %s' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac'], d['e2e']['value']/1e9, d['roofline']['traffic']))"
echo "== bench biased"; timeout 900 python bench.py --scheme biased --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_biased_$T.json 2> gpurun_out/bench_biased_$T.err
tail -1 gpurun_out/bench_biased_$T.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('GEPS %.3f ms/step %.4f frac %.3f' % (d['value']/1e9, d['ms_per_step'], d['roofline']['frac']))"
