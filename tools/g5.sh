export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
bash tools/bench_all.sh r01h
for c in papers friendster; do for inst in 2 4; do
  timeout 1500 python bench.py --config $c --steps 100 --warmup 5 --instances $inst --cpu-seconds 10 > gpurun_out/bench_${c}_i${inst}_r01h.json 2> gpurun_out/bench_${c}_i${inst}_r01h.err; echo "$c inst $inst rc=$?"
  python -c "
import json; d=json.loads(open('gpurun_out/bench_${c}_i${inst}_r01h.json').read().strip().splitlines()[-1]); print('$c', $inst, round(d['value']/1e9,3), 'G edges/s', round(d['ms_per_step'],4), 'ms', 'frac', round(d['roofline']['frac'],3))"
done; done
