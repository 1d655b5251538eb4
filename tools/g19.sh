export PYTHONUNBUFFERED=1
bash tools/profile.sh r01l k_csp
for c in papers friendster; do
  timeout 1500 python bench.py --config $c --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${c}_r01l.json 2> gpurun_out/bench_${c}_r01l.err; echo "$c rc=$?"
  python -c "
import json; d=json.loads(open('gpurun_out/bench_${c}_r01l.json').read().strip().splitlines()[-1]); print('$c', round(d['value']/1e9,3), 'G edges/s', round(d['ms_per_step'],4), 'ms', 'frac', round(d['roofline']['frac'],3), 'e2e', round(d['e2e']['value']/1e9,3))"
done
bash tools/bench_all.sh r01l
