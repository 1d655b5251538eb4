export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 900 python bench.py --steps 100 --warmup 5 --scheme biased --cpu-seconds 5 > gpurun_out/bench_biased_r01i.json 2> gpurun_out/bench_biased_r01i.err; echo "biased rc=$?"; tail -2 gpurun_out/bench_biased_r01i.err
timeout 900 python bench.py --steps 100 --warmup 5 --hot-frac 0.25 --cpu-seconds 5 > gpurun_out/bench_hot25_r01i.json 2> gpurun_out/bench_hot25_r01i.err; echo "hot rc=$?"; tail -2 gpurun_out/bench_hot25_r01i.err
for f in gpurun_out/bench_biased_r01i.json gpurun_out/bench_hot25_r01i.json; do python -c "
import json; d=json.loads(open('$f').read().strip().splitlines()[-1]); print('$f', round(d['value']/1e9,3), d['ms_per_step'], d['roofline'])"; done
{
for P in 2 4 8; do P=$P timeout 300 python tools/virtual_time.py 2>&1 | tail -1; DSP_MULTI_STAGED=1 P=$P timeout 300 python tools/virtual_time.py 2>&1 | tail -1 | sed 's/^/staged: /'; P=$P timeout 300 python tools/phases_multi.py 2>&1 | tail -2; done
} > gpurun_out/multi_virtual_r01.txt 2>&1
cat gpurun_out/multi_virtual_r01.txt
