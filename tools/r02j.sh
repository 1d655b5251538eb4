export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
echo "== bench"; timeout 600 python bench.py --steps 200 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_r02j.json 2> gpurun_out/bench_r02j.err; tail -2 gpurun_out/bench_r02j.err; python -c "import json; d=json.load(open('gpurun_out/bench_r02j.json')); print(d['ms_per_step'], d['roofline']['frac'], d['e2e']['value']/1e9, d['breakdown'])"
echo "== biased phases K=4"; BIASED=1 K=4 timeout 600 python tools/phases_bench.py 8 2>&1 | tail -20
echo "== biased phases K=1"; BIASED=1 K=1 timeout 600 python tools/phases_bench.py 8 2>&1 | tail -20
