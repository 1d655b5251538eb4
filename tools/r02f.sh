export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
echo "== multiprocess"; timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -3
for K in 4 3; do echo "== bench K=$K"; timeout 600 python bench.py --steps 200 --warmup 5 --instances $K --no-cpu-baseline --no-breakdown 2> gpurun_out/b_k$K.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['frac'], d['e2e']['value']/1e9, d['clocks'])"; tail -2 gpurun_out/b_k$K.err; done
echo "== phases bench K=4"; K=4 timeout 600 python tools/phases_bench.py 12 2>&1 | tail -20
