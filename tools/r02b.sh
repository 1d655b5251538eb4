export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
for K in 4 5 6; do echo "== bench K=$K"; timeout 600 python bench.py --steps 200 --warmup 5 --instances $K --no-cpu-baseline --no-breakdown 2> gpurun_out/b_k$K.err | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['frac'], d['e2e']['value']/1e9, d['clocks'])"; tail -2 gpurun_out/b_k$K.err; done
echo "== bench 2 procs same GPU"; DSP_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 30 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_same2.json 2> gpurun_out/bench_same2.err; tail -5 gpurun_out/bench_same2.err; cat gpurun_out/bench_same2.json
