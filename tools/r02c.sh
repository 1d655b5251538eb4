export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -5
echo "== multiprocess"; timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -5
echo "== bench 2 procs same GPU K=1"; DSP_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 30 --warmup 3 --cpu-seconds 10 --instances 1 > gpurun_out/bench_same2_k1.json 2> gpurun_out/bench_same2_k1.err; tail -3 gpurun_out/bench_same2_k1.err; cat gpurun_out/bench_same2_k1.json
echo "== bench 2 procs same GPU K=4"; DSP_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 30 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_same2_k4.json 2> gpurun_out/bench_same2_k4.err; tail -3 gpurun_out/bench_same2_k4.err; cat gpurun_out/bench_same2_k4.json
