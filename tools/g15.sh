export PYTHONUNBUFFERED=1
bash tools/profile.sh r01k k_csp
BENCH_ARGS="--instances 1" SKIP=6 COUNT=2 bash -c 'timeout 1500 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_csp -s 6 -c 2 -o gpurun_out/prof_r01k1 -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline --instances 1 > gpurun_out/prof_r01k1.log 2>&1'; echo "single rc=$?"
