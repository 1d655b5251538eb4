export PYTHONUNBUFFERED=1
BENCH_ARGS="--instances 1" bash tools/profile.sh r01j k_csp
SKIP=2 COUNT=2 timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_gather -s 2 -c 2 -o gpurun_out/prof_r01j_gather -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline --instances 1 > gpurun_out/prof_r01j_gather.log 2>&1; echo "gather rc=$?"
