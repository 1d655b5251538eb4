export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -2
echo "== mp"; timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -2
VARIANTS="main old" ROUNDS=4 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | grep round
echo "== virtual"; timeout 900 python tools/virtual_time.py 2>&1 | tail -9
