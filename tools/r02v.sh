export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests/test_gpu_tiered.py tests/test_gpu_parity.py -m "gpu and not slow" -x -q 2>&1 | tail -3
VARIANTS="main splitdef" ROUNDS=3 EXTRA="--no-cpu-baseline" bash tools/ab_variants.sh 2>&1 | grep round
