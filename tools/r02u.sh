export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
echo "== slow parity"; timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_relabel_hash.py -m "gpu and slow" -x -q 2>&1 | tail -3
echo "== phases K=1"; K=1 timeout 600 python tools/phases_bench.py 10 2>&1 | head -14
echo "== sample alone"; MODES=sample timeout 600 python tools/phases.py 10 2>&1 | head -3
VARIANTS="main" ROUNDS=2 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | grep round
