export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
echo "== multiprocess"; timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -3
