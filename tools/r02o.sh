export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
echo "== virtual"; timeout 900 python tools/virtual_time.py 2>&1 | tail -12
