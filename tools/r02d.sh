export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== multiprocess channels"; timeout 600 python -m pytest tests/test_gpu_multiprocess.py -x -q -k "node-2" 2>&1 | grep -v "^\s*$" | tail -30
echo "== phases bench K=4"; K=4 timeout 600 python tools/phases_bench.py 12 2>&1 | tail -30
echo "== phases bench K=1"; K=1 timeout 600 python tools/phases_bench.py 12 2>&1 | tail -30
