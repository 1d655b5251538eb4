export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== multiprocess channels"; timeout 600 python -m pytest tests/test_gpu_multiprocess.py -x -q -k "node-2" 2>&1 | grep -v "^\s*$" | tail -8
echo "== split row micro"; timeout 300 ./tools/micro/split_row_bench 2>&1 | tail -20
