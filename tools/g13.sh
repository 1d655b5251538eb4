export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for rep in 1 2 3; do
ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed 's/^/direct32 /'
DSP_RELABEL=direct64 ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed 's/^/direct64 /'
done
