export PYTHONUNBUFFERED=1
DIM=4 KS=1,2,3,4 timeout 600 python tools/instances.py 2>&1 | grep "K="
for rep in 1 2; do
ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed 's/^/direct /'
DSP_RELABEL=hash ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed 's/^/hash /'
done
