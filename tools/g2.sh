export PYTHONUNBUFFERED=1
for inst in 4 5 6 7 8 4; do ARGS="--instances $inst" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed "s/^/inst $inst /"; done
