export PYTHONUNBUFFERED=1
for rep in 1 2; do
for k in 3 4 5 6; do ARGS="--instances $k" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed "s/^/K$k /"; done
ARGS="--instances 4" VARIANTS=ipl REPS=1 bash tools/ab_bench.sh | sed "s/^/K4 /"
done
