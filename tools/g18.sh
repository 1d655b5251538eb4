export PYTHONUNBUFFERED=1
for rep in 1 2; do
for lr in 4 8 16 32; do DSP_LANE_ROUNDS=$lr ARGS="" VARIANTS=base REPS=1 bash tools/ab_bench.sh | sed "s/^/lr$lr /"; done
done
