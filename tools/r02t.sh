export PYTHONUNBUFFERED=1
VARIANTS="main hu8 hu2" ROUNDS=3 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | grep round
VARIANTS="main old" ROUNDS=2 EXTRA="--scheme biased --no-cpu-baseline --no-breakdown --steps 100" bash tools/ab_variants.sh 2>&1 | grep round
