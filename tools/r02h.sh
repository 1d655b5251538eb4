export PYTHONUNBUFFERED=1
for v in main nosplit; do
  for lw in 4 8 2; do
    EXTRA="--no-breakdown --loader-warps $lw" VARIANTS="$v" ROUNDS=1 STEPS=200 bash tools/ab_variants.sh | sed "s/^/lw=$lw /"
  done
done
