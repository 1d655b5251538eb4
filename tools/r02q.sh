export PYTHONUNBUFFERED=1
VARIANTS="main old" ROUNDS=3 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | tail -6
for v in main old; do lib=""; [ "$v" = old ] && lib=paper_conf_ppopp_caiz0zszck23_b200/libdsp_old.so
  echo "== $v K=1"; DSP_LIB=$lib K=1 timeout 600 python tools/phases_bench.py 10 2>&1 | head -1
  echo "== $v biased"; DSP_LIB=$lib timeout 600 python bench.py --scheme biased --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['frac'])"
done
