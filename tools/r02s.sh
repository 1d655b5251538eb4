export PYTHONUNBUFFERED=1
VARIANTS="main noinl" ROUNDS=3 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | grep round
for v in main noinl; do lib=""; [ "$v" = noinl ] && lib=paper_conf_ppopp_caiz0zszck23_b200/libdsp_noinl.so
  echo "== $v K=1"; DSP_LIB=$lib K=1 timeout 600 python tools/phases_bench.py 10 2>&1 | head -1
done
