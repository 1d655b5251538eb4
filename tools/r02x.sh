export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
echo "== slow parity"; timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_relabel_hash.py -m "gpu and slow" -x -q 2>&1 | tail -2
for v in main old; do lib=""; [ "$v" = old ] && lib=paper_conf_ppopp_caiz0zszck23_b200/libdsp_old.so
  echo "== $v K=4"; DSP_LIB=$lib K=4 timeout 600 python tools/phases_bench.py 10 2>&1 | head -1
done
VARIANTS="main old" ROUNDS=3 EXTRA="--no-cpu-baseline --no-breakdown" bash tools/ab_variants.sh 2>&1 | grep round
echo "== virtual"; P=2,4 K=1,4 timeout 600 python tools/virtual_time.py 2>&1 | tail -4
