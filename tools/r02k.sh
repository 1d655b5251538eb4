export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -k "biased or hash" 2>&1 | tail -3
echo "== biased phases K=4"; BIASED=1 K=4 timeout 600 python tools/phases_bench.py 8 2>&1 | tail -16
echo "== bench biased"; timeout 600 python bench.py --scheme biased --steps 100 --warmup 5 --no-cpu-baseline --no-breakdown 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['roofline']['frac'], d['value']/1e9)"
echo "== ncu biased"; timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_csp_persistent -s 8 -c 1 -o gpurun_out/prof_biased_r02k -f python bench.py --scheme biased --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_biased_r02k.log 2>&1; echo ncu rc=$?
