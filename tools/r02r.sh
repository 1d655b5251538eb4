export PYTHONUNBUFFERED=1
echo "== tests"; timeout 900 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -3
echo "== multiprocess"; timeout 900 python -m pytest tests/test_gpu_multiprocess.py -x -q 2>&1 | tail -3
echo "== ncu single"; timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 6 -c 1 -o gpurun_out/prof_single_r02b -f python bench.py --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_single_r02b.log 2>&1; echo rc=$?
python tools/ncu_summary.py gpurun_out/prof_single_r02b.ncu-rep "" single_r02b 2>&1 | grep "^| \`"; cp profiles/ncu_single_r02b.md gpurun_out/
