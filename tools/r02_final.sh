#!/bin/bash
# Round-2 closing evidence at one build: tests, every bench line, ncu, sanitizer, phases.
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${TAG:-r02}
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build()" || exit 1
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
echo "== pytest gpu"; timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/gputest_$T.txt
echo "== bench products"; timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err; tail -c 400 gpurun_out/bench_$T.json; echo
echo "== bench reference"; timeout 900 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/bench_reference_$T.json 2>&1; tail -c 300 gpurun_out/bench_reference_$T.json; echo
for sc in biased layer walk; do echo "== bench $sc"; timeout 900 python bench.py --scheme $sc --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${sc}_$T.json 2> gpurun_out/bench_${sc}_$T.err; tail -c 300 gpurun_out/bench_${sc}_$T.json; echo; done
echo "== bench hot25"; timeout 900 python bench.py --hot-frac 0.25 --steps 30 --warmup 3 --cpu-seconds 5 > gpurun_out/bench_hot25_$T.json 2> gpurun_out/bench_hot25_$T.err; tail -c 300 gpurun_out/bench_hot25_$T.json; echo
echo "== bench same-gpu 2 procs"; DSP_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 30 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_same_gpu2_$T.json 2> gpurun_out/bench_same_gpu2_$T.err; tail -c 300 gpurun_out/bench_same_gpu2_$T.json; echo
echo "== phases"; K=4 timeout 600 python tools/phases_bench.py 12 > gpurun_out/phases_bench_$T.txt 2>&1; cat gpurun_out/phases_bench_$T.txt | head -3
echo "== virtual"; timeout 900 python tools/virtual_time.py > gpurun_out/multi_virtual_$T.txt 2>&1; tail -3 gpurun_out/multi_virtual_$T.txt
echo "== ncu launch list"; timeout 900 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/launches_$T.log 2>&1; echo rc=$?
echo "== ncu full"; timeout 1500 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:"k_csp_persistent|k_gather_tma" -s 6 -c 3 -o gpurun_out/prof_$T -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline > gpurun_out/prof_$T.log 2>&1; echo rc=$?
echo "== ncu biased"; timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_csp_persistent -s 8 -c 1 -o gpurun_out/prof_biased_$T -f python bench.py --scheme biased --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_biased_$T.log 2>&1; echo rc=$?
for cfg in papers friendster; do echo "== bench $cfg"; timeout 1500 python bench.py --config $cfg --steps 50 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${cfg}_$T.json 2> gpurun_out/bench_${cfg}_$T.err; tail -c 300 gpurun_out/bench_${cfg}_$T.json; echo; done
