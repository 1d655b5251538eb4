#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${TAG:-r02b}
python -c "from paper_conf_ppopp_caiz0zszck23_b200 import _build; _build.build()" || exit 1
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -2
echo "== pytest gpu"; timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -4 | tee gpurun_out/gputest_$T.txt
echo "== bench products"; timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err; tail -c 300 gpurun_out/bench_$T.json; echo
for sc in biased layer walk; do echo "== bench $sc"; timeout 900 python bench.py --scheme $sc --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${sc}_$T.json 2> gpurun_out/bench_${sc}_$T.err; tail -c 200 gpurun_out/bench_${sc}_$T.json; echo; done
echo "== bench same-gpu 2 procs"; DSP_BENCH_SAME_GPU=1 timeout 900 python bench.py --gpus 2 --steps 30 --warmup 3 --cpu-seconds 10 > gpurun_out/bench_same_gpu2_$T.json 2> gpurun_out/bench_same_gpu2_$T.err; tail -c 200 gpurun_out/bench_same_gpu2_$T.json; echo
echo "== phases"; K=4 timeout 600 python tools/phases_bench.py 12 > gpurun_out/phases_bench_$T.txt 2>&1; head -3 gpurun_out/phases_bench_$T.txt; K=1 timeout 600 python tools/phases_bench.py 12 > gpurun_out/phases_bench_k1_$T.txt 2>&1; head -2 gpurun_out/phases_bench_k1_$T.txt
echo "== ncu launch list"; timeout 900 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/launches_$T.log 2>&1; echo rc=$?
echo "== ncu bench-config launch"; timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 7 -c 2 -o gpurun_out/prof_$T -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_$T.log 2>&1; echo rc=$?
echo "== ncu single"; timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 6 -c 1 -o gpurun_out/prof_single_$T -f python bench.py --instances 1 --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_single_$T.log 2>&1; echo rc=$?
for t in $T single_$T; do python tools/ncu_summary.py gpurun_out/prof_$t.ncu-rep gpurun_out/launches_$T.csv $t > /dev/null 2>&1; cp profiles/ncu_$t.md gpurun_out/; done
cp profiles/ncu_traffic.json gpurun_out/ncu_traffic_box.json
rm -f gpurun_out/prof_$T.ncu-rep
for cfg in papers friendster; do echo "== bench $cfg"; timeout 1500 python bench.py --config $cfg --steps 50 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${cfg}_$T.json 2> gpurun_out/bench_${cfg}_$T.err; tail -c 200 gpurun_out/bench_${cfg}_$T.json; echo; done
ls -la gpurun_out | tail -40
