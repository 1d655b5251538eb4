#!/bin/bash
# closing evidence at the current build (1 GPU): smoke, the whole GPU suite,
# every bench line, the ncu launch list and full captures of the bench-config
# uniform and biased launches
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
T=${TAG:-r02c}
NCU=/usr/local/cuda/bin/ncu
echo "== smoke"; timeout 300 python __graft_entry__.py smoke 2>&1 | tail -1
echo "== pytest gpu"; timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -3 | tee gpurun_out/gputest_$T.txt
echo "== bench products"; timeout 900 python bench.py > gpurun_out/bench_$T.json 2> gpurun_out/bench_$T.err; tail -c 300 gpurun_out/bench_$T.json; echo
for sc in biased layer walk; do echo "== bench $sc"; timeout 900 python bench.py --scheme $sc --steps 100 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${sc}_$T.json 2> gpurun_out/bench_${sc}_$T.err; tail -c 200 gpurun_out/bench_${sc}_$T.json; echo; done
echo "== ncu launch list"; timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$T.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/launches_$T.log 2>&1; echo rc=$?
echo "== ncu bench-config launch"; timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 7 -c 2 -o gpurun_out/prof_$T -f python bench.py --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_$T.log 2>&1; echo rc=$?
echo "== ncu single"; TAG=$T bash tools/ncu_single.sh | tail -1
echo "== ncu biased launch"; timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:"k_csp_persistent" -s 7 -c 2 -o gpurun_out/prof_biased_$T -f python bench.py --scheme biased --steps 12 --warmup 3 --no-cpu-baseline --no-breakdown > gpurun_out/prof_biased_$T.log 2>&1; echo rc=$?
python tools/ncu_summary.py gpurun_out/prof_$T.ncu-rep gpurun_out/launches_$T.csv $T > /dev/null 2>&1; cp profiles/ncu_$T.md gpurun_out/ 2>/dev/null
python tools/ncu_summary.py gpurun_out/prof_biased_$T.ncu-rep "" biased_$T > /dev/null 2>&1; cp profiles/ncu_biased_$T.md gpurun_out/ 2>/dev/null
cp profiles/ncu_traffic.json gpurun_out/ncu_traffic_box.json
rm -f gpurun_out/prof_$T.ncu-rep
for cfg in papers friendster; do echo "== bench $cfg"; timeout 1500 python bench.py --config $cfg --steps 50 --warmup 5 --cpu-seconds 10 > gpurun_out/bench_${cfg}_$T.json 2> gpurun_out/bench_${cfg}_$T.err; tail -c 200 gpurun_out/bench_${cfg}_$T.json; echo; done
ls -la gpurun_out | tail -30
